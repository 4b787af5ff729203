"""Flush-network microbenchmark (dev tool): cycles per call for (P, L)."""
import sys, os, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigmod_shanbhagpm18_b200 import _lib
lib = _lib.load()
lib.topk_debug_netbench.argtypes = [ctypes.c_int] * 5 + [ctypes.c_void_p]
out = (ctypes.c_uint64 * 2)()
for e64 in (0, 1):
    for L in (0, 3, 5, 8, 10):
        for P in (1024, 2048, 4096):
            if P < 2 << L: continue
            for smem_net in ((0, 1) if L <= 8 else (1,)):
                lib.topk_debug_netbench(P, L, e64, smem_net, 20, out)
                print(json.dumps(dict(e64=e64, L=L, P=P, net="smem" if smem_net else "warp", cycles=out[0], phaseA=out[1] if not smem_net else None)), flush=True)
