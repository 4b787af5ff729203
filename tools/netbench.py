"""Flush-network microbenchmark (dev tool): cycles per call for (P, L).
net: warp = exact entry network (wnet.cuh), smem = shared-memory network,
code = code-only network (cnet.cuh)."""
import sys, os, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigmod_shanbhagpm18_b200 import _lib
lib = _lib.load()
lib.topk_debug_netbench.argtypes = [ctypes.c_int] * 5 + [ctypes.c_void_p]
out = (ctypes.c_uint64 * 3)()
nets = sys.argv[1].split(",") if len(sys.argv) > 1 else ["warp", "code", "small"]
code = {"warp": 0, "smem": 1, "code": 4, "small": 5}
for e64 in (0, 1):
    for L in (0, 3, 5, 8, 9, 10):
        for P in (512, 1024, 2048, 4096):
            if P < 2 << L: continue
            for net in nets:
                if net == "warp" and L > 8 or net == "code" and L > 9 or net == "small" and P > 1024: continue
                lib.topk_debug_netbench(P, L, e64, code[net], 20, out)
                print(json.dumps(dict(e64=e64, L=L, P=P, net=net, cycles=out[0],
                                      phaseA=out[1] if net == "warp" else None)), flush=True)
