import sys, os, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigmod_shanbhagpm18_b200 import _lib
lib = _lib.load()
lib.topk_debug_netbench.argtypes = [ctypes.c_int] * 5 + [ctypes.c_void_p]
out = (ctypes.c_uint64 * 2)()
for mode in (2, 3):
    lib.topk_debug_netbench(1024, 0, 0, mode, 20, out)
    print("mode", mode, "cycles per 64 iters", out[0])
for P, L in ((2, 0), (64, 0), (1024, 0), (512, 8), (1024, 8)):
    for net in (0, 1):
        lib.topk_debug_netbench(P, L, 0, net, 20, out)
        print(json.dumps(dict(P=P, L=L, net=["warp", "smem"][net], cycles=out[0])))
