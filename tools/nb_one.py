"""Run one flush-network microbenchmark config (for ncu): P L e64 net iters."""
import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigmod_shanbhagpm18_b200 import _lib
lib = _lib.load()
lib.topk_debug_netbench.argtypes = [ctypes.c_int] * 5 + [ctypes.c_void_p]
out = (ctypes.c_uint64 * 2)()
P, L = int(sys.argv[1]), int(sys.argv[2])
e64 = int(sys.argv[3]) if len(sys.argv) > 3 else 0
net = int(sys.argv[4]) if len(sys.argv) > 4 else 0
iters = int(sys.argv[5]) if len(sys.argv) > 5 else 20
lib.topk_debug_netbench(P, L, e64, net, iters, out)
print(P, L, e64, net, out[0], out[1])
