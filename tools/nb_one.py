import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigmod_shanbhagpm18_b200 import _lib
lib = _lib.load()
lib.topk_debug_netbench.argtypes = [ctypes.c_int] * 5 + [ctypes.c_void_p]
out = (ctypes.c_uint64 * 2)()
P, L = int(sys.argv[1]), int(sys.argv[2])
lib.topk_debug_netbench(P, L, 0, 0, 4, out)
print(P, L, out[0])
