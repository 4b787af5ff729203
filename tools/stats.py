"""Per-launch flush statistics of select_kernel (dev tool)."""
import sys, os, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen, _lib
lib = _lib.load()
lib.topk_debug_stats.argtypes = [ctypes.c_void_p, ctypes.c_int]
n = int(sys.argv[1]); dist = sys.argv[2]; mode = sys.argv[3]
ks = [int(a) for a in sys.argv[4].split(",")]
x = datagen.generate(dist, n, "f32", seed=datagen.config_seed(2), device="cuda")
buf = (ctypes.c_uint64 * 8)()
for k in ks:
    tk.topk(x, k, mode=mode); torch.cuda.synchronize()
    lib.topk_debug_stats(buf, 1)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); tk.topk(x, k, mode=mode); e1.record(); torch.cuda.synchronize()
    lib.topk_debug_stats(buf, 1)
    print(json.dumps(dict(k=k, dist=dist, mode=mode, ms=e0.elapsed_time(e1), flushes=buf[0], survivors=buf[1],
          flush_cyc_per_flush=buf[2] / max(1, buf[0]), deferrals=buf[3], tiles=buf[4])), flush=True)
