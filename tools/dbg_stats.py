"""Per-launch debug counters of a -DTOPK_DEBUG library (dev):
    TOPK_LIB=variants/libtopk_X.so python tools/dbg_stats.py LG DIST K [K ...]
g_stats (select.cuh): flushes, survivors flushed, flush cycles, deferrals, tiles, refreshes,
exact flushes, sentinel outputs -- totals over all CTAs of one launch."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen, _lib
lib = _lib.load()
lib.topk_debug_stats.argtypes = [ctypes.c_void_p, ctypes.c_int]
lg, dist = int(sys.argv[1]), sys.argv[2]
x = datagen.generate(dist, 1 << lg, "f32", seed=datagen.config_seed(2), device="cuda")
names = ["flushes", "survivors", "flush_cyc", "deferrals", "tiles", "refreshes", "exact", "sentinel"]
for k in map(int, sys.argv[3:]):
    tk.topk(x, k); torch.cuda.synchronize()
    h = np.zeros(8, dtype=np.uint64)
    assert lib.topk_debug_stats(h.ctypes.data, 1) == 0
    tk.topk(x, k); torch.cuda.synchronize()
    assert lib.topk_debug_stats(h.ctypes.data, 1) == 0
    d = dict(zip(names, (int(v) for v in h)))
    d["flush_us_per_cta"] = round(d["flush_cyc"] / 1.965e3 / 148, 1)
    print(f"{os.environ.get('TOPK_LIB','')[-16:]} 2^{lg} {dist} k={k}: {d}", flush=True)
