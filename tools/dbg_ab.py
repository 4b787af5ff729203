"""A/B of the c_dbg knobs of a -DTOPK_DEBUG library (dev): CUDA-event median per setting.

    TOPK_LIB=variants/libtopk_dbg.so python tools/dbg_ab.py LG DIST K FLAGS1 FLAGS2 ...
(FLAGS in any int base, e.g. 0 0x2; select.cuh documents the bits).  Debug builds carry
trace/stat instrumentation: compare settings with each other, not with the product."""
import ctypes, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen, _lib
lib = _lib.load()
lg, dist, k = int(sys.argv[1]), sys.argv[2], int(sys.argv[3])
n = 1 << lg
x = datagen.generate(dist, n, "f32", seed=datagen.config_seed(2), device="cuda")
ov, oi = oracle.topk(x.cpu().numpy(), k, True)
for fl in sys.argv[4:]:
    assert lib.topk_debug_flags(ctypes.c_int(int(fl, 0))) == 0
    for _ in range(3):
        v, i = tk.topk(x, k)
    ok = bool(np.array_equal(i.cpu().numpy(), oi))
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(31)]
    ev[0].record()
    for t in range(30):
        tk.topk(x, k)
        ev[t + 1].record()
    torch.cuda.synchronize()
    us = statistics.median(ev[t].elapsed_time(ev[t + 1]) for t in range(30)) * 1e3
    print(f"2^{lg} {dist} k={k} flags={fl}: {us:.1f} us ok={ok}", flush=True)
lib.topk_debug_flags(ctypes.c_int(0))
