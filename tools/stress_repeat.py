"""Repeat one top-k call many times against the oracle (dev): catches nondeterminism."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
dt, lg, k, reps = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
dist = sys.argv[5] if len(sys.argv) > 5 else "uniform"
seed = int(sys.argv[6]) if len(sys.argv) > 6 else None
n = 1 << lg
if os.environ.get("TOPK_DBG"):
    import ctypes
    from paper_conf_sigmod_shanbhagpm18_b200 import _lib
    assert _lib.load().topk_debug_flags(ctypes.c_int(int(os.environ["TOPK_DBG"], 0))) == 0
x = datagen.generate(dist, n, dt, seed=n + 17 if seed is None else seed, device="cuda")
keys = x.cpu().numpy()
ov, oi = oracle.topk(keys, k, True)
bad = 0
for r in range(reps):
    v, i = tk.topk(x, k, True)
    gi = i.cpu().numpy()
    if not np.array_equal(gi, oi):
        bad += 1
        if bad <= 3:
            d = np.nonzero(gi != oi)[0]
            print(f"rep {r}: {len(d)} mismatches, first at {d[:5]}", flush=True)
print(f"{os.environ.get('TOPK_LIB','')[-20:]} dbg={os.environ.get('TOPK_DBG')} {dt} 2^{lg} k={k} {dist} seed={seed}: {bad}/{reps} wrong", flush=True)
