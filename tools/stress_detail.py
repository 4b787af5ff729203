"""Repeat one top-k call, and for every wrong result print which oracle entries are
missing / which extras came in (dev: diagnosing nondeterministic selection errors)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import _lib, datagen
dt, lg, k, reps = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
n = 1 << lg
lib = _lib.load()
dbg = os.environ.get("TOPK_DBG")
if dbg:
    assert lib.topk_debug_flags(ctypes.c_int(int(dbg, 0))) == 0
stats = np.zeros(8, dtype=np.uint64)
lib.topk_debug_stats.argtypes = [ctypes.c_void_p, ctypes.c_int]
x = datagen.generate("uniform", n, dt, seed=n + 17, device="cuda")
keys = x.cpu().numpy()
ov, oi = oracle.topk(keys, 2 * k, True)
order = {int(j): r for r, j in enumerate(oi)}
bad = 0
for r in range(reps):
    if dbg:
        lib.topk_debug_stats(stats.ctypes.data, 1)
    v, i = tk.topk(x, k, True)
    gi = i.cpu().numpy()
    if dbg:
        lib.topk_debug_stats(stats.ctypes.data, 0)
    if np.array_equal(gi, oi[:k]):
        continue
    bad += 1
    miss = sorted(order[int(j)] for j in set(oi[:k].tolist()) - set(gi.tolist()))
    extra = [order.get(int(j), -1) for j in set(gi.tolist()) - set(oi[:k].tolist())]
    sorted_ok = all(order.get(int(a), 1e9) < order.get(int(b), 1e9) for a, b in zip(gi, gi[1:]))
    print(f"rep {r}: missing ranks {miss[:8]} ({len(miss)}) extras ranks {sorted(extra)[:8]} "
          f"({len(extra)}) sorted={sorted_ok} stats={stats.tolist() if dbg else None}", flush=True)
print(f"dbg={dbg} {dt} 2^{lg} k={k}: {bad}/{reps} wrong", flush=True)
