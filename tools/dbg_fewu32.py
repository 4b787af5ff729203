"""Debug: fewdistinct u32 parity under the select kernel's debug switches."""
import sys, os, ctypes
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen, _lib
lib = _lib.load()
buf = (ctypes.c_uint64 * 8)()
n = (1 << 18) + 5
dist = sys.argv[1] if len(sys.argv) > 1 else "fewdistinct"
dt = sys.argv[2] if len(sys.argv) > 2 else "u32"
x = datagen.generate(dist, n, dt, seed=303)
xh = x.view(torch.int32).numpy().view(np.uint32) if dt == "u32" else x.numpy()
for flags in (0, 1, 2, 4, 6, 7):
    lib.topk_debug_flags(flags)
    for k in (1, 64, 1000):
        for largest in (True, False):
            lib.topk_debug_stats(buf, 1)
            v, i = tk.topk(x.cuda(), k, largest)
            torch.cuda.synchronize()
            lib.topk_debug_stats(buf, 1)
            ov, oi = oracle.topk(xh, k, largest)
            gi = i.cpu().numpy()
            ok = np.array_equal(gi, oi)
            print(f"flags={flags} k={k} largest={largest} ok={ok} sentinels={buf[7]} flushes={buf[0]} exact={buf[6]}",
                  "" if ok else f"first bad {np.nonzero(gi != oi)[0][:3]} got {gi[np.nonzero(gi != oi)[0][:3]]} want {oi[np.nonzero(gi != oi)[0][:3]]}", flush=True)
