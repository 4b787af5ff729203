"""KKKV timing + parity spot check (dev; honours TOPK_LIB)."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
n = 1 << 28
ks = [datagen.generate("uniform", n, "f32", seed=datagen.config_seed(7, j), device="cuda") for j in range(3)]
for k in (64, 1024):
    f = lambda: tk.topk_kkk(*ks, k)
    for _ in range(3): f()
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(11)]
    ev[0].record()
    for t in range(10):
        f(); ev[t + 1].record()
    torch.cuda.synchronize()
    us = statistics.median(ev[t].elapsed_time(ev[t + 1]) for t in range(10)) * 1e3
    print(json.dumps({"lib": os.path.basename(os.environ.get("TOPK_LIB", "main")), "k": k, "us": round(us, 1)}), flush=True)
m = 1 << 22
r = tk.topk_kkk(*[c[:m] for c in ks], 300)
o = oracle.topk_kkk(*[c[:m].cpu().numpy() for c in ks], 300)
print("parity", bool(np.array_equal(r[3].cpu().numpy(), o[3])))
