"""8-byte-row query forms timing + parity spot check (dev; honours TOPK_LIB)."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
n4 = 1 << 28
lib = os.path.basename(os.environ.get("TOPK_LIB", "main"))
def med(f):
    for _ in range(3): f()
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(11)]
    ev[0].record()
    for t in range(10):
        f(); ev[t + 1].record()
    torch.cuda.synchronize()
    return round(statistics.median(ev[t].elapsed_time(ev[t + 1]) for t in range(10)) * 1e3, 1)
cnt = datagen.generate("uniform", n4, "u32", seed=datagen.config_seed(6), device="cuda")
tcol = datagen.generate("uniform", n4, "u32", seed=datagen.config_seed(6, 1), device="cuda")
print(json.dumps({"lib": lib, "q1": med(lambda: tk.query(cnt, 50, True, pred=("range", tcol, 0, 1 << 31)))}))
a = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(6, 2), device="cuda")
b = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(6, 3), device="cuda")
print(json.dumps({"lib": lib, "q2": med(lambda: tk.query(a, 50, True, rank_b=b, rank_w=0.5))}))
print(json.dumps({"lib": lib, "kkv": med(lambda: tk.topk_kk(a, b, 64))}))
m = 1 << 22
r = tk.topk_kk(a[:m], b[:m], 300)
o = oracle.topk_kk(a[:m].cpu().numpy(), b[:m].cpu().numpy(), 300)
r2 = tk.query(a[:m], 300, True, rank_b=b[:m], rank_w=0.5)
o2 = oracle.query(a[:m].cpu().numpy(), 300, True, rank_b=b[:m].cpu().numpy(), rank_w=0.5)
print("parity", bool(np.array_equal(r[2].cpu().numpy(), o[2])), bool(np.array_equal(r2[1].cpu().numpy(), o2[1])))
