"""A/B of topk on several distributions (dev tool)."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
n = 1 << 29
ks = [int(a) for a in sys.argv[1].split(",")]
dists = sys.argv[2].split(",")
out = []
for d in dists:
    x = datagen.generate(d, n, "f32", seed=datagen.config_seed(2), device="cuda")
    for k in ks:
        tk.topk(x, k); torch.cuda.synchronize()
        r = []
        for _ in range(5):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); tk.topk(x, k); e1.record(); torch.cuda.synchronize()
            r.append(e0.elapsed_time(e1) * 1000)
        out.append(f"{d[:4]} k={k}: {min(r):.0f}")
    del x
print(" | ".join(out))
