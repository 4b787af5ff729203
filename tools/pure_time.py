import sys, os, json, statistics
sys.path.insert(0, '/root/repo')
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
x = datagen.generate("uniform", 1 << 29, "f32", seed=datagen.config_seed(2), device="cuda")
for k in (1, 8, 32, 64, 256, 1024):
    f = lambda: tk.topk(x, k, mode="pure")
    for _ in range(2): f()
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(6)]
    ev[0].record()
    for t in range(5):
        f(); ev[t + 1].record()
    torch.cuda.synchronize()
    us = statistics.median(ev[t].elapsed_time(ev[t + 1]) for t in range(5)) * 1e3
    print(json.dumps({"k": k, "pure_us": round(us, 1)}), flush=True)
