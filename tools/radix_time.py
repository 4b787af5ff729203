"""CUDA-event timing of radix select vs bitonic top-k on 2^29 uniform f32 (dev tool)."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
x = datagen.generate("uniform", 1 << 29, "f32", seed=datagen.config_seed(2), device="cuda")
for k in (32, 256, 1024):
    for name, f in (("radix", lambda: tk.topk_radix(x, k)), ("bitonic", lambda: tk.topk(x, k))):
        for _ in range(3): f()
        torch.cuda.synchronize()
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(11)]
        ev[0].record()
        for t in range(10):
            f(); ev[t + 1].record()
        torch.cuda.synchronize()
        us = statistics.median(ev[t].elapsed_time(ev[t + 1]) for t in range(10)) * 1e3
        print(json.dumps({"k": k, "impl": name, "us": round(us, 1)}), flush=True)
