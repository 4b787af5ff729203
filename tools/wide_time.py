"""CUDA-event timing of the wide-entry configs (f64, KKV, KKKV, BJ4a) (dev tool)."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
n = 1 << 28
dev = "cuda"
def med(f, it=10):
    for _ in range(3): f()
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(it + 1)]
    ev[0].record()
    for t in range(it):
        f(); ev[t + 1].record()
    torch.cuda.synchronize()
    return statistics.median(ev[t].elapsed_time(ev[t + 1]) for t in range(it)) * 1e3
xd = datagen.generate("uniform", n, "f64", seed=datagen.config_seed(4), device=dev)
for k in (64, 1024):
    print(json.dumps({"cfg": f"f64 k={k}", "us": round(med(lambda: tk.topk(xd, k)), 1)}))
del xd
k1 = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(7), device=dev)
k2 = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(7, 1), device=dev)
k3 = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(7, 2), device=dev)
print(json.dumps({"cfg": "KKV k=64", "us": round(med(lambda: tk.topk_kk(k1, k2, 64)), 1)}))
print(json.dumps({"cfg": "KKKV k=64", "us": round(med(lambda: tk.topk_kkk(k1, k2, k3, 64)), 1)}))
print(json.dumps({"cfg": "KKKV k=1024", "us": round(med(lambda: tk.topk_kkk(k1, k2, k3, 1024)), 1)}))
