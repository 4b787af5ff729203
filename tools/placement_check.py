import statistics, sys
sys.path.insert(0, ".")
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
n = 1 << 29
def med(f):
    for _ in range(3): f()
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(21)]
    ev[0].record()
    for t in range(20):
        f(); ev[t + 1].record()
    torch.cuda.synchronize()
    return round(statistics.median(ev[t].elapsed_time(ev[t + 1]) for t in range(20)) * 1e3, 1)
x = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(2), device="cuda")
print("x uniform", med(lambda: tk.topk(x, 256)))
for d in ("increasing", "decreasing", "fewdistinct"):
    y = datagen.generate(d, n, "f32", seed=datagen.config_seed(3), device="cuda")
    print("second buffer", d, med(lambda: tk.topk(y, 256)))
    x.copy_(y)
    print("first buffer", d, med(lambda: tk.topk(x, 256)))
    del y
