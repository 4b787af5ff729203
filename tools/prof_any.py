"""Run one hot-path op a few times (for an ncu capture of its kernel; dev tool).

    python tools/prof_any.py select|pure|query1|query2|kk|kkk|radix K
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen

op, k = sys.argv[1], int(sys.argv[2])
dev = "cuda"
if op in ("select", "radix", "pure"):
    x = datagen.generate("uniform", 1 << 29, "f32", seed=datagen.config_seed(2), device=dev)
    f = {"select": lambda: tk.topk(x, k), "radix": lambda: tk.topk_radix(x, k),
         "pure": lambda: tk.topk(x, k, mode="pure")}[op]
elif op == "query1":
    n = 1 << 28
    cnt = datagen.generate("uniform", n, "u32", seed=datagen.config_seed(6), device=dev)
    t = datagen.generate("uniform", n, "u32", seed=datagen.config_seed(6, 1), device=dev)
    f = lambda: tk.query(cnt, k, True, pred=("range", t, 0, 1 << 31))
elif op == "query2":
    n = 1 << 28
    a = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(6, 2), device=dev)
    b = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(6, 3), device=dev)
    f = lambda: tk.query(a, k, True, rank_b=b, rank_w=0.5)
elif op == "kk":
    n = 1 << 28
    k1 = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(7), device=dev)
    k2 = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(7, 1), device=dev)
    f = lambda: tk.topk_kk(k1, k2, k)
elif op == "kkk":
    n = 1 << 28
    ks = [datagen.generate("uniform", n, "f32", seed=datagen.config_seed(7, j), device=dev)
          for j in range(3)]
    f = lambda: tk.topk_kkk(*ks, k)
else:
    raise SystemExit(f"unknown op {op}")
for _ in range(4):
    f()
torch.cuda.synchronize()
