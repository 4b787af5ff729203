"""Repeat the query forms / compound keys against the oracle (dev): catches nondeterminism
in their streaming passes (boot sample, flushes, tail)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
lg, reps = int(sys.argv[1]), int(sys.argv[2])
n = (1 << lg) + 4
a, b, c = (datagen.generate("uniform", n, "f32", seed=21 + j) for j in range(3))
col = datagen.generate("uniform", n, "u32", seed=24)
ad, bd, cd, cold = a.cuda(), b.cuda(), c.cuda(), col.cuda()
cases = {
    "kk": (lambda: tk.topk_kk(ad, bd, 300)[2], oracle.topk_kk(a.numpy(), b.numpy(), 300)[2]),
    "kkk": (lambda: tk.topk_kkk(ad, bd, cd, 300)[3],
            oracle.topk_kkk(a.numpy(), b.numpy(), c.numpy(), 300)[3]),
    "rank": (lambda: tk.query(ad, 300, True, rank_b=bd, rank_w=0.5)[1],
             oracle.query(a.numpy(), 300, True, rank_b=b.numpy(), rank_w=0.5)[1]),
    "pred": (lambda: tk.query(ad, 300, True, pred=("range", cold, 0, 1 << 31))[1],
             oracle.query(a.numpy(), 300, True,
                          pred=("range", col.view(torch.int32).numpy().view(np.uint32), 0, 1 << 31))[1]),
}
for name, (f, exp) in cases.items():
    bad = sum(int(not np.array_equal(f().cpu().numpy(), exp)) for _ in range(reps))
    print(f"{name} 2^{lg}+4: {bad}/{reps} wrong", flush=True)
