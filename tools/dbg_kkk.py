import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
for n in (20, 5000, 1 << 20):
    cols = [datagen.generate("fewdistinct", n, "f32", seed=331), datagen.generate("fewdistinct", n, "f32", seed=332),
            datagen.generate("uniform", n, "f32", seed=333)]
    for orders in ((False, True, False), (False, False, False), (False, True, True), (True, True, False), (True, False, True)):
        for k in (1, 4):
            out = tk.topk_kkk(*[c.cuda() for c in cols], k, orders)
            torch.cuda.synchronize()
            r = oracle.topk_kkk(*[c.numpy() for c in cols], k, orders)
            g = out[3].cpu().numpy()
            ok = np.array_equal(g, r[3])
            print(n, orders, k, "OK" if ok else "BAD", g[:4], r[3][:4],
                  [out[j].cpu().numpy()[:2] for j in range(3)], [r[j][:2] for j in range(3)], flush=True)
