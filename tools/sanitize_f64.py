"""f64 k >= 1024 calls for a compute-sanitizer racecheck run (dev)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
lg = int(sys.argv[1]) if len(sys.argv) > 1 else 22
x = datagen.generate("uniform", 1 << lg, "f64", seed=(1 << lg) + 17).cuda()
keys = x.cpu().numpy()
print("gen", flush=True)
for k in (1024, 2048):
    v, i = tk.topk(x, k, True)
    ov, oi = oracle.topk(keys, k, True)
    print(k, np.array_equal(i.cpu().numpy(), oi), flush=True)
