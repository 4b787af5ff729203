"""Launch topk a few times on 2^29 f32 (for ncu capture of the select kernel)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
n = int(sys.argv[1]); k = int(sys.argv[2]); mode = sys.argv[3] if len(sys.argv) > 3 else "filter"
dist = sys.argv[4] if len(sys.argv) > 4 else "uniform"
x = datagen.generate(dist, n, "f32", seed=datagen.config_seed(2), device="cuda")
for _ in range(4):
    tk.topk(x, k, mode=mode)
torch.cuda.synchronize()
