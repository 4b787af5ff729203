"""Small-n device latency (graph-replayed): streaming kernel vs pure kernels, k = 64 / 256
(dev; run with TOPK_PURE_SMALL_N=0 so filter mode stays on the streaming kernel)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
from small_n import graph_us
for lg in (16, 18, 20, 21, 22, 23, 24):
    n = 1 << lg
    x = datagen.generate("uniform", n, "f32", seed=5, device="cuda")
    for k in (64, 256):
        v = torch.empty(k, dtype=torch.float32, device="cuda")
        i = torch.empty(k, dtype=torch.int64, device="cuda")
        ws = tk.Workspace(tk.workspace_bytes(torch.float32, n, k), "cuda")
        row = {"log2n": lg, "k": k}
        for mode in ("filter", "pure"):
            row[mode] = graph_us(lambda: tk.topk(x, k, mode=mode, out=(v, i, None), workspace=ws))
        print(json.dumps(row), flush=True)
