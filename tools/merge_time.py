"""Device latency of the merge kernel (graph-replayed), G sorted runs of k (dev tool)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from small_n import graph_us
for G, k in ((2, 256), (8, 256), (8, 1024), (8, 2048), (64, 256)):
    x = datagen.generate("uniform", G * 65536, "f32", seed=G + k, device="cuda")
    vs, is_ = [], []
    for r in range(G):
        v, i = tk.topk(x[r * 65536:(r + 1) * 65536], k, base=r * 65536)
        vs.append(v)
        is_.append(i)
    cv, ci = torch.cat(vs), torch.cat(is_)
    row = {"G": G, "k": k}
    for sr in (True, False):
        row["sorted" if sr else "any_order"] = graph_us(lambda: tk.merge(cv, ci, k, runs=G, sorted_runs=sr))
    print(json.dumps(row), flush=True)
