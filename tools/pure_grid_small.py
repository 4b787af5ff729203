"""Small-n latency of the pure kernel (graph-replayed, dev; honours TOPK_LIB and
TOPK_PURE_GRID): 2^12 .. 2^22 at k = 8 / 32, plus pure mode k = 256 at 2^20, and a
parity check of each against the oracle."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
from small_n import graph_us
lib = os.path.basename(os.environ.get("TOPK_LIB", "main"))
for lg in (12, 16, 18, 20, 22):
    x = datagen.generate("uniform", 1 << lg, "f32", seed=3, device="cuda")
    ok = all(np.array_equal(tk.topk(x, k)[1].cpu().numpy(), oracle.topk(x.cpu().numpy(), k, True)[1])
             for k in (8, 32))
    row = {"lib": lib, "lg": lg, "ok": ok, "k32": graph_us(lambda: tk.topk(x, 32)),
           "k8": graph_us(lambda: tk.topk(x, 8))}
    if lg == 20:
        row["pure256"] = graph_us(lambda: tk.topk(x, 256, mode="pure"))
    print(json.dumps(row), flush=True)
