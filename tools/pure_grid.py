"""Pure-kernel grid-size A/B for small inputs (dev): graph-timed device latency per env."""
import json, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import json, sys
sys.path.insert(0, "."); sys.path.insert(0, "tools")
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
from small_n import graph_us
out = {}
for lg in (16, 18, 20, 22):
    n = 1 << lg
    x = datagen.generate("uniform", n, "f32", seed=5, device="cuda")
    for k in (8, 32):
        v = torch.empty(k, dtype=torch.float32, device="cuda")
        i = torch.empty(k, dtype=torch.int64, device="cuda")
        ws = tk.Workspace(tk.workspace_bytes(torch.float32, n, k), "cuda")
        out[f"{lg}/{k}"] = graph_us(lambda: tk.topk(x, k, out=(v, i, None), workspace=ws))
print(json.dumps(out))
'''
for g in sys.argv[1:]:
    env = dict(os.environ, TOPK_PURE_GRID=g)
    r = subprocess.run([sys.executable, "-c", CHILD], cwd=ROOT, env=env, capture_output=True, text=True)
    print(g, r.stdout.strip() or r.stderr[-300:], flush=True)
