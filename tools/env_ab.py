"""Runtime-knob A/B (dev tool): time 2^29 f32 top-k (k = 1, 256) in a subprocess per env
setting (TOPK_BLOCK, TOPK_WAVE, TOPK_PERM, TOPK_LIB are read once per process)."""
import json, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import json, statistics, sys
sys.path.insert(0, ".")
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
x = datagen.generate("uniform", 1 << 29, "f32", seed=datagen.config_seed(2), device="cuda")
out = {}
for k in (1, 256, 1024):
    f = lambda: tk.topk(x, k)
    for _ in range(3): f()
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(31)]
    ev[0].record()
    for t in range(30):
        f(); ev[t + 1].record()
    torch.cuda.synchronize()
    out[k] = round(statistics.median(ev[t].elapsed_time(ev[t + 1]) for t in range(30)) * 1e3, 1)
print(json.dumps(out))
'''
for spec in sys.argv[1:]:
    env = dict(os.environ)
    for kv in filter(None, spec.split(",")):
        a, b = kv.split("=")
        env[a] = b
    r = subprocess.run([sys.executable, "-c", CHILD], cwd=ROOT, env=env, capture_output=True, text=True)
    print(spec or "default", r.stdout.strip() or r.stderr[-300:], flush=True)
