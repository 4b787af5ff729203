"""A/B of the select kernel's debug switches (dev tool): b2b us per (flags, dist, k)."""
import sys, os, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen, _lib
lib = _lib.load()
n = 1 << 29
flags_list = [int(a) for a in sys.argv[1].split(",")]
dists = sys.argv[2].split(",")
ks = [int(a) for a in sys.argv[3].split(",")]
for dist in dists:
    x = datagen.generate(dist, n, "f32", seed=datagen.config_seed(2), device="cuda")
    for k in ks:
        ov = torch.empty(k, dtype=torch.float32, device="cuda"); oi = torch.empty(k, dtype=torch.int64, device="cuda")
        f = lambda: tk.topk(x, k, True, out=(ov, oi, None))
        row = {}
        for fl in flags_list:
            lib.topk_debug_flags(fl)
            for _ in range(3): f()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(20): f()
            e1.record(); torch.cuda.synchronize()
            row[fl] = round(e0.elapsed_time(e1) * 1e3 / 20, 1)
        print(json.dumps(dict(dist=dist, k=k, us=row)), flush=True)
    del x
lib.topk_debug_flags(0)
