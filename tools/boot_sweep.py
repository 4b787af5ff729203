"""Sweep the boot-buffer debug knob (select.cuh c_dbg bits 8-9) -- dev tool."""
import sys, os, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen, _lib
lib = _lib.load()
lib.topk_debug_flags.argtypes = [ctypes.c_int]
x = datagen.generate("uniform", 1 << 29, "f32", seed=datagen.config_seed(2), device="cuda")
for dist in ("uniform", "increasing"):
    if dist != "uniform":
        x = datagen.generate(dist, 1 << 29, "f32", seed=datagen.config_seed(3), device="cuda")
    for v in (0, 1, 2):
        lib.topk_debug_flags(v << 8)
        for k in (32, 256, 1024):
            for _ in range(3):
                tk.topk(x, k)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(20):
                tk.topk(x, k)
            e1.record(); torch.cuda.synchronize()
            print(json.dumps({"dist": dist, "boot": 4096 >> v, "k": k, "us": round(e0.elapsed_time(e1) / 20 * 1e3, 1)}), flush=True)
lib.topk_debug_flags(0)
