"""Sweep select.cuh debug knobs (c_dbg) at a few k -- dev tool.
    python tools/knob_sweep.py FLAGS[,FLAGS...] K[,K...]"""
import sys, os, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen, _lib
lib = _lib.load()
lib.topk_debug_flags.argtypes = [ctypes.c_int]
flags = [int(f, 0) for f in sys.argv[1].split(",")]
ks = [int(k) for k in sys.argv[2].split(",")]
x = datagen.generate("uniform", 1 << 29, "f32", seed=datagen.config_seed(2), device="cuda")
for rep in range(2):
    for fl in flags:
        lib.topk_debug_flags(fl)
        out = []
        for k in ks:
            for _ in range(3):
                tk.topk(x, k)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(20):
                tk.topk(x, k)
            e1.record(); torch.cuda.synchronize()
            out.append(f"k{k}={e0.elapsed_time(e1) / 20 * 1e3:.1f}")
        print(hex(fl), " ".join(out), flush=True)
lib.topk_debug_flags(0)
