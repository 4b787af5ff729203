"""Interleaved A/B timing of the TMA probe and topk (dev tool)."""
import sys, os, ctypes, json, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen, _lib
lib = _lib.load()
n = 1 << 29
ks = [int(a) for a in sys.argv[1].split(",")] if len(sys.argv) > 1 else [1, 32, 256]
x = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(2), device="cuda")
sink = torch.zeros(4, dtype=torch.int32, device="cuda")
st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
def t(fn, it=5):
    fn(); torch.cuda.synchronize()
    res = []
    for _ in range(it):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        res.append(e0.elapsed_time(e1) * 1000)
    return res
probe = lambda: lib.topk_probe_read(ctypes.c_void_p(x.data_ptr()), n * 4, 1, 0, 30720, 6, ctypes.c_void_p(sink.data_ptr()), st)
for rep in range(2):
    r = t(probe); print("probe us", [round(v) for v in r])
    for k in ks:
        r = t(lambda: tk.topk(x, k)); print(f"k={k} us", [round(v) for v in r])
