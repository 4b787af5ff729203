"""Kernel time vs the CTA-timeline span (dev tool): is time lost outside the CTAs?"""
import sys, os, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen, _lib
lib = _lib.load()
lib.topk_debug_trace.argtypes = [ctypes.c_int, ctypes.c_void_p]
n = 1 << 29
k = int(sys.argv[1]) if len(sys.argv) > 1 else 256
x = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(2), device="cuda")
ov = torch.empty(k, dtype=torch.float32, device="cuda"); oi = torch.empty(k, dtype=torch.int64, device="cuda")
f = lambda: tk.topk(x, k, True, out=(ov, oi, None))
for _ in range(5): f()
torch.cuda.synchronize()
ts = []
for _ in range(10):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); f(); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1) * 1e3)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(50): f()
e1.record(); torch.cuda.synchronize()
b2b = e0.elapsed_time(e1) * 1e3 / 50
lib.topk_debug_trace(1, None)
f(); torch.cuda.synchronize()
buf = np.zeros((160, 64), dtype=np.uint64)
lib.topk_debug_trace(0, buf.ctypes.data_as(ctypes.c_void_p))
st = [int(buf[c, 1]) & ((1 << 56) - 1) for c in range(148) if buf[c, 0] > 0]
en = [int(buf[c, int(buf[c, 0])]) & ((1 << 56) - 1) for c in range(148) if buf[c, 0] > 0]
# python-side launch cost
import time
torch.cuda.synchronize(); t0 = time.perf_counter()
for _ in range(200): tk.launch_count()
t1 = time.perf_counter()
for _ in range(20): f()
t2 = time.perf_counter(); torch.cuda.synchronize()
print(json.dumps(dict(k=k, single_us=sorted(ts)[len(ts)//2], b2b_us=b2b, span_us=(max(en) - min(st)) / 1e3,
                      start_skew_us=(max(st) - min(st)) / 1e3, host_call_us=(t2 - t1) / 20 * 1e6)))
