"""Per-CTA timeline of one select_kernel launch (dev tool)."""
import sys, os, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen, _lib
lib = _lib.load()
lib.topk_debug_trace.argtypes = [ctypes.c_int, ctypes.c_void_p]
n = int(sys.argv[1]); dist = sys.argv[2]; k = int(sys.argv[3])
x = datagen.generate(dist, n, "f32", seed=datagen.config_seed(2), device="cuda")
for _ in range(3): tk.topk(x, k)
torch.cuda.synchronize()
lib.topk_debug_trace(1, None)
tk.topk(x, k); torch.cuda.synchronize()
buf = np.zeros((160, 64), dtype=np.uint64)
lib.topk_debug_trace(0, buf.ctypes.data_as(ctypes.c_void_p))
t0 = None
rows = []
GHZ = float(os.environ.get("TRACE_GHZ", "1.965"))  # stamps are SM clocks (select.cuh trace)
for c in range(148):
    m = int(buf[c, 0])
    g0, c0 = int(buf[c, 63]), int(buf[c, 62]) & ((1 << 56) - 1)
    ev = [(int(v) >> 56, g0 + ((int(v) & ((1 << 56) - 1)) - c0) / GHZ) for v in buf[c, 1:m + 1]]
    if ev: rows.append(ev)
t0 = min(e[0][1] for e in rows)
names = {1: "start", 2: "fb", 3: "fe", 4: "sEnd", 5: "tail", 6: "end", 7: "refr", 8: "sampled", 9: "ranked", 10: "appended", 11: "tb", 12: "ph0", 13: "ph1", 14: "loaded", 15: "apd",
         16: "cnet", 17: "bnd", 18: "cmp", 19: "wnet", 20: "wait", 21: "lpub", 22: "rank", 23: "r0", 24: "r1", 25: "mask", 26: "apd1"}
for _e in range(32, 64): names[_e] = f"cnt{(_e - 32) * 64}+"
send_c = [(max([t for e, t in ev if e == 4] or [0]), c) for c, ev in enumerate(rows)]
send_c.sort()
tail_c = [c for c, ev in enumerate(rows) if any(e == 5 for e, _ in ev)]
for _, c in send_c[:2] + send_c[-2:] + [(0, c) for c in tail_c]:
    print(c, " ".join(f"{names[e]}@{(t - t0) / 1000:.1f}" for e, t in rows[c]))
fl = [sum(1 for e, _ in ev if e == 2) for ev in rows]
ft = []
for ev in rows:
    b = None
    for e, t in ev:
        if e == 2: b = t
        if e == 3 and b is not None: ft.append((b - t0, t - b)); b = None
send = [t - t0 for ev in rows for e, t in ev if e == 4]
tail = [(t - t0) for ev in rows for e, t in ev if e in (5, 6)]
print(json.dumps(dict(k=k, dist=dist, flushes_per_cta=float(np.mean(fl)), flush_us_mean=float(np.mean([d for _, d in ft])) / 1000,
      first_flush_end_us_max=float(max(b + d for b, d in ft[:1])) / 1000 if ft else 0,
      stream_end_us=[float(min(send)) / 1000, float(np.median(send)) / 1000, float(max(send)) / 1000], tail_us=[x / 1000 for x in tail])))
# histogram of flush begin times
hb = np.histogram([b / 1000 for b, _ in ft], bins=10)
print("flush begin hist (us):", [f"{e:.0f}:{c}" for c, e in zip(hb[0], hb[1])])

