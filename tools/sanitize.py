"""Small (T1-size) calls of every kernel family, for compute-sanitizer memcheck /
racecheck / synccheck runs (tools/gpu_sanitize.sh).  Each result is checked against the
oracle, so a run that completes also proves the answers under the tool."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen


def same(v, i, ov, oi):
    assert np.array_equal(i.cpu().numpy(), oi)
    assert v.cpu().numpy().tobytes() == ov.tobytes()


n = (1 << 20) + 13
for dist in ("uniform", "fewdistinct"):
    x = datagen.generate(dist, n, "f32", seed=11)
    xd = x.cuda()
    for k in (1, 32, 256, 1024):
        same(*tk.topk(xd, k), *oracle.topk(x.numpy(), k, True))
    for k in (8, 32):
        same(*tk.topk(xd, k, mode="pure"), *oracle.topk(x.numpy(), k, True))
    same(*tk.topk(xd, 256, mode="pure"), *oracle.topk(x.numpy(), 256, True))
xd64 = datagen.generate("uniform", 1 << 18, "f64", seed=12)
same(*tk.topk(xd64.cuda(), 64, False), *oracle.topk(xd64.numpy(), 64, False))
# merge kernel (sorted runs and any order), radix select, query form
vs, is_ = [], []
for r in range(4):
    v, i = tk.topk(xd[r * 1000:(r + 1) * 1000 + 500], 100, base=r * 1000)
    vs.append(v)
    is_.append(i)
cv, ci = torch.cat(vs), torch.cat(is_)
ov, oi = oracle.topk(cv.cpu().numpy(), 100, True, idx=ci.cpu().numpy())
same(*tk.merge(cv, ci, 100, runs=4, sorted_runs=True), ov, oi)
same(*tk.merge(cv, ci, 100, runs=4), ov, oi)
xr = datagen.generate("uniform", 1 << 20, "f32", seed=13)
same(*tk.topk_radix(xr.cuda(), 256), *oracle.topk(xr.numpy(), 256, True))
col = datagen.generate("uniform", 1 << 20, "u32", seed=14)
v, i = tk.query(xr.cuda(), 50, True, pred=("range", col.cuda(), 0, 1 << 31))
ov, oi, m = oracle.query(xr.numpy(), 50, True, pred=("range", col.view(torch.int32).numpy().view(np.uint32), 0, 1 << 31))
same(v, i, ov, oi)
# compound keys (KKV: E64 entries, KKKV: E96 entries -- both run the boot sample)
a, b, c = (datagen.generate("uniform", (1 << 20) + 4, "f32", seed=15 + j) for j in range(3))
r = tk.topk_kk(a.cuda(), b.cuda(), 64)
assert np.array_equal(r[2].cpu().numpy(), oracle.topk_kk(a.numpy(), b.numpy(), 64)[2])
r = tk.topk_kkk(a.cuda(), b.cuda(), c.cuda(), 64)
assert np.array_equal(r[3].cpu().numpy(), oracle.topk_kkk(a.numpy(), b.numpy(), c.numpy(), 64)[3])
torch.cuda.synchronize()
print("sanitize workload ok")
