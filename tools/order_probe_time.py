"""Wave-order probe check (dev; honours TOPK_LIB): 2^29 f32 inputs whose order the probe
must classify -- sorted both ways, organ pipe (up then down), sawtooth (8 ramps), uniform --
CUDA-event median of 10 launches at k = 256, checked against the oracle."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
n = 1 << 29
inc = datagen.generate("increasing", n, "f32", seed=datagen.config_seed(3), device="cuda")
cases = {
    "increasing": inc,
    "decreasing": torch.flip(inc, [0]),
    "organ_pipe": torch.cat([inc[0::2], torch.flip(inc[1::2], [0])]),
    "sawtooth8": inc.view(8, -1).t().contiguous().view(-1).view(8, -1).contiguous().view(-1),
    "uniform": datagen.generate("uniform", n, "f32", seed=datagen.config_seed(2), device="cuda"),
}
lib = os.path.basename(os.environ.get("TOPK_LIB", "main"))
for name, x in cases.items():
    f = lambda: tk.topk(x, 256)
    for _ in range(3): f()
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(11)]
    ev[0].record()
    for t in range(10):
        f(); ev[t + 1].record()
    torch.cuda.synchronize()
    us = statistics.median(ev[t].elapsed_time(ev[t + 1]) for t in range(10)) * 1e3
    ok = bool(np.array_equal(f()[1].cpu().numpy(), oracle.topk(x.cpu().numpy(), 256, True)[1]))
    print(json.dumps({"lib": lib, "input": name, "us": round(us, 1), "ok": ok}), flush=True)
    del x
