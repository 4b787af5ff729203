"""Quick CUDA-event timing of topk() on 2^29 f32 uniform for a k sweep (dev tool)."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen

def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 29
    dist = sys.argv[2] if len(sys.argv) > 2 else "uniform"
    modes = sys.argv[3].split(",") if len(sys.argv) > 3 else ["filter"]
    ks = [int(a) for a in sys.argv[4].split(",")] if len(sys.argv) > 4 else [1, 8, 32, 64, 128, 256, 512, 1024]
    x = datagen.generate(dist, n, "f32", seed=datagen.config_seed(2), device="cuda")
    res = []
    for mode in modes:
        for k in ks:
            for _ in range(3):
                tk.topk(x, k, mode=mode)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            it = 10 if mode == "filter" else 2
            e0.record()
            for _ in range(it):
                tk.topk(x, k, mode=mode)
            e1.record(); torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / it
            gbs = n * 4 / ms / 1e6
            res.append(dict(mode=mode, dist=dist, k=k, ms=ms, gbs=gbs, frac=gbs / 6563.2))
            print(json.dumps(res[-1]), flush=True)

main()
