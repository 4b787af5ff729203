"""Small-n latency: filter vs pure kernel (dev tool).  30 launches captured in a CUDA graph
and replayed, so the host-side Python/ctypes cost per call is not in the number."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen


def graph_us(f, reps=30):
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            f()
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(reps):
            f()
    g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / reps * 1e3)
    return round(min(ts), 2)


if __name__ == "__main__":
    for lg in (12, 16, 18, 20, 22, 24, 26):
        n = 1 << lg
        x = datagen.generate("uniform", n, "f32", seed=5, device="cuda")
        for k in (8, 32):
            row = {"log2n": lg, "k": k}
            v = torch.empty(k, dtype=torch.float32, device="cuda")
            i = torch.empty(k, dtype=torch.int64, device="cuda")
            ws = tk.Workspace(tk.workspace_bytes(torch.float32, n, k), "cuda")
            for mode in ("filter", "pure"):
                row[mode] = graph_us(lambda: tk.topk(x, k, mode=mode, out=(v, i, None), workspace=ws))
            print(json.dumps(row), flush=True)
