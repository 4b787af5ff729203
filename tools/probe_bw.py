"""Read-bandwidth probes (dev tool): LDG grid sweep and TMA ring tile/stage sweep."""
import sys, os, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sigmod_shanbhagpm18_b200 import _lib
lib = _lib.load()
nbytes = 1 << 31
x = torch.empty(nbytes // 4, dtype=torch.int32, device="cuda").random_()
sink = torch.zeros(4, dtype=torch.int32, device="cuda")
st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
def run(method, grid, tile, stages, it=10):
    for _ in range(3):
        assert lib.topk_probe_read(ctypes.c_void_p(x.data_ptr()), nbytes, method, grid, tile, stages, ctypes.c_void_p(sink.data_ptr()), st) == 0
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(it):
        lib.topk_probe_read(ctypes.c_void_p(x.data_ptr()), nbytes, method, grid, tile, stages, ctypes.c_void_p(sink.data_ptr()), st)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / it
    print(json.dumps(dict(method=["ldg", "tma"][method], grid=grid, tile=tile, stages=stages, us=ms * 1e3, gbs=nbytes / ms / 1e6)), flush=True)
for g in (148, 296, 592, 1184, 2368):
    run(0, g, 0, 0)
for tile, stages in ((7680, 16), (15360, 8), (15360, 12), (30720, 4), (30720, 6), (30720, 7), (61440, 3), (49152, 4), (16384, 8), (32768, 6)):
    run(1, 0, tile, stages)
for tile, stages in ((15360, 6), (30720, 3)):
    run(1, 296, tile, stages)
