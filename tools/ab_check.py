"""A/B dev tool: parity (vs the oracle, max order, f32) + CUDA-event timing of the select
kernel for every library given, on the same inputs.

    python tools/ab_check.py LIB1 [LIB2 ...]     # TOPK_LIB-style paths ('' = product lib)

Prints one JSON line per (lib, n, dist, k): ok (bit-exact), median us over 20 launches
(back to back; inputs < L2 are not flushed -- this is a relative A/B, not a bench).
"""
import ctypes
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import oracle
from paper_conf_sigmod_shanbhagpm18_b200 import datagen

CASES = [(1 << 20, "uniform", (32, 256)), ((1 << 20) + 13, "fewdistinct", (64, 1024)),
         (1 << 25, "uniform", (64, 256)), (1 << 29, "uniform", (1, 32, 256, 1024, 2048)),
         (1 << 29, "fewdistinct", (256,)), (1 << 29, "increasing", (256,))]


if os.environ.get("AB_CASES"):  # e.g. AB_CASES="29:uniform:1,256,1024;25:uniform:64"
    CASES = []
    for c in os.environ["AB_CASES"].split(";"):
        lg, dist, ks = c.split(":")
        CASES.append((1 << int(lg), dist, tuple(int(k) for k in ks.split(","))))


DT = os.environ.get("AB_DTYPE", "f32")  # f32 | u32 | f64
DC = {"f32": 0, "u32": 1, "f64": 2}[DT]


def load(path):
    lib = ctypes.CDLL(path)
    vp, u64, u32, i32, sz = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int, ctypes.c_size_t
    lib.topk_workspace_bytes.argtypes = [i32, u64, u32]
    lib.topk_workspace_bytes.restype = sz
    lib.topk_select.argtypes = [i32, vp, vp, u64, u64, u32, i32, i32, vp, vp, vp, vp, sz, vp]
    lib.topk_select.restype = i32
    return lib


def main():
    from paper_conf_sigmod_shanbhagpm18_b200 import _build
    libs = [(p or _build.LIB) for p in sys.argv[1:]] or [_build.LIB]
    handles = [load(p) for p in libs]
    st = torch.cuda.current_stream()
    for n, dist, ks in CASES:
        x = datagen.generate(dist, n, DT, seed=datagen.config_seed(2), device="cuda")
        keys = x.cpu().numpy()
        ov, oi = oracle.topk(keys, max(ks), True)
        for k in ks:
            for path, lib in zip(libs, handles):
                ws = torch.zeros(int(lib.topk_workspace_bytes(DC, n, k)), dtype=torch.uint8,
                                 device="cuda")
                v = torch.empty(k, dtype=x.dtype, device="cuda")
                i = torch.empty(k, dtype=torch.int64, device="cuda")

                def f():
                    r = lib.topk_select(DC, x.data_ptr(), None, n, 0, k, 0, 0, v.data_ptr(), None,
                                        i.data_ptr(), ws.data_ptr(), ws.numel(), st.cuda_stream)
                    assert r == 0, r
                for _ in range(3):
                    f()
                torch.cuda.synchronize()
                ok = bool(np.array_equal(i.cpu().numpy(), oi[:k]) and
                          v.cpu().numpy().tobytes() == ov[:k].tobytes())
                ev = [torch.cuda.Event(enable_timing=True) for _ in range(21)]
                ev[0].record()
                for t in range(20):
                    f()
                    ev[t + 1].record()
                torch.cuda.synchronize()
                us = statistics.median(ev[t].elapsed_time(ev[t + 1]) for t in range(20)) * 1e3
                print(json.dumps({"lib": os.path.basename(path), "n": n, "dist": dist, "k": k,
                                  "ok": ok, "us": round(us, 1)}), flush=True)
        del x


if __name__ == "__main__":
    main()
