#!/usr/bin/env python
"""Benchmark of the B200 bitonic top-k hot path (BASELINE.json metric:
"keys/sec and % of HBM roofline, 2^29 f32 top-k (k=1..1024), 1/2/4/8 B200").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--k 256] [--impl ours|reference]

A step is one top-k over one batch of synthetic input resident in HBM (BJ configs[1]:
n = 2^29 uniform f32 per GPU, headline k = 256, max order, values + indices).  With
torchrun (N > 1) every rank owns a 2^29-key shard of a global N * 2^29 input (weak
scaling): local top-k with the shard's base offset, NCCL all-gather of the k
candidates, one merge kernel -- the partitioned scheme of P:34 / P:444.  Rank 0 prints
ONE JSON line.  `--impl reference` times the CPU oracle (the reference arm of this
paper-only tier) on the host cores instead.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "keys/sec and % of HBM roofline, 2^29 f32 top-k (k=1..1024), 1/2/4/8 B200"
N_PER_GPU = 1 << 29
KEY_BYTES = 4
FALLBACK_HBM_GBS = 6650.0  # B200_PROFILING.md fallback (only if MEASURED_PEAKS.json absent)


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)", d
    return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)", {}


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                 "--format=csv,noheader,nounits", "-lms", "20"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
            time.sleep(0.15)
        except FileNotFoundError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc is not None:
            time.sleep(0.05)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4)
                          if len(r) > 4 + i and r[4 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "samples": len(self.rows)}


def dist_env():
    r = int(os.environ.get("RANK", "0"))
    w = int(os.environ.get("WORLD_SIZE", "1"))
    lr = int(os.environ.get("LOCAL_RANK", "0"))
    return r, w, lr


def cpu_baseline(keys_host, k, note):
    """The oracle as it stands on this host's cores (a reported baseline)."""
    import oracle
    t0 = time.perf_counter()
    oracle.topk(keys_host, k, True)
    dt = time.perf_counter() - t0
    return {"value": keys_host.shape[0] / dt, "unit": "keys/s", "cores": oracle.threads(),
            "kind": "oracle", "sample": note, "seconds": dt}


def run_reference(args):
    """--impl reference: the CPU oracle timed on the host (rank 0 only)."""
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import numpy as np
    import oracle
    from paper_conf_sigmod_shanbhagpm18_b200 import datagen
    oracle.build()
    n = 1 << 26  # bounded sample: the first 2^26 rows of the 2^29-key input, every step
    keys = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(2),
                            n_total=N_PER_GPU).numpy()
    for _ in range(args.warmup):
        oracle.topk(keys, args.k, True)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.topk(keys, args.k, True)
        times.append(time.perf_counter() - t0)
    t = sum(times)
    value = n * args.steps / t
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "keys/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * t / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": f"2^29 uniform f32, k={args.k}, max order, values+indices (BJ configs[1])",
                   "n": N_PER_GPU, "k": args.k, "sample_rows": n},
        "cpu_baseline": {"value": value, "unit": "keys/s", "cores": oracle.threads(),
                         "kind": "oracle",
                         "sample": "first 2^26 rows of the 2^29-key input, every step"},
        "e2e": {"value": value, "unit": "keys/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def time_steps(fn, steps, stream, torch):
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(steps):
        fn()
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1)


def run_ours(args):
    import torch
    import torch.distributed as dist

    import paper_conf_sigmod_shanbhagpm18_b200 as tk
    from paper_conf_sigmod_shanbhagpm18_b200 import datagen

    rank, world, lrank = dist_env()
    if world != args.gpus:
        args.gpus = world
    torch.cuda.set_device(lrank)
    dev = torch.device("cuda", lrank)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    n = N_PER_GPU
    k = args.k
    stream = torch.cuda.current_stream(dev)
    x = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(2), device=dev,
                         base=rank * n, n_total=world * n)
    out_v = torch.empty(k, dtype=torch.float32, device=dev)
    out_i = torch.empty(k, dtype=torch.int64, device=dev)

    from paper_conf_sigmod_shanbhagpm18_b200.dist import NcclComm, sharded_topk_native

    comm = NcclComm(device=dev) if world > 1 else None

    def step():
        if world > 1:  # C ABI topk_select_sharded: local top-k (base = shard offset) ->
            # ncclAllGather of the k candidates -> merge kernel, one stream, no host sync
            return sharded_topk_native(x, k, comm, True, base=rank * n,
                                       out=(out_v, out_i, None))
        return tk.topk(x, k, True, base=rank * n, out=(out_v, out_i, None))

    for _ in range(max(3, args.warmup)):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    lc0 = tk.launch_count()
    with ClockSampler(lrank) as clk:
        if world > 1:
            dist.barrier()
        ms = time_steps(step, args.steps, stream, torch)
    launches = tk.launch_count() - lc0
    ms_t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms = float(ms_t.item())
    ms_step = ms / args.steps
    value = world * n / (ms_step / 1e3)

    # ---- e2e: through the C ABI with HOST buffers (topk_select_host: pinned keys streamed
    # in 64 Mi-key chunks overlapping the reductive pass; results copied back)
    hx = torch.empty(n, dtype=torch.float32, pin_memory=True)
    hx.copy_(x)
    hv = torch.empty(k, dtype=torch.float32, pin_memory=True)
    hi = torch.empty(k, dtype=torch.int64, pin_memory=True)
    e2e_steps = max(2, min(args.steps, 5))

    def e2e_step():
        if world > 1:
            raise RuntimeError("unused")
        tk.topk_host(hx, k, True, chunk_keys=1 << 26, out=(hv, hi))

    def e2e_step_sharded():
        xd.copy_(hx, non_blocking=True)
        v, i = sharded_topk_native(xd, k, comm, True, base=rank * n, out=(out_v, out_i, None))
        hv.copy_(v, non_blocking=True)
        hi.copy_(i, non_blocking=True)

    if world > 1:
        xd = torch.empty_like(x)
        fn_e2e = e2e_step_sharded
    else:
        fn_e2e = e2e_step
    fn_e2e()
    ms_e2e = time_steps(fn_e2e, e2e_steps, stream, torch)
    t_e = torch.tensor([ms_e2e], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t_e, op=dist.ReduceOp.MAX)
    e2e_value = world * n / (float(t_e.item()) / e2e_steps / 1e3)
    del hx

    # ---- extra (untimed for the headline): k sweep and distributions on rank 0
    extra = {}
    if rank == 0 and not args.no_sweep:
        sweep = []
        for kk in (1, 8, 32, 64, 128, 256, 512, 1024, 2048):
            f = lambda: tk.topk(x, kk, True)
            for _ in range(3):
                f()
            t = time_steps(f, 10, stream, torch) / 10
            sweep.append({"k": kk, "us": round(t * 1e3, 1), "keys_per_s": n / (t / 1e3)})
        extra["k_sweep_uniform"] = sweep
        # f2: the paper's selection-based method (radix select) on the same
        # input, next to the §7 cost model's predictions with B200 parameters
        from paper_conf_sigmod_shanbhagpm18_b200 import costmodel as cm
        hw = cm.b200(peaks()[0])
        rv = []
        for kk in (32, 256, 1024):
            f = lambda: tk.topk_radix(x, kk, True)
            for _ in range(3):
                f()
            t = time_steps(f, 10, stream, torch) / 10
            tb = next(s_["us"] for s_ in sweep if s_["k"] == kk)
            rv.append({"k": kk, "radix_us": round(t * 1e3, 1), "bitonic_us": tb,
                       "model_radix_us": round(cm.radix_time(n, KEY_BYTES, hw) * 1e6, 1),
                       "model_bitonic_paper_us": round(cm.bitonic_time(n, KEY_BYTES, kk, hw) * 1e6, 1),
                       "model_bitonic_b200_us": round(cm.bitonic_b200_time(n, KEY_BYTES, hw) * 1e6, 1),
                       "model_choice_paper": cm.choose(n, KEY_BYTES, kk, hw),
                       "model_choice_b200": cm.choose_b200(n, KEY_BYTES, kk, hw),
                       "measured_choice": "bitonic" if tb <= t * 1e3 else "radix"})
        extra["radix_vs_bitonic"] = rv
        adv = []
        for d in ("increasing", "decreasing", "fewdistinct", "bucketkiller"):
            xa = datagen.generate(d, n, "f32", seed=datagen.config_seed(3), device=dev)
            f = lambda: tk.topk(xa, 256, True)
            for _ in range(3):
                f()
            t = time_steps(f, 10, stream, torch) / 10
            adv.append({"dist": d, "k": 256, "us": round(t * 1e3, 1), "keys_per_s": n / (t / 1e3)})
            del xa
        extra["adversarial_k256"] = adv
        # the other BJ configs on this GPU (parity-tested in tests/; reported here)
        cfgs = []

        def timed(f, it=10):
            for _ in range(3):
                f()
            return time_steps(f, it, stream, torch) / it

        x1 = datagen.generate("uniform", 1 << 20, "f32", seed=datagen.config_seed(1), device=dev)
        t = timed(lambda: tk.topk(x1, 32, True), 50)
        cfgs.append({"config": "BJ1: 2^20 uniform f32, k=32 (launch-bound)", "us": round(t * 1e3, 1),
                     "keys_per_s": (1 << 20) / (t / 1e3)})
        del x1
        n4 = 1 << 28
        xu = datagen.generate("uniform", n4, "u32", seed=datagen.config_seed(4), device=dev)
        pu = datagen.payload(n4, seed=datagen.config_seed(4), device=dev)
        t = timed(lambda: tk.topk(xu, 64, True, payload=pu))
        cfgs.append({"config": "BJ4a: 2^28 u32 key + u32 payload, DESC LIMIT 64", "us": round(t * 1e3, 1),
                     "keys_per_s": n4 / (t / 1e3), "frac_hbm": n4 * 4 / (t / 1e3) / 1e9 / peaks()[0]})
        del xu, pu
        xd64 = datagen.generate("uniform", n4, "f64", seed=datagen.config_seed(4), device=dev)
        t = timed(lambda: tk.topk(xd64, 64, True))
        cfgs.append({"config": "BJ4b: 2^28 f64, DESC LIMIT 64", "us": round(t * 1e3, 1),
                     "keys_per_s": n4 / (t / 1e3), "frac_hbm": n4 * 8 / (t / 1e3) / 1e9 / peaks()[0]})
        del xd64
        # f1: the paper's §5 query forms fused into the pass (queries 1-3 of
        # §6.8): 2^28 rows, 8 bytes streamed per row (key column + one more column)
        cnt = datagen.generate("uniform", n4, "u32", seed=datagen.config_seed(6), device=dev)
        tcol = datagen.generate("uniform", n4, "u32", seed=datagen.config_seed(6, 1), device=dev)
        lang = (tcol.view(torch.int32) & 63).view(torch.uint32)  # dictionary codes 0..63
        for name, fq in (
                ("query1: WHERE time < 2^31 (sel 0.5) ORDER BY count DESC LIMIT 50 (u32 cols)",
                 lambda: tk.query(cnt, 50, True, pred=("range", tcol, 0, 1 << 31))),
                ("query3: WHERE lang IN (52 of 64 codes, sel 0.81) ORDER BY count DESC LIMIT 50",
                 lambda: tk.query(cnt, 50, True, pred=("in", lang, (1 << 52) - 1)))):
            t = timed(fq)
            cfgs.append({"config": f"f1 {name}", "us": round(t * 1e3, 1),
                         "rows_per_s": n4 / (t / 1e3),
                         "frac_hbm": n4 * 8 / (t / 1e3) / 1e9 / peaks()[0]})
        del cnt, tcol, lang
        a = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(6, 2), device=dev)
        b = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(6, 3), device=dev)
        t = timed(lambda: tk.query(a, 50, True, rank_b=b, rank_w=0.5))
        cfgs.append({"config": "f1 query2: ORDER BY a + 0.5 * b DESC LIMIT 50 (f32 cols)",
                     "us": round(t * 1e3, 1), "rows_per_s": n4 / (t / 1e3),
                     "frac_hbm": n4 * 8 / (t / 1e3) / 1e9 / peaks()[0]})
        # f3: compound keys, KKV (Fig 14's 2^28 tuples): ORDER BY k1, k2 with the
        # 4-byte value gathered through the tuple id; 8 bytes streamed per row
        k1 = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(7), device=dev)
        k2 = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(7, 1), device=dev)
        pv = datagen.payload(n4, seed=datagen.config_seed(7), device=dev)
        t = timed(lambda: tk.topk_kk(k1, k2, 64, True, True, payload=pv))
        cfgs.append({"config": "f3 KKV: 2^28 rows, ORDER BY k1 DESC, k2 DESC LIMIT 64, u32 value",
                     "us": round(t * 1e3, 1), "rows_per_s": n4 / (t / 1e3),
                     "frac_hbm": n4 * 8 / (t / 1e3) / 1e9 / peaks()[0]})
        k3 = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(7, 2), device=dev)
        t = timed(lambda: tk.topk_kkk(k1, k2, k3, 64, payload=pv))
        cfgs.append({"config": "f3 KKKV: 2^28 rows, ORDER BY k1, k2, k3 DESC LIMIT 64, u32 value",
                     "us": round(t * 1e3, 1), "rows_per_s": n4 / (t / 1e3),
                     "frac_hbm": n4 * 12 / (t / 1e3) / 1e9 / peaks()[0]})
        del k1, k2, k3, pv, a, b
        for kk in (32, 256):
            t = timed(lambda: tk.topk(x, kk, True, mode="pure"), 2)
            cfgs.append({"config": f"pure mode (paper's data-independent network on every key), "
                                   f"2^29 f32, k={kk}", "us": round(t * 1e3, 1),
                         "keys_per_s": n / (t / 1e3)})
        if not args.no_big:
            del x
            torch.cuda.empty_cache()
            n5 = 1 << 32
            x5 = datagen.generate("uniform", n5, "f32", seed=datagen.config_seed(5), device=dev)
            t = timed(lambda: tk.topk(x5, 256, True), 5)
            cfgs.append({"config": "BJ5 at G=1: 2^32 uniform f32, k=256 (2 chunks of 2^31 + merge)",
                         "us": round(t * 1e3, 1), "keys_per_s": n5 / (t / 1e3),
                         "frac_hbm": n5 * 4 / (t / 1e3) / 1e9 / peaks()[0]})
            del x5
            x = None
        extra["other_configs"] = cfgs

    if rank == 0:
        hbm, peak_src, mp = peaks()
        gbs = n * KEY_BYTES / (ms_step / 1e3) / 1e9  # this GPU's kernel (+ merge if N > 1)
        traffic = None
        tp = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tp):
            with open(tp) as f:
                traffic = json.load(f).get(f"select_k{k}")
        base_note = "inputs larger than L2 (2 GiB per GPU > 126 MB), no flush needed"
        keys_host = None
        if not args.no_cpu_baseline:
            keys_host = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(2),
                                         base=0, n_total=world * n).numpy()
        line = {
            "metric": METRIC, "value": value, "unit": "keys/s", "n_gpus": world,
            "steps": args.steps, "warmup": max(3, args.warmup), "ms_per_step": ms_step,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"2^29 uniform f32 per GPU, k={k}, max order, values+indices "
                                   f"(BJ configs[1]; N>1: configs[4]-style shards + NCCL gather + merge)",
                       "n_per_gpu": n, "n_total": world * n, "k": k,
                       "parallelism": f"shard{world}" if world > 1 else "single",
                       "l2": base_note},
            "roofline": {"bound": "hbm", "achieved": gbs, "peak": hbm, "unit": "GB/s",
                         "frac": gbs / hbm, "traffic": traffic, "peak_source": peak_src,
                         "frac_of_8tbs_nominal": gbs / 8000.0},
            "clocks": clk.summary(),
            "gpu_launches": launches,
            "e2e": {"value": e2e_value, "unit": "keys/s", "h2d_bytes_per_step": n * KEY_BYTES,
                    "d2h_bytes_per_step": k * (KEY_BYTES + 8),
                    "note": "C-ABI topk_select_host: pinned host keys streamed in 2^26-key "
                            "chunks overlapped with the per-chunk top-k, merge, results to "
                            "host, per step (N>1: copy + sharded top-k)"},
        }
        if keys_host is not None:
            line["cpu_baseline"] = cpu_baseline(keys_host, k, "the full 2^29-key input, once")
        line.update(extra)
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        comm.close()
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--k", type=int, default=256)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-sweep", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-big", action="store_true", help="skip the 2^32-key extra")
    args = ap.parse_args()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
