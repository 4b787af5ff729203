#!/usr/bin/env python
"""Benchmark of the B200 bitonic top-k hot path (BASELINE.json metric:
"keys/sec and % of HBM roofline, 2^29 f32 top-k (k=1..1024), 1/2/4/8 B200").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--k 256] [--impl ours|reference]
                    [--n-total 4294967296]

A step is one top-k over one batch of synthetic input resident in HBM (BJ configs[1]:
n = 2^29 uniform f32 per GPU, headline k = 256, max order, values + indices).  With
torchrun (N > 1) every rank owns a shard of the global input: by default 2^29 keys per
rank (weak scaling, global N * 2^29); with --n-total T the global input is T keys split
over the ranks (strong scaling, BJ configs[4]: T = 2^32 at N = 1/2/4/8).  Each rank runs
the local top-k with its shard's base offset, NCCL all-gathers the k candidates and runs
one merge kernel -- the partitioned scheme of P:34 / P:444.  Rank 0 prints ONE JSON line.
`--impl reference` times the CPU oracle (the reference arm of this paper-only tier) on
the host cores instead.

Besides the headline the line carries, all measured in this run: the median / min step
time, the read-only probe of the same buffer (the paper's "Memory Bandwidth" line,
P:244), the select kernel's DRAM bytes per launch from an ncu subprocess (roofline
`traffic`), the k sweep, the Fig-13 size sweep, the other BJ configs and the
CPU oracle (cores, CPU model, and a one-thread run).
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


def workload(k, world=1, n_total=None):
    """config.workload of both arms."""
    if n_total is None:
        return (f"2^29 uniform f32 per GPU, k={k}, max order, values+indices (BJ configs[1]; "
                f"N>1: weak scaling, configs[4]-style shards + NCCL gather + merge)")
    return (f"{n_total} uniform f32 split over {world} GPU(s), k={k}, max order, "
            f"values+indices (BJ configs[4], strong scaling)")


def shard_plan(rank, world, n_total=None):
    """The rows rank `rank` of `world` owns: weak scaling (n_total None) -- 2^29 per rank,
    global input world * 2^29; strong scaling -- n_total split into contiguous shards.
    Returns (n_total, lo, hi): global rows [lo, hi)."""
    if n_total is None:
        n_total = world * N_PER_GPU
    return n_total, n_total * rank // world, n_total * (rank + 1) // world


def dist_env():
    r = int(os.environ.get("RANK", "0"))
    w = int(os.environ.get("WORLD_SIZE", "1"))
    lr = int(os.environ.get("LOCAL_RANK", "0"))
    return r, w, lr


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def cpu_baseline(keys_host, k):
    """The oracle as it stands on this host's cores (a reported baseline, not a target):
    the full input with every core of the affinity mask (median of 3), and a one-thread
    run on the first 2^26 rows."""
    import numpy as np
    import oracle
    n = keys_host.shape[0]
    ts = []
    for _ in range(3):
        t0 = time.perf_counter()
        oracle.topk(keys_host, k, True)
        ts.append(time.perf_counter() - t0)
    dt = statistics.median(ts)
    n1 = min(n, 1 << 26)
    t0 = time.perf_counter()
    oracle.topk(np.ascontiguousarray(keys_host[:n1]), k, True, threads=1)
    dt1 = time.perf_counter() - t0
    return {"value": n / dt, "unit": "keys/s", "cores": oracle.threads(), "kind": "oracle",
            "sample": f"the full {n}-key input, median of 3 runs", "seconds": dt,
            "cpu_model": cpu_model(),
            "p1": {"value": n1 / dt1, "unit": "keys/s", "cores": 1, "seconds": dt1,
                   "sample": f"first {n1} rows of the same input"}}


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
        "config": {"workload": workload(args.k), "n_per_gpu": N_PER_GPU, "n_total": N_PER_GPU,
                   "k": args.k, "sample_rows": n},
        "cpu_baseline": {"value": value, "unit": "keys/s", "cores": oracle.threads(),
                         "kind": "oracle",
                         "sample": "first 2^26 rows of the 2^29-key input, every step"},
        "e2e": {"value": value, "unit": "keys/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def time_steps(fn, steps, stream, torch, per_step=False):
    """CUDA events on the launching stream around `steps` back-to-back steps (plus one
    event between consecutive steps when per_step: no host synchronisation inside)."""
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(steps + 1 if per_step else 2)]
    ev[0].record(stream)
    for i in range(steps):
        fn()
        if per_step:
            ev[i + 1].record(stream)
    ev[-1].record(stream)
    torch.cuda.synchronize()
    total = ev[0].elapsed_time(ev[-1])
    if not per_step:
        return total
    return total, [ev[i].elapsed_time(ev[i + 1]) for i in range(steps)]


def probe_read(x, stream, torch):
    """The paper's "Memory Bandwidth" line: read the step's own input buffer once,
    no top-k work -- 128-bit loads (16 CTAs/SM) and the select kernel's TMA ring
    (30 KB x 4 stages, 1 CTA/SM).  Best of 10 launches each, GB/s."""
    import ctypes
    from paper_conf_sigmod_shanbhagpm18_b200 import _lib
    lib = _lib.load()
    sink = torch.zeros(4, dtype=torch.int32, device=x.device)
    nbytes = x.numel() * x.element_size() // 16 * 16
    sp = ctypes.c_void_p(stream.cuda_stream)
    out = {}
    for name, method, grid, tile, stages in (("ldg", 0, 16 * torch.cuda.get_device_properties(
            x.device).multi_processor_count, 0, 0), ("tma_ring", 1, 0, 30720, 4)):
        def f():
            st = lib.topk_probe_read(ctypes.c_void_p(x.data_ptr()), nbytes, method, grid, tile,
                                     stages, ctypes.c_void_p(sink.data_ptr()), sp)
            _lib.check(st, "topk_probe_read")
        for _ in range(3):
            f()
        _, per = time_steps(f, 10, stream, torch, per_step=True)
        out[f"{name}_gbs"] = nbytes / (min(per) / 1e3) / 1e9
    out["best_gbs"] = max(out.values())
    out["bytes"] = nbytes
    return out


def graph_us(f, torch, reps=30):
    """Device time per call: `reps` calls captured in a CUDA graph and replayed (min of 5
    replays), so the host-side cost of each Python call is not in the number."""
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
    return min(ts)


def ncu_traffic(k, n, timeout=420):
    """DRAM bytes (read + write) of ONE select_kernel launch on the headline input, from
    an ncu subprocess (`bench.py --ncu-target`) -- the roofline `traffic` of this run.
    None (with the reason) if ncu is unavailable or fails."""
    cmd = ["ncu", "--metrics", "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum",
           "--clock-control", "none", "-k", "regex:select_kernel", "-s", "2", "-c", "1", "--csv",
           sys.executable, os.path.abspath(__file__), "--ncu-target", "--k", str(k), "--n", str(n)]
    try:
        r = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout, cwd=ROOT)
    except (OSError, subprocess.TimeoutExpired) as e:
        return None, f"ncu failed: {type(e).__name__}"
    import csv
    rows = [row for row in csv.reader(r.stdout.splitlines()) if len(row) > 10]
    if len(rows) < 2:
        return None, f"ncu produced no metrics (rc={r.returncode}): {r.stderr.strip()[-200:]}"
    h = rows[0]
    ni, vi, ui = h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
             "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3, "second": 1.0,
             "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1.0}
    m = {row[ni]: float(row[vi].replace(",", "")) * scale.get(row[ui], 1.0) for row in rows[1:]}
    rd, wr = m.get("dram__bytes_read.sum"), m.get("dram__bytes_write.sum")
    if rd is None or wr is None:
        return None, "ncu output lacks dram__bytes_*"
    return {"bytes": rd + wr, "read": rd, "write": wr,
            "ncu_kernel_us": m.get("gpu__time_duration.sum", 0.0) * 1e6}, "ok"


def run_ncu_target(args):
    """Child of ncu_traffic(): the headline launch on the headline input, 3 times."""
    import torch
    import paper_conf_sigmod_shanbhagpm18_b200 as tk
    from paper_conf_sigmod_shanbhagpm18_b200 import datagen
    x = datagen.generate("uniform", args.n, "f32", seed=datagen.config_seed(2), device="cuda",
                         n_total=args.n)
    for _ in range(3):
        tk.topk(x, args.k, True)
    torch.cuda.synchronize()


def size_sweep(tk, datagen, stream, torch, peak, k=64):
    """Fig. 13: data size 2^21 ... 2^29 uniform f32 at fixed k = 64.  Inputs
    that fit the 126 MB L2 (<= 2^25 keys) are timed one launch at a time with the L2
    flushed before each launch (a read of 512 MiB, which leaves clean lines -- a write
    would leave dirty lines whose write-back lands inside the timed launch); larger ones
    back to back."""
    import ctypes
    from paper_conf_sigmod_shanbhagpm18_b200 import _lib
    lib = _lib.load()
    dev = stream.device
    scrub = torch.ones(1 << 27, dtype=torch.int32, device=dev)
    sink = torch.zeros(4, dtype=torch.int32, device=dev)

    def flush_l2():
        _lib.check(lib.topk_probe_read(ctypes.c_void_p(scrub.data_ptr()), scrub.numel() * 4, 0, 0,
                                       0, 0, ctypes.c_void_p(sink.data_ptr()),
                                       ctypes.c_void_p(stream.cuda_stream)), "probe (L2 flush)")

    out = []
    for lg in range(21, 30):
        n = 1 << lg
        x = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(2), device=dev,
                             n_total=1 << 29)
        f = lambda: tk.topk(x, k, True)
        for _ in range(3):
            f()
        if lg <= 25:
            # flush, event, launch, event -- enqueued without a host synchronisation in
            # between: the ~70 us flush keeps the GPU busy while the host enqueues the
            # launch, so the events bracket the device time only (a synchronize before
            # the first event let ~25 us of Python call overhead into the interval)
            torch.cuda.synchronize()
            evs = []
            for _ in range(10):
                flush_l2()
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                f()
                e1.record(stream)
                evs.append((e0, e1))
            torch.cuda.synchronize()
            us = statistics.median(a.elapsed_time(b) for a, b in evs) * 1e3
            l2 = "flushed"
        else:
            _, per = time_steps(f, 10, stream, torch, per_step=True)
            us = statistics.median(per) * 1e3
            l2 = "> L2"
        out.append({"log2n": lg, "k": k, "us": round(us, 2), "keys_per_s": n / (us / 1e6),
                    "frac_hbm": n * 4 / (us / 1e6) / 1e9 / peak, "l2": l2})
        del x
    del scrub
    return out


def run_ours(args):
    import torch
    import torch.distributed as dist

    import paper_conf_sigmod_shanbhagpm18_b200 as tk
    from paper_conf_sigmod_shanbhagpm18_b200 import datagen
    from paper_conf_sigmod_shanbhagpm18_b200.dist import NcclComm, sharded_topk_native

    rank, world, lrank = dist_env()
    if world != args.gpus:
        args.gpus = world
    torch.cuda.set_device(lrank)
    dev = torch.device("cuda", lrank)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    strong = args.n_total is not None
    n_total, lo, hi = shard_plan(rank, world, args.n_total)
    n = hi - lo  # this rank's shard: global rows [lo, hi)
    k = args.k
    stream = torch.cuda.current_stream(dev)
    seed = datagen.config_seed(5 if strong else 2)
    x = datagen.generate("uniform", n, "f32", seed=seed, device=dev, base=lo, n_total=n_total)
    out_v = torch.empty(k, dtype=torch.float32, device=dev)
    out_i = torch.empty(k, dtype=torch.int64, device=dev)
    comm = NcclComm(device=dev) if world > 1 else None

    def step():
        if world > 1:  # C ABI topk_select_sharded: local top-k (base = shard offset) ->
            # ncclAllGather of the k candidates -> merge kernel, one stream, no host sync
            return sharded_topk_native(x, k, comm, True, base=lo, out=(out_v, out_i, None))
        return tk.topk(x, k, True, base=lo, out=(out_v, out_i, None))

    warm = max(3, args.warmup)
    for _ in range(warm):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    lc0 = tk.launch_count()
    with ClockSampler(lrank) as clk:
        if world > 1:
            dist.barrier()
        ms, per = time_steps(step, args.steps, stream, torch, per_step=True)
    launches = tk.launch_count() - lc0
    ms_t = torch.tensor([ms, statistics.median(per), min(per)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms, med, mn = (float(v) for v in ms_t.tolist())
    ms_step = ms / args.steps
    value = n_total / (ms_step / 1e3)

    # ---- e2e: through the C ABI with HOST buffers, copies inside the timed region
    hx = torch.empty(n, dtype=torch.float32, pin_memory=True)
    hx.copy_(x)
    hv = torch.empty(k, dtype=torch.float32, pin_memory=True)
    hi_ = torch.empty(k, dtype=torch.int64, pin_memory=True)
    e2e_steps = max(2, min(args.steps, 5))

    def e2e_step():  # topk_select_host: pinned keys streamed in 2^26-key chunks
        tk.topk_host(hx, k, True, chunk_keys=1 << 26, out=(hv, hi_))

    def e2e_step_sharded():
        xd.copy_(hx, non_blocking=True)
        v, i = sharded_topk_native(xd, k, comm, True, base=lo, out=(out_v, out_i, None))
        hv.copy_(v, non_blocking=True)
        hi_.copy_(i, non_blocking=True)

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
    e2e_value = n_total / (float(t_e.item()) / e2e_steps / 1e3)
    hv_last, hi_last = hv.clone(), hi_.clone()  # the e2e result, read back to the host
    del hx
    if world > 1:
        del xd

    hbm, peak_src, mp = peaks()
    probe = probe_read(x, stream, torch) if rank == 0 else None

    # ---- extras (untimed for the headline; rank 0, N = 1 only)
    extra = {}
    if rank == 0 and world == 1 and not args.no_sweep:
        extra = run_extras(args, tk, datagen, x, stream, torch, hbm)

    if rank == 0:
        x = None
        torch.cuda.empty_cache()
        gbs = n * KEY_BYTES / (ms_step / 1e3) / 1e9  # this GPU's kernel (+ gather/merge if N > 1)
        traffic, why = (None, "skipped (--no-ncu)")
        if world == 1 and not args.no_ncu and not strong:
            traffic, why = ncu_traffic(k, n)
        keys_host = None
        if world == 1 and not args.no_cpu_baseline and not strong:
            keys_host = datagen.generate("uniform", n, "f32", seed=seed, base=0,
                                         n_total=n_total).numpy()
        wl = workload(k, world, n_total if strong else None)
        line = {
            "metric": METRIC, "value": value, "unit": "keys/s", "n_gpus": world,
            "steps": args.steps, "warmup": warm, "ms_per_step": ms_step,
            "ms_per_step_median": med, "ms_per_step_min": mn,
            "higher_is_better": True, "scaling": "strong" if strong else "weak",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": wl, "n_per_gpu": n, "n_total": n_total, "k": k,
                       "parallelism": f"shard{world}" if world > 1 else "single",
                       "l2": "inputs larger than L2 (>= 2 GiB per GPU > 126 MB), no flush needed"},
            "roofline": {"bound": "hbm", "achieved": gbs, "peak": hbm, "unit": "GB/s",
                         "frac": gbs / hbm,
                         "traffic": traffic["bytes"] if traffic else None,
                         "traffic_detail": traffic or why,
                         "algorithmic_bytes": n * KEY_BYTES,
                         "peak_source": peak_src,
                         "probe_gbs": probe["best_gbs"],
                         "frac_of_probe": gbs / probe["best_gbs"],
                         "frac_of_8tbs_nominal": gbs / 8000.0},
            "probe_read": probe,
            "clocks": clk.summary(),
            "gpu_launches": launches,
            "e2e": {"value": e2e_value, "unit": "keys/s", "h2d_bytes_per_step": n * KEY_BYTES,
                    "d2h_bytes_per_step": k * (KEY_BYTES + 8),
                    "note": "C-ABI topk_select_host: pinned host keys streamed in 2^26-key "
                            "chunks overlapped with the per-chunk top-k, merge, results to "
                            "host, per step (N>1: copy + sharded top-k)"},
        }
        if keys_host is not None:
            line["cpu_baseline"] = cpu_baseline(keys_host, k)
        line.update(extra)
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        comm.close()
        dist.destroy_process_group()


def run_extras(args, tk, datagen, x, stream, torch, hbm):
    """k sweep, radix vs bitonic, adversarial inputs, the Fig-13 size sweep, the other BJ
    configs, query forms, compound keys and pure mode -- each reported, parity-tested in
    tests/."""
    dev = x.device
    n = x.numel()
    extra = {}

    def timed(f, it=10):
        for _ in range(3):
            f()
        _, per = time_steps(f, it, stream, torch, per_step=True)
        return statistics.median(per)

    sweep = []
    for kk in (1, 8, 32, 64, 128, 256, 512, 1024, 2048):
        t = timed(lambda: tk.topk(x, kk, True))
        sweep.append({"k": kk, "us": round(t * 1e3, 1), "keys_per_s": n / (t / 1e3),
                      "frac_hbm": n * KEY_BYTES / (t / 1e3) / 1e9 / hbm})
    extra["k_sweep_uniform"] = sweep
    # f2: the paper's selection-based method (radix select) on the same
    # input, next to the §7 cost model's predictions with B200 parameters
    from paper_conf_sigmod_shanbhagpm18_b200 import costmodel as cm
    hw = cm.b200(hbm)
    rv = []
    for kk in (32, 256, 1024):
        t = timed(lambda: tk.topk_radix(x, kk, True))
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
        t = timed(lambda: tk.topk(xa, 256, True))
        adv.append({"dist": d, "k": 256, "us": round(t * 1e3, 1), "keys_per_s": n / (t / 1e3),
                    "frac_hbm": n * KEY_BYTES / (t / 1e3) / 1e9 / hbm})
        del xa
    extra["adversarial_k256"] = adv
    extra["size_sweep_k64"] = size_sweep(tk, datagen, stream, torch, hbm)
    cfgs = []
    x1 = datagen.generate("uniform", 1 << 20, "f32", seed=datagen.config_seed(1), device=dev)
    t = timed(lambda: tk.topk(x1, 32, True), 50)
    cfgs.append({"config": "BJ1: 2^20 uniform f32, k=32 (per Python call, back to back: host-bound)",
                 "us": round(t * 1e3, 2), "keys_per_s": (1 << 20) / (t / 1e3)})
    v1 = torch.empty(32, dtype=torch.float32, device=dev)
    i1 = torch.empty(32, dtype=torch.int64, device=dev)
    ws1 = tk.Workspace(tk.workspace_bytes(torch.float32, 1 << 20, 32), dev)
    t = graph_us(lambda: tk.topk(x1, 32, True, out=(v1, i1, None), workspace=ws1), torch)
    cfgs.append({"config": "BJ1: 2^20 uniform f32, k=32 (device latency: 30 calls replayed from a "
                           "CUDA graph, L2-resident)", "us": round(t, 2),
                 "keys_per_s": (1 << 20) / (t / 1e6)})
    x1 = None
    del x1
    n4 = 1 << 28
    xu = datagen.generate("uniform", n4, "u32", seed=datagen.config_seed(4), device=dev)
    pu = datagen.payload(n4, seed=datagen.config_seed(4), device=dev)
    t = timed(lambda: tk.topk(xu, 64, True, payload=pu))
    cfgs.append({"config": "BJ4a: 2^28 u32 key + u32 payload, DESC LIMIT 64", "us": round(t * 1e3, 1),
                 "keys_per_s": n4 / (t / 1e3), "frac_hbm": n4 * 4 / (t / 1e3) / 1e9 / hbm})
    del xu, pu
    xd64 = datagen.generate("uniform", n4, "f64", seed=datagen.config_seed(4), device=dev)
    t = timed(lambda: tk.topk(xd64, 64, True))
    cfgs.append({"config": "BJ4b: 2^28 f64, DESC LIMIT 64", "us": round(t * 1e3, 1),
                 "keys_per_s": n4 / (t / 1e3), "frac_hbm": n4 * 8 / (t / 1e3) / 1e9 / hbm})
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
                     "rows_per_s": n4 / (t / 1e3), "frac_hbm": n4 * 8 / (t / 1e3) / 1e9 / hbm})
    del cnt, tcol, lang
    a = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(6, 2), device=dev)
    b = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(6, 3), device=dev)
    t = timed(lambda: tk.query(a, 50, True, rank_b=b, rank_w=0.5))
    cfgs.append({"config": "f1 query2: ORDER BY a + 0.5 * b DESC LIMIT 50 (f32 cols)",
                 "us": round(t * 1e3, 1), "rows_per_s": n4 / (t / 1e3),
                 "frac_hbm": n4 * 8 / (t / 1e3) / 1e9 / hbm})
    # f3: compound keys, KKV / KKKV: the 4-byte value gathered through the
    # tuple id; 8 / 12 bytes streamed per row
    k1 = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(7), device=dev)
    k2 = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(7, 1), device=dev)
    pv = datagen.payload(n4, seed=datagen.config_seed(7), device=dev)
    t = timed(lambda: tk.topk_kk(k1, k2, 64, True, True, payload=pv))
    cfgs.append({"config": "f3 KKV: 2^28 rows, ORDER BY k1 DESC, k2 DESC LIMIT 64, u32 value",
                 "us": round(t * 1e3, 1), "rows_per_s": n4 / (t / 1e3),
                 "frac_hbm": n4 * 8 / (t / 1e3) / 1e9 / hbm})
    k3 = datagen.generate("uniform", n4, "f32", seed=datagen.config_seed(7, 2), device=dev)
    t = timed(lambda: tk.topk_kkk(k1, k2, k3, 64, payload=pv))
    cfgs.append({"config": "f3 KKKV: 2^28 rows, ORDER BY k1, k2, k3 DESC LIMIT 64, u32 value",
                 "us": round(t * 1e3, 1), "rows_per_s": n4 / (t / 1e3),
                 "frac_hbm": n4 * 12 / (t / 1e3) / 1e9 / hbm})
    del k1, k2, k3, pv, a, b
    for kk in (32, 256, 1024):
        t = timed(lambda: tk.topk(x, kk, True, mode="pure"), 3)
        cfgs.append({"config": f"pure mode (paper's data-independent network on every key), "
                               f"2^29 f32, k={kk}", "us": round(t * 1e3, 1),
                     "keys_per_s": n / (t / 1e3), "frac_hbm": n * KEY_BYTES / (t / 1e3) / 1e9 / hbm})
    extra["other_configs"] = cfgs
    if not args.no_big:
        free, _ = torch.cuda.mem_get_info(dev)
        n5 = 1 << 32
        if free > n5 * 4 + (1 << 30):
            x5 = datagen.generate("uniform", n5, "f32", seed=datagen.config_seed(5), device=dev)
            t = timed(lambda: tk.topk(x5, 256, True), 5)
            cfgs.append({"config": "BJ5 at G=1: 2^32 uniform f32, k=256 (2 chunks of 2^31 + merge)",
                         "us": round(t * 1e3, 1), "keys_per_s": n5 / (t / 1e3),
                         "frac_hbm": n5 * 4 / (t / 1e3) / 1e9 / hbm})
            del x5
    return extra


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
    ap.add_argument("--no-ncu", action="store_true", help="skip the ncu traffic subprocess")
    ap.add_argument("--n-total", type=int, default=None,
                    help="strong scaling: global keys split over the ranks (e.g. 4294967296)")
    ap.add_argument("--ncu-target", action="store_true", help=argparse.SUPPRESS)
    ap.add_argument("--n", type=int, default=N_PER_GPU, help=argparse.SUPPRESS)
    args = ap.parse_args()
    if args.ncu_target:
        run_ncu_target(args)
    elif args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
