"""Summarise ncu captures into profiles/ (committed evidence).

    python tools/summarize_profiles.py ROUND   # reads gpurun_out/, writes profiles/

* launches_<round>.csv      -> profiles/launches_<round>.md (per-kernel launch list)
* prof_select_k*_<round>    -> profiles/ncu_select_k*_<round>.md (key --set full metrics)
                              profiles/traffic.json (dram bytes read+write per launch,
                              read by bench.py for the roofline "traffic" field)
"""
import csv
import glob
import json
import os
import re
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.environ.get("PROF_IN", os.path.join(ROOT, "gpurun_out"))
PROF = os.environ.get("PROF_OUT", os.path.join(ROOT, "profiles"))

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__bytes_read.sum.per_second", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size", "launch__shared_mem_per_block_dynamic",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
    "smsp__thread_inst_executed_per_inst_executed.ratio",
    "smsp__sass_average_branch_targets_threads_uniform.pct",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "sm__cycles_elapsed.avg.per_second", "lts__t_bytes.sum",
    "sm__issue_active.avg.pct_of_peak_sustained_elapsed",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
]


def raw(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(txt.splitlines()))
    h, units, vals = rows[0], rows[1], rows[2]
    return {h[i]: (vals[i], units[i]) for i in range(len(h))}


def stalls(rep):
    d = raw(rep)
    out = {}
    for name, (v, _) in d.items():
        m = re.match(r"smsp__pcsamp_warps_issue_stalled_(\w+)$", name)
        if m and not name.endswith("not_issued"):
            try:
                out[m.group(1)] = int(float(v))
            except ValueError:
                pass
    return dict(sorted(out.items(), key=lambda kv: -kv[1])[:8])


def to_bytes(v, unit):
    f = float(v.replace(",", ""))
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)


def main(rnd):
    os.makedirs(PROF, exist_ok=True)
    traffic_path = os.path.join(PROF, "traffic_summary.json")  # (bench.py measures its own)
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    for rep in sorted(glob.glob(os.path.join(OUT, f"prof_select_k*_{rnd}.ncu-rep"))):
        k = re.search(r"_k(\d+)_", rep).group(1)
        d = raw(rep)
        lines = [f"# ncu --set full: select_kernel, 2^29 uniform f32, k={k} ({rnd})", "",
                 "Command: `ncu --set full --clock-control none --import-source on "
                 f"-k regex:select_kernel -s 3 -c 1 python tools/prof_one.py 536870912 {k}` "
                 "(one launch after 3 warm-ups; cold-cache, replayed ~40x: compare shares, "
                 "not absolute times).", "", "| metric | unit | value |", "|---|---|---|"]
        for key in KEYS:
            if key in d:
                lines.append(f"| {key} | {d[key][1]} | {d[key][0]} |")
        st = stalls(rep)
        lines += ["", "Top warp-stall reasons (pc samples):", "",
                  "| reason | samples |", "|---|---|"] + [f"| {a} | {b} |" for a, b in st.items()]
        rd = to_bytes(*d["dram__bytes_read.sum"])
        wr = to_bytes(*d["dram__bytes_write.sum"])
        lines += ["", f"DRAM traffic per launch: {rd + wr:.4g} B (algorithmic: "
                      f"{(1 << 29) * 4:.4g} B = 2^29 keys x 4 B)."]
        with open(os.path.join(PROF, f"ncu_select_k{k}_{rnd}.md"), "w") as f:
            f.write("\n".join(lines) + "\n")
        traffic[f"select_k{k}"] = rd + wr
    # other captures: prof_<tag>_<round>.ncu-rep + gpurun_out/prof_meta.json
    # {tag: {"desc", "cmd", "alg_bytes"}}
    meta_p = os.path.join(OUT, "prof_meta.json")
    meta = json.load(open(meta_p)) if os.path.exists(meta_p) else {}
    for tag, m in meta.items():
        rep = os.path.join(OUT, f"prof_{tag}_{rnd}.ncu-rep")
        if not os.path.exists(rep):
            continue
        d = raw(rep)
        lines = [f"# ncu --set full: {m['desc']} ({rnd})", "", f"Command: `{m['cmd']}` (cold-cache, "
                 "replayed ~40x: compare shares, not absolute times).", "",
                 "| metric | unit | value |", "|---|---|---|"]
        for key in KEYS:
            if key in d:
                lines.append(f"| {key} | {d[key][1]} | {d[key][0]} |")
        st = stalls(rep)
        lines += ["", "Top warp-stall reasons (pc samples):", "",
                  "| reason | samples |", "|---|---|"] + [f"| {a} | {b} |" for a, b in st.items()]
        rd = to_bytes(*d["dram__bytes_read.sum"])
        wr = to_bytes(*d["dram__bytes_write.sum"])
        lines += ["", f"DRAM traffic per launch: {rd + wr:.4g} B (algorithmic: "
                      f"{m['alg_bytes']:.4g} B)."]
        with open(os.path.join(PROF, f"ncu_{tag}_{rnd}.md"), "w") as f:
            f.write("\n".join(lines) + "\n")
        traffic[tag] = rd + wr
    with open(traffic_path, "w") as f:
        json.dump(traffic, f, indent=1)
    lp = os.path.join(OUT, f"launches_{rnd}.csv")
    if os.path.exists(lp):
        rows = [r for r in csv.reader(open(lp)) if len(r) > 10]
        if not rows:
            rows = [["Kernel Name", "Metric Value"]]
        h = rows[0]
        ki, vi = h.index("Kernel Name"), h.index("Metric Value")
        agg = defaultdict(list)
        for r in rows[1:]:
            try:
                name = re.sub(r"\(.*", "", r[ki])
                v = float(r[vi].replace(",", ""))
                if "select_kernel" in name:  # the timed step vs the e2e leg's 2^26-key chunks
                    name += " [2^29-key step]" if v > 150e3 else " [e2e: 2^26-key chunk]"
                agg[name].append(v)
            except ValueError:
                pass
        tot = sum(sum(v) for v in agg.values())
        lines = [f"# Launch list of `bench.py --steps 20 --warmup 3` ({rnd})", "",
                 "`ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'select_kernel|merge_kernel' -c 60` "
                 "(only this library's kernels; per-launch times are cold-cache and serialised). "
                 "The timed step (N=1) is exactly one select_kernel launch over 2^29 keys (share of "
                 "the step: 1.0); the e2e leg adds one launch per 2^26-key host chunk + one merge.",
                 "", "| kernel | launches | mean us | share of our kernel time |", "|---|---|---|---|"]
        for name, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
            lines.append(f"| {name} | {len(v)} | {sum(v) / len(v) / 1e3:.1f} | {sum(v) / tot:.3f} |")
        with open(os.path.join(PROF, f"launches_{rnd}.md"), "w") as f:
            f.write("\n".join(lines) + "\n")
    print(open(traffic_path).read())


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "r1")
