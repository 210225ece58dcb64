#!/usr/bin/env python
"""Summarise ncu captures for profiles/ (run here, on the CPU box, on reports fetched from
gpurun_out/).

  python tools/ncu_summary.py full   <report.ncu-rep> <config> <alg_bytes_per_launch> > profiles/X.md
  python tools/ncu_summary.py launches <launches.csv>                                  > profiles/Y.md

`full` also merges {config: {dram_bytes_per_launch, ...}} into profiles/ncu_traffic.json, the
file bench.py reads for roofline.traffic.
"""
import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram__bytes.sum.per_second",
    "lts__t_sector_hit_rate.pct", "lts__t_bytes.sum", "l1tex__t_bytes.sum",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size", "launch__occupancy_limit_registers",
    "launch__occupancy_limit_shared_mem", "smsp__cycles_active.avg", "sm__cycles_elapsed.avg.per_second",
    "smsp__average_warp_latency_issue_stalled_long_scoreboard", "smsp__inst_executed.sum",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "lts__t_sectors_op_red.sum", "lts__t_sectors_op_atom.sum",
]


def to_bytes(val, unit):
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    return float(val) * scale.get(unit, 1)


def raw_rows(rep):
    if rep.endswith(".csv"):  # a `--page raw --csv` export made on the GPU box
        out = open(rep).read()
    else:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    hdr, units, rows = r[0], r[1], r[2:]
    return hdr, units, rows


def full(rep, config, alg_bytes, variant=None, rnd=None):
    hdr, units, rows = raw_rows(rep)
    print(f"# ncu --set full: {os.path.basename(rep)} ({config})\n")
    traffic_all = []
    per_kernel = defaultdict(list)
    for row in rows:
        d = dict(zip(hdr, row))
        u = dict(zip(hdr, units))
        name = d.get("Kernel Name", "?")
        print(f"## {name}\n")
        print("| metric | unit | value |\n|---|---|---|")
        for k in KEYS:
            if k in d:
                print(f"| {k} | {u.get(k, '')} | {d[k]} |")
        rb = to_bytes(d["dram__bytes_read.sum"], u["dram__bytes_read.sum"])
        wb = to_bytes(d["dram__bytes_write.sum"], u["dram__bytes_write.sum"])
        t = rb + wb
        traffic_all.append(t)
        per_kernel[name].append(t)
        print(f"\nDRAM traffic per launch: {t / 1e9:.4f} GB; algorithmic bytes per launch: {alg_bytes / 1e9:.4f} GB; "
              f"traffic / algorithmic = {t / alg_bytes:.4f}\n")
    # one step = one launch of every distinct kernel of the fp_* call (variant 17: producer,
    # consumer, finalize): the step's traffic is the sum of their per-launch means
    kern = {k: int(sum(v) / len(v)) for k, v in per_kernel.items()}
    step = sum(kern.values())
    if os.environ.get("NCU_STEP_ALL"):  # the capture is exactly one step (variant 20: a launch per block)
        kern = {k: int(sum(v)) for k, v in per_kernel.items()}
        step = int(sum(traffic_all))
    print(f"\nDRAM traffic per step (sum over the {len(kern)} kernels): {step / 1e9:.4f} GB; "
          f"traffic / algorithmic = {step / alg_bytes:.4f}\n")
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    db = json.load(open(p)) if os.path.exists(p) else {}
    db[config] = {"dram_bytes_per_step": step, "algorithmic_bytes_per_step": int(alg_bytes),
                  "kernels": kern, "file": os.path.basename(rep), "variant": variant, "round": rnd}
    json.dump(db, open(p, "w"), indent=1, sort_keys=True)


def launches(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    hdr = rows[0]
    idx = {k: i for i, k in enumerate(hdr)}
    agg = defaultdict(list)
    for r in rows[1:]:
        if r[idx["Metric Name"]] != "gpu__time_duration.sum":
            continue
        agg[r[idx["Kernel Name"]]].append(float(r[idx["Metric Value"]]))
    total = sum(sum(v) for v in agg.values())
    print(f"# launch list: {os.path.basename(path)} (ncu --metrics gpu__time_duration.sum, cold-cache, serialised)\n")
    print("| kernel | launches | mean us | share of listed time |\n|---|---|---|---|")
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        print(f"| `{k[:110]}` | {len(v)} | {sum(v) / len(v) / 1e3:.1f} | {100 * sum(v) / total:.1f}% |")


if __name__ == "__main__":
    if sys.argv[1] == "full":
        full(sys.argv[2], sys.argv[3], float(sys.argv[4]), int(sys.argv[5]) if len(sys.argv) > 5 else None,
             sys.argv[6] if len(sys.argv) > 6 else None)
    else:
        launches(sys.argv[2])
