#!/usr/bin/env python
"""Dense plan probe (C2 by default): time fp_dense_ex plans (VS, TL, grid) with CUDA events,
median of N, each result checked against the chooser's.  python tools/dense_probe.py [config]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import paper_conf_ppopp_asharitbrcks15_b200 as fp  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2"
dev = torch.device("cuda:0")
cfg, inp = bench.build_inputs(name, 0, 1, dev)
fdt = fp.FP_F64 if cfg["dtype"] == "f64" else fp.FP_F32
run = lambda L=None: fp.dense(inp["X"], inp["y"], inp["v"], inp["z"], cfg["alpha"], cfg["beta"], w=inp["w"], launch=L)
base = fp.choose(False, fp.row_stats_dense(cfg["m"], cfg["n"]), fdt, 0)
run()
torch.cuda.synchronize()
ref = inp["w"].double().cpu().numpy().copy()
s = torch.cuda.current_stream()


def t(L, reps=20):
    ts = []
    for i in range(reps + 3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        run(L)
        b.record(s)
        torch.cuda.synchronize()
        if i >= 3:
            ts.append(a.elapsed_time(b))
    return float(np.median(ts))


print("chooser", base.as_dict(), f"{t(base):.4f} ms")
n = cfg["n"]
for vs in (4, 8, 16, 32):
    tl = max(1, (n + vs - 1) // vs)
    for grid in (296, 444, 592, 888):
        L = fp.fp_launch()
        L.variant, L.vs, L.tl, L.bs, L.grid = 1, vs, tl, 256, grid
        try:
            ms = t(L)
            w = inp["w"].double().cpu().numpy()
            rel = np.linalg.norm(w - ref) / np.linalg.norm(ref)
            print(f"vs={vs} tl={tl} grid={grid}: {ms:.4f} ms  rel {rel:.1e}")
        except fp.FusedPatError as e:
            print(f"vs={vs} tl={tl} grid={grid}: {str(e)[:70]}")
for tl in (4, 8, 16, 32):
    for grid in (148, 296, 592, 888, 1184):
        L = fp.fp_launch()
        L.variant, L.vs, L.tl, L.bs, L.grid = 2, 256, tl, 256, grid
        try:
            ms = t(L)
            w = inp["w"].double().cpu().numpy()
            rel = np.linalg.norm(w - ref) / np.linalg.norm(ref)
            print(f"CTA variant tl={tl} grid={grid}: {ms:.4f} ms  rel {rel:.1e}")
        except fp.FusedPatError as e:
            print(f"CTA variant tl={tl} grid={grid}: {str(e)[:70]}")
