#!/usr/bin/env python
"""C1 latency probe: time fp_dense_ex plans on the C1 problem with a cold L2 (flush between
calls), median of N.  python tools/c1_probe.py"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import paper_conf_ppopp_asharitbrcks15_b200 as fp  # noqa: E402

dev = torch.device("cuda:0")
cfg, inp = bench.build_inputs("C1", 0, 1, dev)
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
run = lambda L=None: fp.dense(inp["X"], inp["y"], inp["v"], inp["z"], cfg["alpha"], cfg["beta"], w=inp["w"], launch=L)
st = fp.row_stats_dense(cfg["m"], cfg["n"])
base = fp.choose(False, st, fp.FP_F64, 0)
print("chooser", base.as_dict())


def t(L, reps=40, cold=True):
    ts = []
    s = torch.cuda.current_stream()
    for i in range(reps + 5):
        if cold:
            flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        run(L)
        b.record(s)
        torch.cuda.synchronize()
        if i >= 5:
            ts.append(a.elapsed_time(b) * 1e3)
    return float(np.median(ts))


print("chooser cold us", t(base), "warm us", t(base, cold=False))
for vs in (8, 16, 32):
    for tl in (4, 8, 16):
        if vs * tl < cfg["n"] or tl * 8 > 256:
            continue
        for grid in (16, 32, 64, 125, 148, 296):
            L = fp.fp_launch()
            L.variant, L.vs, L.tl, L.bs, L.grid = 1, vs, tl, 256, grid
            try:
                print(f"vs={vs} tl={tl} grid={grid}: cold {t(L):.2f} us  warm {t(L, cold=False):.2f} us")
            except fp.FusedPatError as e:
                print(f"vs={vs} tl={tl} grid={grid}: {str(e)[:60]}")
