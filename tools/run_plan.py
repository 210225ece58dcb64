#!/usr/bin/env python
"""Run one config with an explicit launch plan (fp_csr_ex / fp_dense_ex) a few times -- a
short target for `ncu -k regex:... ` captures of a specific kernel variant.

  python tools/run_plan.py --config C3 --variant 6 --vs 32 --tl 8 --grid 592 --reps 3
"""
import argparse
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
import paper_conf_ppopp_asharitbrcks15_b200 as fp  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--variant", type=int, required=True)
    ap.add_argument("--vs", type=int, default=32)
    ap.add_argument("--tl", type=int, default=0)
    ap.add_argument("--grid", type=int, default=592)
    ap.add_argument("--reps", type=int, default=3)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    cfg, inp = bench.build_inputs(a.config, 0, 1, dev)
    L = fp.fp_launch()
    L.variant, L.vs, L.tl, L.bs, L.grid = a.variant, a.vs, a.tl, 256, a.grid
    for _ in range(a.reps):
        if cfg["fmt"] == "csr":
            fp.csr(inp["rowptr"], inp["colidx"], inp["val"], cfg["n"], inp["y"], inp["v"], inp["z"], cfg["alpha"],
                   cfg["beta"], w=inp["w"], launch=L)
        else:
            fp.dense(inp["X"], inp["y"], inp["v"], inp["z"], cfg["alpha"], cfg["beta"], w=inp["w"], launch=L)
    torch.cuda.synchronize()
    print("ok")


if __name__ == "__main__":
    main()
