#!/usr/bin/env python
"""Launch-parameter sweep (the Fig. 6 method of PAPER.md, on B200): time the
fused kernel over a grid of plans through fp_csr_ex / fp_dense_ex and report where the
chooser's plan (fp_choose) ranks.  Every plan's result is checked against the chooser's
result (normwise, the north_star tolerance) -- correctness never depends on the plan.

  python tools/sweep.py --config C3 [--reps 5] [--out profiles/sweep_C3.json]
"""
import argparse
import itertools
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
import paper_conf_ppopp_asharitbrcks15_b200 as fp  # noqa: E402
import synth  # noqa: E402

TOL = {"f64": 1e-11, "f32": 2e-5}


def time_call(fn, reps):
    s = torch.cuda.current_stream()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        fn()
        b.record(s)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return float(np.median(ts))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default=None)
    ap.add_argument("--variants", default=None, help="comma-separated subset of variants to sweep")
    ap.add_argument("--grids", default="74,148,222,296,370,444,592,740,888,1184,1776,2368")
    ap.add_argument("--replicas", default="1,2,4,8,16", help="copies of w for the L2-red variants (large n)")
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    cfg, inp = bench.build_inputs(args.config, 0, 1, dev)
    n, dt = cfg["n"], cfg["dtype"]
    alpha, beta = cfg["alpha"], cfg["beta"]
    xb, alg = bench.algorithmic_bytes(cfg, cfg["m"], inp["nnz_local"])
    csr = cfg["fmt"] == "csr"
    fdt = fp.FP_F64 if dt == "f64" else fp.FP_F32
    if csr:
        st = fp.fp_row_stats()
        st.m, st.n, st.nnz = cfg["m"], n, inp["nnz_local"]
        st.mean = st.nnz / st.m
        base = fp.choose(True, st, fdt, 0)
        run = lambda L=None: fp.csr(inp["rowptr"], inp["colidx"], inp["val"], n, inp["y"], inp["v"], inp["z"], alpha,
                                    beta, w=inp["w"], launch=L)
    else:
        st = fp.row_stats_dense(cfg["m"], n)
        base = fp.choose(False, st, fdt, 0)
        run = lambda L=None: fp.dense(inp["X"], inp["y"], inp["v"], inp["z"], alpha, beta, w=inp["w"], launch=L)
    run()
    torch.cuda.synchronize()
    ref = inp["w"].double().cpu().numpy().copy()
    t_base = time_call(lambda: run(base), args.reps)

    grids = [int(g) for g in args.grids.split(",")]
    if csr:
        vsk = [(1, 2), (1, 4), (1, 12), (1, 16), (2, 2), (2, 4), (2, 8), (4, 2), (4, 4), (8, 1), (8, 2), (16, 1),
               (16, 2), (32, 2), (32, 4)]
        space = [(var, vs, k) for var in (3, 4, 5, 11) for vs, k in vsk]   # CSR-vector, Eq. (4)'s VS x K
        space += [(var, 32, nb) for var in (6, 7, 8, 12) for nb in (2, 4, 8)]   # flat kernels: k = NB tiles
        space += [(16, 32, 8), (18, 32, 8)]   # flat + y prefix + L2 reds; flat-4 + fixed-point partial
        if dt == "f32":
            space += [(17, 32, 8)]            # binned scatter
        if cfg["n"] <= 2048:
            space += [(10, vs, k) for vs, k in ((4, 4), (8, 2), (16, 2), (32, 4))]   # owner-computes
    else:
        space = [(base.variant, base.vs, base.tl)]
    if args.variants:
        keep = {int(v) for v in args.variants.split(",")}
        space = [s for s in space if s[0] in keep]
    # the L2-red variants also sweep the copies of w their reds spread over (fp_launch.cluster)
    reps_l2 = [int(r) for r in args.replicas.split(",")] if csr and cfg["n"] > 8192 else [0]
    space = [(var, vs, k, (r if var in (4, 7, 16) else 0)) for (var, vs, k) in space
             for r in (reps_l2 if var in (4, 7, 16) else [0])]
    rows = []
    for (var, vs, k, rep), g in itertools.product(space, grids):
        L = fp.fp_launch()
        L.variant, L.vs, L.tl, L.bs, L.grid = var, vs, k, (1024 if var in (16, 17) else 256), g
        L.cluster = rep
        try:
            ms = time_call(lambda: run(L), args.reps)
        except fp.FusedPatError as e:
            rows.append(dict(variant=var, vs=vs, k=k, grid=g, replicas=rep, ms=None, err=str(e)[:80]))
            continue
        w = inp["w"].double().cpu().numpy()
        rel = float(np.linalg.norm(w - ref) / max(np.linalg.norm(ref), 1e-300))
        rows.append(dict(variant=var, vs=vs, k=k, grid=g, replicas=rep, ms=ms, gbs=xb / ms / 1e6, rel_vs_chooser=rel,
                         ok=rel <= TOL[dt]))
    timed = sorted([r for r in rows if r["ms"] is not None], key=lambda r: r["ms"])
    rank = sum(1 for r in timed if r["ms"] < t_base) + 1
    best = timed[0]
    # the paper's quality claim: the model's choice within 2 % of the best setting and
    # in the top 1 % of all settings
    out = dict(config=args.config, chooser=base.as_dict(), chooser_ms=t_base, chooser_gbs=xb / t_base / 1e6,
               best=best, chooser_rank=rank, settings=len(timed), chooser_vs_best=t_base / best["ms"],
               within_2pct=t_base <= 1.02 * best["ms"], top_1pct=rank <= max(1, int(0.01 * len(timed) + 0.5)),
               columns=bench.COLS,
               all_ok=all(r.get("ok", True) for r in rows), results=rows)
    print(json.dumps({k: v for k, v in out.items() if k != "results"}))
    if args.out:
        json.dump(out, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
