#!/usr/bin/env python
"""C5 variance probe: per-pass times of the fused op on the C5 matrix and per-solve CG times."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import paper_conf_ppopp_asharitbrcks15_b200 as fp  # noqa: E402
import synth  # noqa: E402

dev = torch.device("cuda:0")
cfg, inp = bench.build_inputs("C5", 0, 1, dev)
labels = synth.vector(cfg["m"], "f64", seed=synth.config_seed("C5"), stream=synth.S_LABEL, device=dev)
s = torch.cuda.current_stream()


def ev(fn, k):
    out = []
    for _ in range(k):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        fn()
        b.record(s)
        torch.cuda.synchronize()
        out.append(a.elapsed_time(b))
    return np.round(out, 2).tolist()


print("X ptr", hex(inp["X"].data_ptr()), "bytes", inp["X"].numel() * 8)
print("pass ms", ev(lambda: fp.dense(inp["X"], inp["y"], None, inp["z"], 1.0, 1e-3, w=inp["w"]), 30))
print("solve ms", ev(lambda: fp.cg_linreg_dense(inp["X"], labels, eps=1e-3, max_iter=20, tol=0.0), 5))
print("pass ms", ev(lambda: fp.dense(inp["X"], inp["y"], None, inp["z"], 1.0, 1e-3, w=inp["w"]), 10))
if len(sys.argv) > 1:  # with nvidia-smi polling as bench.py's clock sampler does
    smi = bench.ClockSampler(0)
    smi.start()
    print("solve ms (nvidia-smi -lms 100 running)", ev(lambda: fp.cg_linreg_dense(inp["X"], labels, eps=1e-3, max_iter=20, tol=0.0), 10))
    print(smi.stop())
    print("solve ms (after)", ev(lambda: fp.cg_linreg_dense(inp["X"], labels, eps=1e-3, max_iter=20, tol=0.0), 5))
