#!/usr/bin/env python
"""Probe: time CSR plans on synthetic matrices of a chosen shape (device-generated), to see
what bounds a kernel.  python tools/split_probe.py m n dtype lengths-json plan[,plan...]
plan = variant:cluster (variant 13) or variant:vs:k (fp_csr_ex plans); 'auto' = chooser."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_asharitbrcks15_b200 as fp  # noqa: E402
import synth  # noqa: E402


def main():
    m, n, dt = int(sys.argv[1]), int(sys.argv[2]), sys.argv[3]
    lengths = tuple(json.loads(sys.argv[4]))
    dev = torch.device("cuda:0")
    rp, ci, va = synth.csr(m, n, dt, lengths, seed=7, device=dev)
    y = synth.vector(n, dt, seed=7, stream=synth.S_Y, device=dev)
    v = synth.vector(m, dt, kind="pos", seed=7, stream=synth.S_V, device=dev)
    z = synth.vector(n, dt, seed=7, stream=synth.S_Z, device=dev)
    nnz = va.shape[0]
    for spec in sys.argv[5].split(","):
        parts = spec.split(":")
        L = None
        if parts[0] != "auto":
            L = fp.fp_launch()
            L.variant = int(parts[0])
            if L.variant == 13:
                L.cluster = int(parts[1])
            else:
                L.vs, L.tl, L.bs, L.grid = int(parts[1]), int(parts[2]), 256, 0
        P = fp.CsrPlan(rp, ci, n, va.dtype, launch=L) if (L is None or L.variant == 13) else None
        run = (lambda: P(va, y, v, z, 1.0, 1.0)) if P else (lambda: fp.csr(rp, ci, va, n, y, v, z, 1.0, 1.0, launch=L))
        for _ in range(2):
            run()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(5):
            run()
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / 5
        lb = P.launch.as_dict() if P else L.as_dict()
        print(f"{m}x{n} {dt} {lengths} nnz={nnz} plan={spec} -> {ms:.3f} ms  "
              f"{nnz * (4 + va.element_size()) / ms / 1e6:.0f} GB/s  [{lb['variant_name']} cs={lb['cluster']} "
              f"tl={lb['tl']} grid={lb['grid']}]", flush=True)


if __name__ == "__main__":
    main()
