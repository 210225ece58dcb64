#!/usr/bin/env python
"""Small-shape driver for compute-sanitizer (memcheck / racecheck / synccheck): every kernel
family once -- dense vector / CTA / cluster, CSR vector (shared / L2 / private / owner /
fixed-point / cp.async stream), flat (shared / L2 / private / fixed / 1024-thread with a y
prefix), flat-4 with the fixed-point partial (18), the binned scatter (17: producer, consumer,
finalize), the packed plans (19: k_pk1 with its TMA ring, the cooperative k_pk; 20: L2 blocks
with hot columns and long rows, and their pack kernels), the peer exchange (one-rank local group), the L2-replica fold, the column-split plan, the row epilogues, CG and TRON drivers --
on tiny inputs.

  compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_ppopp_asharitbrcks15_b200 as fp  # noqa: E402
import synth  # noqa: E402


def main():
    dev = torch.device("cuda:0")
    for dt in ("f64", "f32"):
        for (m, n) in ((300, 33), (257, 128), (70, 3000), (9, 20000)):
            X = synth.dense(m, n, dt, seed=1, device=dev)
            y = synth.vector(n, dt, seed=1, device=dev)
            v = synth.vector(m, dt, kind="pos", seed=1, stream=synth.S_V, device=dev)
            z = synth.vector(n, dt, seed=1, stream=synth.S_Z, device=dev)
            fp.dense(X, y, v, z, 0.5, 1.5)
            fp.dense(X, None, v, None, 1.0, 0.0)
            p = torch.empty(m, dtype=X.dtype, device=dev)
            fp.dense_epi(X, y, v, None, 1.0, 0.0, fp.FP_EPI_LINEAR, row_out=p)
        rp, ci, va = synth.csr(2000, 700, dt, ("powerlaw", 2.0, 3.0), seed=2, device=dev)
        y = synth.vector(700, dt, seed=2, device=dev)
        v = synth.vector(2000, dt, kind="pos", seed=2, stream=synth.S_V, device=dev)
        z = synth.vector(700, dt, seed=2, stream=synth.S_Z, device=dev)
        experimental = b"+experimental" in fp.lib().fp_version()
        for var, vs, tl in ((3, 8, 2), (3, 4, 4), (4, 32, 4), (5, 8, 2), (6, 32, 4), (7, 32, 8), (8, 32, 2),
                            (10, 8, 2), (11, 4, 4), (12, 32, 4), (14, 4, 4), (15, 4, 4), (16, 32, 8), (18, 32, 8)):
            if var in (10, 12, 14, 15) and not experimental:
                continue
            L = fp.fp_launch()
            L.variant, L.vs, L.tl, L.bs, L.grid = var, vs, tl, 1024 if var == 16 else 256, 13
            fp.csr(rp, ci, va, 700, y, v, z, 1.0, 1.0, launch=L)  # 4/7/16: w replicated over L2, folded
        # variant 16 with a partial y prefix in shared memory (n beyond the ~56K / 28K staged)
        nw = 60000 if dt == "f32" else 30000
        rpw, ciw, vaw = synth.csr(500, nw, dt, ("powerlaw", 2.0, 3.0), seed=5, device=dev)
        yw = synth.vector(nw, dt, seed=5, device=dev)
        L = fp.fp_launch()
        L.variant, L.vs, L.tl, L.bs, L.grid = 16, 32, 8, 1024, 7
        fp.csr(rpw, ciw, vaw, nw, yw, None, yw, 1.0, 1.0, launch=L)
        # variant 17 (binned scatter, fp32): one and two column blocks, long + empty rows
        if dt == "f32":
            for nb, nn in ((1, 700), (2, 90000)):
                rpb, cib, vab = synth.csr(3000, nn, dt, ("powerlaw", 2.0, 3.0), seed=6, device=dev)
                yb = synth.vector(nn, dt, seed=6, device=dev)
                zb = synth.vector(nn, dt, seed=6, stream=synth.S_Z, device=dev)
                vb = synth.vector(3000, dt, kind="pos", seed=6, stream=synth.S_V, device=dev)
                L = fp.fp_launch()
                L.variant, L.vs, L.tl, L.bs, L.grid, L.cluster = 17, 32, 8, 1024, 5, nb
                fp.csr(rpb, cib, vab, nn, yb, vb, zb, 1.0, 1.0, launch=L)
                fp.csr(rpb, cib, vab, nn, None, vb, None, 2.0, 0.0, launch=L)
        # packed plans: variant 19 (one block: k_pk1 with the TMA tile ring; fp32 two blocks: the
        # cooperative k_pk) and variant 20 (L2 blocks, forced small; hot columns; long rows)
        rpp, cip, vap = synth.csr(3000, 1500, dt, ("uniform", 0, 700), seed=8, device=dev)
        yp = synth.vector(1500, dt, seed=8, device=dev)
        vp = synth.vector(3000, dt, kind="pos", seed=8, stream=synth.S_V, device=dev)
        P1 = fp.CsrPlan(rpp, cip, 1500, vap.dtype)
        P1.pack(vap)
        P1(None, yp, vp, yp, 1.0, 1.0)
        P1(None, None, vp, None, 2.0, 0.0)
        if dt == "f32":
            rq, cq, vq = synth.csr(4000, 60000, dt, ("powerlaw", 2.0, 3.0), seed=9, device=dev)
            yq = synth.vector(60000, dt, seed=9, device=dev)
            os.environ["FP_PK_GROUPS"] = "2"
            P2 = fp.CsrPlan(rq, cq, 60000, vq.dtype)
            P2.pack(vq)
            del os.environ["FP_PK_GROUPS"]
            P2(None, yq, None, yq, 1.0, 1.0)
        rl, cl, vl = synth.csr(3000, 20000, dt, ("powerlaw", 2.5, 9.5), seed=10, device=dev, col_skew=2)
        yl = synth.vector(20000, dt, seed=10, device=dev)
        vl2 = synth.vector(3000, dt, kind="pos", seed=10, stream=synth.S_V, device=dev)
        os.environ.update(FP_PK_L2="1", FP_L2B_BW="6000", FP_L2B_HOT="50")
        P3 = fp.CsrPlan(rl, cl, 20000, vl.dtype)
        P3.pack(vl)
        for k in ("FP_PK_L2", "FP_L2B_BW", "FP_L2B_HOT"):
            del os.environ[k]
        P3(None, yl, vl2, yl, 1.0, 1.0)
        P3(None, None, vl2, None, 1.0, 0.0)
        # the peer exchange (one-rank local group: the same kernels, a trivially met barrier)
        g = fp.LocalGroup(1, 0, max_bytes=700 * 8)
        fp.csr_dist(g.comms[0], rp, ci, va, 700, y, v, z, 1.0, 1.0)
        g.comms[0].allreduce(y.clone())
        torch.cuda.synchronize()
        g.close()
        # CSR plan with the column split of variant 13 (cluster of 2)
        F = fp.fp_launch()
        F.variant, F.cluster = 13, 2
        P = fp.CsrPlan(rp, ci, 700, va.dtype, launch=F)
        P(va, y, v, z, 1.0, 1.0)
        lab = torch.where(synth.vector(2000, dt, seed=3, device=dev) > 0, 1.0, -1.0).to(va.dtype)
        D = torch.empty(2000, dtype=va.dtype, device=dev)
        loss = torch.zeros(1, dtype=torch.float64, device=dev)
        fp.csr_epi(rp, ci, va, 700, y, lab, y, 1.0, 1.0, fp.FP_EPI_LOGISTIC, c=1.0, row_out=D, scalar_out=loss)
        Xc = synth.dense(500, 40, dt, seed=4, device=dev)
        b = synth.vector(500, dt, seed=4, device=dev)
        fp.cg_linreg_dense(Xc, b, max_iter=3, tol=0.0)
        fp.logreg_tron_dense(Xc, torch.where(b > 0, 1.0, -1.0).to(b.dtype), max_iter=2)
    torch.cuda.synchronize()
    print("sanitize driver ok")


if __name__ == "__main__":
    main()
