"""The fused multi-GPU exchange over peer memory (FP_COMM_PEER, csrc/comm.cu), exercised with
2..8 ranks on ONE GPU through fp_comm_init_local_group -- the same kernels (epoch flags with
system-scope release/acquire, a one-warp barrier, the rank-ordered sum of the ranks'
partials) that run across GPUs on CUDA-IPC-mapped buffers.

Row a11 / SURVEY 8(e): Eq. (1) is a sum over rows (Eq. 2/3), so X row-partitioned
over ranks needs exactly one exchange of the n-vector partials; beta*z is added once (R18).
Each simulated rank runs in its own host thread on its own stream.  On one device no kernel
waits for another rank's launch (B200_PROFILING: separate launches that spin on one another may
never run together): each rank publishes its flag, synchronises its stream and meets the others
on the host, and only then launches its barrier, whose flags are already set (comm.cu
peer_finish).  Checked: integer twins bit-exact against the full-matrix oracle, every rank holding
the identical bits, three calls in a row (both parities of the double-buffered partials),
fp_allreduce, and the CG driver with a peer communicator against the single-GPU CG.
"""
import threading

import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_asharitbrcks15_b200 as fp
import synth
from _util import assert_bitexact

pytestmark = pytest.mark.gpu


def run_ranks(P, fn):
    """fn(rank, stream) in P threads; returns the per-rank results (re-raises the first error)."""
    out, err = [None] * P, []

    def body(r):
        try:
            s = torch.cuda.Stream(device=0)
            with torch.cuda.stream(s):
                out[r] = fn(r, s)
            s.synchronize()
        except Exception as e:  # noqa: BLE001 -- reported below
            err.append((r, e))

    th = [threading.Thread(target=body, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(120)
    assert not any(t.is_alive() for t in th), "a rank did not finish (barrier deadlock?)"
    if err:
        raise err[0][1]
    return out


@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("fmt,dt", [("csr", "f32"), ("csr", "f64"), ("dense", "f64")])
def test_peer_dist_bitexact(cuda_dev, P, fmt, dt):
    m, n = 24_011, (3000 if fmt == "csr" else 96)
    y = synth.vector(n, dt, kind="int_small", seed=P, stream=synth.S_Y)
    z = synth.vector(n, dt, kind="int_small", seed=P, stream=synth.S_Z)
    v = synth.vector(m, dt, kind="int_pos", seed=P, stream=synth.S_V)
    if fmt == "csr":
        rp, ci, va = synth.csr(m, n, dt, ("powerlaw", 2.5, 13.64), kind="int_pm12", seed=P)
        full, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, -2.0)
        b = fp.shard_rows_csr(rp, P)
        shards = [fp.shard_slice_csr(rp, ci, va, v, b, r) for r in range(P)]
        shards = [tuple(t.contiguous().to(cuda_dev) for t in sh) for sh in shards]
    else:
        X = synth.dense(m, n, dt, kind="int_pm12", seed=P)
        full, _ = oracle.dense(X, y, v, z, 1.0, -2.0)
        b = fp.shard_rows_dense(m, P)
        shards = [(X[b[r]:b[r + 1]].contiguous().to(cuda_dev), v[b[r]:b[r + 1]].to(cuda_dev)) for r in range(P)]
    yd, zd = y.to(cuda_dev), z.to(cuda_dev)
    # each shard's local-pass kernel once, serially: its first launch loads the kernel (lazy
    # module loading synchronises the device, which would wait on another rank's spinning barrier)
    for r in range(P):
        if fmt == "csr":
            lrp, lci, lva, lv = shards[r]
            fp.csr(lrp, lci, lva, n, yd, lv, zd, 1.0, -2.0)
        else:
            fp.dense(shards[r][0], yd, shards[r][1], zd, 1.0, -2.0)
    torch.cuda.synchronize()
    g = fp.LocalGroup(P, 0, max_bytes=n * 8)
    try:
        for rep in range(3):
            def fn(r, s):
                if fmt == "csr":
                    lrp, lci, lva, lv = shards[r]
                    return fp.csr_dist(g.comms[r], lrp, lci, lva, n, yd, lv, zd, 1.0, -2.0, stream=s)
                Xl, vl = shards[r]
                return fp.dense_dist(g.comms[r], Xl, yd, vl, zd, 1.0, -2.0, stream=s)
            ws = run_ranks(P, fn)
            torch.cuda.synchronize()
            assert not g.timed_out()
            for r in range(P):
                assert torch.equal(ws[r], ws[0]), f"rank {r} differs from rank 0 (call {rep})"
            assert_bitexact(ws[0], full, f"peer {fmt} {dt} P={P} call {rep}")
    finally:
        g.close()


def test_peer_allreduce_rank_order(cuda_dev):
    P, n = 5, 100_003
    vecs = [torch.randn(n, dtype=torch.float64, generator=torch.Generator().manual_seed(r)) for r in range(P)]
    ref = vecs[0].numpy().copy()
    for r in range(1, P):
        ref = ref + vecs[r].numpy()  # the kernel's order: ((v0 + v1) + v2) + ...
    g = fp.LocalGroup(P, 0, max_bytes=n * 8)
    try:
        bufs = [t.to(cuda_dev) for t in vecs]
        run_ranks(P, lambda r, s: g.comms[r].allreduce(bufs[r], stream=s))
        torch.cuda.synchronize()
        for r in range(P):
            assert np.array_equal(bufs[r].cpu().numpy(), ref)
    finally:
        g.close()


def test_peer_cg_matches_single_gpu(cuda_dev):
    P, m, n = 4, 20_000, 50
    X = synth.dense(m, n, "f64", kind="colscaled", seed=14)
    lab = synth.vector(m, "f64", seed=14, stream=synth.S_LABEL)
    w1, it1, h1 = fp.cg_linreg_dense(X.to(cuda_dev), lab.to(cuda_dev), eps=1e-3, max_iter=10, tol=0.0)
    b = fp.shard_rows_dense(m, P)
    Xs = [X[b[r]:b[r + 1]].contiguous().to(cuda_dev) for r in range(P)]
    ls = [lab[b[r]:b[r + 1]].to(cuda_dev) for r in range(P)]
    g = fp.LocalGroup(P, 0, max_bytes=n * 8)
    try:
        res = run_ranks(P, lambda r, s: fp.cg_linreg_dense(Xs[r], ls[r], eps=1e-3, max_iter=10, tol=0.0,
                                                           comm=g.comms[r], stream=s))
        torch.cuda.synchronize()
        assert not g.timed_out()
        for r in range(P):
            w, it, h = res[r]
            assert it == it1 == 10
            assert torch.equal(w, res[0][0]), "ranks disagree on the CG iterate"
            np.testing.assert_allclose(h.numpy(), h1.numpy(), rtol=1e-8)
            assert float((w - w1).norm() / w1.norm()) < 1e-8
    finally:
        g.close()


@pytest.mark.parametrize("P", [2, 4])
@pytest.mark.parametrize("packed", [True, False, "l2"])
def test_peer_plan_dist_bitexact(cuda_dev, monkeypatch, P, packed):
    """fp_csr_plan_dist: every rank runs its shard's plan (packed copy: variant 19 or 20, or the
    unpacked plan) and the peer exchange; every rank bit-identical and bit-exact against the
    full-matrix oracle on an integer twin, over three calls.  The ranks share one GPU here, so
    the packed passes (cooperative launches) use 4 CTA groups each (FP_PK_GROUPS)."""
    m, n = 30_011, 60_000
    y = synth.vector(n, "f32", kind="int_small", seed=P, stream=synth.S_Y)
    z = synth.vector(n, "f32", kind="int_small", seed=P, stream=synth.S_Z)
    v = synth.vector(m, "f32", kind="int_pos", seed=P, stream=synth.S_V)
    rp, ci, va = synth.csr(m, n, "f32", ("powerlaw", 2.5, 13.64), kind="int_pm12", seed=P)
    full, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, -2.0)
    b = fp.shard_rows_csr(rp, P)
    shards = [tuple(t.contiguous().to(cuda_dev) for t in fp.shard_slice_csr(rp, ci, va, v, b, r)) for r in range(P)]
    monkeypatch.setenv("FP_PK_GROUPS", "4")
    if packed == "l2":  # variant 20 (L2-sized column blocks, forced small) on every rank's shard
        monkeypatch.setenv("FP_PK_L2", "1")
        monkeypatch.setenv("FP_L2B_BW", "7000")
        monkeypatch.setenv("FP_L2B_HOT", "40")
    plans = []
    for lrp, lci, lva, lv in shards:
        pl = fp.CsrPlan(lrp, lci, n, torch.float32)
        if packed:
            pl.pack(lva)
        plans.append(pl)
    torch.cuda.synchronize()
    yd, zd = y.to(cuda_dev), z.to(cuda_dev)
    for r in range(P):  # load the kernels before the ranks run concurrently
        plans[r](None if packed else shards[r][2], yd, shards[r][3], zd, 1.0, -2.0)
    torch.cuda.synchronize()
    g = fp.LocalGroup(P, 0, max_bytes=n * 8)
    try:
        for rep in range(3):
            def fn(r, s):
                return plans[r].dist(g.comms[r], None if packed else shards[r][2], yd, shards[r][3], zd, 1.0, -2.0,
                                     stream=s)
            ws = run_ranks(P, fn)
            torch.cuda.synchronize()
            assert not g.timed_out()
            for r in range(P):
                assert torch.equal(ws[r], ws[0]), f"rank {r} differs from rank 0 (call {rep})"
            assert_bitexact(ws[0], full, f"plan dist packed={packed} P={P} call {rep}")
    finally:
        g.close()
