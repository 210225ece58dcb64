"""GPU parity of variant 19 (FP_VAR_CSR_PACKED, csr_packed.cu) against the fp64 oracle.

The packed plan (fp_csr_plan_pack) splits the columns into CS = 1/2/4/8 blocks, one CTA per
block and SM holding y and the partial w of its block in shared memory (SURVEY 8 rows a3/a7/
a9/a10 at large n); the row dots of Eq. (2) are completed across the CTAs of a group
(one tagged word per row through L2), the scatter of Eq. (3) (Alg. 2 l.13-14) runs
from the registers that hold the row, into a 32-bit fixed-point partial (reading R25).
Checked here, at sizes the oracle finishes in seconds:
* integer twins bit-exact for every block count, every instance (with/without y, v, beta*z),
  power-law / binomial / long rows (segments beyond the 256-entry register window), empty rows,
  non-canonical rows (i.i.d. columns: unsorted, repeats), ragged m;
* the int32 wrap and the terms beyond the CTA's cap carried by the fp64 spill;
* U[-1,1) fp32 data within the north_star 2e-5 normwise tolerance, rows scaled by 2^+-30;
* IEEE propagation of Inf/NaN terms (reading R8);
* determinism (bit-identical reruns), re-packing with new values, CUDA-graph replays (the
  per-call exchange tag lives in device memory);
* what it refuses (exec without values on an unpacked plan); fp64 wider than one block takes
  variant 20's L2-sized column blocks (csr_l2block.cu), tested at the end;
* the single-block pass (k_pk1, fp32 and fp64) on C3/S3-shaped matrices.
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_asharitbrcks15_b200 as fp
import synth
from _util import assert_bitexact, assert_parity

pytestmark = pytest.mark.gpu


def make(m, n, lengths, seed, kind, col_skew=0):
    rp, ci, va = synth.csr(m, n, "f32", lengths, kind=kind, seed=seed, col_skew=col_skew)
    integer = kind.startswith("int")
    y = synth.vector(n, "f32", kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Y)
    v = synth.vector(m, "f32", kind="int_pos" if integer else "pos", seed=seed, stream=synth.S_V)
    z = synth.vector(n, "f32", kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Z)
    return rp, ci, va, y, v, z


def packed_plan(dev, rp, ci, va, n, blocks=0, monkeypatch=None):
    if monkeypatch is not None:
        monkeypatch.setenv("FP_PK_CS", str(blocks))
    plan = fp.CsrPlan(rp.to(dev), ci.to(dev), n, torch.float32)
    plan.pack(va.to(dev))
    torch.cuda.synchronize()
    if monkeypatch is not None:
        monkeypatch.delenv("FP_PK_CS")
    return plan


def run(plan, dev, y, v, z, alpha, beta):
    cu = lambda t: None if t is None else t.to(dev)
    w = plan(None, cu(y), cu(v), cu(z), alpha, beta)
    torch.cuda.synchronize()
    return w


INSTANCES = lambda y, v, z: ((y, v, z, 1.0, 1.0), (y, None, None, 2.0, 0.0), (None, v, z, -1.0, 0.5),
                             (y, v, z, 0.5, -2.0))


@pytest.mark.parametrize("n,blocks", [(1000, 1), (1000, 2), (40_000, 2), (100_000, 4), (100_000, 8),
                                      (150_000, 8), (57_001, 4)])
@pytest.mark.parametrize("lengths", [("powerlaw", 2.5, 13.64), ("binomial", 0.01), ("uniform", 0, 1500)])
def test_packed_integer_twin_bitexact(cuda_dev, monkeypatch, n, blocks, lengths):
    m = 20_011 if lengths[0] != "uniform" else 2_003
    if lengths[0] == "binomial":
        lengths = ("binomial", min(0.01, 200.0 / n))
    if lengths[0] == "uniform":
        lengths = ("uniform", 0, min(1500, n))
    rp, ci, va, y, v, z = make(m, n, lengths, seed=n % 97 + blocks, kind="int_pm12")
    plan = packed_plan(cuda_dev, rp, ci, va, n, blocks, monkeypatch)
    info = plan.pack_info
    assert info["blocks"] == blocks and info["entries"] >= ci.numel()
    assert plan.launch.variant == 19 and plan.launch.cluster == blocks
    for args in INSTANCES(y, v, z):
        ref, mag = oracle.csr(m, n, rp, ci, va, *args)
        assert mag.max() < 2**24
        w = run(plan, cuda_dev, *args)
        assert_bitexact(w, ref, f"packed n={n} cs={blocks} {lengths} y={args[0] is not None}")


@pytest.mark.parametrize("blocks", [2, 4])
def test_packed_edge_shapes(cuda_dev, monkeypatch, blocks):
    """m = 1, m < 32, ragged m, empty rows (lengths from 0), one row longer than n/2, nnz = 0."""
    n = 50_000
    for m, lengths in ((1, ("uniform", 1, 40)), (5, ("uniform", 0, 3)), (33, ("uniform", 0, 9)),
                       (1000, ("uniform", 0, 2)), (7, ("uniform", 26_000, 40_000))):
        rp, ci, va, y, v, z = make(m, n, lengths, seed=m, kind="int_pm12")
        plan = packed_plan(cuda_dev, rp, ci, va, n, blocks, monkeypatch)
        for args in INSTANCES(y, v, z):
            ref, _ = oracle.csr(m, n, rp, ci, va, *args)
            w = run(plan, cuda_dev, *args)
            assert_bitexact(w, ref, f"packed edge m={m} {lengths} cs={blocks}")
    # nnz = 0: w = beta z
    m = 50
    rp = torch.zeros(m + 1, dtype=torch.int64)
    ci = torch.zeros(0, dtype=torch.int32)
    va = torch.zeros(0, dtype=torch.float32)
    y = torch.ones(n)
    z = torch.arange(n, dtype=torch.float32)
    plan = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), n, torch.float32)
    w = plan(va.to(cuda_dev), y.to(cuda_dev), None, z.to(cuda_dev), 1.0, 2.0)
    assert torch.equal(w.cpu(), 2 * z)


@pytest.mark.parametrize("blocks", [4, 8])
def test_packed_noncanonical_rows(cuda_dev, monkeypatch, blocks):
    """i.i.d. columns: unsorted rows with repeated columns (reading R7: duplicates summed)."""
    m, n = 10_000, 80_000
    rp, ci, va, y, v, z = make(m, n, ("powerlaw", 2.0, 20.0), seed=11, kind="int_pm12", col_skew=-1)
    plan = packed_plan(cuda_dev, rp, ci, va, n, blocks, monkeypatch)
    for args in INSTANCES(y, v, z):
        ref, _ = oracle.csr(m, n, rp, ci, va, *args)
        w = run(plan, cuda_dev, *args)
        assert_bitexact(w, ref, f"packed iid cs={blocks}")


def test_packed_int32_wrap_and_cap_spill(cuda_dev):
    """Every row holds column 0 and n-1 with the largest same-sign term: each CTA's int32 sum of
    those columns wraps many times (carried through the fp64 spill); a late row 64x larger than
    everything before it goes beyond the CTA's cap (spilled)."""
    m, n = 60_000, 90_000
    rp, ci, va = synth.csr(m, n, "f32", ("uniform", 2, 12), kind="int_pm12", seed=5)
    rp, ci, va = rp.clone(), ci.clone(), va.clone()
    ci[rp[:-1]] = 0
    ci[rp[1:] - 1] = n - 1
    va[rp[:-1]] = 2.0
    va[rp[1:] - 1] = 2.0
    va[rp[m - 7]:rp[m - 6]] *= 64.0
    y = torch.zeros(n, dtype=torch.float32)
    y[0] = 3.0
    y[n - 1] = 3.0
    v = torch.full((m,), 3.0)
    ref, _ = oracle.csr(m, n, rp, ci, va, y, v, None, 1.0, 0.0)
    assert abs(ref[0]) > 2**21
    plan = packed_plan(cuda_dev, rp, ci, va, n)
    w = run(plan, cuda_dev, y, v, None, 1.0, 0.0)
    assert_bitexact(w, ref, "packed wraps")


@pytest.mark.parametrize("n", [100_000, 30_000])
def test_packed_float_parity_deterministic(cuda_dev, n):
    m = 40_000
    rp, ci, va, y, v, z = make(m, n, ("powerlaw", 2.5, 13.64), seed=7, kind="uniform")
    plan = packed_plan(cuda_dev, rp, ci, va, n)
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    w = run(plan, cuda_dev, y, v, z, 1.0, 1.0)
    err = assert_parity(w, ref, mag, torch.float32, f"packed float n={n}")
    assert err < 2e-6, f"fixed-point error {err:.2e} well inside the tolerance expected"
    w2 = run(plan, cuda_dev, y, v, z, 1.0, 1.0)
    assert torch.equal(w, w2), "the packed sum must be order-independent (bit-identical reruns)"


def test_packed_dynamic_range(cuda_dev):
    """Rows scaled by 2^+-30 at random: terms far beyond the first round's cap (spill) and far
    below the quantum (rounded): the normwise bound still holds."""
    m, n = 30_000, 70_000
    rp, ci, va, y, v, z = make(m, n, ("powerlaw", 2.5, 13.64), seed=8, kind="uniform")
    g = torch.Generator().manual_seed(3)
    sc = torch.pow(2.0, torch.randint(-30, 31, (m,), generator=g).float())
    va = va * torch.repeat_interleave(sc, (rp[1:] - rp[:-1]))
    plan = packed_plan(cuda_dev, rp, ci, va, n)
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    w = run(plan, cuda_dev, y, v, z, 1.0, 1.0)
    assert_parity(w, ref, mag, torch.float32, "packed dynamic range")


def test_packed_nonfinite_propagates(cuda_dev):
    m, n = 5000, 80_000
    rp, ci, va, y, v, z = make(m, n, ("powerlaw", 2.5, 13.64), seed=9, kind="uniform")
    va = va.clone()
    va[100] = float("inf")
    va[2000] = float("nan")
    plan = packed_plan(cuda_dev, rp, ci, va, n)
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    w = run(plan, cuda_dev, y, v, z, 1.0, 1.0)
    assert_parity(w, ref, mag, torch.float32, "packed non-finite")


def test_packed_repack_unpacked_exec_alpha0(cuda_dev):
    """pack again with new values; exec with val on a packed plan runs the unpacked path; alpha
    = 0 writes beta z; exec without val on an unpacked plan and a forced 16-block pack are refused."""
    m, n = 8000, 100_000
    rp, ci, va, y, v, z = make(m, n, ("powerlaw", 2.5, 13.64), seed=4, kind="int_pm12")
    plan = packed_plan(cuda_dev, rp, ci, va, n)
    va2 = -2 * va
    plan.pack(va2.to(cuda_dev))
    ref, _ = oracle.csr(m, n, rp, ci, va2, y, v, z, 1.0, 1.0)
    assert_bitexact(run(plan, cuda_dev, y, v, z, 1.0, 1.0), ref, "repacked")
    ref1, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    w = plan(va.to(cuda_dev), y.to(cuda_dev), v.to(cuda_dev), z.to(cuda_dev), 1.0, 1.0)
    torch.cuda.synchronize()
    assert_bitexact(w, ref1, "packed plan, exec with val")
    w0 = run(plan, cuda_dev, y, v, z, 0.0, 3.0)
    assert torch.equal(w0.cpu(), 3 * z)
    plain = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), n, torch.float32)
    with pytest.raises(fp.FusedPatError):
        plain(None, y.to(cuda_dev), v.to(cuda_dev), z.to(cuda_dev), 1.0, 1.0)
    rp64, ci64, va64 = synth.csr(500, 60_000, "f64", ("uniform", 0, 20), seed=3)
    p64 = fp.CsrPlan(rp64.to(cuda_dev), ci64.to(cuda_dev), 60_000, torch.float64)
    with pytest.raises(fp.FusedPatError):  # more than 8 shared-memory blocks forced
        import os
        os.environ["FP_PK_CS"] = "16"
        try:
            p64.pack(va64.to(cuda_dev))
        finally:
            del os.environ["FP_PK_CS"]


def test_packed_graph_replay(cuda_dev):
    """A captured exec replayed many times (the exchange tag is a device counter advanced by the
    finalize, so replays never read a previous call's row partials)."""
    m, n = 20_000, 100_000
    rp, ci, va, y, v, z = make(m, n, ("powerlaw", 2.5, 13.64), seed=12, kind="int_pm12")
    plan = packed_plan(cuda_dev, rp, ci, va, n)
    ref, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    yd, vd, zd = y.to(cuda_dev), v.to(cuda_dev), z.to(cuda_dev)
    w = torch.empty(n, device=cuda_dev)
    s = torch.cuda.Stream(device=cuda_dev)
    s.wait_stream(torch.cuda.current_stream(cuda_dev))
    with torch.cuda.stream(s):
        plan(None, yd, vd, zd, 1.0, 1.0, w=w)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        plan(None, yd, vd, zd, 1.0, 1.0, w=w)
    for i in range(5):
        w.zero_()
        g.replay()
        torch.cuda.synchronize()
        assert_bitexact(w, ref, f"graph replay {i}")


# ------------------------------------------------------------------ the single-block pass (k_pk1), fp32 and fp64
@pytest.mark.parametrize("dt", ["f32", "f64"])
@pytest.mark.parametrize("lengths", [("binomial", 0.01), ("powerlaw", 2.5, 13.64), ("uniform", 0, 700)])
def test_packed1_integer_twin_bitexact(cuda_dev, dt, lengths):
    """One column block (small n, C3/S3 shapes): every tile loaded once, dot / q / scatter from the
    same registers; long rows (beyond the 256-entry window) streamed twice.  fp64: the 64-bit
    fixed point in two int32 limbs.  Integer twins bit-exact, every instance."""
    m, n = (20_011, 1000) if lengths[0] != "uniform" else (4_001, 1000)
    tdt = torch.float64 if dt == "f64" else torch.float32
    rp, ci, va = synth.csr(m, n, dt, lengths, kind="int_pm12", seed=21)
    y = synth.vector(n, dt, kind="int_small", seed=21, stream=synth.S_Y)
    v = synth.vector(m, dt, kind="int_pos", seed=21, stream=synth.S_V)
    z = synth.vector(n, dt, kind="int_small", seed=21, stream=synth.S_Z)
    plan = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), n, tdt)
    plan.pack(va.to(cuda_dev))
    assert plan.launch.variant == 19 and plan.launch.cluster == 1
    for args in INSTANCES(y, v, z):
        ref, mag = oracle.csr(m, n, rp, ci, va, *args)
        assert mag.max() < 2**24
        w = run(plan, cuda_dev, *args)
        assert_bitexact(w, ref, f"packed1 {dt} {lengths} y={args[0] is not None}")


@pytest.mark.parametrize("dt", ["f32", "f64"])
def test_packed1_float_parity(cuda_dev, dt):
    """U[-1,1) data (C3 rows) plus rows scaled by 2^+-30: the north_star tolerance (1e-11 fp64,
    2e-5 fp32); reruns bit-identical."""
    m, n = 30_000, 1000
    tdt = torch.float64 if dt == "f64" else torch.float32
    rp, ci, va = synth.csr(m, n, dt, ("binomial", 0.01), seed=8)
    y = synth.vector(n, dt, seed=8, stream=synth.S_Y)
    v = synth.vector(m, dt, kind="pos", seed=8, stream=synth.S_V)
    z = synth.vector(n, dt, seed=8, stream=synth.S_Z)
    plan = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), n, tdt)
    plan.pack(va.to(cuda_dev))
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    w = run(plan, cuda_dev, y, v, z, 1.0, 1.0)
    assert_parity(w, ref, mag, tdt, f"packed1 {dt}")
    assert torch.equal(w, run(plan, cuda_dev, y, v, z, 1.0, 1.0))
    g = torch.Generator().manual_seed(5)
    sc = torch.pow(2.0, torch.randint(-30, 31, (m,), generator=g).to(tdt))
    va2 = va * torch.repeat_interleave(sc, (rp[1:] - rp[:-1]))
    plan.pack(va2.to(cuda_dev))
    ref, mag = oracle.csr(m, n, rp, ci, va2, y, v, z, 1.0, 1.0)
    assert_parity(run(plan, cuda_dev, y, v, z, 1.0, 1.0), ref, mag, tdt, f"packed1 {dt} dynamic range")


def test_packed1_nonfinite_and_wide_fp64(cuda_dev):
    """Inf / NaN propagate (reading R8); an fp64 matrix too wide for one block packs into L2 blocks."""
    m, n = 3000, 800
    rp, ci, va = synth.csr(m, n, "f64", ("binomial", 0.02), seed=9)
    y = synth.vector(n, "f64", seed=9, stream=synth.S_Y)
    va = va.clone()
    va[50] = float("inf")
    va[700] = float("nan")
    plan = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), n, torch.float64)
    plan.pack(va.to(cuda_dev))
    ref, mag = oracle.csr(m, n, rp, ci, va, y, None, None, 1.0, 0.0)
    assert_parity(run(plan, cuda_dev, y, None, None, 1.0, 0.0), ref, mag, torch.float64, "packed1 non-finite")
    rp, ci, va = synth.csr(200, 40_000, "f64", ("uniform", 0, 20), seed=3)
    p64 = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), 40_000, torch.float64)
    p64.pack(va.to(cuda_dev))  # too wide for one shared-memory block: variant 20's L2 blocks
    assert p64.launch.variant == 20


# ------------------------------------------------------------------ variant 20: L2-sized column blocks
def l2_plan(dev, monkeypatch, rp, ci, va, n, bw, tdt):
    monkeypatch.setenv("FP_PK_L2", "1")
    monkeypatch.setenv("FP_L2B_BW", str(bw))
    plan = fp.CsrPlan(rp.to(dev), ci.to(dev), n, tdt)
    plan.pack(va.to(dev))
    torch.cuda.synchronize()
    monkeypatch.delenv("FP_PK_L2")
    monkeypatch.delenv("FP_L2B_BW")
    assert plan.launch.variant == 20
    return plan


@pytest.mark.parametrize("dt", ["f32", "f64"])
@pytest.mark.parametrize("n,bw", [(5000, 1000), (20_000, 3001), (4096, 4096)])
@pytest.mark.parametrize("lengths,skew", [(("powerlaw", 2.5, 13.64), 0), (("binomial", 0.004), 0),
                                          (("uniform", 0, 1500), 0), (("powerlaw", 2.5, 9.5), 2)])
@pytest.mark.parametrize("hot", [None, "40"])
def test_l2block_integer_twin_bitexact(cuda_dev, monkeypatch, dt, n, bw, lengths, skew, hot):
    """Variant 20 (csr_l2block.cu): the columns in blocks of bw (here small, so that a test-sized
    matrix spans several blocks, a ragged last block, one block), row dots accumulated over the
    blocks, the heaviest block fused (q and its scatter from the same registers), the others
    re-read; rows longer than a 256-entry chunk split into partial chunks; empty rows; Zipf-like
    columns (skew); hot columns (more than `hot` nonzeros: scattered by column).  Integer twins:
    every sum exact in fp64 / below 2^24 in fp32, so bit-exact whatever the red order."""
    m = 6_007 if lengths[0] != "uniform" else 1_501
    tdt = torch.float64 if dt == "f64" else torch.float32
    if hot is not None:
        monkeypatch.setenv("FP_L2B_HOT", hot)
    rp, ci, va = synth.csr(m, n, dt, lengths, kind="int_pm12", seed=31, col_skew=skew)
    y = synth.vector(n, dt, kind="int_small", seed=31, stream=synth.S_Y)
    v = synth.vector(m, dt, kind="int_pos", seed=31, stream=synth.S_V)
    z = synth.vector(n, dt, kind="int_small", seed=31, stream=synth.S_Z)
    plan = l2_plan(cuda_dev, monkeypatch, rp, ci, va, n, bw, tdt)
    assert plan.launch.cluster == (n + bw - 1) // bw
    for args in INSTANCES(y, v, z):
        ref, mag = oracle.csr(m, n, rp, ci, va, *args)
        if dt == "f32" and mag.max() >= 2**24:
            continue
        w = run(plan, cuda_dev, *args)
        assert_bitexact(w, ref, f"l2block {dt} n={n} bw={bw} {lengths} y={args[0] is not None}")


@pytest.mark.parametrize("dt", ["f32", "f64"])
def test_l2block_float_parity_skewed(cuda_dev, monkeypatch, dt):
    """U[-1,1) data on KDD-shaped rows (power-law lengths, Zipf-like columns: most nonzeros in
    the first block, which then runs fused), the north_star tolerance (1e-11 fp64, 2e-5 fp32);
    rows scaled by 2^+-30."""
    m, n = 40_000, 200_000
    tdt = torch.float64 if dt == "f64" else torch.float32
    rp, ci, va = synth.csr(m, n, dt, ("powerlaw", 2.5, 9.5), seed=12, col_skew=2)
    y = synth.vector(n, dt, seed=12, stream=synth.S_Y)
    v = synth.vector(m, dt, kind="pos", seed=12, stream=synth.S_V)
    z = synth.vector(n, dt, seed=12, stream=synth.S_Z)
    plan = l2_plan(cuda_dev, monkeypatch, rp, ci, va, n, 25_000, tdt)
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    assert_parity(run(plan, cuda_dev, y, v, z, 1.0, 1.0), ref, mag, tdt, f"l2block {dt}")
    g = torch.Generator().manual_seed(6)
    sc = torch.pow(2.0, torch.randint(-30, 31, (m,), generator=g).to(tdt))
    va2 = va * torch.repeat_interleave(sc, (rp[1:] - rp[:-1]))
    plan.pack(va2.to(cuda_dev))  # re-pack unforced: fp32 -> shared-memory blocks, fp64 -> one L2 block
    ref, mag = oracle.csr(m, n, rp, ci, va2, y, v, z, 1.0, 1.0)
    assert_parity(run(plan, cuda_dev, y, v, z, 1.0, 1.0), ref, mag, tdt, f"l2block {dt} dynamic range")


def test_l2block_chosen_for_wide_fp64_and_nonfinite(cuda_dev):
    """fp64 wider than one shared-memory block packs into L2 blocks without forcing (the
    round-2 refusal is gone); Inf / NaN propagate (reading R8)."""
    m, n = 3000, 40_000
    rp, ci, va = synth.csr(m, n, "f64", ("uniform", 0, 60), seed=3)
    va = va.clone()
    va[10] = float("inf")
    va[4000] = float("nan")
    y = synth.vector(n, "f64", seed=3, stream=synth.S_Y)
    plan = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), n, torch.float64)
    plan.pack(va.to(cuda_dev))
    assert plan.launch.variant == 20 and plan.launch.cluster == 1
    ref, mag = oracle.csr(m, n, rp, ci, va, y, None, None, 1.0, 0.0)
    assert_parity(run(plan, cuda_dev, y, None, None, 1.0, 0.0), ref, mag, torch.float64, "l2block non-finite")


def test_l2block_graph_replay(cuda_dev, monkeypatch):
    """The L2-block launches captured in a CUDA graph and replayed: same result each replay."""
    m, n = 5000, 9000
    rp, ci, va = synth.csr(m, n, "f64", ("powerlaw", 2.5, 13.64), kind="int_pm12", seed=4)
    y = synth.vector(n, "f64", kind="int_small", seed=4, stream=synth.S_Y)
    v = synth.vector(m, "f64", kind="int_pos", seed=4, stream=synth.S_V)
    z = synth.vector(n, "f64", kind="int_small", seed=4, stream=synth.S_Z)
    plan = l2_plan(cuda_dev, monkeypatch, rp, ci, va, n, 2000, torch.float64)
    ref, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    yd, vd, zd = y.to(cuda_dev), v.to(cuda_dev), z.to(cuda_dev)
    w = torch.empty(n, dtype=torch.float64, device=cuda_dev)
    s = torch.cuda.Stream(device=cuda_dev)
    with torch.cuda.stream(s):
        plan(None, yd, vd, zd, 1.0, 1.0, w=w)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        plan(None, yd, vd, zd, 1.0, 1.0, w=w)
    for i in range(3):
        w.zero_()
        g.replay()
        torch.cuda.synchronize()
        assert_bitexact(w, ref, f"l2block graph replay {i}")


def test_pack_detail_counts(cuda_dev, monkeypatch):
    """fp_csr_plan_pack_detail reports what an exec does: variant 20's hot columns and their
    nonzeros equal a host count of the columns above the threshold; the entries streamed count
    the fused block once and the others twice; variant 19 streams its copy once in 2 launches."""
    m, n, thr = 6000, 30_000, 120
    rp, ci, va = synth.csr(m, n, "f64", ("powerlaw", 2.5, 9.5), seed=17, col_skew=2)
    monkeypatch.setenv("FP_L2B_HOT", str(thr))
    plan = l2_plan(cuda_dev, monkeypatch, rp, ci, va, n, 7000, torch.float64)
    d, info = plan.pack_detail, plan.pack_info
    counts = np.bincount(ci.numpy(), minlength=n)
    assert d["variant"] == 20 and d["blocks"] == info["blocks"] == 5
    assert d["hot_columns"] == int((counts > thr).sum()) > 0
    assert d["hot_entries"] == int(counts[counts > thr].sum())
    per_block = np.bincount(ci.numpy() // 7000, minlength=5)
    assert d["fused_block"] == int(np.argmax(per_block))
    assert info["entries"] < d["entries_streamed"] <= 2 * info["entries"] + d["hot_entries"]
    assert d["launches"] == 2 * (5 - 1) + 5  # init, 4 dots, fused, q, 4 scatters, partial, hot
    rp, ci, va = synth.csr(m, 1000, "f32", ("binomial", 0.01), seed=17)
    p19 = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), 1000, torch.float32)
    p19.pack(va.to(cuda_dev))
    d = p19.pack_detail
    assert d["variant"] == 19 and d["entries_streamed"] == p19.pack_info["entries"] and d["launches"] == 2


@pytest.mark.parametrize("dt", ["f32", "f64"])
def test_packed1_unaligned_v_and_w_alias_z(cuda_dev, dt):
    """k_pk1 takes v with its tile copy only when v is 16-byte aligned: a v that starts one
    element into its buffer runs the global-load path, same bits; w may alias z (in place)."""
    m, n = 7_001, 1000
    tdt = torch.float64 if dt == "f64" else torch.float32
    rp, ci, va = synth.csr(m, n, dt, ("binomial", 0.01), kind="int_pm12", seed=23)
    y = synth.vector(n, dt, kind="int_small", seed=23, stream=synth.S_Y)
    v = synth.vector(m, dt, kind="int_pos", seed=23, stream=synth.S_V)
    z = synth.vector(n, dt, kind="int_small", seed=23, stream=synth.S_Z)
    plan = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), n, tdt)
    plan.pack(va.to(cuda_dev))
    ref, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 2.0)
    vbuf = torch.zeros(m + 1, dtype=tdt, device=cuda_dev)
    vbuf[1:] = v.to(cuda_dev)
    vu = vbuf[1:]
    assert vu.data_ptr() % 16 != 0
    w = plan(None, y.to(cuda_dev), vu, z.to(cuda_dev), 1.0, 2.0)
    torch.cuda.synchronize()
    assert_bitexact(w, ref, f"packed1 {dt} unaligned v")
    zw = z.to(cuda_dev).clone()
    plan(None, y.to(cuda_dev), v.to(cuda_dev), zw, 1.0, 2.0, w=zw)
    torch.cuda.synchronize()
    assert_bitexact(zw, ref, f"packed1 {dt} w aliases z")


@pytest.mark.parametrize("dt,n,ns", [("f64", 1000, "0"), ("f64", 1000, "1"), ("f64", 1000, "2"), ("f32", 1000, "2"),
                                     ("f64", 12_000, None), ("f32", 23_000, None)])
def test_packed1_ring_depths_and_widest_block(cuda_dev, monkeypatch, dt, n, ns):
    """k_pk1 with every ring depth (0: windows from global memory, fp64 too) and at the widest
    single block (the ring no longer fits next to y and the partial w): integer twins bit-exact,
    long rows included."""
    m = 3_001
    tdt = torch.float64 if dt == "f64" else torch.float32
    rp, ci, va = synth.csr(m, n, dt, ("uniform", 0, 400), kind="int_pm12", seed=29)
    y = synth.vector(n, dt, kind="int_small", seed=29, stream=synth.S_Y)
    v = synth.vector(m, dt, kind="int_pos", seed=29, stream=synth.S_V)
    z = synth.vector(n, dt, kind="int_small", seed=29, stream=synth.S_Z)
    if ns is not None:
        monkeypatch.setenv("FP_PK1_NS", ns)
    plan = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), n, tdt)
    plan.pack(va.to(cuda_dev))
    assert plan.launch.variant == 19 and plan.launch.cluster == 1
    for args in ((y, v, z, 1.0, 1.0), (None, v, z, -1.0, 0.5)):
        ref, mag = oracle.csr(m, n, rp, ci, va, *args)
        if dt == "f32" and mag.max() >= 2**24:
            continue
        assert_bitexact(run(plan, cuda_dev, *args), ref, f"packed1 {dt} n={n} ns={ns}")
