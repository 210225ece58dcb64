"""GPU parity of variant 17 (FP_VAR_CSR_BINNED, csr_binned.cu) against the fp64 oracle.

The large-n CSR path of SURVEY 8 rows a7/a10: the scatter of Eq. (3) (Alg. 2 l.13-14, P:220-
221) goes through column-block bins and a shared-memory fixed-point reduction instead of
per-nonzero global atomics.  Checked here, at sizes the oracle finishes in seconds:
* integer twins bit-exact for 1 and 2 column blocks, every instance (with/without y, v, beta*z),
  forced producer grids, rows longer than the 256-nonzero batch (warp-per-row path);
* the int32 wrap carried into hi[] (columns hit by thousands of same-sign maximal terms);
* U[-1,1) fp32 data within the north_star 2e-5 normwise tolerance;
* IEEE propagation of Inf/NaN terms (reading R8) through the spill vector;
* determinism: the fixed-point sum is order-independent, so repeated calls are bit-identical;
* the chooser picks it for the C4 shape.
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_asharitbrcks15_b200 as fp
import synth
from _util import assert_bitexact, assert_parity

pytestmark = pytest.mark.gpu


def make(m, n, lengths, seed, kind):
    rp, ci, va = synth.csr(m, n, "f32", lengths, kind=kind, seed=seed)
    integer = kind.startswith("int")
    y = synth.vector(n, "f32", kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Y)
    v = synth.vector(m, "f32", kind="int_pos" if integer else "pos", seed=seed, stream=synth.S_V)
    z = synth.vector(n, "f32", kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Z)
    return rp, ci, va, y, v, z


def launch(nbin, grid=0):
    L = fp.fp_launch()
    L.variant, L.vs, L.tl, L.bs, L.grid, L.cluster = 17, 32, 8, 1024, grid, nbin
    return L


def run(dev, rp, ci, va, n, y, v, z, alpha, beta, L):
    cu = lambda t: None if t is None else t.to(dev)
    w = fp.csr(cu(rp), cu(ci), cu(va), n, cu(y), cu(v), cu(z), alpha, beta, launch=L)
    torch.cuda.synchronize()
    return w


@pytest.mark.parametrize("n,nbin", [(1000, 1), (40_000, 1), (40_000, 2), (100_000, 2), (113_000, 2)])
@pytest.mark.parametrize("lengths", [("powerlaw", 2.5, 13.64), ("binomial", 0.01), ("uniform", 0, 600)])
def test_binned_integer_twin_bitexact(cuda_dev, n, nbin, lengths):
    m = 30_000 if lengths[0] != "binomial" else 8_000
    if lengths[0] == "binomial":
        lengths = ("binomial", min(0.01, 200.0 / n))
    if lengths[0] == "uniform" and n < 10_000:
        m = 3_000  # keep every column sum below 2^24 (fp32 integer twin exact in any order)
    rp, ci, va, y, v, z = make(m, n, lengths, seed=n % 101 + nbin, kind="int_pm12")
    for args in ((y, v, z, 1.0, 1.0), (y, None, None, 2.0, 0.0), (None, v, z, -1.0, 0.5), (y, v, z, 0.5, -2.0)):
        ref, mag = oracle.csr(m, n, rp, ci, va, *args)
        assert mag.max() < 2**24
        w = run(cuda_dev, rp, ci, va, n, *args, launch(nbin))
        assert_bitexact(w, ref, f"binned n={n} nbin={nbin} {lengths} y={args[0] is not None}")


@pytest.mark.parametrize("grid", [1, 7, 148, 300])
def test_binned_forced_grids_bitexact(cuda_dev, grid):
    m, n = 20_011, 70_000
    rp, ci, va, y, v, z = make(m, n, ("powerlaw", 2.0, 3.0), seed=grid, kind="int_pm12")
    ref, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    w = run(cuda_dev, rp, ci, va, n, y, v, z, 1.0, 1.0, launch(2, grid))
    assert_bitexact(w, ref, f"binned grid={grid}")


def test_binned_int32_wrap_carries(cuda_dev):
    """Every row holds column 0 (and n-1) with the same sign and the largest |term|: each
    consumer's int32 accumulator for those columns wraps many times (hi[] carries)."""
    m, n = 60_000, 90_000
    rp, ci, va = synth.csr(m, n, "f32", ("uniform", 2, 12), kind="int_pm12", seed=5)
    rp, ci, va = rp.clone(), ci.clone(), va.clone()
    starts, ends = rp[:-1], rp[1:] - 1
    ci[starts] = 0
    ci[ends] = n - 1
    va[starts] = 2.0
    va[ends] = 2.0
    # keep rows canonical (sorted): first entry 0, last n-1, middle entries strictly inside
    y = torch.zeros(n, dtype=torch.float32)
    y[0] = 3.0
    y[n - 1] = 3.0
    v = torch.full((m,), 3.0)
    ref, _ = oracle.csr(m, n, rp, ci, va, y, v, None, 1.0, 0.0)
    assert abs(ref[0]) > 2**21  # ~800 maximal terms per consumer: the int32 sum wraps ~10 times
    w = run(cuda_dev, rp, ci, va, n, y, v, None, 1.0, 0.0, launch(2))
    assert_bitexact(w, ref, "binned wraps")


@pytest.mark.parametrize("n,nbin", [(100_000, 2), (60_000, 2), (30_000, 1)])
def test_binned_float_parity(cuda_dev, n, nbin):
    m = 40_000
    rp, ci, va, y, v, z = make(m, n, ("powerlaw", 2.5, 13.64), seed=7, kind="uniform")
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    w = run(cuda_dev, rp, ci, va, n, y, v, z, 1.0, 1.0, launch(nbin))
    assert_parity(w, ref, mag, torch.float32, f"binned float n={n}")
    w2 = run(cuda_dev, rp, ci, va, n, y, v, z, 1.0, 1.0, launch(nbin))
    assert torch.equal(w, w2), "fixed-point reduction must be order-independent (bit-identical reruns)"


def test_binned_nonfinite_propagates(cuda_dev):
    m, n = 5000, 80_000
    rp, ci, va, y, v, z = make(m, n, ("powerlaw", 2.5, 13.64), seed=9, kind="uniform")
    va = va.clone()
    va[100] = float("inf")
    va[2000] = float("nan")
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    w = run(cuda_dev, rp, ci, va, n, y, v, z, 1.0, 1.0, launch(2))
    assert_parity(w, ref, mag, torch.float32, "binned non-finite")


def test_binned_refuses_what_it_cannot_do(cuda_dev):
    """fp64, a row epilogue, or n beyond two blocks of one SM's shared memory: FP_ERR_UNSUPPORTED
    through an explicit plan (the chooser never picks variant 17 there)."""
    m, n = 2000, 150_000
    rp, ci, va, y, v, z = make(m, n, ("uniform", 0, 20), seed=3, kind="uniform")
    with pytest.raises(fp.FusedPatError):
        run(cuda_dev, rp, ci, va, n, y, v, z, 1.0, 1.0, launch(2))
    rp, ci, va = synth.csr(m, 5000, "f64", ("uniform", 0, 20), seed=3)
    y = synth.vector(5000, "f64", seed=3)
    with pytest.raises(fp.FusedPatError):
        run(cuda_dev, rp, ci, va, 5000, y, None, None, 1.0, 0.0, launch(1))


def test_binned_chosen_for_c4_shape(cuda_dev):
    st = fp.fp_row_stats()
    st.m, st.n, st.nnz = 50_000_000, 100_000, 2_000_000_000
    st.mean = 40.0
    L = fp.choose(True, st, fp.FP_F32, 0)
    assert (L.variant, L.cluster, L.bs, L.tl) == (17, 2, 1024, 8)


# ------------------------------------------------------------------ variant 18 (flat-4, fixed-point CTA partial)
DT = {"f64": torch.float64, "f32": torch.float32}


def launch18(grid=0, variant=18):
    L = fp.fp_launch()
    L.variant, L.vs, L.tl, L.bs, L.grid = variant, 32, 8, 256, grid
    return L


def make_dt(m, n, dt, lengths, seed, kind):
    rp, ci, va = synth.csr(m, n, dt, lengths, kind=kind, seed=seed)
    integer = kind.startswith("int")
    y = synth.vector(n, dt, kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Y)
    v = synth.vector(m, dt, kind="int_pos" if integer else "pos", seed=seed, stream=synth.S_V)
    z = synth.vector(n, dt, kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Z)
    return rp, ci, va, y, v, z


@pytest.mark.parametrize("variant", [18])
@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("lengths", [("binomial", 0.01), ("powerlaw", 2.0, 3.0), ("uniform", 0, 600), ("uniform", 0, 3)])
@pytest.mark.parametrize("grid", [0, 1, 37])
def test_flat4_fixed_bitexact(cuda_dev, variant, dt, lengths, grid):
    """Variant 18 on integer twins: bit-exact for every instance, short rows (flat batches of 4
    nonzeros per lane), rows beyond 128 (warp-per-row steps), empty rows, forced grids."""
    m, n = (20_000, 1000) if lengths[0] != "uniform" or lengths[2] < 100 else (3_000, 1000)
    rp, ci, va, y, v, z = make_dt(m, n, dt, lengths, seed=grid + 3, kind="int_pm12")
    for args in ((y, v, z, 1.0, 1.0), (None, v, None, -1.0, 0.0), (y, None, z, 2.0, -0.5)):
        ref, mag = oracle.csr(m, n, rp, ci, va, *args)
        assert mag.max() < (2**24 if dt == "f32" else 2**53)
        w = run(cuda_dev, rp, ci, va, n, *args, launch18(grid, variant))
        assert_bitexact(w, ref, f"variant {variant} {dt} {lengths} grid={grid} y={args[0] is not None}")


@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_flat4_fixed_misaligned_slices(cuda_dev, dt):
    """colidx / val starting 1..3 entries past a 16-byte boundary (row-shard slices): the 4-entry
    groups follow the common misalignment."""
    m, n = 5000, 800
    rp, ci, va, y, v, z = make_dt(m, n, dt, ("binomial", 0.02), seed=5, kind="int_pm12")
    ref, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    for off in (1, 2, 3):
        cib = torch.zeros(ci.numel() + 4, dtype=torch.int32)
        vab = torch.zeros(va.numel() + 4, dtype=va.dtype)
        cib[off:off + ci.numel()] = ci
        vab[off:off + va.numel()] = va
        cid, vad = cib.to(cuda_dev), vab.to(cuda_dev)
        w = fp.csr(rp.to(cuda_dev), cid[off:off + ci.numel()], vad[off:off + va.numel()], n, y.to(cuda_dev),
                   v.to(cuda_dev), z.to(cuda_dev), 1.0, 1.0, launch=launch18())
        torch.cuda.synchronize()
        assert_bitexact(w, ref, f"flat4 misaligned by {off}")


@pytest.mark.parametrize("variant", [18])
@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_flat4_fixed_float_parity(cuda_dev, variant, dt):
    """U[-1,1) data, C3-shaped rows, plus rows scaled by 2^+-30 (terms far beyond / below the
    CTA's cap exponent take the fp64 spill / round to the fixed grid): north_star tolerance."""
    m, n = 30_000, 1000
    rp, ci, va, y, v, z = make_dt(m, n, dt, ("binomial", 0.01), seed=8, kind="uniform")
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    w = run(cuda_dev, rp, ci, va, n, y, v, z, 1.0, 1.0, launch18(0, variant))
    assert_parity(w, ref, mag, DT[dt], "flat4 fixed float")
    scale = torch.ones(m, dtype=va.dtype)
    scale[::97] = 2.0**30
    scale[1::89] = 2.0**-30
    rows = torch.repeat_interleave(torch.arange(m), rp[1:] - rp[:-1])
    va2 = va * scale[rows]
    ref, mag = oracle.csr(m, n, rp, ci, va2, y, v, z, 1.0, 1.0)
    w = run(cuda_dev, rp, ci, va2, n, y, v, z, 1.0, 1.0, launch18(0, variant))
    assert_parity(w, ref, mag, DT[dt], "flat4 fixed wide range")


def test_binned_host_streaming_accumulates_chunks(cuda_dev):
    """fp_csr_host (P:151 streaming) on a matrix of ~3 chunks of 512 MB: every chunk runs the
    binned plan (variant 17, > 16M nonzeros) with accumulate = 1 after the first (the finalize
    adds into w); integer twin bit-exact against the oracle over the whole matrix."""
    m, n = 4_000_000, 100_000
    rp, ci, va = synth.csr(m, n, "f32", ("powerlaw", 2.5, 13.64), kind="int_pm12", seed=41)
    assert int(rp[-1]) > 2 * (512 << 20) // 8  # at least three chunks
    y = synth.vector(n, "f32", kind="int_small", seed=41, stream=synth.S_Y)
    v = synth.vector(m, "f32", kind="int_pos", seed=41, stream=synth.S_V)
    z = synth.vector(n, "f32", kind="int_small", seed=41, stream=synth.S_Z)
    # v = 1, beta = 0 keep every partial sum below 2^24 (fp32 twin exact in any order, also
    # across the chunk boundaries where the finalize adds into the fp32 w)
    ref, mag = oracle.csr(m, n, rp, ci, va, y, None, None, 1.0, 0.0)
    assert mag.max() < 2**24
    w = fp.csr_host(rp, ci, va, n, y, None, None, 1.0, 0.0)
    assert_bitexact(w, ref, "binned host streaming")
