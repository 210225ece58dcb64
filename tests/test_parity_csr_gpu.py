"""GPU parity of fp_csr (through the C ABI) against the fp64 oracle.

Row-length mixes of the paper's workloads (uniform Binomial rows at density 0.01, P:411;
power-law KDD-like skew) at sizes the oracle finishes in seconds, both the shared-
memory (small n) and L2 (large n) variants, every VS of Eq. (4) forced
through fp_csr_ex, rows longer than the register cache (tail re-read path), empty rows,
duplicates/unsorted columns (reading R7), integer twins bit-exact, dense-vs-CSR agreement,
device-side structure validation and row statistics."""
import numpy as np
import pytest
import scipy.sparse as sp
import torch

import oracle
import paper_conf_ppopp_asharitbrcks15_b200 as fp
import synth
from _util import TOL, assert_bitexact, assert_parity, skip_unbuilt

pytestmark = pytest.mark.gpu

DT = {"f64": torch.float64, "f32": torch.float32}


def make_csr(m, n, dt, lengths, seed, kind="uniform"):
    rp, ci, va = synth.csr(m, n, dt, lengths, kind=kind, seed=seed)
    integer = kind.startswith("int")
    y = synth.vector(n, dt, kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Y)
    v = synth.vector(m, dt, kind="int_pos" if integer else "pos", seed=seed, stream=synth.S_V)
    z = synth.vector(n, dt, kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Z)
    return rp, ci, va, y, v, z


def gpu_csr(dev, rp, ci, va, n, y, v, z, alpha, beta, launch=None):
    cu = lambda t: None if t is None else t.to(dev)
    w = fp.csr(cu(rp), cu(ci), cu(va), n, cu(y), cu(v), cu(z), alpha, beta, launch=launch)
    torch.cuda.synchronize()
    return w


CASES = [
    # m, n, lengths
    (20000, 1000, ("binomial", 0.01)),          # C3 shape, scaled down (smem path)
    (5000, 300, ("binomial", 0.05)),
    (3000, 100, ("uniform", 0, 3)),             # very short rows, many empty
    (20000, 100000, ("powerlaw", 2.5, 13.64)),  # C4 shape, scaled down (L2 path)
    (4000, 4000, ("powerlaw", 2.0, 5.0)),       # heavy rows up to n (tail re-read)
    (2000, 700, ("uniform", 30, 200)),          # rows longer than VS*K
    (1, 50, ("fixed", 50)),
]


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("m,n,lengths", CASES)
@pytest.mark.parametrize("inst", ["full", "xty", "xtxy", "xtxy_bz"])
def test_csr_instances(cuda_dev, dt, m, n, lengths, inst):
    rp, ci, va, y, v, z = make_csr(m, n, dt, lengths, seed=m + n)
    I = {"full": (y, v, z, 0.75, -1.25), "xty": (None, v, None, -2.0, 0.0), "xtxy": (y, None, None, 1.0, 0.0),
         "xtxy_bz": (y, None, z, 1.0, 0.5)}[inst]
    ref, mag = oracle.csr(m, n, rp, ci, va, *I)
    w = gpu_csr(cuda_dev, rp, ci, va, n, *I)
    assert_parity(w, ref, mag, DT[dt], f"{dt} {m}x{n} {lengths} {inst}")


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("variant", [3, 4, 5, 11])
@pytest.mark.parametrize("vs", [1, 2, 4, 8, 16, 32])
def test_csr_every_vs_and_variant_bitexact(cuda_dev, dt, variant, vs):
    """fp_csr_ex with every VS of Eq. (4) and both aggregation variants: integer twins
    must equal the oracle bit for bit (structure handling is exact)."""
    m, n = 3000, 500
    rp, ci, va, y, v, z = make_csr(m, n, dt, ("uniform", 0, 70), seed=vs, kind="int_pm12")
    ref, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    L = fp.fp_launch()
    L.variant, L.vs, L.bs, L.grid = variant, vs, 256, 37
    w = gpu_csr(cuda_dev, rp, ci, va, n, y, v, z, 1.0, 1.0, launch=L)
    assert_bitexact(w, ref, f"vs={vs} variant={variant}")


@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_csr_integer_twin_powerlaw_bitexact(cuda_dev, dt):
    m, n = 30000, 2000
    rp, ci, va, y, v, z = make_csr(m, n, dt, ("powerlaw", 2.5, 13.64), seed=77, kind="int_pm12")
    A = sp.csr_matrix((va.double().numpy(), ci.numpy(), rp.numpy()), shape=(m, n))
    bound = float((abs(A).T @ (v.double().numpy() * (abs(A) @ np.abs(y.double().numpy())))).max())
    if dt == "f32" and bound >= 2**24:
        pytest.skip("fp32 twin beyond the exactness bound")
    ref, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 2.0, -1.0)
    w = gpu_csr(cuda_dev, rp, ci, va, n, y, v, z, 2.0, -1.0)
    assert_bitexact(w, ref, "powerlaw twin")


def test_dense_vs_csr_bitexact(cuda_dev):
    """The same integer matrix through fp_dense and fp_csr gives identical w."""
    m, n = 4000, 96
    rp, ci, va, y, v, z = make_csr(m, n, "f64", ("binomial", 0.3), seed=5, kind="int_pm12")
    D = torch.zeros((m, n), dtype=torch.float64)
    rows = torch.repeat_interleave(torch.arange(m), rp[1:] - rp[:-1])
    D[rows, ci.long()] = va
    wc = gpu_csr(cuda_dev, rp, ci, va, n, y, v, z, 1.0, 1.0)
    wd = fp.dense(D.to(cuda_dev), y.to(cuda_dev), v.to(cuda_dev), z.to(cuda_dev), 1.0, 1.0)
    assert torch.equal(wc.cpu(), wd.cpu())


def test_duplicates_and_unsorted_columns(cuda_dev):
    """Reading R7: non-canonical CSR, duplicates summed (== scipy sum_duplicates())."""
    rng = np.random.default_rng(3)
    m, n = 500, 64
    lens = rng.integers(0, 40, m)
    rp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    ci = rng.integers(0, n, rp[-1]).astype(np.int32)               # unsorted, with duplicates
    va = rng.integers(-2, 3, rp[-1]).astype(np.float64)
    y, v, z = rng.integers(-3, 4, n).astype(np.float64), rng.integers(1, 4, m).astype(np.float64), np.ones(n)
    A = sp.csr_matrix((va.copy(), ci.copy(), rp.copy()), shape=(m, n))  # scipy dedups in place
    A.sum_duplicates()
    ref = A.T @ (v * (A @ y)) + z
    w = gpu_csr(cuda_dev, torch.from_numpy(rp), torch.from_numpy(ci), torch.from_numpy(va), n, torch.from_numpy(y),
                torch.from_numpy(v), torch.from_numpy(z), 1.0, 1.0)
    assert_bitexact(w, ref, "duplicates")


@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_csr_edge_cases(cuda_dev, dt):
    tdt = DT[dt]
    n = 40
    z = synth.vector(n, dt, seed=2).to(cuda_dev)
    rp0 = torch.zeros(1, dtype=torch.int64, device=cuda_dev)      # m == 0
    e_i = torch.zeros(0, dtype=torch.int32, device=cuda_dev)
    e_v = torch.zeros(0, dtype=tdt, device=cuda_dev)
    w = fp.csr(rp0, e_i, e_v, n, None, None, z, 1.0, 3.0)
    assert torch.equal(w, (3.0 * z.double()).to(tdt))
    rpz = torch.zeros(11, dtype=torch.int64, device=cuda_dev)     # nnz == 0, all rows empty
    w = fp.csr(rpz, e_i, e_v, n, torch.ones(n, dtype=tdt, device=cuda_dev), torch.ones(10, dtype=tdt,
               device=cuda_dev), z, 1.0, 1.0)
    assert torch.equal(w, z)
    # Inf in y on a column no stored entry touches must not leak through padded lanes
    rp, ci, va, y, v, _ = make_csr(2000, n, dt, ("uniform", 0, 5), seed=1)
    used = set(ci.tolist())
    free = [j for j in range(n) if j not in used]
    if free:
        y[free[0]] = float("inf")
        y[0] = y[0] if 0 in used else float("inf")
        ref, mag = oracle.csr(2000, n, rp, ci, va, y, v, None, 1.0, 0.0)
        w = gpu_csr(cuda_dev, rp, ci, va, n, y, v, None, 1.0, 0.0)
        assert_parity(w, ref, mag, tdt, "inf in untouched y")


def test_validate_and_row_stats(cuda_dev):
    rp, ci, va = synth.csr(10000, 500, "f64", ("powerlaw", 2.5, 3.0), seed=4)
    rpd, cid = rp.to(cuda_dev), ci.to(cuda_dev)
    fp.csr_validate(rpd, cid, 500)
    bad = cid.clone()
    bad[123] = 500
    with pytest.raises(fp.FusedPatError):
        fp.csr_validate(rpd, bad, 500)
    sd, sh = fp.row_stats_device(rpd), fp.row_stats_host(rp)
    for k in ("m", "nnz", "max_len", "min_len", "empty_rows"):
        assert getattr(sd, k) == getattr(sh, k)
    assert list(sd.hist_log2) == list(sh.hist_log2)


def test_csr_plan_c3_c4(cuda_dev):
    """B200 plan for the C3/C4 shapes: Eq. (4) VS from mu, smem vs L2 aggregation by n."""
    st = fp.fp_row_stats()
    st.m, st.n, st.nnz = 20_000_000, 1000, 200_000_000
    st.mean = 10.0
    L = fp.choose(True, st, fp.FP_F64, 0)
    # fp64, y + w on chip: the flat-4 kernel with the fixed-point CTA partial (variant 18, the
    # best of 936 settings in profiles/r02_sweep_C3.json); fp32: CSR-vector with the CTA-shared
    # partial, Eq. (4)'s VS = 8 bin run as 4 lanes x 4 cached entries (profiles/r02_sweep_S3.json)
    assert (L.variant, L.bs) == (18, 256)
    L = fp.choose(True, st, fp.FP_F32, 0)
    assert (L.vs, L.tl, L.variant) == (4, 4, 3)
    st.m, st.n, st.nnz = 50_000_000, 100_000, 2_000_000_000
    st.mean = 40.0
    L = fp.choose(True, st, fp.FP_F32, 0)
    # flat producer (one 1024-thread CTA per SM, 56 % of y in smem) writing column-block bins
    # that a fixed-point shared-memory consumer reduces (variant 17, 2 bins of 50K columns)
    assert L.variant == 17 and L.tl == 8 and L.bs == 1024 and L.cluster == 2


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("variant", [6, 7, 8, 12])
@pytest.mark.parametrize("nb", [2, 4, 8])
@pytest.mark.parametrize("lengths", [("uniform", 0, 70), ("powerlaw", 2.0, 3.0), ("binomial", 0.02)])
def test_csr_flat_bitexact(cuda_dev, dt, variant, nb, lengths):
    """Flat kernels (lanes on consecutive nonzeros, rows longer than 32*NB take the warp-per-
    row path): integer twins bit-exact for every instance."""
    skip_unbuilt(variant)
    m, n = 4000, 600
    rp, ci, va, y, v, z = make_csr(m, n, dt, lengths, seed=nb + variant, kind="int_pm12")
    L = fp.fp_launch()
    L.variant, L.vs, L.tl, L.bs, L.grid = variant, 32, nb, 256, 59
    for args in ((y, v, z, 1.0, 1.0), (None, v, None, -1.0, 0.0), (y, None, None, 2.0, 0.0)):
        ref, _ = oracle.csr(m, n, rp, ci, va, *args)
        w = gpu_csr(cuda_dev, rp, ci, va, n, *args, launch=L)
        assert_bitexact(w, ref, f"flat variant={variant} nb={nb} {lengths}")


@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_kdd_like_skewed_columns(cuda_dev, dt):
    """NEXT-2 shape, scaled: power-law rows, Zipf-like column popularity over a wide n (the L2
    path with hot columns contending on the same w entries); integer twin bit-exact in fp64."""
    m, n = 60000, 2_000_000
    rp, ci, va = synth.csr(m, n, dt, ("powerlaw", 2.5, 9.5, 20000), seed=21, col_skew=2)
    y = synth.vector(n, dt, seed=21, stream=synth.S_Y)
    v = synth.vector(m, dt, kind="pos", seed=21, stream=synth.S_V)
    z = synth.vector(n, dt, seed=21, stream=synth.S_Z)
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    w = gpu_csr(cuda_dev, rp, ci, va, n, y, v, z, 1.0, 1.0)
    assert_parity(w, ref, mag, DT[dt], "kdd-like")
    if dt == "f64":
        rp, ci, va = synth.csr(m, n, dt, ("powerlaw", 2.5, 9.5, 20000), seed=22, col_skew=2, kind="int_pm12")
        yi = synth.vector(n, dt, kind="int_small", seed=22, stream=synth.S_Y)
        vi = synth.vector(m, dt, kind="int_pos", seed=22, stream=synth.S_V)
        ref, _ = oracle.csr(m, n, rp, ci, va, yi, vi, None, 1.0, 0.0)
        w = gpu_csr(cuda_dev, rp, ci, va, n, yi, vi, None, 1.0, 0.0)
        assert_bitexact(w, ref, "kdd-like twin")


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("vs,k", [(4, 4), (8, 2), (16, 2), (32, 4)])
@pytest.mark.parametrize("n", [700, 2000])
def test_csr_owner_bitexact(cuda_dev, dt, vs, k, n):
    """Owner-computes aggregation (variant 10): queues, drains, spills -- integer twins exact,
    including heavy rows (power-law) that overflow the queues into the CAS spill partial."""
    skip_unbuilt(10)
    m = 6000
    for lengths in (("binomial", 0.01), ("powerlaw", 2.0, 4.0)):
        rp, ci, va, y, v, z = make_csr(m, n, dt, lengths, seed=vs + n, kind="int_pm12")
        L = fp.fp_launch()
        L.variant, L.vs, L.tl, L.bs, L.grid = 10, vs, k, 256, 23
        for args in ((y, v, z, 1.0, 1.0), (None, v, None, -1.0, 0.0)):
            ref, _ = oracle.csr(m, n, rp, ci, va, *args)
            w = gpu_csr(cuda_dev, rp, ci, va, n, *args, launch=L)
            assert_bitexact(w, ref, f"owner vs={vs} k={k} n={n} {lengths}")


def _single_column(m, v_of_row, dt):
    rp = torch.arange(m + 1, dtype=torch.int64)
    ci = torch.zeros(m, dtype=torch.int32)
    va = torch.ones(m, dtype=DT[dt])
    v = torch.tensor([v_of_row(r) for r in range(m)], dtype=DT[dt])
    return rp, ci, va, torch.ones(1, dtype=DT[dt]), v


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("variant,vs,tl", [(11, 1, 2), (11, 8, 2), (12, 32, 4)])
def test_fixed_point_limb_moves_and_spill_bitexact(cuda_dev, dt, variant, vs, tl):
    """Fixed-point partial (fixacc.cuh) on one CTA and one column: the first rows set the cap
    exponent from terms of 1 (cap 2^7); then 40k terms of 63 push the high limb past 2^29
    (value-preserving moves into the fp64 spill) and terms of 1000 exceed the cap (spill
    path).  Integers: the sum is exact, so w must equal the oracle bit for bit."""
    skip_unbuilt(variant)
    m = 60000  # one CTA of 8 warps: warp w owns rows [7500 w, 7500 (w + 1)); each starts with 256 rows of 1
    rp, ci, va, y, v = _single_column(m, lambda r: 1.0 if r % 7500 < 256 else (1000.0 if r % 97 == 0 else 63.0), dt)
    ref, _ = oracle.csr(m, 1, rp, ci, va, y, v, None, 1.0, 0.0)
    L = fp.fp_launch()
    L.variant, L.vs, L.tl, L.bs, L.grid = variant, vs, tl, 256, 1
    w = gpu_csr(cuda_dev, rp, ci, va, 1, y, v, None, 1.0, 0.0, launch=L)
    assert_bitexact(w, ref, f"fixed moves variant={variant}")


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("variant", [11, 12])
def test_fixed_point_wide_dynamic_range(cuda_dev, dt, variant):
    """Rows scaled by 2^k, k uniform in [-40, 40] (terms spanning ~2^160): the fixed-point
    partial keeps the stated normwise tolerance (small terms round to the CTA's grid, large
    ones spill to fp64; DESIGN reading R21)."""
    skip_unbuilt(variant)
    m, n = 30000, 800
    rp, ci, va, y, v, z = make_csr(m, n, dt, ("binomial", 0.01), seed=41)
    k = torch.from_numpy(np.random.default_rng(41).integers(-40, 41, m)).double()
    v = (v.double() * torch.pow(2.0, k)).to(DT[dt])
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    L = fp.fp_launch()
    L.variant, L.vs, L.tl, L.bs, L.grid = variant, 8 if variant == 11 else 32, 2 if variant == 11 else 4, 256, 148
    w = gpu_csr(cuda_dev, rp, ci, va, n, y, v, z, 1.0, 1.0, launch=L)
    assert_parity(w, ref, mag, DT[dt], f"fixed wide range variant={variant}")


STREAM_VSK = [(2, 4), (4, 4), (8, 2), (16, 2), (32, 4)]


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("variant", [14, 15])
@pytest.mark.parametrize("vsk", STREAM_VSK)
@pytest.mark.parametrize("lengths", [("uniform", 0, 70), ("powerlaw", 2.5, 13.64), ("binomial", 0.01)])
def test_csr_stream_bitexact(cuda_dev, dt, variant, vsk, lengths):
    """Stream variants (csr_stream.cuh: cp.async two-stage row stream): batches that overflow
    the stage (rows read from global), rows longer than VS*K, empty rows, an nnz that is not a
    multiple of the 16-byte chunk (zero-filled tail), warps with no rows -- integer twins must
    equal the oracle bit for bit, with and without y."""
    skip_unbuilt(variant)
    m, n = 7001, 1000
    rp, ci, va, y, v, z = make_csr(m, n, dt, lengths, seed=vsk[0] * 10 + vsk[1], kind="int_pm12")
    vs, k = vsk
    for yy, grid in ((y, 37), (None, 148), (y, 1)):
        ref, _ = oracle.csr(m, n, rp, ci, va, yy, v, z, 1.0, 1.0)
        L = fp.fp_launch()
        L.variant, L.vs, L.tl, L.bs, L.grid = variant, vs, k, 256, grid
        w = gpu_csr(cuda_dev, rp, ci, va, n, yy, v, z, 1.0, 1.0, launch=L)
        assert_bitexact(w, ref, f"stream variant={variant} vs={vs} k={k} y={yy is not None} grid={grid}")


@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_csr_stream_misaligned_falls_back(cuda_dev, dt):
    """colidx / val not 16-byte aligned: variant 14 runs as variant 3 (same result)."""
    m, n = 2000, 300
    rp, ci, va, y, v, z = make_csr(m, n, dt, ("binomial", 0.05), seed=3, kind="int_pm12")
    nnz = int(rp[-1])
    ci2 = torch.cat([torch.zeros(1, dtype=ci.dtype), ci])
    va2 = torch.cat([torch.zeros(1, dtype=va.dtype), va])
    ref, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    dev = cuda_dev
    ci_d, va_d = ci2.to(dev)[1:], va2.to(dev)[1:]
    assert ci_d.data_ptr() % 16 != 0 and ci_d.numel() == nnz
    L = fp.fp_launch()
    L.variant, L.vs, L.tl, L.bs, L.grid = 14, 4, 4, 256, 64
    w = fp.csr(rp.to(dev), ci_d, va_d, n, y.to(dev), v.to(dev), z.to(dev), 1.0, 1.0, launch=L)
    assert_bitexact(w.cpu(), ref, "misaligned stream fallback")


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("variant", [14, 15])
def test_csr_stream_float_parity(cuda_dev, dt, variant):
    """Full-precision C3-shaped inputs (scaled down): normwise tolerance of north_star."""
    skip_unbuilt(variant)
    m, n = 200_000, 1000
    rp, ci, va, y, v, z = make_csr(m, n, dt, ("binomial", 0.01), seed=9)
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 0.75, -1.25)
    L = fp.fp_launch()
    L.variant, L.vs, L.tl, L.bs, L.grid = variant, 4, 4, 256, 0
    w = gpu_csr(cuda_dev, rp, ci, va, n, y, v, z, 0.75, -1.25, launch=L)
    assert_parity(w, ref, mag, DT[dt], f"stream float variant={variant}")


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("n", [1000, 60_000, 120_000])
def test_csr_flat_l2_wide_bitexact(cuda_dev, dt, n):
    """Variant 16 (1024-thread flat CTA, reds into L2, a y prefix of ~220 KB in shared memory):
    y fully staged (n = 1000), partly staged (fp32 n = 60K fits, fp64 does not; n = 120K
    splits both) -- integer twins bit-exact, with and without y."""
    m = 20_000
    rp, ci, va, y, v, z = make_csr(m, n, dt, ("powerlaw", 2.5, 13.64), seed=n % 97, kind="int_pm12")
    for yy in (y, None):
        ref, _ = oracle.csr(m, n, rp, ci, va, yy, v, z, 1.0, -1.0)
        L = fp.fp_launch()
        L.variant, L.vs, L.tl, L.bs, L.grid = 16, 32, 8, 1024, 0
        w = gpu_csr(cuda_dev, rp, ci, va, n, yy, v, z, 1.0, -1.0, launch=L)
        assert_bitexact(w, ref, f"wide flat n={n} y={yy is not None}")
