"""GPU parity of the column-split cluster kernel (FP_VAR_CSR_COLSPLIT, csr_colsplit.cuh) run
through a CSR plan (fp_csr_plan_create / fp_csr_plan_exec) against the fp64 oracle.

The split serves n too wide for one SM (C4: n = 1e5, P:427's large-n regime): CTA k of a
cluster holds column block k of y and w; every row is cut into CS segments at the block
bounds (offsets precomputed by the plan).  Covered: the C4 shape scaled down (chooser's own
plan), every cluster size forced on integer twins (bit-exact: any dropped, duplicated or
misplaced segment entry changes w), every instance of Table 1, rows longer than the register
tiles (re-read path), empty rows and ragged batches, in-place w == z, and the refusal of a
forced split on non-canonical rows (reading R7)."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_asharitbrcks15_b200 as fp
import synth
from _util import assert_bitexact, assert_parity

pytestmark = pytest.mark.gpu

DT = {"f64": torch.float64, "f32": torch.float32}


def make(m, n, dt, lengths, seed, kind="uniform"):
    rp, ci, va = synth.csr(m, n, dt, lengths, kind=kind, seed=seed)
    integer = kind.startswith("int")
    y = synth.vector(n, dt, kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Y)
    v = synth.vector(m, dt, kind="int_pos" if integer else "pos", seed=seed, stream=synth.S_V)
    z = synth.vector(n, dt, kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Z)
    return rp, ci, va, y, v, z


def forced(cs):
    L = fp.fp_launch()
    L.variant, L.cluster = 13, cs
    return L


def run_plan(dev, rp, ci, va, n, args, launch=None):
    cu = lambda t: None if t is None else t.to(dev)
    P = fp.CsrPlan(cu(rp), cu(ci), n, va.dtype, launch=launch)
    y, v, z, alpha, beta = args
    w = P(cu(va), cu(y), cu(v), cu(z), alpha, beta)
    torch.cuda.synchronize()
    return P, w


@pytest.mark.parametrize("dt", ["f32", "f64"])
def test_c4_shape_chooser_plan(cuda_dev, dt):
    """C4 shape scaled to the oracle (power-law rows, n = 1e5): the chooser's plan (flat + L2,
    1024-thread CTAs with a y prefix in shared memory)
    and, for fp32, the forced column split (y and w blocks of 25K columns in 4 CTAs; fp64 at
    this n does not fit a cluster) -- both within the north_star tolerance."""
    m, n = 20000, 100000
    rp, ci, va, y, v, z = make(m, n, dt, ("powerlaw", 2.5, 13.64), seed=404)
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
    P, w = run_plan(cuda_dev, rp, ci, va, n, (y, v, z, 1.0, 1.0))
    assert P.launch.variant == 16 and P.launch.bs == 1024
    assert_parity(w, ref, mag, DT[dt], "C4-shape chooser plan")
    if dt == "f32":
        P, w = run_plan(cuda_dev, rp, ci, va, n, (y, v, z, 1.0, 1.0), launch=forced(4))
        assert P.launch.variant == 13 and P.launch.cluster == 4
        assert_parity(w, ref, mag, DT[dt], "C4-shape column split")


@pytest.mark.parametrize("dt", ["f32", "f64"])
@pytest.mark.parametrize("cs", [2, 4, 8])
@pytest.mark.parametrize("lengths", [("binomial", 0.01), ("powerlaw", 2.0, 3.0), ("uniform", 0, 5)])
def test_forced_split_integer_twins_bitexact(cuda_dev, dt, cs, lengths):
    m, n = 7001, 3000  # ragged last batch
    rp, ci, va, y, v, z = make(m, n, dt, lengths, seed=cs * 7 + len(lengths), kind="int_pm12")
    for args in ((y, v, z, 1.0, 1.0), (None, v, None, -2.0, 0.0), (y, None, None, 1.0, 0.0), (y, v, z, 0.5, -2.0)):
        P, w = run_plan(cuda_dev, rp, ci, va, n, args, launch=forced(cs))
        assert P.launch.variant == 13 and P.launch.cluster == cs
        ref, _ = oracle.csr(m, n, rp, ci, va, *args)
        assert_bitexact(w, ref, f"split cs={cs} {lengths} y={args[0] is not None}")


@pytest.mark.parametrize("dt", ["f32", "f64"])
def test_split_long_rows_beyond_register_tiles(cuda_dev, dt):
    """Rows up to n = 4000 long: a warp's block segment exceeds the NB = 8 register tiles (256
    entries) and the tail is re-read for the scatter; also whole rows inside one block."""
    m, n = 3000, 4000
    rp, ci, va, y, v, z = make(m, n, dt, ("powerlaw", 1.6, 20.0), seed=9, kind="int_pm12")
    for cs in (2, 4):
        P, w = run_plan(cuda_dev, rp, ci, va, n, (y, v, z, 1.0, 1.0), launch=forced(cs))
        ref, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
        assert_bitexact(w, ref, f"long rows cs={cs}")


@pytest.mark.parametrize("dt", ["f32", "f64"])
def test_split_real_values_and_inplace(cuda_dev, dt):
    m, n = 30000, 20000
    rp, ci, va, y, v, z = make(m, n, dt, ("binomial", 0.002), seed=31)
    ref, mag = oracle.csr(m, n, rp, ci, va, y, v, z, 0.75, -1.25)
    P = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), n, DT[dt], launch=forced(2))
    zd = z.to(cuda_dev).clone()
    w = P(va.to(cuda_dev), y.to(cuda_dev), v.to(cuda_dev), zd, 0.75, -1.25, w=zd)  # w aliases z
    torch.cuda.synchronize()
    assert_parity(w, ref, mag, DT[dt], "split in-place")
    w2 = P(va.to(cuda_dev), y.to(cuda_dev), v.to(cuda_dev), z.to(cuda_dev), 0.75, -1.25)  # plan reuse
    assert_parity(w2, ref, mag, DT[dt], "split reuse")


def test_split_empty_rows_and_edge_shapes(cuda_dev):
    dt = "f64"
    for m, n in ((1, 4), (33, 5), (5000, 64)):
        rp, ci, va, y, v, z = make(m, n, dt, ("uniform", 0, 3), seed=m, kind="int_pm12")
        P, w = run_plan(cuda_dev, rp, ci, va, n, (y, v, z, 1.0, 1.0), launch=forced(2))
        ref, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 1.0, 1.0)
        assert_bitexact(w, ref, f"edge {m}x{n}")


def test_split_refuses_noncanonical_rows(cuda_dev):
    rng = np.random.default_rng(5)
    m, n = 400, 300
    lens = rng.integers(0, 30, m)
    rp = torch.from_numpy(np.concatenate([[0], np.cumsum(lens)]).astype(np.int64))
    ci = torch.from_numpy(rng.integers(0, n, int(rp[-1])).astype(np.int32))  # unsorted, duplicates
    with pytest.raises(fp.FusedPatError) as e:
        fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), n, torch.float64, launch=forced(2))
    assert e.value.status == 4  # FP_ERR_INVALID_CSR
    P = fp.CsrPlan(rp.to(cuda_dev), ci.to(cuda_dev), n, torch.float64)  # chooser: no split
    assert P.launch.variant != 13
