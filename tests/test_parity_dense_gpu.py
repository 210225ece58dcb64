"""GPU parity of fp_dense (through the C ABI) against the fp64 oracle, element by element.

Sizes span several CTAs/tiles plus ragged tails; every Table-1 instance; both
dtypes; the vector (VS <= 32) and CTA (VS = BS) variants; 32-byte-aligned (LDG.256) and
misaligned (scalar) rows; padded ld; edge cases of readings R2-R10.  Integer
twins (exact in any summation order) must match bit for bit."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_asharitbrcks15_b200 as fp
import synth
from _util import TOL, assert_bitexact, assert_parity

pytestmark = pytest.mark.gpu

DT = {"f64": torch.float64, "f32": torch.float32}
INSTANCES = {
    "full": dict(y=True, v=True, z=True, alpha=0.75, beta=-1.25),      # Table 1 row 5
    "xty": dict(y=False, v=True, z=False, alpha=-2.0, beta=0.0),       # row 1: alpha X^T y (y passed as v)
    "xtxy": dict(y=True, v=False, z=False, alpha=1.0, beta=0.0),       # row 2
    "xtvxy": dict(y=True, v=True, z=False, alpha=1.0, beta=0.0),       # row 3
    "xtxy_bz": dict(y=True, v=False, z=True, alpha=1.0, beta=0.5),     # row 4
}


def make(m, n, dt, seed, kind="uniform", ld=None):
    X = synth.dense(m, n, dt, kind=kind, seed=seed, ld=ld)
    vk = "int_pos" if kind.startswith("int") else "pos"
    yk = "int_small" if kind.startswith("int") else "uniform"
    y = synth.vector(n, dt, kind=yk, seed=seed, stream=synth.S_Y)
    v = synth.vector(m, dt, kind=vk, seed=seed, stream=synth.S_V)
    z = synth.vector(n, dt, kind=yk, seed=seed, stream=synth.S_Z)
    return X, y, v, z


def run_both(X, y, v, z, inst, dev, n=None):
    m = X.shape[0]
    n = X.shape[1] if n is None else n
    I = INSTANCES[inst]
    yy, vv, zz = (y if I["y"] else None), (v if I["v"] else None), (z if I["z"] else None)
    ref, mag = oracle.dense_ld(X.contiguous(), m, n, X.shape[1], yy, vv, zz, I["alpha"], I["beta"])
    Xd = X.to(dev)
    cu = lambda t: None if t is None else t.to(dev)
    w = fp.dense(Xd[:, :n] if n != X.shape[1] else Xd, cu(yy), cu(vv), cu(zz), I["alpha"], I["beta"])
    torch.cuda.synchronize()
    return w, ref, mag


SHAPES = [(1, 1), (7, 3), (33, 8), (1000, 100), (4099, 128), (3001, 33), (1234, 257), (513, 1000), (300, 2048),
          (2000, 17), (777, 64)]


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("m,n", SHAPES)
@pytest.mark.parametrize("inst", list(INSTANCES))
def test_dense_instances(cuda_dev, dt, m, n, inst):
    X, y, v, z = make(m, n, dt, seed=m * 7 + n)
    w, ref, mag = run_both(X, y, v, z, inst, cuda_dev)
    assert_parity(w, ref, mag, DT[dt], f"{dt} {m}x{n} {inst}")


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("m,n", [(5000, 2500), (301, 4100), (64, 8000), (3, 16384)])
def test_dense_cta_variant(cuda_dev, dt, m, n):
    """Wide rows (VS = BS > 32, Alg. 3 l.16-22 two-level reduce)."""
    if dt == "f64" and n > 8192:
        pytest.skip("beyond the fp64 register-resident limit")
    X, y, v, z = make(m, n, dt, seed=n)
    w, ref, mag = run_both(X, y, v, z, "full", cuda_dev)
    assert_parity(w, ref, mag, DT[dt], f"cta {dt} {m}x{n}")


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("m,n", [(2000, 100), (999, 128), (4097, 1000), (100, 3000)])
def test_dense_integer_twins_bitexact(cuda_dev, dt, m, n):
    """Integer-valued inputs: every summation order is exact, so GPU == oracle bitwise."""
    X, y, v, z = make(m, n, dt, seed=3, kind="int_pm12")
    # fp32 exactness bound: sum_r |X_rj v_r p_r| < 2^24
    bound = float((X.double().abs().T @ (v.double().abs() * (X.double().abs() @ y.double().abs()))).max())
    if dt == "f32" and bound >= 2**24:
        pytest.skip("fp32 twin exceeds the exactness bound")
    w, ref, _ = run_both(X, y, v, z, "full", cuda_dev)
    assert_bitexact(w, ref, f"twin {dt} {m}x{n}")


@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_padded_ld_nan_padding_not_read(cuda_dev, dt):
    m, n, ld = 3000, 100, 136
    X, y, v, z = make(m, n, dt, seed=5, ld=ld)        # columns n..ld-1 hold NaN
    w, ref, mag = run_both(X, y, v, z, "full", cuda_dev, n=n)
    assert torch.isfinite(w).all()
    assert_parity(w, ref, mag, DT[dt], "padded ld")


@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_misaligned_rows_scalar_path(cuda_dev, dt):
    """ld*sizeof(T) not a multiple of 32 (and X offset by one element): scalar-load kernels."""
    m, n = 2001, 77
    X, y, v, z = make(m, n + 1, dt, seed=9)
    Xd = X.to(cuda_dev)[:, 1:]                          # misaligned base, ld = n+1
    ref, mag = oracle.dense(X[:, 1:].contiguous(), y[1:].contiguous(), v, z[1:].contiguous(), 0.75, -1.25)
    w = fp.dense(Xd, y[1:].contiguous().to(cuda_dev), v.to(cuda_dev), z[1:].contiguous().to(cuda_dev), 0.75, -1.25)
    assert_parity(w, ref, mag, DT[dt], "misaligned")


@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_edge_cases(cuda_dev, dt):
    tdt = DT[dt]
    n = 50
    z = synth.vector(n, dt, seed=1).to(cuda_dev)
    # m == 0 -> w = beta z
    X0 = torch.empty((0, n), dtype=tdt, device=cuda_dev)
    w = fp.dense(X0, torch.ones(n, dtype=tdt, device=cuda_dev), None, z, 1.0, 2.0)
    assert torch.equal(w, (2.0 * z.double()).to(tdt))
    # alpha == 0 -> X/y/v not read (NaN there must not leak)
    Xn = torch.full((10, n), float("nan"), dtype=tdt, device=cuda_dev)
    w = fp.dense(Xn, torch.full((n,), float("nan"), dtype=tdt, device=cuda_dev), None, z, 0.0, -1.0)
    assert torch.equal(w, -z)
    # beta == 0 -> z not read
    X, y, v, _ = make(100, n, dt, seed=2)
    w = fp.dense(X.to(cuda_dev), y.to(cuda_dev), v.to(cuda_dev), torch.full((n,), float("nan"), dtype=tdt,
                 device=cuda_dev), 1.0, 0.0)
    assert torch.isfinite(w).all()
    # n == 0 -> no-op
    fp.dense(torch.empty((5, 0), dtype=tdt, device=cuda_dev), torch.empty(0, dtype=tdt, device=cuda_dev))
    # w aliases z (in place, BLAS style)
    X, y, v, z0 = make(700, n, dt, seed=4)
    ref, mag = oracle.dense(X, y, v, z0, 0.5, 3.0)
    zz = z0.to(cuda_dev).clone()
    fp.dense(X.to(cuda_dev), y.to(cuda_dev), v.to(cuda_dev), zz, 0.5, 3.0, w=zz)
    assert_parity(zz, ref, mag, tdt, "w aliases z")
    # overlapping w and y is rejected
    buf = torch.zeros(2 * n, dtype=tdt, device=cuda_dev)
    with pytest.raises(fp.FusedPatError):
        fp.dense(X.to(cuda_dev), buf[:n], None, None, 1.0, 0.0, w=buf[n // 2: n // 2 + n])


def test_repeated_calls_and_streams(cuda_dev):
    """Workspace is re-zeroed by the finaliser: back-to-back calls, and calls on a side stream."""
    X, y, v, z = make(5000, 128, "f32", seed=8)
    ref, mag = oracle.dense(X, y, v, z, 1.0, 1.0)
    Xd, yd, vd, zd = (t.to(cuda_dev) for t in (X, y, v, z))
    for _ in range(5):
        w = fp.dense(Xd, yd, vd, zd, 1.0, 1.0)
        assert_parity(w, ref, mag, torch.float32, "repeat")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        w2 = fp.dense(Xd, yd, vd, zd, 1.0, 1.0)
    s.synchronize()
    assert_parity(w2, ref, mag, torch.float32, "side stream")


@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_plan_overrides_agree(cuda_dev, dt):
    """Correctness never depends on the plan: other VS / grid choices give the same result."""
    m, n = 3000, 24
    X, y, v, z = make(m, n, dt, seed=11, kind="int_pm12")
    ref, _ = oracle.dense(X, y, v, z, 1.0, 1.0)
    Xd, yd, vd, zd = (t.to(cuda_dev) for t in (X, y, v, z))
    e = 32 // X.element_size()
    for vs in (4, 8, 16, 32):
        if vs * e < n:
            continue
        for grid in (1, 7, 148, 1000):
            L = fp.fp_launch()
            L.variant, L.vs, L.bs, L.tl, L.grid = 1, vs, 256, e, grid
            w = fp.dense(Xd, yd, vd, zd, 1.0, 1.0, launch=L)
            assert_bitexact(w, ref, f"vs={vs} grid={grid}")


def test_plan_reports(cuda_dev):
    st = fp.row_stats_dense(10_000_000, 128)
    L = fp.choose(False, st, fp.FP_F32, 0)
    assert L.variant == 1 and L.vs == 16 and L.tl == 8 and L.grid % 148 == 0
    st = fp.row_stats_dense(4_000_000, 1000)
    L = fp.choose(False, st, fp.FP_F64, 0)
    assert L.variant == 1 and L.vs == 32 and L.tl == 32


@pytest.mark.parametrize("dt,m,n", [("f32", 500, 20000), ("f32", 97, 70001), ("f32", 64, 131072),
                                    ("f64", 300, 10000), ("f64", 61, 40000), ("f64", 33, 65536)])
def test_dense_cluster_variant(cuda_dev, dt, m, n):
    """Rows wider than one CTA's registers: thread-block cluster of CS CTAs, the row's dot
    reduced through DSMEM (NEXT-4 wide-n dense; the paper's fallback was two gemv)."""
    X, y, v, z = make(m, n, dt, seed=n + m)
    st = fp.row_stats_dense(m, n)
    L = fp.choose(False, st, fp.FP_F32 if dt == "f32" else fp.FP_F64, 0)
    assert L.variant == 9 and L.cluster in (2, 4, 8)
    w, ref, mag = run_both(X, y, v, z, "full", cuda_dev)
    assert_parity(w, ref, mag, DT[dt], f"cluster {dt} {m}x{n}")
    Xi, yi, vi, zi = make(m, n, dt, seed=7, kind="int_pm12")
    w, ref, _ = run_both(Xi, yi, vi, zi, "full", cuda_dev)
    if dt == "f64":
        assert_bitexact(w, ref, f"cluster twin {m}x{n}")


@pytest.mark.parametrize("dt,ldpad", [("f32", 0), ("f32", 4), ("f32", 1), ("f64", 2), ("f64", 0)])
@pytest.mark.parametrize("inst", ["xty", "xtvxy", "full"])
def test_dense_cluster_instances_ld(cuda_dev, dt, ldpad, inst):
    """Cluster variant over Table-1 instances (incl. row 1, no y: YM=0) and padded row strides:
    ld = n+4 fp32 / n+2 fp64 keeps 16-byte rows (bulk-copy ring), ld = n+1 fp32 falls back to
    scalar loads (register-only cluster kernel)."""
    m, n = 203, 30001 if dt == "f32" else 17003
    X, y, v, z = make(m, n, dt, seed=ldpad + 11, ld=n + ldpad if ldpad else None)
    st = fp.row_stats_dense(m, n)
    L = fp.choose(False, st, fp.FP_F32 if dt == "f32" else fp.FP_F64, 0)
    assert L.variant == 9
    w, ref, mag = run_both(X, y, v, z, inst, cuda_dev, n=n)
    assert_parity(w, ref, mag, DT[dt], f"cluster {dt} ld+{ldpad} {inst}")


def test_dense_cluster_register_kernel(cuda_dev, tmp_path):
    """The register-only cluster kernel (FP_CLUSTER_TMA=0: per-row cluster barrier, x held in
    registers; the path taken for rows that are not 16-byte aligned) on 16-byte-aligned rows,
    in a subprocess because the switch is read once per process; parity against the oracle
    like the default bulk-copy ring kernel."""
    import os
    import subprocess
    import sys
    m, n = 150, 40000
    script = tmp_path / "regk.py"
    script.write_text(
        "import sys, torch, synth, paper_conf_ppopp_asharitbrcks15_b200 as fp\n"
        f"m, n = {m}, {n}\n"
        "X = synth.dense(m, n, 'f32', seed=5).cuda()\n"
        "y = synth.vector(n, 'f32', seed=5, stream=synth.S_Y).cuda()\n"
        "v = synth.vector(m, 'f32', kind='pos', seed=5, stream=synth.S_V).cuda()\n"
        "L = fp.choose(False, fp.row_stats_dense(m, n), fp.FP_F32, 0)\n"
        "assert L.variant == 9 and L.tl * 4 == 256, L.as_dict()\n"
        "w = fp.dense(X, y, v, None, 1.0, 0.0)\n"
        "torch.save(w.cpu(), sys.argv[1])\n")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, FP_CLUSTER_TMA="0", PYTHONPATH=root)
    out = tmp_path / "w.pt"
    subprocess.run([sys.executable, str(script), str(out)], check=True, env=env, cwd=root, timeout=300)
    w = torch.load(out)
    X = synth.dense(m, n, "f32", seed=5)
    y = synth.vector(n, "f32", seed=5, stream=synth.S_Y)
    v = synth.vector(m, "f32", kind="pos", seed=5, stream=synth.S_V)
    ref, mag = oracle.dense(X, y, v, None, 1.0, 0.0)
    assert_parity(w, ref, mag, torch.float32, "cluster register kernel")
    L = fp.choose(False, fp.row_stats_dense(m, n), fp.FP_F32, 0)
    assert L.tl * 4 <= 128  # default process: the bulk-copy ring kernel
