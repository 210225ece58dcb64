"""Pins for the fp64 oracle (oracle/oracle.c) against things OTHER than itself.

Each test cites what fixes the expected value: exact rational arithmetic, an explicit
brute-force Gram matrix, numpy/scipy textbook expressions, closed forms and invariants of
Eq. (1), and the readings R2-R10 of DESIGN.md.  A plausible mistake in the
oracle (dropped term, wrong sign, transposed operand, wrong index, alpha/beta misplaced,
v applied to the wrong side) makes at least one of these fail -- the exact-dyadic pins alone
distinguish all of them, since every instance there is computed without rounding.
"""
from fractions import Fraction

import numpy as np
import pytest
import scipy.sparse as sp

import oracle

RNG = np.random.default_rng(20150207)


def dyadic(shape, rng, den=8, lo=-8, hi=8):
    return rng.integers(lo, hi + 1, size=shape).astype(np.float64) / den


def exact_pattern(X, y, v, z, alpha, beta):
    """Eq. (1) in exact rational arithmetic (Python Fractions), straight from the definition."""
    m, n = X.shape
    Xf = [[Fraction(float(X[r, c])) for c in range(n)] for r in range(m)]
    if y is None:
        p = [Fraction(1)] * m
    else:
        yf = [Fraction(float(t)) for t in y]
        p = [sum((Xf[r][c] * yf[c] for c in range(n)), Fraction(0)) for r in range(m)]
    q = [p[r] * (Fraction(float(v[r])) if v is not None else 1) for r in range(m)]
    w = []
    for c in range(n):
        acc = sum((Xf[r][c] * q[r] for r in range(m)), Fraction(0))
        t = Fraction(float(alpha)) * acc
        if beta != 0:
            t += Fraction(float(beta)) * Fraction(float(z[c]))
        w.append(t)
    return w


# ---------------------------------------------------------------- exact arithmetic pins
@pytest.mark.parametrize("case", range(12))
def test_exact_dyadic_dense(case):
    """Dyadic inputs with few bits: every product and partial sum is exact in fp64, so the
    oracle must EQUAL the exact rational result (Eq. 1 evaluated exactly)."""
    rng = np.random.default_rng(case)
    m, n = int(rng.integers(1, 13)), int(rng.integers(1, 13))
    X = dyadic((m, n), rng)
    y, v, z = dyadic(n, rng), dyadic(m, rng), dyadic(n, rng)
    alpha, beta = [(0.75, -1.25), (1.0, 0.0), (-2.0, 0.5), (0.5, 2.0)][case % 4]
    inst = case % 3  # 0 full, 1 v omitted, 2 y omitted (Table 1 row 1)
    yy = None if inst == 2 else y
    vv = None if inst == 1 else v
    zz = z if beta != 0 else None
    exp = exact_pattern(X, yy, vv, zz, alpha, beta)
    for threads in (1, 3):
        w, _ = oracle.dense(X, yy, vv, zz, alpha, beta, threads=threads)
        assert [Fraction(float(t)) for t in w] == exp


def test_exact_dyadic_csr():
    rng = np.random.default_rng(7)
    m, n = 11, 9
    X = dyadic((m, n), rng)
    X[rng.random((m, n)) < 0.5] = 0.0
    X[3, :] = 0.0  # an empty row
    A = sp.csr_matrix(X)
    y, v, z = dyadic(n, rng), dyadic(m, rng), dyadic(n, rng)
    exp = exact_pattern(X, y, v, z, 0.75, -1.25)
    w, _ = oracle.csr(m, n, A.indptr, A.indices, A.data, y, v, z, 0.75, -1.25, threads=2)
    assert [Fraction(float(t)) for t in w] == exp


def test_random_fp64_within_rounding_bound():
    """Full-precision inputs: |w - w_exact| <= 8u * mag (componentwise; compensated sums)."""
    rng = np.random.default_rng(11)
    m, n = 10, 7
    X = rng.uniform(-1, 1, (m, n))
    y, v, z = rng.uniform(-1, 1, n), rng.uniform(0, 0.25, m), rng.uniform(-1, 1, n)
    exp = exact_pattern(X, y, v, z, 0.3, -0.7)
    w, mag = oracle.dense(X, y, v, z, 0.3, -0.7, threads=1)
    u = np.finfo(np.float64).eps / 2
    for j in range(n):
        err = abs(Fraction(float(w[j])) - exp[j])
        assert err <= Fraction(8 * u * mag[j])


# ---------------------------------------------------------------- brute force / textbook
def test_bruteforce_gram():
    """Explicit G = X^T diag(v) X (n x n), then w = alpha G y + beta z (a different evaluation
    order than Eq. 2/3: the Gram matrix is formed first)."""
    rng = np.random.default_rng(3)
    m, n = 300, 17
    X = rng.uniform(-1, 1, (m, n))
    y, v, z = rng.uniform(-1, 1, n), rng.uniform(0, 0.25, m), rng.uniform(-1, 1, n)
    G = np.zeros((n, n))
    for r in range(m):
        G += v[r] * np.outer(X[r], X[r])
    ref = 0.75 * G @ y - 1.25 * z
    w, mag = oracle.dense(X, y, v, z, 0.75, -1.25)
    assert np.max(np.abs(w - ref) / mag) < 1e-13


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_numpy_textbook_dense(dtype):
    rng = np.random.default_rng(4)
    m, n = 1000, 100
    X = rng.uniform(-1, 1, (m, n)).astype(dtype)
    y, v, z = (rng.uniform(-1, 1, n).astype(dtype), rng.uniform(0, .25, m).astype(dtype),
               rng.uniform(-1, 1, n).astype(dtype))
    Xd, yd, vd, zd = (a.astype(np.float64) for a in (X, y, v, z))
    ref = 0.75 * Xd.T @ (vd * (Xd @ yd)) - 1.25 * zd
    w, mag = oracle.dense(X, y, v, z, 0.75, -1.25)
    assert np.linalg.norm(w - ref) / np.linalg.norm(ref) < 1e-14


def test_scipy_textbook_csr():
    rng = np.random.default_rng(5)
    m, n = 5000, 300
    A = sp.random(m, n, density=0.02, format="csr", random_state=5, data_rvs=lambda k: rng.uniform(-1, 1, k))
    y, v, z = rng.uniform(-1, 1, n), rng.uniform(0, .25, m), rng.uniform(-1, 1, n)
    ref = 1.5 * (A.T @ (v * (A @ y))) + 0.5 * z
    w, _ = oracle.csr(m, n, A.indptr, A.indices, A.data, y, v, z, 1.5, 0.5)
    assert np.linalg.norm(w - ref) / np.linalg.norm(ref) < 1e-14
    # Table 1 row 1: alpha X^T y  (y == NULL, the length-m vector passed as v)
    w1, _ = oracle.csr(m, n, A.indptr, A.indices, A.data, None, v, None, -2.0, 0.0)
    ref1 = -2.0 * (A.T @ v)
    assert np.linalg.norm(w1 - ref1) / np.linalg.norm(ref1) < 1e-14


# ---------------------------------------------------------------- closed forms
def test_identity_and_diagonal():
    rng = np.random.default_rng(6)
    n = 13
    y, v, z = rng.uniform(-1, 1, n), rng.uniform(0, 1, n), rng.uniform(-1, 1, n)
    w, _ = oracle.dense(np.eye(n), y, v, z, 2.0, -0.5)
    np.testing.assert_array_equal(w, 2.0 * (v * y) - 0.5 * z)          # X = I
    d = dyadic(n, rng)
    w, _ = oracle.dense(np.diag(d), y, v, z, 1.0, 1.0)
    np.testing.assert_allclose(w, d * d * v * y + z, rtol=1e-15, atol=1e-16)  # X = D


def test_ones_and_rank1():
    rng = np.random.default_rng(8)
    m, n = 40, 9
    y, v, z = rng.uniform(-1, 1, n), rng.uniform(0, 1, m), rng.uniform(-1, 1, n)
    w, _ = oracle.dense(np.ones((m, n)), y, v, z, 0.5, 3.0)
    np.testing.assert_allclose(w, 0.5 * v.sum() * y.sum() + 3.0 * z, rtol=1e-13)
    a, b = rng.uniform(-1, 1, m), rng.uniform(-1, 1, n)
    w, mag = oracle.dense(np.outer(a, b), y, v, z, -1.0, 0.0)
    ref = -1.0 * np.sum(v * a * a) * (b @ y) * b
    assert np.max(np.abs(w - ref) / mag) < 1e-14


def test_alpha_zero_does_not_read_X_and_v_zero():
    """R3: alpha == 0 -> w = beta z exactly, X/y/v not read (NaN there must not leak)."""
    m, n = 5, 4
    X = np.full((m, n), np.nan)
    z = np.arange(n, dtype=np.float64)
    w, _ = oracle.dense(X, np.full(n, np.nan), np.full(m, np.nan), z, 0.0, -2.0)
    np.testing.assert_array_equal(w, -2.0 * z)
    # v = 0 -> w = beta z
    rng = np.random.default_rng(1)
    w, _ = oracle.dense(rng.uniform(-1, 1, (m, n)), rng.uniform(-1, 1, n), np.zeros(m), z, 1.0, 1.0)
    np.testing.assert_array_equal(w, z)


def test_beta_zero_does_not_read_z():
    rng = np.random.default_rng(2)
    X = rng.uniform(-1, 1, (6, 3))
    y = rng.uniform(-1, 1, 3)
    w, _ = oracle.dense(X, y, None, np.full(3, np.nan), 1.0, 0.0)
    assert np.all(np.isfinite(w))
    with pytest.raises(ValueError):
        oracle.dense(X, y, None, None, 1.0, 1.0)  # R4: z omitted requires beta == 0


def test_edge_shapes():
    w, _ = oracle.dense(np.zeros((0, 5)), np.ones(5), None, np.arange(5.0), 1.0, 2.0)   # m = 0 -> beta z
    np.testing.assert_array_equal(w, 2.0 * np.arange(5.0))
    w, _ = oracle.dense(np.zeros((4, 0)), np.zeros(0), None, None, 1.0, 0.0)            # n = 0
    assert w.shape == (0,)
    rp = np.zeros(4, np.int64)                                                          # nnz = 0
    w, _ = oracle.csr(3, 5, rp, np.zeros(0, np.int32), np.zeros(0), np.ones(5), np.ones(3), np.ones(5), 1.0, 1.0)
    np.testing.assert_array_equal(w, np.ones(5))


# ---------------------------------------------------------------- invariants
def int_twin(m, n, rng):
    X = rng.choice([-2.0, -1.0, 1.0, 2.0], size=(m, n))
    return X, rng.integers(-3, 4, n).astype(float), rng.integers(1, 4, m).astype(float), rng.integers(-3, 4, n).astype(float)


def test_linearity_exact_on_integer_twins():
    rng = np.random.default_rng(9)
    X, y1, v, z = int_twin(50, 20, rng)
    y2 = rng.integers(-3, 4, 20).astype(float)
    T = lambda yy: oracle.dense(X, yy, v, None, 1.0, 0.0)[0]
    np.testing.assert_array_equal(T(y1 + 2 * y2), T(y1) + 2 * T(y2))                 # linear in y
    w_ab, _ = oracle.dense(X, y1, v, z, 2.0, -3.0)
    np.testing.assert_array_equal(w_ab, 2.0 * T(y1) - 3.0 * z)                        # alpha, beta placement


def test_symmetry_and_psd():
    """T = X^T diag(v) X is symmetric: u.T(y) = y.T(u); PSD for v >= 0 with
    y.T(y) = sum_i v_i (X y)_i^2 computed independently."""
    rng = np.random.default_rng(10)
    m, n = 400, 25
    X = rng.uniform(-1, 1, (m, n))
    v = rng.uniform(0, 1, m)
    y, u = rng.uniform(-1, 1, n), rng.uniform(-1, 1, n)
    Ty, Tu = oracle.dense(X, y, v, None, 1, 0)[0], oracle.dense(X, u, v, None, 1, 0)[0]
    assert abs(u @ Ty - y @ Tu) <= 1e-12 * abs(u @ Ty)
    quad = sum(v[i] * float(np.dot(X[i], y)) ** 2 for i in range(m))
    assert y @ Ty > 0 and abs(y @ Ty - quad) <= 1e-12 * quad


def test_permutations():
    rng = np.random.default_rng(12)
    m, n = 200, 30
    X, y, v, z = rng.uniform(-1, 1, (m, n)), rng.uniform(-1, 1, n), rng.uniform(0, 1, m), rng.uniform(-1, 1, n)
    w, mag = oracle.dense(X, y, v, z, 0.5, 0.25)
    pr = rng.permutation(m)
    w2, _ = oracle.dense(X[pr], y, v[pr], z, 0.5, 0.25)                               # rows with v
    assert np.max(np.abs(w2 - w) / mag) < 1e-14
    pc = rng.permutation(n)
    w3, _ = oracle.dense(X[:, pc], y[pc], v, z[pc], 0.5, 0.25)                        # columns
    assert np.max(np.abs(w3 - w[pc]) / mag[pc]) < 1e-14


def test_shard_sum_decomposition():
    """8(e): sum over row shards with beta = 0, plus beta z once, equals the full result
    (exactly on integer twins) -- the multi-GPU decomposition, pinned on CPU."""
    rng = np.random.default_rng(13)
    X, y, v, z = int_twin(97, 23, rng)
    full, _ = oracle.dense(X, y, v, z, 2.0, -1.0)
    bounds = [0, 13, 50, 51, 97]
    acc = -1.0 * z
    for a, b in zip(bounds[:-1], bounds[1:]):
        acc = acc + oracle.dense(X[a:b], y, v[a:b], None, 2.0, 0.0)[0]
    np.testing.assert_array_equal(acc, full)


def test_dense_vs_csr_agree():
    rng = np.random.default_rng(14)
    X, y, v, z = int_twin(60, 40, rng)
    X[rng.random(X.shape) < 0.7] = 0.0
    A = sp.csr_matrix(X)
    wd, _ = oracle.dense(X, y, v, z, 1.0, 1.0)
    wc, _ = oracle.csr(60, 40, A.indptr, A.indices, A.data, y, v, z, 1.0, 1.0)
    np.testing.assert_array_equal(wd, wc)


def test_csr_duplicates_summed():
    """R7: non-canonical CSR (unsorted, duplicate columns) == its sum_duplicates() form."""
    indptr = np.array([0, 3, 3, 6], np.int64)
    indices = np.array([2, 0, 2, 1, 1, 0], np.int32)
    data = np.array([1.0, 2.0, -3.0, 0.5, 0.25, 4.0])
    A = sp.csr_matrix((data, indices, indptr), shape=(3, 3))
    B = A.copy()
    B.sum_duplicates()
    y, v, z = np.array([1.0, -2.0, 3.0]), np.array([2.0, 1.0, -1.0]), np.array([1.0, 1.0, 1.0])
    wa, _ = oracle.csr(3, 3, indptr, indices, data, y, v, z, 1.0, 1.0)
    wb, _ = oracle.csr(3, 3, B.indptr, B.indices, B.data, y, v, z, 1.0, 1.0)
    np.testing.assert_array_equal(wa, wb)
    np.testing.assert_array_equal(wa, B.T @ (v * (B @ y)) + z)


def test_thread_count_independent():
    rng = np.random.default_rng(15)
    X = rng.uniform(-1, 1, (3000, 50))
    y, v = rng.uniform(-1, 1, 50), rng.uniform(0, 1, 3000)
    w1, mag = oracle.dense(X, y, v, None, 1.0, 0.0, threads=1)
    w8, _ = oracle.dense(X, y, v, None, 1.0, 0.0, threads=8)
    assert np.max(np.abs(w1 - w8) / mag) < 1e-15
