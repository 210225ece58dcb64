"""Pins for the oracle's Listing-1 CG (reading R19 in DESIGN.md).

Expected values come from numpy.linalg.solve of the normal equations (the fixed point CG
must reach), from the CG theory facts (exact convergence in <= n steps for SPD systems in
exact arithmetic; monotone A-norm error), and from the stopping rule nr2 <= nr2_0 * tol^2.
"""
import numpy as np
import scipy.sparse as sp

import oracle


def test_cg_converges_to_normal_equations_dense():
    rng = np.random.default_rng(1)
    m, n = 400, 12
    X = rng.uniform(-1, 1, (m, n))
    b = rng.uniform(-1, 1, m)
    eps = 1e-3
    w, iters, hist = oracle.cg_linreg_dense(X, b, eps=eps, max_iter=100, tol=1e-12)
    ref = np.linalg.solve(X.T @ X + eps * np.eye(n), X.T @ b)
    assert np.linalg.norm(w - ref) / np.linalg.norm(ref) < 1e-10
    assert iters <= n + 3                      # SPD n x n: <= n steps up to rounding
    assert hist[-1] <= hist[0] * 1e-24         # stopping rule nr2 <= nr2_0 tol^2
    assert np.all(hist[1:] < hist[0])


def test_cg_converges_csr_and_matches_dense_form():
    rng = np.random.default_rng(2)
    m, n = 800, 30
    A = sp.random(m, n, density=0.2, format="csr", random_state=3, data_rvs=lambda k: rng.uniform(-1, 1, k))
    b = rng.uniform(-1, 1, m)
    w, iters, _ = oracle.cg_linreg_csr(m, n, A.indptr, A.indices, A.data, b, eps=1e-3, max_iter=200, tol=1e-12)
    D = A.toarray()
    ref = np.linalg.solve(D.T @ D + 1e-3 * np.eye(n), D.T @ b)
    assert np.linalg.norm(w - ref) / np.linalg.norm(ref) < 1e-10
    wd, itd, _ = oracle.cg_linreg_dense(D, b, eps=1e-3, max_iter=200, tol=1e-12)
    assert itd == iters and np.linalg.norm(wd - w) / np.linalg.norm(w) < 1e-12


def test_cg_fixed_iterations_and_tol_zero():
    """C5 runs a fixed iteration count with tol = 0: exactly max_iter iterations happen,
    and the A-norm error decreases monotonically (CG optimality)."""
    rng = np.random.default_rng(4)
    m, n = 300, 40
    X = rng.uniform(-1, 1, (m, n)) * (2.0 ** rng.integers(-4, 5, n))
    b = rng.uniform(-1, 1, m)
    H = X.T @ X + 1e-3 * np.eye(n)
    ref = np.linalg.solve(H, X.T @ b)
    errs = []
    for k in range(1, 8):
        w, iters, _ = oracle.cg_linreg_dense(X, b, eps=1e-3, max_iter=k, tol=0.0)
        assert iters == k
        e = w - ref
        errs.append(e @ H @ e)
    assert all(errs[i + 1] < errs[i] for i in range(len(errs) - 1))


def test_cg_first_iterate_closed_form():
    """After one step from w0 = 0: w1 = a p0 with p0 = X^T b, a = |p0|^2 / p0.H p0."""
    rng = np.random.default_rng(5)
    X = rng.uniform(-1, 1, (50, 6))
    b = rng.uniform(-1, 1, 50)
    H = X.T @ X + 1e-3 * np.eye(6)
    p0 = X.T @ b
    w1 = (p0 @ p0) / (p0 @ H @ p0) * p0
    w, iters, hist = oracle.cg_linreg_dense(X, b, eps=1e-3, max_iter=1, tol=0.0)
    np.testing.assert_allclose(w, w1, rtol=1e-13)
    np.testing.assert_allclose(hist[0], p0 @ p0, rtol=1e-14)
