"""Pins for the oracle's logistic regression (reading R20: L2-regularised LR by TRON, the
method the paper cites for LogReg, P:58 / [24]).  Expected values come from things other
than the oracle: closed forms at w = 0, central finite differences of f (for g) and of g
(for the Hessian weights D), and an independent minimiser (scipy L-BFGS on the same f)."""
import numpy as np
import scipy.optimize as so
import scipy.sparse as sp

import oracle


def problem(m=300, n=12, seed=0):
    rng = np.random.default_rng(seed)
    X = rng.uniform(-1, 1, (m, n))
    wt = rng.normal(size=n)
    y = np.where(X @ wt + 0.3 * rng.normal(size=m) > 0, 1.0, -1.0)
    return X, y


def f_plain(X, y, C, w):  # the objective, written independently with numpy
    t = y * (X @ w)
    return 0.5 * w @ w + C * np.sum(np.logaddexp(0.0, -t))


def test_closed_form_at_zero():
    X, y = problem()
    C = 2.0
    f, g, D = oracle.logreg_fgd_dense(X, y, C, np.zeros(X.shape[1]))
    assert abs(f - C * X.shape[0] * np.log(2.0)) < 1e-12 * f
    np.testing.assert_allclose(g, -0.5 * C * X.T @ y, rtol=1e-13, atol=1e-13)   # sigma(0) = 1/2
    np.testing.assert_allclose(D, np.full(X.shape[0], C / 4), rtol=1e-15)


def test_gradient_and_hessian_by_finite_differences():
    X, y = problem(seed=1)
    C = 0.7
    rng = np.random.default_rng(2)
    w = rng.normal(size=X.shape[1]) * 0.5
    f, g, D = oracle.logreg_fgd_dense(X, y, C, w)
    assert abs(f - f_plain(X, y, C, w)) < 1e-12 * abs(f)
    h = 1e-6
    fd = np.array([(f_plain(X, y, C, w + h * e) - f_plain(X, y, C, w - h * e)) / (2 * h) for e in np.eye(len(w))])
    np.testing.assert_allclose(g, fd, rtol=1e-6, atol=1e-7)
    s = rng.normal(size=len(w))
    gp = oracle.logreg_fgd_dense(X, y, C, w + h * s)[1]
    gm = oracle.logreg_fgd_dense(X, y, C, w - h * s)[1]
    Hs = s + X.T @ (D * (X @ s))
    np.testing.assert_allclose(Hs, (gp - gm) / (2 * h), rtol=1e-5, atol=1e-6)


def test_tron_matches_independent_minimiser():
    X, y = problem(seed=3)
    C = 1.0
    w, iters, hist = oracle.logreg_tron_dense(X, y, C=C, eps=1e-10, max_iter=100)
    res = so.minimize(lambda w_: f_plain(X, y, C, w_), np.zeros(X.shape[1]),
                      jac=lambda w_: w_ + X.T @ (C * (1 / (1 + np.exp(-y * (X @ w_))) - 1) * y),
                      method="L-BFGS-B", options=dict(gtol=1e-12, ftol=1e-15, maxiter=10000))
    assert np.linalg.norm(w - res.x) / np.linalg.norm(res.x) < 1e-7
    assert np.all(np.diff(hist) < 0)          # accepted steps decrease f
    assert 1 <= iters <= 30


def test_tron_csr_equals_dense():
    X, y = problem(m=500, n=20, seed=4)
    X[np.random.default_rng(5).random(X.shape) < 0.6] = 0.0
    A = sp.csr_matrix(X)
    wd, itd, _ = oracle.logreg_tron_dense(X, y, C=0.5, eps=1e-8)
    wc, itc, _ = oracle.logreg_tron_csr(500, 20, A.indptr, A.indices, A.data, y, C=0.5, eps=1e-8)
    assert itd == itc
    np.testing.assert_allclose(wc, wd, rtol=1e-12, atol=1e-14)
