"""GPU tests of the row epilogues (fp_*_epi) and the TRON logistic-regression driver (reading
R20, NEXT-1) against the fp64 oracle."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_asharitbrcks15_b200 as fp
import synth
from _util import TOL, assert_parity

pytestmark = pytest.mark.gpu
DT = {"f64": torch.float64, "f32": torch.float32}


def labels_for(Xd, seed):
    """labels in {-1,+1} from a planted model (host numpy, test infrastructure)"""
    rng = np.random.default_rng(seed)
    wt = rng.normal(size=Xd.shape[1])
    return np.where(Xd @ wt + 0.5 * rng.normal(size=Xd.shape[0]) > 0, 1.0, -1.0)


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("m,n", [(5000, 64), (3001, 128), (2000, 1000), (300, 20000)])
def test_logistic_epilogue_dense(cuda_dev, dt, m, n):
    X = synth.dense(m, n, dt, seed=m)
    y = torch.from_numpy(labels_for(X.double().numpy(), m)).to(DT[dt])
    w = synth.vector(n, dt, seed=m, stream=synth.S_Y) * 0.2
    C = 1.5
    f_ref, g_ref, D_ref = oracle.logreg_fgd_dense(X, y, C, w.double().numpy())
    Xd, yd, wd = X.to(cuda_dev), y.to(cuda_dev), w.to(cuda_dev)
    D = torch.empty(m, dtype=DT[dt], device=cuda_dev)
    loss = torch.zeros(1, dtype=torch.float64, device=cuda_dev)
    g = fp.dense_epi(Xd, wd, yd, wd, 1.0, 1.0, fp.FP_EPI_LOGISTIC, c=C, row_out=D, scalar_out=loss)
    torch.cuda.synchronize()
    f = 0.5 * float(wd.double() @ wd.double()) + C * float(loss)
    _, mag = oracle.dense(X, w, None, w, 1.0, 1.0)
    assert_parity(g, g_ref, np.abs(g_ref) + 1.0, DT[dt], "logistic gradient")
    rt = 1e-12 if dt == "f64" else 2e-5
    np.testing.assert_allclose(D.double().cpu().numpy(), D_ref, rtol=rt * 10, atol=rt)
    assert abs(f - f_ref) <= rt * 10 * abs(f_ref)


@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_logistic_epilogue_csr(cuda_dev, dt):
    m, n = 20000, 500
    rp, ci, va = synth.csr(m, n, dt, ("binomial", 0.03), seed=3)
    import scipy.sparse as sp
    A = sp.csr_matrix((va.double().numpy(), ci.numpy(), rp.numpy()), shape=(m, n))
    rng = np.random.default_rng(1)
    y = torch.from_numpy(np.where(A @ rng.normal(size=n) > 0, 1.0, -1.0)).to(DT[dt])
    w = synth.vector(n, dt, seed=3, stream=synth.S_Y) * 0.3
    C = 0.8
    f_ref, g_ref, D_ref = oracle.logreg_fgd_csr(m, n, rp, ci, va, y, C, w.double().numpy())
    D = torch.empty(m, dtype=DT[dt], device=cuda_dev)
    loss = torch.zeros(1, dtype=torch.float64, device=cuda_dev)
    wd = w.to(cuda_dev)
    g = fp.csr_epi(rp.to(cuda_dev), ci.to(cuda_dev), va.to(cuda_dev), n, wd, y.to(cuda_dev), wd, 1.0, 1.0,
                   fp.FP_EPI_LOGISTIC, c=C, row_out=D, scalar_out=loss)
    torch.cuda.synchronize()
    assert_parity(g, g_ref, np.abs(g_ref) + 1.0, DT[dt], "csr logistic gradient")
    rt = 1e-12 if dt == "f64" else 2e-5
    np.testing.assert_allclose(D.double().cpu().numpy(), D_ref, rtol=rt * 10, atol=rt)
    f = 0.5 * float(wd.double() @ wd.double()) + C * float(loss)
    assert abs(f - f_ref) <= rt * 10 * abs(f_ref)


def test_linear_epilogue_writes_Xy(cuda_dev):
    m, n = 7000, 100
    X = synth.dense(m, n, "f64", seed=9)
    yv = synth.vector(n, "f64", seed=9)
    v = synth.vector(m, "f64", kind="pos", seed=9, stream=synth.S_V)
    Xd = X.to(cuda_dev)
    p = torch.empty(m, dtype=torch.float64, device=cuda_dev)
    w = fp.dense_epi(Xd, yv.to(cuda_dev), v.to(cuda_dev), None, 1.0, 0.0, fp.FP_EPI_LINEAR, row_out=p)
    torch.cuda.synchronize()
    ref_p = X.numpy() @ yv.numpy()
    assert np.max(np.abs(p.cpu().numpy() - ref_p)) <= 1e-12 * np.max(np.abs(X.numpy()) @ np.abs(yv.numpy()))
    ref, mag = oracle.dense(X, yv, v, None, 1.0, 0.0)
    assert_parity(w, ref, mag, torch.float64, "linear epilogue w")


@pytest.mark.parametrize("fmt", ["dense", "csr"])
def test_tron_matches_oracle(cuda_dev, fmt):
    m, n, C = 20000, 80, 1.0
    if fmt == "dense":
        X = synth.dense(m, n, "f64", seed=11)
        y = torch.from_numpy(labels_for(X.numpy(), 11))
        w_ref, it_ref, f_ref = oracle.logreg_tron_dense(X, y, C=C, eps=1e-6, max_iter=50)
        w, it, fh = fp.logreg_tron_dense(X.to(cuda_dev), y.to(cuda_dev), C=C, eps=1e-6, max_iter=50)
    else:
        rp, ci, va = synth.csr(m, n, "f64", ("binomial", 0.2), seed=12)
        import scipy.sparse as sp
        A = sp.csr_matrix((va.numpy(), ci.numpy(), rp.numpy()), shape=(m, n))
        y = torch.from_numpy(labels_for(A.toarray(), 12))
        w_ref, it_ref, f_ref = oracle.logreg_tron_csr(m, n, rp, ci, va, y, C=C, eps=1e-6, max_iter=50)
        w, it, fh = fp.logreg_tron_csr(rp.to(cuda_dev), ci.to(cuda_dev), va.to(cuda_dev), n, y.to(cuda_dev), C=C,
                                       eps=1e-6, max_iter=50)
    torch.cuda.synchronize()
    # Derived bounds instead of iterate-by-iterate slack: f(w) = |w|^2/2 + C sum log(1+e^-y x.w)
    # has Hessian I + C X^T D X >= I, so it is 1-strongly convex and for any w
    #   |w - w*| <= |g(w)|   and   0 <= f(w) - f* <= |g(w)|^2 / 2,
    # hence |w_gpu - w_ref| <= |g(w_gpu)| + |g(w_ref)| and |f(w_gpu) - f(w_ref)| <= (|g_gpu|^2 +
    # |g_ref|^2) / 2, with g and f evaluated by the oracle (fp64) at both points.
    wg = w.cpu().numpy()
    if fmt == "dense":
        fg, gg, _ = oracle.logreg_fgd_dense(X, y, C, wg)
        fr, gr, _ = oracle.logreg_fgd_dense(X, y, C, w_ref)
    else:
        fg, gg, _ = oracle.logreg_fgd_csr(m, n, rp, ci, va, y, C, wg)
        fr, gr, _ = oracle.logreg_fgd_csr(m, n, rp, ci, va, y, C, w_ref)
    ng, nr = np.linalg.norm(gg), np.linalg.norm(gr)
    g0 = np.linalg.norm(oracle.logreg_fgd_dense(X, y, C, np.zeros(n))[1] if fmt == "dense" else
                        oracle.logreg_fgd_csr(m, n, rp, ci, va, y, C, np.zeros(n))[1])
    assert ng <= 1e-6 * g0 * 1.01, "GPU TRON stopped before |g| <= eps |g0| (its stopping rule)"
    rnd = 1e-12 * (np.linalg.norm(w_ref) + abs(fr))  # fp64 evaluation of the bounds themselves
    assert np.linalg.norm(wg - w_ref) <= ng + nr + rnd
    assert abs(fg - fr) <= 0.5 * (ng**2 + nr**2) + rnd
    assert abs(float(fh[-1]) - fg) <= 1e-10 * abs(fg)  # the driver's own f at its final w


def test_tron_fp32_converges(cuda_dev):
    m, n = 20000, 64
    X = synth.dense(m, n, "f32", seed=13)
    y = torch.from_numpy(labels_for(X.double().numpy(), 13)).float()
    w_ref, _, f_ref = oracle.logreg_tron_dense(X.double(), y.double(), C=1.0, eps=1e-8, max_iter=100)
    w, it, fh = fp.logreg_tron_dense(X.to(cuda_dev), y.to(cuda_dev), C=1.0, eps=1e-3, max_iter=100)
    assert abs(float(fh[-1]) - f_ref[-1]) <= 1e-4 * abs(f_ref[-1])
