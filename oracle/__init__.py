"""ORACLE -- test infrastructure only (see oracle.c header).

Plain fp64 CPU reference of PAPER.md Eq. (1), row-decomposed per Eq. (2)/(3)
(P:142-147), beta*z / alpha placement per Algorithm 2, and the
Listing-1 CG driver.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py`` (cpu_baseline leg and ``--impl reference``) may import this package.
The product (``paper_conf_ppopp_asharitbrcks15_b200``) never imports it.

Pins (tests/test_oracle_*.py): exact Fraction arithmetic on dyadic inputs, explicit
X^T diag(v) X brute force, closed forms (identity, diagonal, ones, rank-1, alpha=0, v=0),
invariants (linearity, symmetry, PSD, permutations, shard-sum), numpy/scipy textbook
cross-checks, and CG convergence to numpy.linalg.solve.  Parity status per function is
listed in DESIGN.md ("Oracle pins"); no function is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

F32, F64 = 0, 1


def _lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make -C {os.path.dirname(_HERE)} oracle` "
                               "(or __graft_entry__.build())")
        lib = ctypes.CDLL(path)
        i64, dbl, vp, ci = ctypes.c_int64, ctypes.c_double, ctypes.c_void_p, ctypes.c_int
        lib.oracle_dense.argtypes = [i64, i64, vp, i64, vp, vp, vp, dbl, dbl, ci, ci, vp, vp]
        lib.oracle_csr.argtypes = [i64, i64, vp, vp, vp, vp, vp, vp, dbl, dbl, ci, ci, vp, vp]
        lib.oracle_cg_linreg_dense.argtypes = [i64, i64, vp, i64, vp, dbl, ci, dbl, ci, ci, vp, vp, vp]
        lib.oracle_cg_linreg_csr.argtypes = [i64, i64, vp, vp, vp, vp, dbl, ci, dbl, ci, ci, vp, vp, vp]
        lib.oracle_logreg_fgd_dense.argtypes = [i64, i64, vp, i64, vp, dbl, vp, ci, ci, vp, vp, vp]
        lib.oracle_logreg_fgd_csr.argtypes = [i64, i64, vp, vp, vp, vp, dbl, vp, ci, ci, vp, vp, vp]
        lib.oracle_logreg_tron_dense.argtypes = [i64, i64, vp, i64, vp, dbl, dbl, ci, ci, ci, ci, vp, vp, vp]
        lib.oracle_logreg_tron_csr.argtypes = [i64, i64, vp, vp, vp, vp, dbl, dbl, ci, ci, ci, ci, vp, vp, vp]
        for f in (lib.oracle_dense, lib.oracle_csr, lib.oracle_cg_linreg_dense, lib.oracle_cg_linreg_csr,
                  lib.oracle_logreg_fgd_dense, lib.oracle_logreg_fgd_csr, lib.oracle_logreg_tron_dense,
                  lib.oracle_logreg_tron_csr):
            f.restype = ci
        _LIB = lib
    return _LIB


def _np(a):
    """Accept numpy arrays or CPU torch tensors; return a C-contiguous numpy array (no copy if possible)."""
    if a is None:
        return None
    if hasattr(a, "detach"):
        a = a.detach()
        if a.device.type != "cpu":
            raise ValueError("oracle inputs must live on the host")
        a = a.numpy()
    return np.ascontiguousarray(a)


def _dtype_code(a):
    if a.dtype == np.float64:
        return F64
    if a.dtype == np.float32:
        return F32
    raise TypeError(f"unsupported dtype {a.dtype}")


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def default_threads():
    return max(1, os.cpu_count() or 1)


def dense(X, y, v, z, alpha, beta, threads=None):
    """w = alpha * X^T (v (.) (X y)) + beta z for dense row-major X (m x ld, first n = len-of-w
    columns used when X is 2-D with shape (m, n)).  Returns (w, mag) as fp64 numpy arrays;
    mag = |alpha| |X|^T (|v| (.) |X| |y|) + |beta| |z| (componentwise scale)."""
    X = _np(X)
    m, n = X.shape
    return dense_ld(X, m, n, n, y, v, z, alpha, beta, threads)


def dense_ld(X, m, n, ld, y, v, z, alpha, beta, threads=None):
    X, y, v, z = _np(X), _np(y), _np(v), _np(z)
    dt = _dtype_code(X)
    for a in (y, v, z):
        if a is not None and a.dtype != X.dtype:
            raise TypeError("all operands must share X's dtype")
    w = np.zeros(max(n, 0), np.float64)
    mag = np.zeros(max(n, 0), np.float64)
    rc = _lib().oracle_dense(m, n, _ptr(X), ld, _ptr(y), _ptr(v), _ptr(z), float(alpha), float(beta), dt,
                             threads or default_threads(), _ptr(w), _ptr(mag))
    if rc != 0:
        raise ValueError(f"oracle_dense rc={rc}")
    return w, mag


def csr(m, n, rowptr, colidx, val, y, v, z, alpha, beta, threads=None):
    rowptr = _np(rowptr).astype(np.int64, copy=False)
    colidx = _np(colidx).astype(np.int32, copy=False)
    val, y, v, z = _np(val), _np(y), _np(v), _np(z)
    dt = _dtype_code(val)
    w = np.zeros(max(n, 0), np.float64)
    mag = np.zeros(max(n, 0), np.float64)
    rc = _lib().oracle_csr(m, n, _ptr(rowptr), _ptr(colidx), _ptr(val), _ptr(y), _ptr(v), _ptr(z), float(alpha),
                           float(beta), dt, threads or default_threads(), _ptr(w), _ptr(mag))
    if rc != 0:
        raise ValueError(f"oracle_csr rc={rc}")
    return w, mag


def cg_linreg_dense(X, labels, eps=1e-3, max_iter=100, tol=1e-6, threads=None):
    """Listing 1.  Returns (w, iters, nr2_history)."""
    X, labels = _np(X), _np(labels)
    m, n = X.shape
    w = np.zeros(n, np.float64)
    it = ctypes.c_int(0)
    hist = np.zeros(max_iter + 1, np.float64)
    rc = _lib().oracle_cg_linreg_dense(m, n, _ptr(X), n, _ptr(labels), float(eps), int(max_iter), float(tol),
                                       _dtype_code(X), threads or default_threads(), _ptr(w), ctypes.byref(it),
                                       _ptr(hist))
    if rc != 0:
        raise ValueError(f"oracle_cg_linreg_dense rc={rc}")
    return w, it.value, hist[: it.value + 1]


def logreg_fgd_dense(X, labels, C, w, threads=None):
    """(f, g, D) of L2-regularised logistic regression at w (reading R20)."""
    X, labels = _np(X), _np(labels)
    m, n = X.shape
    w = np.ascontiguousarray(w, dtype=np.float64)
    f = ctypes.c_double(0.0)
    g, D = np.zeros(n), np.zeros(m)
    rc = _lib().oracle_logreg_fgd_dense(m, n, _ptr(X), n, _ptr(labels), float(C), _ptr(w), _dtype_code(X),
                                        threads or default_threads(), ctypes.byref(f), _ptr(g), _ptr(D))
    if rc != 0:
        raise ValueError(f"oracle_logreg_fgd_dense rc={rc}")
    return f.value, g, D


def logreg_fgd_csr(m, n, rowptr, colidx, val, labels, C, w, threads=None):
    rowptr = _np(rowptr).astype(np.int64, copy=False)
    colidx = _np(colidx).astype(np.int32, copy=False)
    val, labels = _np(val), _np(labels)
    w = np.ascontiguousarray(w, dtype=np.float64)
    f = ctypes.c_double(0.0)
    g, D = np.zeros(n), np.zeros(m)
    rc = _lib().oracle_logreg_fgd_csr(m, n, _ptr(rowptr), _ptr(colidx), _ptr(val), _ptr(labels), float(C), _ptr(w),
                                      _dtype_code(val), threads or default_threads(), ctypes.byref(f), _ptr(g),
                                      _ptr(D))
    if rc != 0:
        raise ValueError(f"oracle_logreg_fgd_csr rc={rc}")
    return f.value, g, D


def logreg_tron_dense(X, labels, C=1.0, eps=1e-3, max_iter=50, max_cg=250, threads=None):
    """TRON (reading R20).  Returns (w, iters, f_history)."""
    X, labels = _np(X), _np(labels)
    m, n = X.shape
    w = np.zeros(n)
    it = ctypes.c_int(0)
    hist = np.full(max_iter + 1, np.nan)
    rc = _lib().oracle_logreg_tron_dense(m, n, _ptr(X), n, _ptr(labels), float(C), float(eps), int(max_iter),
                                         int(max_cg), _dtype_code(X), threads or default_threads(), _ptr(w),
                                         ctypes.byref(it), _ptr(hist))
    if rc != 0:
        raise ValueError(f"oracle_logreg_tron_dense rc={rc}")
    return w, it.value, hist[: it.value + 1]


def logreg_tron_csr(m, n, rowptr, colidx, val, labels, C=1.0, eps=1e-3, max_iter=50, max_cg=250, threads=None):
    rowptr = _np(rowptr).astype(np.int64, copy=False)
    colidx = _np(colidx).astype(np.int32, copy=False)
    val, labels = _np(val), _np(labels)
    w = np.zeros(n)
    it = ctypes.c_int(0)
    hist = np.full(max_iter + 1, np.nan)
    rc = _lib().oracle_logreg_tron_csr(m, n, _ptr(rowptr), _ptr(colidx), _ptr(val), _ptr(labels), float(C),
                                       float(eps), int(max_iter), int(max_cg), _dtype_code(val),
                                       threads or default_threads(), _ptr(w), ctypes.byref(it), _ptr(hist))
    if rc != 0:
        raise ValueError(f"oracle_logreg_tron_csr rc={rc}")
    return w, it.value, hist[: it.value + 1]


def cg_linreg_csr(m, n, rowptr, colidx, val, labels, eps=1e-3, max_iter=100, tol=1e-6, threads=None):
    rowptr = _np(rowptr).astype(np.int64, copy=False)
    colidx = _np(colidx).astype(np.int32, copy=False)
    val, labels = _np(val), _np(labels)
    w = np.zeros(n, np.float64)
    it = ctypes.c_int(0)
    hist = np.zeros(max_iter + 1, np.float64)
    rc = _lib().oracle_cg_linreg_csr(m, n, _ptr(rowptr), _ptr(colidx), _ptr(val), _ptr(labels), float(eps),
                                     int(max_iter), float(tol), _dtype_code(val), threads or default_threads(),
                                     _ptr(w), ctypes.byref(it), _ptr(hist))
    if rc != 0:
        raise ValueError(f"oracle_cg_linreg_csr rc={rc}")
    return w, it.value, hist[: it.value + 1]
