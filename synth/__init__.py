"""Seeded synthetic input generators (shared by tests, the oracle side and bench.py).

Counter-based (synth_core.h): every element is a pure function of (seed, stream, global
index), so host arrays (libsynth_host.so, OpenMP) and device arrays (libsynth_cuda.so)
are bit-identical, and a row shard equals the corresponding slice of the full matrix.
This module computes none of the method's arithmetic.  Recipes per config: DESIGN.md
"Input recipe" (PAPER.md P:411 synthetic CSR at density 0.01, P:465 HIGGS-like dense,
P:427 KDD-like skew).
"""
from __future__ import annotations

import ctypes
import math
import os

import numpy as np
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
_HOST = None
_CUDA = None

F32, F64 = 0, 1
S_X, S_Y, S_V, S_Z, S_LEN, S_COL, S_VAL, S_COLSCALE, S_LABEL, S_AUX = range(1, 11)
KINDS = {"uniform": 0, "pos": 1, "int_pm12": 2, "int_small": 3, "int_pos": 4, "colscaled": 5, "dyadic": 6}
BASE_SEED = 20150207  # PPoPP'15 opening day

i64, u64, vp, ci = ctypes.c_int64, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_int


def _host():
    global _HOST
    if _HOST is None:
        path = os.path.join(_HERE, "libsynth_host.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build()")
        lib = ctypes.CDLL(path)
        lib.synth_dense.argtypes = [i64, i64, i64, i64, ci, ci, u64, u64, vp]
        lib.synth_vector.argtypes = [i64, i64, ci, ci, u64, u64, vp]
        lib.synth_row_lengths.argtypes = [i64, i64, vp, i64, u64, vp]
        lib.synth_rowptr.argtypes = [i64, vp, vp]
        lib.synth_csr_fill.argtypes = [i64, i64, i64, i64, vp, ci, ci, ci, u64, vp, vp]
        lib.synth_fnv1a.argtypes = [vp, i64]
        lib.synth_fnv1a.restype = u64
        _HOST = lib
    return _HOST


def _cuda():
    global _CUDA
    if _CUDA is None:
        path = os.path.join(_HERE, "libsynth_cuda.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build()")
        lib = ctypes.CDLL(path)
        lib.synth_dense_cuda.argtypes = [i64, i64, i64, i64, ci, ci, u64, u64, vp, vp]
        lib.synth_vector_cuda.argtypes = [i64, i64, ci, ci, u64, u64, vp, vp]
        lib.synth_row_lengths_cuda.argtypes = [i64, i64, vp, i64, u64, vp, vp]
        lib.synth_rowptr_cuda.argtypes = [i64, vp, vp, vp, ctypes.POINTER(ctypes.c_size_t), vp]
        lib.synth_csr_fill_cuda.argtypes = [i64, i64, i64, vp, ci, ci, ci, u64, vp, vp, vp]
        _CUDA = lib
    return _CUDA


def _tdt(dtype):
    if dtype in (torch.float64, "f64", np.float64):
        return torch.float64, F64
    if dtype in (torch.float32, "f32", np.float32):
        return torch.float32, F32
    raise TypeError(dtype)


def _stream_ptr(device):
    return ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)


def _check(rc, what):
    if rc != 0:
        raise RuntimeError(f"{what} failed rc={rc}")


def dense(m, n, dtype, kind="uniform", seed=BASE_SEED, stream=S_X, ld=None, device="cpu", row0=0):
    """Rows [row0, row0+m) of the seeded matrix as a row-major (m, ld) tensor; element (r, c) =
    value(hash(seed, stream, r*n+c)) (global r); padding columns (c >= n) are NaN."""
    ld = n if ld is None else ld
    tdt, code = _tdt(dtype)
    out = torch.empty((m, ld), dtype=tdt, device=device)
    if out.is_cuda:
        _check(_cuda().synth_dense_cuda(m, n, ld, row0, code, KINDS[kind], seed, stream, ctypes.c_void_p(out.data_ptr()),
                                        _stream_ptr(out.device)), "synth_dense_cuda")
    else:
        _check(_host().synth_dense(m, n, ld, row0, code, KINDS[kind], seed, stream, ctypes.c_void_p(out.data_ptr())),
               "synth_dense")
    return out


def vector(length, dtype, kind="uniform", seed=BASE_SEED, stream=S_Y, i0=0, device="cpu"):
    tdt, code = _tdt(dtype)
    out = torch.empty((length,), dtype=tdt, device=device)
    if out.is_cuda:
        _check(_cuda().synth_vector_cuda(length, i0, code, KINDS[kind], seed, stream,
                                         ctypes.c_void_p(out.data_ptr()), _stream_ptr(out.device)),
               "synth_vector_cuda")
    else:
        _check(_host().synth_vector(length, i0, code, KINDS[kind], seed, stream, ctypes.c_void_p(out.data_ptr())),
               "synth_vector")
    return out


def length_table(spec, n):
    """Inverse-CDF thresholds (uint64, length lmax+1) for the row-length distribution.

    spec: ("binomial", p)            L ~ Binomial(n, p)               (density p)
          ("powerlaw", a, xmin)      L = min(n, floor(xmin (1-u)^(-1/(a-1))))  (KDD-like skew)
          ("fixed", L)               every row has L entries
          ("uniform", lo, hi)        L ~ U{lo..hi}
    """
    kind = spec[0]
    if kind == "fixed":
        L = int(spec[1])
        cdf = np.zeros(L + 1)
        cdf[L] = 1.0
    elif kind == "uniform":
        lo, hi = int(spec[1]), int(spec[2])
        cdf = np.zeros(hi + 1)
        cdf[lo:] = (np.arange(lo, hi + 1) - lo + 1) / (hi - lo + 1)
    elif kind == "binomial":
        from scipy.stats import binom
        p = float(spec[1])
        cdf = binom.cdf(np.arange(n + 1), n, p)
    elif kind == "powerlaw":
        # optional 4th entry caps the length (min(cap, n)); the table then has cap+1 entries
        a, xmin = float(spec[1]), float(spec[2])
        cap = min(n, int(spec[3])) if len(spec) > 3 else n
        L = np.arange(cap + 1, dtype=np.float64)
        cdf = np.where(L + 1 > xmin, 1.0 - (xmin / (L + 1)) ** (a - 1), 0.0)
    else:
        raise ValueError(spec)
    cdf = np.clip(cdf, 0.0, 1.0)
    thr = (np.floor(cdf * 2.0**53).astype(np.uint64) << np.uint64(11))
    thr[-1] = np.uint64(2**64 - 1)
    thr = np.maximum.accumulate(thr)
    return thr


def csr(m, n, dtype, lengths, kind="uniform", seed=BASE_SEED, row0=0, device="cpu", col_skew=0):
    """CSR (rowptr int64[m+1], colidx int32[nnz], val[nnz]) for rows [row0, row0+m) of the
    seeded matrix.  Columns are distinct and sorted (stratified-uniform, synth_core.h).
    A shard (row0 > 0) is bit-identical to the slice of the full matrix (its val/col hash index
    is the GLOBAL nnz index, found from the row lengths of rows [0, row0)).
    col_skew > 0 draws Zipf-like skewed columns (synth_core.h syn_column_skew, u^(2^col_skew));
    col_skew < 0 draws i.i.d. uniform columns (unsorted, repeats possible: syn_column_iid)."""
    tdt, code = _tdt(dtype)
    thr = length_table(lengths, n)
    lmax = len(thr) - 1
    if lmax > n:
        raise ValueError("row-length table exceeds n")
    nnz0 = 0
    if row0 > 0:
        lens0 = np.empty(row0, np.int64)
        _check(_host().synth_row_lengths(row0, 0, thr.ctypes.data_as(vp), lmax, seed, lens0.ctypes.data_as(vp)),
               "synth_row_lengths")
        nnz0 = int(lens0.sum())
    if str(device).startswith("cuda"):
        dev = torch.device(device)
        lib = _cuda()
        s = _stream_ptr(dev)
        thr_d = torch.from_numpy(thr.view(np.int64)).to(dev)
        lens = torch.empty(m, dtype=torch.int64, device=dev)
        rowptr = torch.empty(m + 1, dtype=torch.int64, device=dev)
        _check(lib.synth_row_lengths_cuda(m, row0, ctypes.c_void_p(thr_d.data_ptr()), lmax, seed,
                                          ctypes.c_void_p(lens.data_ptr()), s), "synth_row_lengths_cuda")
        tb = ctypes.c_size_t(0)
        _check(lib.synth_rowptr_cuda(m, None, None, None, ctypes.byref(tb), s), "synth_rowptr_cuda(query)")
        temp = torch.empty(max(int(tb.value), 1), dtype=torch.uint8, device=dev)
        _check(lib.synth_rowptr_cuda(m, ctypes.c_void_p(lens.data_ptr()), ctypes.c_void_p(rowptr.data_ptr()),
                                     ctypes.c_void_p(temp.data_ptr()), ctypes.byref(tb), s), "synth_rowptr_cuda")
        del lens, temp
        nnz = int(rowptr[-1].item())
        colidx = torch.empty(nnz, dtype=torch.int32, device=dev)
        val = torch.empty(nnz, dtype=tdt, device=dev)
        _check(lib.synth_csr_fill_cuda(m, n, nnz0, ctypes.c_void_p(rowptr.data_ptr()), code, KINDS[kind], col_skew, seed,
                                       ctypes.c_void_p(colidx.data_ptr()), ctypes.c_void_p(val.data_ptr()), s),
               "synth_csr_fill_cuda")
        return rowptr, colidx, val
    lib = _host()
    lens = np.empty(m, np.int64)
    _check(lib.synth_row_lengths(m, row0, thr.ctypes.data_as(vp), lmax, seed, lens.ctypes.data_as(vp)),
           "synth_row_lengths")
    rowptr = np.empty(m + 1, np.int64)
    lib.synth_rowptr(m, lens.ctypes.data_as(vp), rowptr.ctypes.data_as(vp))
    nnz = int(rowptr[-1])
    colidx = np.empty(nnz, np.int32)
    val = np.empty(nnz, np.float64 if code == F64 else np.float32)
    _check(lib.synth_csr_fill(m, n, row0, nnz0, rowptr.ctypes.data_as(vp), code, KINDS[kind], col_skew, seed,
                              colidx.ctypes.data_as(vp), val.ctypes.data_as(vp)), "synth_csr_fill")
    return torch.from_numpy(rowptr), torch.from_numpy(colidx), torch.from_numpy(val)


def fnv1a(t):
    """FNV-1a checksum of a host tensor's bytes."""
    t = t.contiguous()
    if t.is_cuda:
        t = t.cpu()
    return int(_host().synth_fnv1a(ctypes.c_void_p(t.data_ptr()), t.numel() * t.element_size()))


# ---- the benchmark configurations (BASELINE.json configs) -----------------------
CONFIGS = {
    # name: format, dtype, m, n, row-length spec (csr), instance scalars
    "C1": dict(fmt="dense", dtype="f64", m=1000, n=100, alpha=0.75, beta=-1.25, use_v=True, use_z=True,
               xkind="uniform", desc="dense fp64 1000x100 full pattern"),
    "C2": dict(fmt="dense", dtype="f32", m=10_000_000, n=128, alpha=1.0, beta=0.0, use_v=False, use_z=False,
               xkind="uniform", desc="dense fp32 10Mx128, X^T(Xy)"),
    "C3": dict(fmt="csr", dtype="f64", m=20_000_000, n=1000, lengths=("binomial", 0.01), alpha=1.0, beta=1.0,
               use_v=True, use_z=True, xkind="uniform", desc="CSR fp64 20Mx1000 density 0.01, full with v"),
    "C4": dict(fmt="csr", dtype="f32", m=50_000_000, n=100_000, lengths=("powerlaw", 2.5, 13.64), alpha=1.0,
               beta=1.0, use_v=True, use_z=True, xkind="uniform", desc="CSR fp32 50Mx100K power-law, full with v"),
    "C5": dict(fmt="dense", dtype="f64", m=4_000_000, n=1000, alpha=1.0, beta=1e-3, use_v=False, use_z=True,
               xkind="colscaled", desc="dense fp64 4Mx1000 CG iteration X^T(Xp)+eps p"),
    # NEXT rows, not BASELINE.json configs:
    # NEXT-2: KDD2010-shaped ultra-wide CSR (15.0M x 29.9M, 424M nnz at P:419-427): power-law rows of
    # mean ~28, w and y (240 MB fp64) beyond L2 -> the flat L2/HBM-red path.
    "K1": dict(fmt="csr", dtype="f64", m=15_009_374, n=29_890_095, lengths=("powerlaw", 2.5, 9.5, 1_000_000),
               alpha=1.0, beta=1.0, use_v=True, use_z=True, xkind="uniform", col_skew=2,
               desc="CSR fp64 KDD-shaped 15Mx29.9M power-law rows (mean ~28), Zipf-like columns (u^4), full with v"),
    # C3's matrix in fp32 (chooser evidence for fp32 small-n CSR; not a BASELINE.json config)
    "S3": dict(fmt="csr", dtype="f32", m=20_000_000, n=1000, lengths=("binomial", 0.01), alpha=1.0, beta=1.0,
               use_v=True, use_z=True, xkind="uniform", desc="CSR fp32 20Mx1000 density 0.01, full with v"),
    # NEXT-4: dense rows wider than one CTA's registers (thread-block cluster kernel)
    "W1": dict(fmt="dense", dtype="f32", m=40_000, n=65_536, alpha=1.0, beta=0.0, use_v=False, use_z=False,
               xkind="uniform", desc="dense fp32 40000x65536 wide rows, X^T(Xy)"),
}


def config_seed(name):
    return BASE_SEED + int(name[1:])
