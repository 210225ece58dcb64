"""Python binding of libfusedpat (include/fusedpat.h) -- argument marshalling only.

The fused pattern of Ashari et al., PPoPP'15, Eq. (1):

    w = alpha * X^T (v (.) (X y)) + beta * z

Every step runs in the CUDA library (``libfusedpat.so``, sm_100a); this module only turns
torch tensors into pointers/sizes and status codes into exceptions.  PyTorch provides device
memory, streams and process groups.  There is no CPU fallback: importing works without a GPU
(so the ABI can be inspected), but any compute call without a CUDA device fails loudly.

Low-level names mirror the C ABI one to one (``fp_dense``, ``fp_csr``, ``fp_choose`` ...);
the tensor-level helpers ``dense``, ``csr``, ``cg_linreg_*`` and the ``Comm`` class are thin
conveniences over them.
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libfusedpat.so")

FP_F32, FP_F64 = 0, 1
STATUS = {0: "FP_OK", 1: "FP_ERR_INVALID_ARG", 2: "FP_ERR_UNSUPPORTED", 3: "FP_ERR_ALIAS", 4: "FP_ERR_INVALID_CSR",
          5: "FP_ERR_CUDA", 6: "FP_ERR_NCCL", 7: "FP_ERR_NOMEM"}
VARIANTS = {1: "dense_vector", 2: "dense_cta", 3: "csr_vector_smem", 4: "csr_vector_l2", 5: "csr_vector_private",
            6: "csr_flat_smem", 7: "csr_flat_l2", 8: "csr_flat_private", 9: "dense_cluster", 10: "csr_owner",
            11: "csr_vector_fixed", 12: "csr_flat_fixed", 13: "csr_colsplit_cluster",
            14: "csr_stream_smem", 15: "csr_stream_fixed", 16: "csr_flat_l2_wide", 17: "csr_binned",
            18: "csr_flat4_fixed", 19: "csr_packed", 20: "csr_l2block"}


class FusedPatError(RuntimeError):
    def __init__(self, status, where, detail):
        self.status = status
        super().__init__(f"{where}: {STATUS.get(status, status)}: {detail}")


class fp_row_stats(ctypes.Structure):
    _fields_ = [("m", ctypes.c_int64), ("n", ctypes.c_int64), ("nnz", ctypes.c_int64), ("mean", ctypes.c_double),
                ("max_len", ctypes.c_int64), ("min_len", ctypes.c_int64), ("empty_rows", ctypes.c_int64),
                ("hist_log2", ctypes.c_int64 * 64)]


class fp_device_profile(ctypes.Structure):
    _fields_ = [(k, ctypes.c_int) for k in (
        "sm_count", "max_threads_per_sm", "max_threads_per_block", "max_blocks_per_sm", "regs_per_sm",
        "max_regs_per_thread", "reg_alloc_unit", "warp_alloc_granularity", "smem_per_sm", "smem_per_block",
        "smem_alloc_unit", "warp_size")]


class fp_launch(ctypes.Structure):
    _fields_ = [("variant", ctypes.c_int), ("vs", ctypes.c_int), ("bs", ctypes.c_int), ("tl", ctypes.c_int),
                ("grid", ctypes.c_int), ("blocks_per_sm", ctypes.c_int), ("rows_per_vector", ctypes.c_int64),
                ("smem_bytes", ctypes.c_int), ("regs_per_thread", ctypes.c_int), ("concurrent_warps", ctypes.c_int),
                ("cluster", ctypes.c_int)]

    def as_dict(self):
        d = {k: getattr(self, k) for k, _ in self._fields_}
        d["variant_name"] = VARIANTS.get(self.variant, "?")
        return d


_i64, _dbl, _vp, _int = ctypes.c_int64, ctypes.c_double, ctypes.c_void_p, ctypes.c_int
_P = ctypes.POINTER

# name -> (restype, argtypes)
_SIGS = {
    "fp_status_string": (ctypes.c_char_p, [_int]),
    "fp_last_error": (ctypes.c_char_p, []),
    "fp_version": (ctypes.c_char_p, []),
    "fp_dense": (_int, [_i64, _i64, _vp, _i64, _vp, _vp, _vp, _dbl, _dbl, _vp, _int, _vp]),
    "fp_csr": (_int, [_i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _dbl, _dbl, _vp, _int, _vp]),
    "fp_dense_ex": (_int, [_i64, _i64, _vp, _i64, _vp, _vp, _vp, _dbl, _dbl, _vp, _int, _P(fp_launch), _vp]),
    "fp_csr_ex": (_int, [_i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _dbl, _dbl, _vp, _int, _P(fp_launch), _vp]),
    "fp_device_profile_query": (_int, [_int, _P(fp_device_profile)]),
    "fp_device_profile_kepler": (_int, [_P(fp_device_profile)]),
    "fp_row_stats_host": (_int, [_i64, _vp, _P(fp_row_stats)]),
    "fp_row_stats_device": (_int, [_i64, _vp, _P(fp_row_stats), _vp]),
    "fp_row_stats_dense": (_int, [_i64, _i64, _P(fp_row_stats)]),
    "fp_choose_paper": (_int, [_int, _P(fp_row_stats), _int, _P(fp_device_profile), _int, _int, _int, _P(fp_launch)]),
    "fp_choose": (_int, [_int, _P(fp_row_stats), _int, _int, _P(fp_launch)]),
    "fp_csr_validate": (_int, [_i64, _i64, _i64, _vp, _vp, _vp]),
    "fp_csr_plan_create": (_int, [_i64, _i64, _i64, _vp, _vp, _int, _P(fp_launch), _P(_vp), _vp]),
    "fp_csr_plan_exec": (_int, [_vp, _vp, _vp, _vp, _vp, _dbl, _dbl, _vp, _vp]),
    "fp_csr_plan_launch": (_int, [_vp, _P(fp_launch)]),
    "fp_csr_plan_destroy": (_int, [_vp]),
    "fp_csr_plan_pack": (_int, [_vp, _vp, _vp]),
    "fp_csr_plan_dist": (_int, [_vp, _vp, _vp, _vp, _vp, _vp, _dbl, _dbl, _vp, _vp]),
    "fp_csr_plan_pack_info": (_int, [_vp, _P(_i64), _P(_i64), _P(_int), _P(_int)]),
    "fp_csr_plan_pack_detail": (_int, [_vp, _P(_i64)]),
    "fp_dense_host": (_int, [_i64, _i64, _vp, _i64, _vp, _vp, _vp, _dbl, _dbl, _vp, _int, _int]),
    "fp_csr_host": (_int, [_i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _dbl, _dbl, _vp, _int, _int]),
    "fp_release_workspace": (_int, []),
    "fp_probe_rates": (_int, [_i64, _i64, _vp, _vp]),
    "fp_comm_get_unique_id": (_int, [_vp]),
    "fp_comm_init": (_int, [_P(_vp), _int, _int, _vp, _int]),
    "fp_comm_destroy": (_int, [_vp]),
    "fp_comm_rank": (_int, [_vp]),
    "fp_comm_size": (_int, [_vp]),
    "fp_allreduce": (_int, [_vp, _vp, _i64, _int, _vp]),
    "fp_comm_enable_peer": (_int, [_vp, _i64, _vp]),
    "fp_comm_enable_nvls": (_int, [_vp, _i64, _vp]),
    "fp_comm_set_mode": (_int, [_vp, _int]),
    "fp_comm_mode": (_int, [_vp]),
    "fp_comm_init_local_group": (_int, [_int, _int, _i64, _vp]),
    "fp_comm_timed_out": (_int, [_vp]),
    "fp_shard_rows_dense": (_int, [_i64, _int, _vp]),
    "fp_shard_rows_csr": (_int, [_i64, _vp, _int, _vp]),
    "fp_dense_dist": (_int, [_i64, _i64, _vp, _i64, _vp, _vp, _vp, _dbl, _dbl, _vp, _int, _vp, _vp]),
    "fp_csr_dist": (_int, [_i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _dbl, _dbl, _vp, _int, _vp, _vp]),
    "fp_dense_epi": (_int, [_i64, _i64, _vp, _i64, _vp, _vp, _vp, _dbl, _dbl, _vp, _int, _int, _dbl, _vp, _vp, _vp]),
    "fp_csr_epi": (_int, [_i64, _i64, _i64, _vp, _vp, _vp, _vp, _vp, _vp, _dbl, _dbl, _vp, _int, _int, _dbl, _vp, _vp,
                          _vp]),
    "fp_logreg_tron_dense": (_int, [_i64, _i64, _vp, _i64, _vp, _dbl, _dbl, _int, _int, _vp, _P(_int), _vp, _int, _vp,
                                    _vp]),
    "fp_logreg_tron_csr": (_int, [_i64, _i64, _i64, _vp, _vp, _vp, _vp, _dbl, _dbl, _int, _int, _vp, _P(_int), _vp,
                                  _int, _vp, _vp]),
    "fp_cg_linreg_dense": (_int, [_i64, _i64, _vp, _i64, _vp, _dbl, _int, _dbl, _vp, _P(_int), _vp, _int, _vp, _vp]),
    "fp_cg_linreg_csr": (_int, [_i64, _i64, _i64, _vp, _vp, _vp, _vp, _dbl, _int, _dbl, _vp, _P(_int), _vp, _int, _vp,
                                _vp]),
}

_lib = None


def lib():
    """Load libfusedpat.so (raises if it was not built -- there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: build it with __graft_entry__.build() (or `make fusedpat`)")
        L = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_GLOBAL)
        for name, (res, args) in _SIGS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def exported_symbols():
    return sorted(_SIGS)


def _check(status, where):
    if status != 0:
        detail = lib().fp_last_error().decode(errors="replace")
        raise FusedPatError(status, where, detail)


def _call(name, *args):
    _check(getattr(lib(), name)(*args), name)


# expose the raw C functions under their C names (checked: raise FusedPatError on failure)
def _make_raw(name):
    def f(*args):
        r = getattr(lib(), name)(*args)
        if _SIGS[name][0] is _int and name not in ("fp_comm_rank", "fp_comm_size", "fp_comm_mode",
                                                    "fp_comm_timed_out"):
            _check(r, name)
        return r
    f.__name__ = name
    f.__doc__ = f"Checked ctypes call of the C ABI function {name} (include/fusedpat.h)."
    return f


for _n in _SIGS:
    globals()[_n] = _make_raw(_n)


# ------------------------------------------------------------------------------- tensor level
def _dt(t):
    if t.dtype == torch.float64:
        return FP_F64
    if t.dtype == torch.float32:
        return FP_F32
    raise TypeError(f"unsupported dtype {t.dtype} (float32 / float64)")


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream(device, stream=None):
    if stream is not None:
        return ctypes.c_void_p(stream.cuda_stream)
    return ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)


def _require_cuda(*ts):
    for t in ts:
        if t is not None and not t.is_cuda:
            raise ValueError("libfusedpat device entry points take CUDA tensors (use fp_*_host for host buffers)")


def _vec(t, length, dtype, name):
    if t is None:
        return None
    if t.dim() != 1 or t.shape[0] != length or t.dtype != dtype or not t.is_contiguous():
        raise ValueError(f"{name} must be a contiguous 1-D {dtype} tensor of length {length}")
    return t


def dense(X, y=None, v=None, z=None, alpha=1.0, beta=0.0, w=None, launch=None, stream=None):
    """w = alpha X^T (v (.) (X y)) + beta z for a dense row-major X (m x n, row stride >= n).
    y=None selects alpha X^T v (Table 1 row 1); v=None means v = 1; returns w."""
    _require_cuda(X, y, v, z, w)
    if X.dim() != 2 or X.stride(1) != 1:
        raise ValueError("X must be 2-D row-major (stride(1) == 1)")
    m, n = X.shape
    ld = X.stride(0) if m > 1 else n
    y, v, z = _vec(y, n, X.dtype, "y"), _vec(v, m, X.dtype, "v"), _vec(z, n, X.dtype, "z")
    if w is None:
        w = torch.empty(n, dtype=X.dtype, device=X.device)
    _vec(w, n, X.dtype, "w")
    s = _stream(X.device, stream)
    if launch is None:
        _call("fp_dense", m, n, _ptr(X), ld, _ptr(y), _ptr(v), _ptr(z), float(alpha), float(beta), _ptr(w), _dt(X), s)
    else:
        _call("fp_dense_ex", m, n, _ptr(X), ld, _ptr(y), _ptr(v), _ptr(z), float(alpha), float(beta), _ptr(w), _dt(X),
              ctypes.byref(launch), s)
    return w


def csr(rowptr, colidx, val, n, y=None, v=None, z=None, alpha=1.0, beta=0.0, w=None, launch=None, stream=None):
    """CSR variant: rowptr int64[m+1], colidx int32[nnz], val[nnz]."""
    _require_cuda(rowptr, colidx, val, y, v, z, w)
    if rowptr.dtype != torch.int64 or colidx.dtype != torch.int32:
        raise TypeError("rowptr must be int64 and colidx int32")
    m = rowptr.shape[0] - 1
    nnz = val.shape[0]
    y, v, z = _vec(y, n, val.dtype, "y"), _vec(v, m, val.dtype, "v"), _vec(z, n, val.dtype, "z")
    if w is None:
        w = torch.empty(n, dtype=val.dtype, device=val.device)
    _vec(w, n, val.dtype, "w")
    s = _stream(val.device, stream)
    args = (m, n, nnz, _ptr(rowptr), _ptr(colidx), _ptr(val), _ptr(y), _ptr(v), _ptr(z), float(alpha), float(beta),
            _ptr(w), _dt(val))
    if launch is None:
        _call("fp_csr", *args, s)
    else:
        _call("fp_csr_ex", *args, ctypes.byref(launch), s)
    return w


class CsrPlan:
    """fp_csr_plan: the once-per-matrix analysis of a CSR structure (launch parameters and, for
    wide n, the column split of the cluster kernel).  Keeps rowptr/colidx alive; the structure
    must not change while the plan is used.  ``plan(val, y, v, z, alpha, beta, w)`` evaluates
    Eq. (1) on the plan's matrix."""

    def __init__(self, rowptr, colidx, n, dtype, launch=None, stream=None):
        _require_cuda(rowptr, colidx)
        if rowptr.dtype != torch.int64 or colidx.dtype != torch.int32:
            raise TypeError("rowptr must be int64 and colidx int32")
        self.rowptr, self.colidx, self.n = rowptr, colidx, int(n)
        self.m, self.nnz = rowptr.shape[0] - 1, colidx.shape[0]
        self.dtype = dtype
        self._h = ctypes.c_void_p()
        fdt = FP_F64 if dtype == torch.float64 else FP_F32
        _call("fp_csr_plan_create", self.m, self.n, self.nnz, _ptr(rowptr), _ptr(colidx), fdt,
              None if launch is None else ctypes.byref(launch), ctypes.byref(self._h), _stream(rowptr.device, stream))

    @property
    def launch(self):
        L = fp_launch()
        _call("fp_csr_plan_launch", self._h, ctypes.byref(L))
        return L

    def pack(self, val, stream=None):
        """fp_csr_plan_pack: the column-blocked copy of the matrix with values ``val`` (variant 19, or
        variant 20's L2-sized column blocks when n is too wide for shared-memory blocks);
        afterwards ``plan(None, y, ...)`` evaluates Eq. (1) on the copy."""
        _require_cuda(val)
        if val.dtype != self.dtype or val.shape[0] != self.nnz:
            raise ValueError(f"val must be {self.dtype}[{self.nnz}]")
        _call("fp_csr_plan_pack", self._h, _ptr(val), _stream(val.device, stream))
        self._packed_dev = val.device

    @property
    def pack_info(self):
        nt, ne, cs, gr = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int(), ctypes.c_int()
        _call("fp_csr_plan_pack_info", self._h, ctypes.byref(nt), ctypes.byref(ne), ctypes.byref(cs),
              ctypes.byref(gr))
        return {"tiles": nt.value, "entries": ne.value, "blocks": cs.value, "groups": gr.value}

    @property
    def pack_detail(self):
        """fp_csr_plan_pack_detail: what one exec of the packed copy does (the roofline's inputs)."""
        out = (ctypes.c_int64 * 8)()
        _call("fp_csr_plan_pack_detail", self._h, out)
        keys = ("variant", "blocks", "fused_block", "hot_columns", "hot_entries", "entries_streamed",
                "launches", "reserved")
        return dict(zip(keys, (int(x) for x in out)))

    def __call__(self, val, y=None, v=None, z=None, alpha=1.0, beta=0.0, w=None, stream=None):
        """Eq. (1) on the plan's matrix with values ``val``; ``val=None`` uses the packed copy."""
        _require_cuda(val, y, v, z, w)
        if val is not None and (val.dtype != self.dtype or val.shape[0] != self.nnz):
            raise ValueError(f"val must be {self.dtype}[{self.nnz}]")
        dev = val.device if val is not None else self.rowptr.device
        y, v, z = _vec(y, self.n, self.dtype, "y"), _vec(v, self.m, self.dtype, "v"), _vec(z, self.n, self.dtype, "z")
        if w is None:
            w = torch.empty(self.n, dtype=self.dtype, device=dev)
        _vec(w, self.n, self.dtype, "w")
        _call("fp_csr_plan_exec", self._h, _ptr(val), _ptr(y), _ptr(v), _ptr(z), float(alpha), float(beta), _ptr(w),
              _stream(dev, stream))
        return w

    def dist(self, comm, val, y=None, v=None, z=None, alpha=1.0, beta=0.0, w=None, stream=None):
        """fp_csr_plan_dist: this plan is the rank's row shard; every rank gets the full w
        (``val=None``: the packed copy)."""
        _require_cuda(val, y, v, z, w)
        dev = val.device if val is not None else self.rowptr.device
        y, v, z = _vec(y, self.n, self.dtype, "y"), _vec(v, self.m, self.dtype, "v"), _vec(z, self.n, self.dtype, "z")
        if w is None:
            w = torch.empty(self.n, dtype=self.dtype, device=dev)
        _vec(w, self.n, self.dtype, "w")
        _call("fp_csr_plan_dist", self._h, comm.handle, _ptr(val), _ptr(y), _ptr(v), _ptr(z), float(alpha), float(beta),
              _ptr(w), _stream(dev, stream))
        return w

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            lib().fp_csr_plan_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def dense_host(X, y=None, v=None, z=None, alpha=1.0, beta=0.0, w=None, device=0):
    """Host-buffer entry (fp_dense_host): X, y, v, z, w are CPU tensors; rows stream through HBM."""
    for t in (X, y, v, z, w):
        if t is not None and t.is_cuda:
            raise ValueError("fp_dense_host takes host tensors")
    m, n = X.shape
    ld = X.stride(0) if m > 1 else n
    if w is None:
        w = torch.empty(n, dtype=X.dtype)
    _call("fp_dense_host", m, n, _ptr(X), ld, _ptr(y), _ptr(v), _ptr(z), float(alpha), float(beta), _ptr(w), _dt(X),
          int(device))
    return w


def csr_host(rowptr, colidx, val, n, y=None, v=None, z=None, alpha=1.0, beta=0.0, w=None, device=0):
    m = rowptr.shape[0] - 1
    if w is None:
        w = torch.empty(n, dtype=val.dtype)
    _call("fp_csr_host", m, n, val.shape[0], _ptr(rowptr), _ptr(colidx), _ptr(val), _ptr(y), _ptr(v), _ptr(z),
          float(alpha), float(beta), _ptr(w), _dt(val), int(device))
    return w


# ------------------------------------------------------------------------------- chooser
def row_stats_host(rowptr):
    st = fp_row_stats()
    rp = rowptr.detach().cpu().contiguous()
    _call("fp_row_stats_host", rp.shape[0] - 1, _ptr(rp), ctypes.byref(st))
    return st


def row_stats_device(rowptr, stream=None):
    st = fp_row_stats()
    _call("fp_row_stats_device", rowptr.shape[0] - 1, _ptr(rowptr), ctypes.byref(st), _stream(rowptr.device, stream))
    return st


def row_stats_dense(m, n):
    st = fp_row_stats()
    _call("fp_row_stats_dense", m, n, ctypes.byref(st))
    return st


def kepler_profile():
    p = fp_device_profile()
    _call("fp_device_profile_kepler", ctypes.byref(p))
    return p


def device_profile(device=0):
    p = fp_device_profile()
    _call("fp_device_profile_query", int(device), ctypes.byref(p))
    return p


def choose_paper(is_csr, stats, dtype, profile, regs_per_thread=43, regs_dense_tl1=23, regs_dense_tl40=255):
    """The paper's analytical model (Section 3.3) -- defaults are its profiled register counts."""
    L = fp_launch()
    _call("fp_choose_paper", int(bool(is_csr)), ctypes.byref(stats), dtype, ctypes.byref(profile),
          int(regs_per_thread), int(regs_dense_tl1), int(regs_dense_tl40), ctypes.byref(L))
    return L


def choose(is_csr, stats, dtype, device=0):
    """The B200 plan the kernels launch."""
    L = fp_launch()
    _call("fp_choose", int(bool(is_csr)), ctypes.byref(stats), dtype, int(device), ctypes.byref(L))
    return L


def csr_validate(rowptr, colidx, n, stream=None):
    _call("fp_csr_validate", rowptr.shape[0] - 1, n, colidx.shape[0], _ptr(rowptr), _ptr(colidx),
          _stream(rowptr.device, stream))


# ------------------------------------------------------------------------------- multi-GPU
def shard_rows_dense(m, nranks):
    b = (ctypes.c_int64 * (nranks + 1))()
    _call("fp_shard_rows_dense", m, nranks, ctypes.cast(b, ctypes.c_void_p))
    return list(b)


def shard_rows_csr(rowptr_host, nranks):
    rp = rowptr_host.detach().cpu().contiguous()
    if rp.dtype != torch.int64:
        raise TypeError("rowptr must be int64")
    b = (ctypes.c_int64 * (nranks + 1))()
    _call("fp_shard_rows_csr", rp.shape[0] - 1, _ptr(rp), nranks, ctypes.cast(b, ctypes.c_void_p))
    return list(b)


class Comm:
    """NCCL communicator owned by libfusedpat, bootstrapped through torch.distributed:
    rank 0 creates the 128-byte unique id, broadcast_object_list ships it to every rank."""

    def __init__(self, device=None, group=None):
        import torch.distributed as dist

        self.rank, self.size = dist.get_rank(group), dist.get_world_size(group)
        self.device = torch.cuda.current_device() if device is None else int(device)
        uid = (ctypes.c_ubyte * 128)()
        if self.rank == 0:
            _call("fp_comm_get_unique_id", ctypes.cast(uid, ctypes.c_void_p))
        obj = [bytes(uid)]
        dist.broadcast_object_list(obj, src=0, group=group)
        uid = (ctypes.c_ubyte * 128).from_buffer_copy(obj[0])
        h = ctypes.c_void_p()
        _call("fp_comm_init", ctypes.byref(h), self.size, self.rank, ctypes.cast(uid, ctypes.c_void_p), self.device)
        self.handle = h

    def close(self):
        if self.handle:
            _call("fp_comm_destroy", self.handle)
            self.handle = None

    def allreduce(self, t, stream=None):
        _call("fp_allreduce", self.handle, _ptr(t), t.numel(), _dt(t), _stream(t.device, stream))
        return t

    def timed_out(self):
        """fp_comm_timed_out: True if a peer / NVLS barrier of this communicator gave up waiting."""
        return lib().fp_comm_timed_out(self.handle) == 1

    def enable_peer(self, max_bytes, stream=None):
        """Collective: switch this communicator to the fused peer-memory exchange
        (FP_COMM_PEER, include/fusedpat.h) for vectors of up to max_bytes."""
        _call("fp_comm_enable_peer", self.handle, int(max_bytes), _stream(torch.device("cuda", self.device), stream))

    def enable_nvls(self, max_bytes, stream=None):
        """Collective: switch to the NVSwitch multicast exchange (FP_COMM_NVLS)."""
        _call("fp_comm_enable_nvls", self.handle, int(max_bytes), _stream(torch.device("cuda", self.device), stream))

    def set_mode(self, mode):
        _call("fp_comm_set_mode", self.handle, int(mode))

    @property
    def mode(self):
        return lib().fp_comm_mode(self.handle)


FP_COMM_NCCL, FP_COMM_PEER, FP_COMM_NVLS = 0, 1, 2


def probe_rates(n, smem_elems=1000, device=None):
    """fp_probe_rates: live random-access throughputs (ops/s) -- gather_l2, red_l2, atom_smem_u32,
    atom_smem_f64, gather_smem_f64 (include/fusedpat.h)."""
    r = (ctypes.c_double * 5)()
    dev = torch.device("cuda", torch.cuda.current_device() if device is None else device)
    _call("fp_probe_rates", int(n), int(smem_elems), ctypes.cast(r, ctypes.c_void_p), _stream(dev, None))
    return dict(zip(("gather_l2", "red_l2", "atom_smem_u32", "atom_smem_f64", "gather_smem_f64"), list(r)))


class LocalGroup:
    """fp_comm_init_local_group: `nranks` peer-exchange communicators on ONE device (a single
    process, no NCCL) -- the same fused exchange as across GPUs, between plain allocations.
    Drive the ranks concurrently (one host thread per rank): a rank's call returns once every
    rank reached its exchange (they meet on the host; no kernel waits for another rank's launch)."""

    def __init__(self, nranks, device=0, max_bytes=1 << 22):
        arr = (ctypes.c_void_p * nranks)()
        _call("fp_comm_init_local_group", int(nranks), int(device), int(max_bytes), ctypes.cast(arr, ctypes.c_void_p))
        self.comms = []
        for r in range(nranks):
            c = Comm.__new__(Comm)
            c.rank, c.size, c.device, c.handle = r, nranks, int(device), ctypes.c_void_p(arr[r])
            self.comms.append(c)

    def timed_out(self):
        return any(lib().fp_comm_timed_out(c.handle) == 1 for c in self.comms)

    def close(self):
        for c in self.comms:
            c.close()


def dense_dist(comm, X_local, y=None, v_local=None, z=None, alpha=1.0, beta=0.0, w=None, stream=None):
    m, n = X_local.shape
    ld = X_local.stride(0) if m > 1 else n
    if w is None:
        w = torch.empty(n, dtype=X_local.dtype, device=X_local.device)
    _call("fp_dense_dist", m, n, _ptr(X_local), ld, _ptr(y), _ptr(v_local), _ptr(z), float(alpha), float(beta),
          _ptr(w), _dt(X_local), comm.handle, _stream(X_local.device, stream))
    return w


def csr_dist(comm, rowptr_local, colidx_local, val_local, n, y=None, v_local=None, z=None, alpha=1.0, beta=0.0,
             w=None, stream=None):
    m = rowptr_local.shape[0] - 1
    if w is None:
        w = torch.empty(n, dtype=val_local.dtype, device=val_local.device)
    _call("fp_csr_dist", m, n, val_local.shape[0], _ptr(rowptr_local), _ptr(colidx_local), _ptr(val_local), _ptr(y),
          _ptr(v_local), _ptr(z), float(alpha), float(beta), _ptr(w), _dt(val_local), comm.handle,
          _stream(val_local.device, stream))
    return w


# ------------------------------------------------------------------------------- drivers
def cg_linreg_dense(X, labels, eps=1e-3, max_iter=100, tol=1e-6, comm=None, stream=None):
    """Listing 1 with the fused op.  Returns (w, iters, nr2_history)."""
    _require_cuda(X, labels)
    m, n = X.shape
    ld = X.stride(0) if m > 1 else n
    w = torch.empty(n, dtype=X.dtype, device=X.device)
    it = ctypes.c_int(0)
    hist = torch.zeros(max_iter + 1, dtype=torch.float64)
    _call("fp_cg_linreg_dense", m, n, _ptr(X), ld, _ptr(labels), float(eps), int(max_iter), float(tol), _ptr(w),
          ctypes.byref(it), _ptr(hist), _dt(X), comm.handle if comm else None, _stream(X.device, stream))
    return w, it.value, hist[: it.value + 1]


def cg_linreg_csr(rowptr, colidx, val, n, labels, eps=1e-3, max_iter=100, tol=1e-6, comm=None, stream=None):
    _require_cuda(rowptr, colidx, val, labels)
    m = rowptr.shape[0] - 1
    w = torch.empty(n, dtype=val.dtype, device=val.device)
    it = ctypes.c_int(0)
    hist = torch.zeros(max_iter + 1, dtype=torch.float64)
    _call("fp_cg_linreg_csr", m, n, val.shape[0], _ptr(rowptr), _ptr(colidx), _ptr(val), _ptr(labels), float(eps),
          int(max_iter), float(tol), _ptr(w), ctypes.byref(it), _ptr(hist), _dt(val), comm.handle if comm else None,
          _stream(val.device, stream))
    return w, it.value, hist[: it.value + 1]


# ------------------------------------------------------------------------------- host sharding
def shard_slice_csr(rowptr, colidx, val, v, bounds, rank):
    """Rank `rank`'s rows [bounds[rank], bounds[rank+1]) of a CSR matrix: rowptr rebased to 0,
    colidx/val/v sliced (views where possible).  Pure host/tensor indexing, no arithmetic of
    the method."""
    r0, r1 = int(bounds[rank]), int(bounds[rank + 1])
    a, b = int(rowptr[r0]), int(rowptr[r1])
    rp = rowptr[r0:r1 + 1] - a
    return rp, colidx[a:b], val[a:b], (None if v is None else v[r0:r1])


# ------------------------------------------------------------------------------- row epilogues
FP_EPI_LINEAR, FP_EPI_LOGISTIC = 0, 1


def dense_epi(X, y, v, z, alpha, beta, epilogue, c=1.0, row_out=None, scalar_out=None, w=None, stream=None):
    """fp_dense_epi: the fused pass with a row epilogue (see include/fusedpat.h)."""
    _require_cuda(X, y, v, z, w, row_out, scalar_out)
    m, n = X.shape
    ld = X.stride(0) if m > 1 else n
    if w is None:
        w = torch.empty(n, dtype=X.dtype, device=X.device)
    _call("fp_dense_epi", m, n, _ptr(X), ld, _ptr(y), _ptr(v), _ptr(z), float(alpha), float(beta), _ptr(w), _dt(X),
          int(epilogue), float(c), _ptr(row_out), _ptr(scalar_out), _stream(X.device, stream))
    return w


def csr_epi(rowptr, colidx, val, n, y, v, z, alpha, beta, epilogue, c=1.0, row_out=None, scalar_out=None, w=None,
            stream=None):
    _require_cuda(rowptr, colidx, val, y, v, z, w, row_out, scalar_out)
    m = rowptr.shape[0] - 1
    if w is None:
        w = torch.empty(n, dtype=val.dtype, device=val.device)
    _call("fp_csr_epi", m, n, val.shape[0], _ptr(rowptr), _ptr(colidx), _ptr(val), _ptr(y), _ptr(v), _ptr(z),
          float(alpha), float(beta), _ptr(w), _dt(val), int(epilogue), float(c), _ptr(row_out), _ptr(scalar_out),
          _stream(val.device, stream))
    return w


def logreg_tron_dense(X, labels, C=1.0, eps=1e-3, max_iter=50, max_cg=250, comm=None, stream=None):
    """TRON logistic regression (reading R20).  Returns (w, iters, f_history)."""
    _require_cuda(X, labels)
    m, n = X.shape
    ld = X.stride(0) if m > 1 else n
    w = torch.empty(n, dtype=X.dtype, device=X.device)
    it = ctypes.c_int(0)
    hist = torch.full((max_iter + 1,), float("nan"), dtype=torch.float64)
    _call("fp_logreg_tron_dense", m, n, _ptr(X), ld, _ptr(labels), float(C), float(eps), int(max_iter), int(max_cg),
          _ptr(w), ctypes.byref(it), _ptr(hist), _dt(X), comm.handle if comm else None, _stream(X.device, stream))
    return w, it.value, hist[: it.value + 1]


def logreg_tron_csr(rowptr, colidx, val, n, labels, C=1.0, eps=1e-3, max_iter=50, max_cg=250, comm=None,
                    stream=None):
    _require_cuda(rowptr, colidx, val, labels)
    m = rowptr.shape[0] - 1
    w = torch.empty(n, dtype=val.dtype, device=val.device)
    it = ctypes.c_int(0)
    hist = torch.full((max_iter + 1,), float("nan"), dtype=torch.float64)
    _call("fp_logreg_tron_csr", m, n, val.shape[0], _ptr(rowptr), _ptr(colidx), _ptr(val), _ptr(labels), float(C),
          float(eps), int(max_iter), int(max_cg), _ptr(w), ctypes.byref(it), _ptr(hist), _dt(val),
          comm.handle if comm else None, _stream(val.device, stream))
    return w, it.value, hist[: it.value + 1]
