"""Full-size parity at BASELINE.json's configs (C1-C5, plus S3 and the KDD-shaped K1), in the
launch configuration bench.py times (same entry point, same plan: the packed copy for CSR) and
through the unpacked chooser plan: the device-generated input is copied to the host and
the fp64 oracle evaluates the whole matrix on the host cores.  fp64 integer twins of C1, C3
and C5 are exact in any summation order and must match bit for bit; the fp32 configs (C2,
C4) are checked against the north_star tolerance."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ppopp_asharitbrcks15_b200 as fp
import synth
from _util import assert_bitexact, assert_parity

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


def gen(name, dev, kind=None):
    cfg = synth.CONFIGS[name]
    seed = synth.config_seed(name)
    m, n, dt = cfg["m"], cfg["n"], cfg["dtype"]
    xk = kind or cfg["xkind"]
    integer = xk.startswith("int")
    d = {}
    if cfg["fmt"] == "dense":
        d["X"] = synth.dense(m, n, dt, kind=xk, seed=seed, device=dev)
    else:
        d["rp"], d["ci"], d["va"] = synth.csr(m, n, dt, cfg["lengths"], kind=xk, seed=seed, device=dev)
    d["y"] = synth.vector(n, dt, kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Y, device=dev)
    d["v"] = synth.vector(m, dt, kind="int_pos" if integer else "pos", seed=seed, stream=synth.S_V,
                          device=dev) if cfg["use_v"] else None
    d["z"] = synth.vector(n, dt, kind="int_small" if integer else "uniform", seed=seed, stream=synth.S_Z,
                          device=dev) if cfg["use_z"] else None
    return cfg, d


def run_gpu(cfg, d):
    if cfg["fmt"] == "dense":
        w = fp.dense(d["X"], d["y"], d["v"], d["z"], cfg["alpha"], cfg["beta"])
    else:
        w = fp.csr(d["rp"], d["ci"], d["va"], cfg["n"], d["y"], d["v"], d["z"], cfg["alpha"], cfg["beta"])
    torch.cuda.synchronize()
    return w.cpu()


def run_oracle(cfg, d):
    h = {k: (None if t is None else t.cpu()) for k, t in d.items()}
    if cfg["fmt"] == "dense":
        return oracle.dense(h["X"], h["y"], h["v"], h["z"], cfg["alpha"], cfg["beta"])
    return oracle.csr(cfg["m"], cfg["n"], h["rp"], h["ci"], h["va"], h["y"], h["v"], h["z"], cfg["alpha"],
                      cfg["beta"])


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
def test_fullsize_parity(cuda_dev, name):
    cfg, d = gen(name, cuda_dev)
    w = run_gpu(cfg, d)
    ref, mag = run_oracle(cfg, d)
    del d
    torch.cuda.empty_cache()
    assert_parity(w, ref, mag, w.dtype, f"{name} full size")


@pytest.mark.parametrize("name", ["C1", "C3", "C5"])
def test_fullsize_integer_twin_bitexact(cuda_dev, name):
    """fp64 configs with integer-valued X, y, v, z: sums stay below 2^53, so every order is
    exact -- any dropped, duplicated or misplaced row/nonzero changes a bit."""
    cfg, d = gen(name, cuda_dev, kind="int_pm12")
    w = run_gpu(cfg, d)
    ref, _ = run_oracle(cfg, d)
    del d
    torch.cuda.empty_cache()
    assert_bitexact(w, ref, f"{name} integer twin")


def run_gpu_packed(cfg, d):
    """bench.py's CSR launch: a plan (fp_csr_plan_create) with its packed copy (fp_csr_plan_pack:
    variant 19's shared-memory column blocks, or variant 20's L2 blocks when n is wider)."""
    plan = fp.CsrPlan(d["rp"], d["ci"], cfg["n"], d["va"].dtype)
    plan.pack(d["va"])
    w = plan(None, d["y"], d["v"], d["z"], cfg["alpha"], cfg["beta"])
    torch.cuda.synchronize()
    return w.cpu(), plan.launch.variant


@pytest.mark.parametrize("name,variant", [("C3", 19), ("C4", 19), ("S3", 19), ("K1", 20)])
def test_fullsize_packed_parity(cuda_dev, name, variant):
    """The packed plans bench.py times, at full size, against the fp64 oracle (north_star
    tolerance); K1 is the KDD-shaped 15M x 29.9M matrix on variant 20."""
    cfg, d = gen(name, cuda_dev)
    w, var = run_gpu_packed(cfg, d)
    assert var == variant
    ref, mag = run_oracle(cfg, d)
    del d
    torch.cuda.empty_cache()
    assert_parity(w, ref, mag, w.dtype, f"{name} packed full size")


@pytest.mark.parametrize("name", ["C3", "K1"])
def test_fullsize_packed_integer_twin_bitexact(cuda_dev, name):
    """fp64 packed plans on integer twins: exact in any order (K1: the hot-column sums stay below
    2^53), so bit-exact against the oracle."""
    cfg, d = gen(name, cuda_dev, kind="int_pm12")
    w, _ = run_gpu_packed(cfg, d)
    ref, _ = run_oracle(cfg, d)
    del d
    torch.cuda.empty_cache()
    assert_bitexact(w, ref, f"{name} packed integer twin")


def test_generator_host_equals_device(cuda_dev):
    """The inputs above are generated on the device; the counter-based generator must give
    the identical bytes on the host (synth_host.c vs synth_cuda.cu)."""
    for dt in ("f32", "f64"):
        for kind in ("uniform", "pos", "int_pm12", "colscaled"):
            a = synth.dense(3001, 77, dt, kind=kind, seed=9, row0=123, ld=80)
            b = synth.dense(3001, 77, dt, kind=kind, seed=9, row0=123, ld=80, device=cuda_dev).cpu()
            assert torch.equal(torch.nan_to_num(a, 7.0), torch.nan_to_num(b, 7.0)), (dt, kind)
        h = synth.csr(20000, 100000, dt, ("powerlaw", 2.5, 13.64), seed=4, row0=777)
        g = synth.csr(20000, 100000, dt, ("powerlaw", 2.5, 13.64), seed=4, row0=777, device=cuda_dev)
        for x, y in zip(h, g):
            assert torch.equal(x, y.cpu())
