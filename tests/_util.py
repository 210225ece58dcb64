"""Shared test helpers: tolerances (BASELINE.json north_star) and the normwise check."""
import numpy as np
import torch

# north_star: normwise relative error <= 1e-11 (fp64) / 2e-5 (fp32)
TOL = {torch.float64: 1e-11, torch.float32: 2e-5}


def normwise_err(w_gpu, w_ref, mag):
    w = w_gpu.detach().cpu().double().numpy()
    d = np.linalg.norm(w - w_ref)
    den = np.linalg.norm(w_ref)
    if den == 0:
        den = np.linalg.norm(mag)
    if den == 0:
        return float(d)
    return float(d / den)


def assert_parity(w_gpu, w_ref, mag, dtype, what=""):
    w = w_gpu.detach().cpu().double().numpy()
    assert np.all(np.isfinite(w) == np.isfinite(w_ref)), f"{what}: non-finite pattern differs"
    fin = np.isfinite(w_ref)
    err = normwise_err(torch.from_numpy(w[fin]), w_ref[fin], mag[fin])
    assert err <= TOL[dtype], f"{what}: normwise rel err {err:.3e} > {TOL[dtype]:.0e}"
    return err


def assert_bitexact(w_gpu, w_ref, what=""):
    w = w_gpu.detach().cpu().double().numpy()
    bad = np.nonzero(w != w_ref)[0]
    assert bad.size == 0, f"{what}: {bad.size} entries differ, first at {bad[:5]}: {w[bad[:5]]} vs {w_ref[bad[:5]]}"


EXPERIMENTAL_VARIANTS = (10, 12, 14, 15)  # built only with FP_EXPERIMENTAL=1 (Makefile)


def skip_unbuilt(variant):
    """Skip a test of a CSR variant the library was built without (never chosen by the plan)."""
    import pytest

    import paper_conf_ppopp_asharitbrcks15_b200 as fp

    if variant in EXPERIMENTAL_VARIANTS and b"+experimental" not in fp.lib().fp_version():
        pytest.skip(f"variant {variant} is built only with FP_EXPERIMENTAL=1")
