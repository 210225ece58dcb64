"""Generator self-checks (host side): determinism, shard == slice, structure, distributions."""
import numpy as np
import pytest
import torch

import synth


def test_dense_deterministic_and_padding_nan():
    a = synth.dense(50, 7, "f64", ld=9, seed=3)
    b = synth.dense(50, 7, "f64", ld=9, seed=3)
    assert torch.equal(a[:, :7], b[:, :7])
    assert torch.isnan(a[:, 7:]).all()
    assert (a[:, :7].abs() <= 1).all()
    c = synth.dense(50, 7, "f32", seed=3)
    assert c.dtype == torch.float32 and (c.abs() <= 1).all()


def test_value_kinds_exact_ranges():
    v = synth.vector(100000, "f64", kind="pos", seed=1).numpy()
    assert v.min() > 0 and v.max() <= 0.25
    i = synth.vector(10000, "f32", kind="int_pm12", seed=1).numpy()
    assert set(np.unique(i)) == {-2.0, -1.0, 1.0, 2.0}
    s = synth.vector(10000, "f64", kind="int_small", seed=1).numpy()
    assert set(np.unique(s)) == set(range(-3, 4))
    u = synth.vector(200000, "f64", kind="uniform", seed=2).numpy()
    assert -1 <= u.min() and u.max() < 1 and abs(u.mean()) < 0.01


@pytest.mark.parametrize("spec,n,mean", [(("binomial", 0.01), 1000, 10.0), (("powerlaw", 2.5, 13.64), 100000, 40.0),
                                         (("fixed", 5), 20, 5.0), (("uniform", 0, 6), 50, 3.0)])
def test_csr_structure(spec, n, mean):
    m = 20000
    rp, ci, va = synth.csr(m, n, "f32", spec, seed=5)
    rp, ci = rp.numpy(), ci.numpy()
    lens = np.diff(rp)
    assert rp[0] == 0 and np.all(lens >= 0)
    assert abs(lens.mean() - mean) / mean < 0.06
    assert ci.min() >= 0 and ci.max() < n
    for r in range(0, m, 997):                     # sorted, distinct
        row = ci[rp[r]:rp[r + 1]]
        assert np.all(np.diff(row) > 0)


def test_powerlaw_tail_shape():
    """SURVEY 8(d) C4 recipe: ~26.6% of rows > 32 holding ~64% of nnz; min length 13."""
    rp, _, _ = synth.csr(200000, 100000, "f32", ("powerlaw", 2.5, 13.64), seed=9)
    lens = np.diff(rp.numpy())
    assert lens.min() == 13
    big = lens > 32
    assert 0.24 < big.mean() < 0.29
    assert 0.58 < lens[big].sum() / lens.sum() < 0.70


def test_shard_equals_slice():
    m, n = 3000, 200
    rp, ci, va = synth.csr(m, n, "f64", ("binomial", 0.05), seed=11)
    r0, r1 = 1234, 2500
    srp, sci, sva = synth.csr(r1 - r0, n, "f64", ("binomial", 0.05), seed=11, row0=r0)
    a, b = int(rp[r0]), int(rp[r1])
    assert torch.equal(srp, rp[r0:r1 + 1] - a)
    assert torch.equal(sci, ci[a:b]) and torch.equal(sva, va[a:b])


def test_fnv_checksum_stable():
    x = synth.vector(1000, "f64", seed=1)
    assert synth.fnv1a(x) == synth.fnv1a(x.clone())


def test_skewed_columns_sorted_distinct_and_skewed():
    m, n = 5000, 1_000_000
    rp, ci, _ = synth.csr(m, n, "f32", ("powerlaw", 2.5, 9.5, 100000), seed=3, col_skew=2)
    rp, ci = rp.numpy(), ci.numpy()
    for r in range(0, m, 97):
        row = ci[rp[r]:rp[r + 1]]
        assert np.all(np.diff(row) > 0) and row.min() >= 0 and row.max() < n
    # popularity decreases with the column index: the first 1 % of columns take far more than 1 %
    assert (ci < n // 100).mean() > 0.2
