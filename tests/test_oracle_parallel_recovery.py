"""Parallel recovery oracle (P:457 on Eq. 2) pinned to the sequential
replay: bit-exact where every sum is exact in fp32, within BASELINE's fp32 tolerance otherwise."""
import numpy as np
import pytest

import oracle
from oracle import parallel_recovery as pr


def chain(n, R, B, nnz, lr, seed, dyadic=False, t0=0):
    rng = np.random.default_rng(seed)
    recs = []
    for q in range(R):
        diffs = []
        for _ in range(B):
            idx = np.sort(rng.choice(n, nnz, replace=False)).astype(np.uint32)
            if dyadic:     # small multiples of 2^-8: every fp32 sum and product below is exact
                val = (rng.integers(-64, 65, nnz) / 256.0).astype(np.float32)
            else:
                val = rng.standard_normal(nnz).astype(np.float32) * np.float32(1e-2)
            diffs.append((idx, val))
        recs.append(oracle.batch_merge(diffs, np.float32(lr), oracle.SUM, n, 0, n, t0 + q * B, 1))
    return recs


def sequential(x, recs, n):
    st = {"x": x.copy(), "m": None, "v": None, "n": n, "lo": 0, "hi": n, "t": 0, "adam_step": 0,
          "momentum_initialized": 0}
    oracle.replay({"kind": "sgd"}, st, recs)
    return st


@pytest.mark.parametrize("R", [1, 2, 5, 9])
def test_exact_when_sums_are_exact(R):
    n = 5000
    recs = chain(n, R, 3, 400, 2.0 ** -4, seed=R, dyadic=True)
    x = (np.random.default_rng(0).integers(-512, 513, n) / 1024.0).astype(np.float32)
    par = {"x": x.copy(), "lo": 0, "hi": n, "t": 0}
    pr.replay_parallel(par, recs)
    seq = sequential(x, recs, n)
    assert np.array_equal(par["x"].view(np.uint32), seq["x"].view(np.uint32))
    assert par["t"] == seq["t"] == 3 * R


@pytest.mark.parametrize("R", [2, 8, 32])
def test_within_tolerance_of_sequential(R):
    n = 20000
    recs = chain(n, R, 4, 800, 0.1, seed=100 + R)
    x = (np.random.default_rng(1).standard_normal(n) * 0.05).astype(np.float32)
    par = {"x": x.copy(), "lo": 0, "hi": n, "t": 0}
    pr.replay_parallel(par, recs)
    seq = sequential(x, recs, n)
    np.testing.assert_allclose(par["x"], seq["x"], rtol=1e-6, atol=1e-7)
    touched = np.unique(np.concatenate([oracle.parse_record(r)["idx"] for r in recs]))
    untouched = np.setdiff1d(np.arange(n), touched)
    assert np.array_equal(par["x"][untouched], x[untouched])     # C^F untouched off the union


def test_rejects_non_constant_lr():
    n = 1000
    r1 = chain(n, 1, 2, 50, 0.1, seed=1)[0]
    r2 = chain(n, 1, 2, 50, 0.2, seed=2, t0=2)[0]
    with pytest.raises(AssertionError):
        pr.replay_parallel({"x": np.zeros(n, np.float32), "lo": 0, "hi": n, "t": 0}, [r1, r2])
