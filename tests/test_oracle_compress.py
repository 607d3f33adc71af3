"""Pins of oracle O1 (compress = exact top-k of |g + r| with error feedback).

Comp(G_{i,t}) is Alg.1 line 4; the paper's operator is "sparsification"
 at ratio rho. Top-k by magnitude with ties to the lower index and the
error-feedback residual come from BASELINE.json north_star (SURVEY.md §8(c) readings #1-#8).

Pins (none of them re-runs the oracle's nth_element-on-composite-key procedure):
  * brute force: full Python sort by (-|a|, index) on small n, many seeds / tie-heavy sets;
  * exhaustive: for n <= 6, every k-subset is tested against the defining order property and
    exactly one subset satisfies it — the oracle's;
  * library: the selected magnitudes equal torch.topk's values;
  * invariants: fp32(emitted) + r' == g + r exactly for every i (EF conservation);
    k == n (fp32 values) => r' == 0; bf16 values: Sterbenz-exact residual, torch's bf16 RNE;
  * the hand-derived worked example in tests/golden/worked_example.json.
"""
import itertools
import json
import os

import numpy as np
import pytest
import torch

import oracle
from workloads import adversarial

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "worked_example.json")))


def mag_key(a):
    return a.view(np.uint32) & np.uint32(0x7FFFFFFF)


def brute_topk(a, k):
    key = mag_key(a)
    order = sorted(range(a.size), key=lambda i: (-int(key[i]), i))
    return np.array(sorted(order[:k]), dtype=np.uint32)


def test_worked_example():
    for rk in ("rank0", "rank1"):
        ex = GOLD[rk]
        g = np.array(ex["g"], np.float32)
        r = np.array(ex["r"], np.float32)
        idx, val, rn = oracle.compress(g, r, GOLD["k"])
        assert idx.tolist() == ex["idx"]
        assert val.tolist() == ex["val"]
        if "r_new" in ex:
            assert rn.tolist() == ex["r_new"]


@pytest.mark.parametrize("kind", ["normal", "grid", "coarse", "zeros90", "allzero", "denormal",
                                  "huge"])
@pytest.mark.parametrize("n", [1, 3, 17, 256, 1000, 4099])
def test_brute_force_sort(kind, n):
    for seed in range(3):
        g = adversarial(kind, n, seed).numpy()
        r = adversarial(kind, n, seed + 100).numpy() * np.float32(0.5)
        a = g + r
        for k in sorted({1, max(1, n // 100), max(1, n // 7), n // 2 or 1, n}):
            idx, val, rn = oracle.compress(g, r, k)
            assert np.array_equal(idx, brute_topk(a, k))
            assert np.array_equal(val.view(np.uint32), a[idx].view(np.uint32))
            # EF conservation, exact: emitted + r' == a (bitwise on the sum's value)
            dense = np.zeros(n, np.float32)
            dense[idx] = val
            fin = np.isfinite(a)
            assert np.all((dense + rn)[fin] == a[fin])
            assert np.all(rn[idx].view(np.uint32) == 0)            # +0 on S
            mask = np.ones(n, bool); mask[idx] = False
            assert np.array_equal(rn[mask].view(np.uint32), a[mask].view(np.uint32))


def test_exhaustive_tie_patterns():
    """For n <= 6 over magnitudes {0, 1, 2} with signs, every k: exactly one k-subset S
    satisfies 'every member precedes every non-member' — and it is the oracle's."""
    vals = [0.0, -0.0, 1.0, -1.0, 2.0]
    cases = 0
    for n in (1, 2, 3, 4, 5):
        for combo in itertools.product(vals, repeat=n):
            a = np.array(combo, np.float32)
            key = mag_key(a)
            for k in range(1, n + 1):
                idx, _, _ = oracle.compress(a, np.zeros(n, np.float32), k)
                valid = []
                for S in itertools.combinations(range(n), k):
                    sset = set(S)
                    ok = all((key[i] > key[j]) or (key[i] == key[j] and i < j)
                             for i in sset for j in range(n) if j not in sset)
                    if ok:
                        valid.append(S)
                assert len(valid) == 1
                assert tuple(idx.tolist()) == valid[0]
                cases += 1
    assert cases > 5000


def test_selected_magnitudes_match_torch_topk():
    for seed in range(5):
        g = adversarial("normal", 50_000, seed).numpy()
        r = adversarial("normal", 50_000, seed + 9).numpy() * np.float32(0.1)
        k = 500
        idx, val, _ = oracle.compress(g, r, k)
        ref = torch.topk(torch.from_numpy(np.abs(g + r)), k).values.numpy()
        assert np.array_equal(np.sort(np.abs(val)), np.sort(ref))


def test_k_equals_n_clears_residual():
    g = adversarial("normal", 999, 3).numpy()
    r = adversarial("grid", 999, 4).numpy()
    idx, val, rn = oracle.compress(g, r, 999)
    assert np.array_equal(idx, np.arange(999, dtype=np.uint32))
    assert np.all(rn.view(np.uint32) == 0)
    assert np.array_equal(val, g + r)


def test_error_feedback_over_iterations():
    """Over T iterations, the residual carries exactly what was not emitted (per step exact)."""
    n, k = 5000, 50
    r = np.zeros(n, np.float32)
    emitted_idx = set()
    for t in range(10):
        g = adversarial("normal", n, 1000 + t).numpy() * np.float32(1e-3)
        a = g + r
        idx, val, r = oracle.compress(g, r, k)
        dense = np.zeros(n, np.float32); dense[idx] = val
        assert np.array_equal(dense + r, a)
        emitted_idx |= set(idx.tolist())
    assert len(emitted_idx) > k                                   # residual rotates selection


def test_bf16_values_sterbenz_residual():
    """bf16 wire values: val = RNE(a) (torch's conversion is the library pin); the residual
    a - fp32(val) is exact, so fp32(val) + r' == a bit-for-bit (reading #8)."""
    g = (adversarial("normal", 20_000, 5).numpy()
         * np.exp(np.linspace(-20, 20, 20_000)).astype(np.float32))
    r = adversarial("normal", 20_000, 6).numpy() * np.float32(1e-3)
    k = 2000
    idx, val16, rn = oracle.compress(g, r, k, vdt=oracle.BF16)
    a = g + r
    ref16 = torch.from_numpy(a[idx]).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(val16, ref16)
    v32 = oracle.bf16_bits_to_f32(val16)
    assert np.array_equal(v32 + rn[idx], a[idx])
    # float64 check that the fp32 subtraction a - fp32(val) was exact
    assert np.array_equal(rn[idx].astype(np.float64), a[idx].astype(np.float64) - v32.astype(np.float64))


def test_bf16_gradient_input_widening():
    g32 = adversarial("normal", 4096, 8).numpy()
    g16 = torch.from_numpy(g32).to(torch.bfloat16)
    gbits = g16.view(torch.int16).numpy().view(np.uint16)
    r = adversarial("grid", 4096, 9).numpy() * np.float32(1e-2)
    idx, val, rn = oracle.compress(gbits, r, 40)
    a = g16.to(torch.float32).numpy() + r
    assert np.array_equal(idx, brute_topk(a, 40))
    assert np.array_equal(val, a[idx])


def test_invalid_arguments():
    g = np.ones(4, np.float32)
    with pytest.raises(oracle.OracleError):
        oracle.compress(g, np.zeros(4, np.float32), 0)
    with pytest.raises(oracle.OracleError):
        oracle.compress(g, np.zeros(4, np.float32), 5)


def test_pairs_layout():
    idx = np.array([1, 5, 9], np.uint32)
    val = np.array([1.5, -2.0, 0.25], np.float32)
    b = oracle.pairs_pack(idx, val)
    assert b.size == 16 + 16
    assert np.array_equal(b[:12].view(np.uint32), idx) and np.all(b[12:16] == 0)
    assert np.array_equal(b[16:28].view(np.float32), val) and np.all(b[28:] == 0)
    b16 = oracle.pairs_pack(idx, np.array([1, 2, 3], np.uint16), oracle.BF16)
    assert b16.size == 32 and np.array_equal(b16[16:22].view(np.uint16), [1, 2, 3])
