"""Configuration model (§3.5): the oracle pinned to
calculus and a hand-derived example, then the C-ABI (host-only, runs on CPU) against the oracle."""
import json
import math
import os

import numpy as np
import pytest

from oracle import config_model as cm

HERE = os.path.dirname(os.path.abspath(__file__))


def models(count=40, seed=3):
    rng = np.random.default_rng(seed)
    out = []
    for _ in range(count):
        out.append({"N": float(rng.integers(1, 1025)), "M": 10 ** rng.uniform(2, 6),
                    "W": 10 ** rng.uniform(6, 11), "S": 10 ** rng.uniform(7, 12), "T": 10 ** rng.uniform(4, 7),
                    "R_F": 10 ** rng.uniform(-1, 2), "R_D": 10 ** rng.uniform(-3, 1)})
    return out


# ---- oracle pins -----------------------------------------------------------------------------
def test_golden_example():
    g = json.load(open(os.path.join(HERE, "golden", "config_model_example.json")))
    f, b = cm.optimal_point(g["model"])
    assert f == pytest.approx(g["f_star"], rel=1e-15) and b == pytest.approx(g["b_star"], rel=1e-15)
    for fv, bv, w in g["wasted"]:
        assert cm.wasted_time(g["model"], fv, bv) == pytest.approx(w, rel=1e-15)


@pytest.mark.parametrize("m", models(12))
def test_partials_vanish_at_optimum(m):
    """Eq. 4: both first-order partials of Eq. 3 are zero at Eq. 5's point (central
    finite differences of the oracle's Eq. 3, relative to the terms' scale)."""
    f, b = cm.optimal_point(m)
    for var, x in (("f", f), ("b", b)):
        h = x * 1e-5
        if var == "f":
            d = (cm.wasted_time(m, f + h, b) - cm.wasted_time(m, f - h, b)) / (2 * h)
            scale = m["N"] * m["T"] * m["S"] / m["W"]          # size of the steady-state term's slope
        else:
            d = (cm.wasted_time(m, f, b + h) - cm.wasted_time(m, f, b - h)) / (2 * h)
            scale = m["N"] * m["T"] / m["M"] / 2                # size of the b/2 term's slope
        assert abs(d) <= 1e-5 * scale, (var, d, scale)


@pytest.mark.parametrize("m", models(6, seed=9))
def test_brute_force_minimum(m):
    """A log-spaced grid search of Eq. 3 finds its minimum next to Eq. 5's point, and Eq. 3 is
    U-shaped in each variable through it (the shape of Table 1's rows and columns)."""
    f0, b0 = cm.optimal_point(m)
    fs = f0 * np.logspace(-1, 1, 201)
    bs = b0 * np.logspace(-1, 1, 201)
    W = np.array([[cm.wasted_time(m, f, b) for b in bs] for f in fs])
    i, j = np.unravel_index(np.argmin(W), W.shape)
    assert abs(i - 100) <= 1 and abs(j - 100) <= 1
    row, col = W[100], W[:, 100]
    assert np.all(np.diff(row[:100]) < 0) and np.all(np.diff(row[100:]) > 0)
    assert np.all(np.diff(col[:100]) < 0) and np.all(np.diff(col[100:]) > 0)


@pytest.mark.parametrize("m", [{"N": 8, "M": 2000.0, "W": 1e9, "S": 5e9, "T": 1e5, "R_F": 30.0, "R_D": 0.5},
                               {"N": 64, "M": 500.0, "W": 2e10, "S": 1e9, "T": 1e6, "R_F": 5.0, "R_D": 0.05},
                               {"N": 2, "M": 50.0, "W": 1e8, "S": 4e9, "T": 1e4, "R_F": 60.0, "R_D": 2.0}])
def test_best_integer_rule(m):
    F, B = cm.best_integer(m)
    f0, b0 = cm.optimal_point(m)
    assert B in (math.floor(b0), math.ceil(b0))
    # brute force over a wide integer neighbourhood: nothing does better
    best = cm.wasted_time(m, 1 / F, B)
    for Fi in range(max(1, F - 200), F + 201):
        for Bi in range(1, min(Fi, 2 * B + 10) + 1):
            assert cm.wasted_time(m, 1 / Fi, Bi) >= best * (1 - 1e-12), (Fi, Bi)


# ---- C-ABI vs oracle (host-only calls: no GPU needed) -------------------------------------------
@pytest.fixture(scope="module")
def ld():
    from paper_conf_sc_yaolhlzz25_b200 import build
    build.build()
    import paper_conf_sc_yaolhlzz25_b200 as mod
    return mod


@pytest.mark.parametrize("m", models(40, seed=5))
def test_abi_matches_oracle(ld, m):
    r = ld.optimal_config(m)
    f0, b0 = cm.optimal_point(m)
    assert r["f_star"] == pytest.approx(f0, rel=1e-12) and r["b_star"] == pytest.approx(b0, rel=1e-12)
    for f, b in ((f0, b0), (f0 * 3, b0 / 2), (1e-3, 7.0)):
        assert ld.wasted_time(m, f, b) == pytest.approx(cm.wasted_time(m, f, b), rel=1e-12)
    F, B = cm.best_integer(m)
    if (r["fcf"], r["B"]) != (F, B):      # only a last-bit tie may pick differently
        wa = cm.wasted_time(m, 1 / r["fcf"], r["B"])
        wo = cm.wasted_time(m, 1 / F, B)
        assert wa == pytest.approx(wo, rel=1e-12)


def test_abi_rejects_bad_models(ld):
    good = {"N": 8, "M": 2000.0, "W": 1e9, "S": 5e9, "T": 1e5, "R_F": 30.0, "R_D": 0.5}
    for key in good:
        for bad in (0.0, -1.0, float("nan"), float("inf")):
            m = dict(good, **{key: bad})
            with pytest.raises(ld.LowDiffError):
                ld.optimal_config(m)
    with pytest.raises(ld.LowDiffError):
        ld.wasted_time(good, 0.0, 2.0)
    with pytest.raises(ld.LowDiffError):
        ld.wasted_time(good, 0.1, float("nan"))
