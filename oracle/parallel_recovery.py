"""Parallel recovery — ORACLE, TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

PAPER.md §4.4 "Parallel recovery module": instead of merging the n differential
checkpoints into the full checkpoint one by one (Eq. 2: M_n = C^F + C^D_1 + ... + C^D_n),
the differentials are merged among themselves and the result is merged into C^F, so that
~log n (here: one) merges touch C^F. For plain SGD (weight decay 0) with one constant lr the
differential of iteration t is -lr * G~_t, so on SUM records (reading #13):

    D = v_1 + v_2 + ... + v_R          per index, fp32, record order, absent terms skipped
    x = x - lr * D                     fp32: one multiply, one subtract per touched index

Plain numpy float32 (IEEE round-to-nearest per operation); `np.add.at` visits the records in
order, and each record holds an index at most once, so every index's sum is a left fold in
record order.
"""
from __future__ import annotations

import numpy as np

from . import SUM, parse_record


def replay_parallel(state: dict, records: list[np.ndarray]) -> dict:
    """state: {"x" float32 array over [lo, hi), "lo", "hi", "t"}; records: SUM record bytes of one
    contiguous chain with one constant lr. Updates x in place and advances t."""
    x, lo = state["x"], int(state["lo"])
    recs = [parse_record(r) for r in records]
    lr = None
    for h in recs:
        assert h["mode"] == SUM, "parallel recovery: SUM records only"
        for v in h["lr"]:
            lr = v if lr is None else lr
            assert v == lr, "parallel recovery: one constant lr"
    if not recs:
        return state
    D = np.zeros(x.size, np.float32)
    touched = np.zeros(x.size, bool)
    for h in recs:                                    # the differentials merged among themselves
        p = h["idx"].astype(np.int64) - lo
        first = ~touched[p]
        D[p[first]] = h["val"][first]                 # absent terms are skipped, not added as +0
        np.add.at(D, p[~first], h["val"][~first])
        touched[p] = True
    p = np.nonzero(touched)[0]
    x[p] = x[p] - np.float32(lr) * D[p]               # merged once into the checkpoint
    state["t"] = int(state["t"]) + sum(h["B"] for h in recs)
    return state
