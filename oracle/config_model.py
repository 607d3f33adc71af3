"""Checkpointing configuration model — ORACLE, TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Plain fp64 Python written from PAPER.md §3.5 "Optimizing Checkpointing Configuration"
(P:318-350). Time is in units of one training iteration: the paper counts the wasted work of b
batched iterations as b/2 and the number of full checkpoints during training as f x T
(P:327), so f is full checkpoints per iteration and T, M, R_F, R_D are in iterations
(reading #29).

  wasted_time(m, f, b)   Eq. 3, term by term as the bullet list P:325-333 builds it
  optimal_point(m)       Eq. 5
  best_integer(m)        reading #30: the integer (FCF = 1/f iterations, B), FCF >= B >= 1, that
                         minimises Eq. 3. Eq. 3 is convex in FCF for fixed b and its minimum over
                         FCF is convex in b with its minimum at b*, so B is floor/ceil(b*) and,
                         for each B, FCF is floor/ceil of the b = B solution of Eq. 4's first
                         equation, 1/f_B = sqrt(2 S M B / (R_D W)) (clamped to >= B);
                         ties -> smaller FCF, then smaller B
"""
from __future__ import annotations

import math

KEYS = ("N", "M", "W", "S", "T", "R_F", "R_D")


def wasted_time(m: dict, f: float, b: float) -> float:
    N, M, W, S, T, R_F, R_D = (float(m[k]) for k in KEYS)
    failures = T / M                                   # "number of failures"
    full_write = S / W                                 # "time of writing a full checkpoint"
    n_full = f * T                                     # "number of full checkpoints"
    merges = 0.5 * (1.0 / f * 1.0 / b - 1.0)           # "number of merging operations on average"
    recovery = N * failures * ((R_F + R_D * merges) + b / 2.0)   # total recovery overhead
    steady = N * full_write * n_full                   # total steady state overhead
    return recovery + steady                           # Eq. 3


def optimal_point(m: dict) -> tuple[float, float]:
    M, W, S, R_D = (float(m[k]) for k in ("M", "W", "S", "R_D"))
    f_star = (R_D * W ** 2 / (4.0 * S ** 2 * M ** 2)) ** (1.0 / 3.0)
    b_star = (2.0 * S * R_D * M / W) ** (1.0 / 3.0)
    return f_star, b_star


def best_integer(m: dict) -> tuple[int, int]:
    M, W, S, R_D = (float(m[k]) for k in ("M", "W", "S", "R_D"))
    _, b_star = optimal_point(m)
    best = None
    for B in sorted({max(1, math.floor(b_star)), max(1, math.ceil(b_star))}):
        F_B = math.sqrt(2.0 * S * M * B / (R_D * W))   # dT/df = 0 at b = B (Eq. 4, first line)
        for F in sorted({max(B, math.floor(F_B)), max(B, math.ceil(F_B))}):
            key = (wasted_time(m, 1.0 / F, B), F, B)
            if best is None or key < best:
                best = key
    return best[1], best[2]
