"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle's tests.

This module holds NO arithmetic of the method (no selection, no coalescing, no merging,
no optimizer step). It only draws inputs with the shapes and value structure of the
paper's workloads (Table 2(b); SURVEY.md §8(d) "Synthetic gradient
structure"):

* segments = the model's real parameter tensors in ``named_parameters()`` order
  (``shapes.json``, written by ``scripts/gen_shapes.py`` on ``device="meta"``);
* each segment s has a fixed scale sigma_s = 10**u_s, u_s ~ U[-4, -1] (seeded per config),
  so layer heterogeneity concentrates the top-k the way real gradients do;
* g_{p,t}[i] = sigma_s(i) * (sqrt(1/2) z_shared(t, i) + sqrt(1/2) z_p(t, i)),
  z ~ N(0, 1): ranks are correlated, as data-parallel gradients of one loss are;
* bf16 gradients (config C4) are the fp32 draw rounded to bf16 by torch (RNE).

Seeds: seed_c = 101 * c; shared part s = (seed_c << 32) | t; rank part
s = (seed_c << 32) | ((p + 1) << 20) | t; per-segment scales s = seed_c.
"""
from __future__ import annotations

import json
import math
import os
from dataclasses import dataclass, field

import torch

_SHAPES = json.load(open(os.path.join(os.path.dirname(__file__), "shapes.json")))


@dataclass(frozen=True)
class Config:
    """One BASELINE.json config (configs[c-1]), made concrete as in SURVEY.md §8(d)."""
    cid: int
    name: str
    model: str
    rho: float
    B: int
    P: int
    gdt: str                  # "f32" | "bf16"  (gradient dtype on the wire into compress)
    vdt: str                  # value dtype of the packed pairs
    opt: str                  # "sgd" | "momentum" | "adam"
    K: int                    # replay chain length (iterations)
    merge: str                # "sum" | "stack"
    hyper: dict = field(default_factory=dict)

    @property
    def segments(self) -> list[int]:
        return _SHAPES[self.model]

    @property
    def n(self) -> int:
        return sum(self.segments)

    @property
    def k(self) -> int:
        return k_for_density(self.n, self.rho)

    @property
    def seed(self) -> int:
        return 101 * self.cid


def k_for_density(n: int, rho: float) -> int:
    """k = max(1, min(n, floor(rho * n))) in double (SURVEY.md §8(c) reading #2)."""
    return max(1, min(n, int(math.floor(rho * n))))


CONFIGS = {
    1: Config(1, "C1-resnet20", "resnet20", 0.01, 4, 1, "f32", "f32", "sgd", 8, "sum",
              {"lr": 0.1}),
    2: Config(2, "C2-resnet50", "resnet50", 0.01, 8, 8, "f32", "f32", "momentum", 16, "stack",
              {"lr": 0.1, "momentum": 0.9, "dampening": 0.0, "nesterov": 0}),
    3: Config(3, "C3-vgg16", "vgg16", 0.001, 16, 1, "f32", "f32", "adam", 16, "stack",
              {"lr": 1e-4, "beta1": 0.9, "beta2": 0.999, "eps": 1e-8}),
    4: Config(4, "C4-bert-large", "bert_large", 0.01, 8, 1, "bf16", "bf16", "adam", 32, "stack",
              {"lr": 1e-4, "beta1": 0.9, "beta2": 0.999, "eps": 1e-8}),
    5: Config(5, "C5-gpt2-xl", "gpt2_xl", 0.001, 32, 8, "f32", "f32", "adam", 32, "stack",
              {"lr": 1e-4, "beta1": 0.9, "beta2": 0.999, "eps": 1e-8}),
}


def shard_bounds(n: int, P: int, p: int) -> tuple[int, int]:
    """Contiguous index shard of rank p: [floor(p n / P), floor((p+1) n / P)) (reading #22)."""
    return (p * n) // P, ((p + 1) * n) // P


def _gen(device, seed: int) -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed(seed & ((1 << 63) - 1))
    return g


def segment_sigmas(cfg: Config, device="cpu") -> torch.Tensor:
    """Per-element scale sigma_s(i), fp32, length n (segments repeated)."""
    g = _gen("cpu", cfg.seed)
    u = torch.rand(len(cfg.segments), generator=g, dtype=torch.float64) * 3.0 - 4.0
    sig = torch.pow(10.0, u).to(torch.float32)
    reps = torch.tensor(cfg.segments, dtype=torch.int64)
    return torch.repeat_interleave(sig, reps).to(device)


def gradient(cfg: Config, rank: int, t: int, device="cpu", sigmas: torch.Tensor | None = None,
             n: int | None = None) -> torch.Tensor:
    """Synthetic DP gradient g_{rank,t} of config cfg (optionally only its first n elements)."""
    assert 0 <= t < (1 << 20) and 0 <= rank < 2047
    n = cfg.n if n is None else n
    if sigmas is None:
        sigmas = segment_sigmas(cfg, device)
    sigmas = sigmas[:n]
    z_s = torch.randn(n, generator=_gen(device, (cfg.seed << 32) | t), device=device)
    z_p = torch.randn(n, generator=_gen(device, (cfg.seed << 32) | ((rank + 1) << 20) | t),
                      device=device)
    h = math.sqrt(0.5)
    g = sigmas * (z_s * h + z_p * h)
    if cfg.gdt == "bf16":
        g = g.to(torch.bfloat16)
    return g


def full_checkpoint(cfg: Config, lo: int, hi: int, device="cpu", seed_offset: int = 0):
    """Synthetic full checkpoint shard (x, m|buf, v) per SURVEY.md §8(d) table.

    Returns dict with fp32 tensors x, m, v (v None for momentum/sgd), and step counters.
    """
    n = hi - lo
    g = _gen(device, (cfg.seed << 32) | (0xFFFFF - seed_offset))
    if cfg.opt == "sgd":
        x = torch.randn(n, generator=g, device=device) * 0.05
        return {"x": x, "m": None, "v": None, "adam_step": 0, "momentum_initialized": 0}
    if cfg.opt == "momentum":
        x = torch.randn(n, generator=g, device=device) * 0.02
        buf = torch.randn(n, generator=g, device=device) * 1e-3
        return {"x": x, "m": buf, "v": None, "adam_step": 0, "momentum_initialized": 1}
    x = torch.randn(n, generator=g, device=device) * 0.02
    m = torch.randn(n, generator=g, device=device) * 1e-4
    v = m * m + 1e-10
    return {"x": x, "m": m, "v": v, "adam_step": 1000, "momentum_initialized": 0}


# ---------------------------------------------------------------------------------------
# Correctness-only input sets (never timed)
# ---------------------------------------------------------------------------------------

def adversarial(kind: str, n: int, seed: int = 0) -> torch.Tensor:
    """fp32 CPU vectors with ties, zeros, signed zeros, denormals and huge magnitudes."""
    g = _gen("cpu", 7919 * seed + 17)
    if kind == "grid":          # values on a 2^-12 grid in [-1, 1]: many exact ties
        return (torch.randint(-4096, 4097, (n,), generator=g).to(torch.float32) / 4096.0)
    if kind == "coarse":        # very few distinct magnitudes: massive ties
        return torch.randint(-3, 4, (n,), generator=g).to(torch.float32) * 0.5
    if kind == "zeros90":       # 90% exact zeros (both signs)
        x = torch.randn(n, generator=g)
        mask = torch.rand(n, generator=g) < 0.9
        x[mask] = 0.0
        neg = torch.rand(n, generator=g) < 0.5
        x[mask & neg] = -0.0
        return x
    if kind == "allzero":
        x = torch.zeros(n)
        x[torch.rand(n, generator=g) < 0.5] = -0.0
        return x
    if kind == "denormal":
        x = torch.randn(n, generator=g) * 1e-39
        return x
    if kind == "huge":
        x = torch.randn(n, generator=g)
        big = torch.rand(n, generator=g) < 0.01
        x[big] = torch.sign(x[big]) * 1e38
        return x
    if kind == "normal":
        return torch.randn(n, generator=g)
    raise ValueError(kind)
