"""Diagnostics: sampled threshold quality over many EF iterations of a workload (GPU).

    python scripts/diag_compress.py [--config 3] [--iters 300] [--cycle 16]
Prints, every few iterations, the candidates found vs k, the capacity, and whether the exact
full-array fallback ran.
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_yaolhlzz25_b200 as ld  # noqa: E402
from workloads import CONFIGS, gradient, segment_sigmas  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=3)
ap.add_argument("--iters", type=int, default=300)
ap.add_argument("--cycle", type=int, default=16)
ap.add_argument("--every", type=int, default=16)
a = ap.parse_args()
cfg = CONFIGS[a.config]
dev = torch.device("cuda", 0)
sig = segment_sigmas(cfg, dev)
grads = [gradient(cfg, 0, t, dev, sigmas=sig) for t in range(a.cycle)]
r = torch.zeros(cfg.n, device=dev)
fallbacks = 0
for it in range(a.iters):
    ld.compress(grads[it % a.cycle], r, cfg.k, vdt=cfg.vdt)
    st = ld.compress_stats(cfg.n, cfg.k)
    fallbacks += st["fallback"]
    rescans = locals().get("rescans", 0) + st["rescan"]
    if it < 20 or it % a.every == 0 or st["path"]:
        import struct
        f = lambda key: struct.unpack("<f", struct.pack("<I", int(key)))[0]
        print(f"it {it:4d} cand/k {st['candidates'] / cfg.k:7.3f} cap/k {st['capacity'] / cfg.k:6.2f} "
              f"path {st['path']} t_est {f(st['t_est']):.6g} kstar {f(st['kstar']):.6g} "
              f"ratio {f(st['t_est']) / max(f(st['kstar']), 1e-30):.4f} S {st['fine_shift']} inbin {st['inbin']} "
              f"ties {st['ties_kept']} t2 {f(st['t2']):.6g} cand2/k {st['candidates2'] / cfg.k:.3f}", flush=True)
print(f"fallbacks: {fallbacks} rescans: {rescans} / {a.iters}")
print(ld.compress_counters(cfg.n, cfg.k))
