"""Warm compress loop for ncu captures (GPU): python scripts/prof_compress.py [--config 3] [--iters 40]
Cycles the bench's resident gradients through one residual and one workspace, so the launches after
the first few are the error-feedback steady state the bench times."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_yaolhlzz25_b200 as ld  # noqa: E402
from workloads import CONFIGS, gradient, segment_sigmas  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=3)
ap.add_argument("--iters", type=int, default=40)
ap.add_argument("--cycle", type=int, default=16)
a = ap.parse_args()
cfg = CONFIGS[a.config]
dev = torch.device("cuda", 0)
sig = segment_sigmas(cfg, dev)
grads = [gradient(cfg, 0, t, dev, sigmas=sig) for t in range(a.cycle)]
del sig
r = torch.zeros(cfg.n, device=dev)
ws = torch.empty(ld.compress_workspace_size(cfg.n, cfg.k), dtype=torch.uint8, device=dev)
pairs = torch.empty(ld.pairs_bytes(cfg.k, cfg.vdt), dtype=torch.uint8, device=dev)
for it in range(a.iters):
    ld.compress(grads[it % a.cycle], r, cfg.k, vdt=cfg.vdt, pairs=pairs, ws=ws)
torch.cuda.synchronize()
print(ld.compress_counters(ws=ws))
