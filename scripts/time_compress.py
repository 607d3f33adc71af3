"""Per-call device time of lowdiff_compress in the error-feedback steady state (GPU), measured as
the bench does its build phase: B calls captured in one CUDA graph, replayed and timed with CUDA
events. python scripts/time_compress.py [--config 3] [--cycle 16] [--reps 20]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_yaolhlzz25_b200 as ld  # noqa: E402
from workloads import CONFIGS, gradient, segment_sigmas  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=3)
ap.add_argument("--cycle", type=int, default=16)
ap.add_argument("--reps", type=int, default=20)
a = ap.parse_args()
cfg = CONFIGS[a.config]
dev = torch.device("cuda", 0)
sig = segment_sigmas(cfg, dev)
grads = [gradient(cfg, 0, t, dev, sigmas=sig) for t in range(a.cycle)]
del sig
r = torch.zeros(cfg.n, device=dev)
ws = torch.empty(ld.compress_workspace_size(cfg.n, cfg.k), dtype=torch.uint8, device=dev)
pairs = torch.empty(ld.pairs_bytes(cfg.k, cfg.vdt), dtype=torch.uint8, device=dev)


def loop():
    for g in grads:
        ld.compress(g, r, cfg.k, vdt=cfg.vdt, pairs=pairs, ws=ws)


for _ in range(6):
    loop()
torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    loop()
g.replay()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(a.reps):
    g.replay()
e1.record()
torch.cuda.synchronize()
per_call = e0.elapsed_time(e1) / (a.reps * len(grads)) * 1e3
# eager, events around each call
ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in grads]
for j, gg in enumerate(grads):
    ev[j][0].record()
    ld.compress(gg, r, cfg.k, vdt=cfg.vdt, pairs=pairs, ws=ws)
    ev[j][1].record()
torch.cuda.synchronize()
eager = sum(x.elapsed_time(y) for x, y in ev) / len(grads) * 1e3
gsz = 2 if cfg.gdt == "bf16" else 4
print(json.dumps({"config": cfg.name, "n": cfg.n, "k": cfg.k, "graph_us_per_call": per_call, "eager_us_per_call": eager,
                  "floor_us": (gsz + 8) * cfg.n / 6456.2e9 * 1e6, "counters": ld.compress_counters(ws=ws)}))
