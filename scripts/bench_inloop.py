#!/usr/bin/env python
"""In-loop checkpointing overhead (the paper's Exp. 1 analogue, P:537-539,
without datasets): per-iteration time of the LowDiff training step (compress -> sync -> live
optimizer update through the replay kernel) with and without the checkpoint side (ring, batch
merge every B iterations, async D2H staging, full checkpoint every FCF iterations), on synthetic
gradients of a BASELINE config (resident pool: no model forward/backward in the timed loop).

    python scripts/bench_inloop.py --config 3 --iters 64 > gpurun_out/inloop.json
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_sc_yaolhlzz25_b200.loop import LowDiffLoop  # noqa: E402
from workloads import CONFIGS, gradient, segment_sigmas  # noqa: E402


def run(cfg, iters, checkpoint, grads, dev, fcf):
    w = torch.zeros(cfg.n, device=dev)
    opt = {"kind": cfg.opt, **{k: v for k, v in cfg.hyper.items() if k != "lr"}}
    loop = LowDiffLoop(w, opt, lr=cfg.hyper["lr"], rho=cfg.rho, B=cfg.B, full_every=fcf,
                       checkpoint=checkpoint)
    for t in range(cfg.B):                       # warm-up: one batch
        loop.step(grads[t % len(grads)])
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for t in range(iters):
        loop.step(grads[t % len(grads)])
    e1.record()
    loop.copy_stream.synchronize()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / iters, (time.perf_counter() - t0) * 1e3 / iters


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--iters", type=int, default=64)
    ap.add_argument("--fcf", type=int, default=0, help="full checkpoint every FCF iterations (default 4B)")
    a = ap.parse_args()
    cfg = CONFIGS[a.config]
    dev = torch.device("cuda", 0)
    sig = segment_sigmas(cfg, dev)
    grads = [gradient(cfg, 0, t, dev, sigmas=sig).float() for t in range(4)]
    fcf = a.fcf or 4 * cfg.B
    off_dev, off_wall = run(cfg, a.iters, False, grads, dev, fcf)
    on_dev, on_wall = run(cfg, a.iters, True, grads, dev, fcf)
    big = cfg.B * (1 << 20)                      # one full checkpoint at t = 0 (in the warm-up) only
    diff_dev, diff_wall = run(cfg, a.iters, True, grads, dev, big)
    print(json.dumps({"config": cfg.name, "n": cfg.n, "B": cfg.B, "fcf": fcf, "iters": a.iters,
                      "no_checkpoint_ms_per_iter": {"device": off_dev, "wall": off_wall},
                      "lowdiff_ms_per_iter": {"device": on_dev, "wall": on_wall},
                      "diff_only_ms_per_iter": {"device": diff_dev, "wall": diff_wall},
                      "overhead_ms_per_iter": on_dev - off_dev,
                      "diff_overhead_ms_per_iter": diff_dev - off_dev,
                      "overhead_pct_wall": 100 * (on_wall - off_wall) / off_wall}, indent=1))


if __name__ == "__main__":
    main()
