#!/usr/bin/env python
"""LowDiff+ (NEXT-4, §5, Alg. 2) on one B200: a synthetic MLP trained on synthetic data
(no dataset), per-iteration time of forward + backward + GPU Adam update (lowdiff_dense_update)
without and with the LowDiff+ checkpoint side (layer-wise D2H snapshots on a copy stream + the CPU
replica update on the host's cores); the GPU update kernel against HBM (28 B per parameter for
fp32 Adam) and the host replica update's throughput.

    python scripts/bench_plus.py --width 4096 --layers 8 --batch 256 --iters 30 > gpurun_out/plus.json
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_yaolhlzz25_b200 as ld  # noqa: E402
from paper_conf_sc_yaolhlzz25_b200.plus import LowDiffPlus  # noqa: E402


def make_model(width, layers, seed=0):
    torch.manual_seed(seed)
    mods = []
    for _ in range(layers):
        mods += [torch.nn.Linear(width, width), torch.nn.GELU()]
    return torch.nn.Sequential(*mods).cuda()


def run(args, checkpoint):
    model = make_model(args.width, args.layers)
    plus = LowDiffPlus(model, {"kind": "adam"}, lr=1e-4, threads=args.threads, checkpoint=checkpoint)
    x = torch.randn(args.batch, args.width, device="cuda")
    y = torch.randn(args.batch, args.width, device="cuda")

    def it():
        plus.zero_grad()
        loss = torch.nn.functional.mse_loss(model(x), y)
        loss.backward()
        plus.step()

    for _ in range(args.warmup):
        it()
    if checkpoint:
        plus.flush()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    e0.record()
    for _ in range(args.iters):
        it()
    e1.record()
    torch.cuda.synchronize()
    dev_ms = e0.elapsed_time(e1) / args.iters
    if checkpoint:
        plus.flush()
    wall_ms = (time.perf_counter() - t0) * 1e3 / args.iters
    n = plus.n
    plus.close() if checkpoint else None
    return n, dev_ms, wall_ms


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--width", type=int, default=4096)
    ap.add_argument("--layers", type=int, default=8)
    ap.add_argument("--batch", type=int, default=256)
    ap.add_argument("--iters", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--threads", type=int, default=0)
    a = ap.parse_args()
    n, off_dev, off_wall = run(a, False)
    _, on_dev, on_wall = run(a, True)
    # the GPU update kernel alone (HBM roofline) and the host update alone
    st = {"x": torch.zeros(n, device="cuda"), "m": torch.zeros(n, device="cuda"), "v": torch.ones(n, device="cuda"),
          "n": n, "lo": 0, "hi": n, "t": 0, "adam_step": 0, "momentum_initialized": 0}
    g = torch.randn(n, device="cuda")
    for _ in range(3):
        ld.dense_update(st, {"kind": "adam"}, g, 1e-4)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        ld.dense_update(st, {"kind": "adam"}, g, 1e-4)
    e1.record()
    torch.cuda.synchronize()
    du_ms = e0.elapsed_time(e1) / 20
    peaks = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                        "MEASURED_PEAKS.json")))
    hs = {"x": torch.zeros(n), "m": torch.zeros(n), "v": torch.ones(n), "n": n, "lo": 0, "hi": n, "t": 0,
          "adam_step": 0, "momentum_initialized": 0}
    hg = torch.randn(n)
    threads = a.threads or os.cpu_count()
    ld.host_update(hs, {"kind": "adam"}, hg, 1e-4, threads)
    t0 = time.perf_counter()
    for _ in range(5):
        ld.host_update(hs, {"kind": "adam"}, hg, 1e-4, threads)
    hu_ms = (time.perf_counter() - t0) * 1e3 / 5
    print(json.dumps({
        "model": f"MLP {a.layers} x Linear({a.width}, {a.width}) + GELU, batch {a.batch}, fp32, Adam",
        "params": n, "iters": a.iters,
        "no_checkpoint_ms_per_iter": {"device": off_dev, "wall": off_wall},
        "lowdiff_plus_ms_per_iter": {"device": on_dev, "wall": on_wall},
        "overhead_pct_wall": 100 * (on_wall - off_wall) / off_wall,
        "dense_update": {"ms": du_ms, "alg_bytes": 28 * n, "achieved_gbs": 28 * n / du_ms / 1e6,
                         "hbm_frac": 28 * n / du_ms / 1e6 / peaks["hbm_gbs"]},
        "host_update": {"ms": hu_ms, "threads": threads, "params_per_s": n / hu_ms * 1e3,
                        "host_gbs": 28 * n / hu_ms / 1e6},
        "snapshot_d2h_bytes_per_iter": 4 * n}, indent=1))


if __name__ == "__main__":
    main()
