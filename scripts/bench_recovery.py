#!/usr/bin/env python
"""Sequential vs parallel recovery on the GPU, plain SGD over SUM
records (the chains parallel recovery applies to): C1's chain (2 records of B = 4 at rho = 0.01) and
longer chains at C2/C3 sizes. Records are built by the library's own batch merge from synthetic
sparse differentials; times are CUDA events around the replay call (records device-resident).

    python scripts/bench_recovery.py > gpurun_out/recovery.json
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_yaolhlzz25_b200 as ld  # noqa: E402
from workloads import CONFIGS  # noqa: E402


def records(n, k, B, R, dev, seed=0):
    g = torch.Generator(device=dev)
    g.manual_seed(seed)
    recs = []
    for q in range(R):
        diffs = []
        for _ in range(B):
            idx = torch.randperm(n, generator=g, device=dev)[:k].sort().values.to(torch.int32)
            val = torch.randn(k, generator=g, device=dev) * 1e-2
            diffs.append((idx, val, torch.tensor([k], dtype=torch.int64, device=dev), k, 0.1))
        rec, nb = ld.batch_merge(diffs, "sum", n, 0, n, q * B, 1)
        nbytes = ld.record_bytes(nb, rec.numel())
        head = torch.empty(80 + 4 * B + 16, dtype=torch.uint8, pin_memory=True)
        head[:80 + 4 * B].copy_(rec[:80 + 4 * B])
        recs.append((rec[:nbytes].clone(), head, nbytes))
    return recs


def timed(fn, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    dev = torch.device("cuda", 0)
    out = []
    for name, n, rho, B, R in (("C1-resnet20 chain", CONFIGS[1].n, 0.01, 4, 2),
                               ("C2-shaped SGD chain", CONFIGS[2].n, 0.01, 8, 8),
                               ("C3-shaped SGD chain", CONFIGS[3].n, 0.001, 16, 16)):
        k = max(1, int(rho * n))
        recs = records(n, k, B, R, dev)
        x0 = torch.randn(n, device=dev) * 0.05
        x = torch.empty_like(x0)
        views = [(r, h) for r, h, _ in recs]

        def run(parallel):
            st = {"x": x, "m": None, "v": None, "x0": x0, "n": n, "lo": 0, "hi": n, "t": 0, "adam_step": 0,
                  "momentum_initialized": 0}
            (ld.replay_parallel if parallel else ld.replay)(st, {"kind": "sgd"}, views)

        t_seq, t_par = timed(lambda: run(False)), timed(lambda: run(True))
        rec_bytes = sum(nb for _, _, nb in recs)
        out.append({"chain": name, "n": n, "records": R, "B": B, "k": k, "record_bytes": rec_bytes,
                    "sequential_ms": t_seq, "parallel_ms": t_par,
                    "merges_touching_checkpoint": {"sequential": R, "parallel": 1},
                    "note": "both load C^F (x0 -> x copy, 8n bytes) inside the call"})
    print(json.dumps({"recovery": out}, indent=1))


if __name__ == "__main__":
    main()
