"""Sync (Alg. 1 line 5; "Allgather") at N ranks: ncclAllGather + coalesce vs the
fused peer-memory version (lowdiff_p2p_*), same inputs, per-rank device time (max over ranks).

    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 \
        scripts/bench_sync.py --config 3 [--iters 50]

Each rank compresses its own seeded gradient once; the timed loop repeats only the Sync of those
pairs into the rank's shard [lo, hi), so the numbers isolate the exchange + coalesce. Prints one
JSON line from rank 0. On one GPU (LOWDIFF_BENCH_DEVICE=0, several ranks) the contexts time-slice
and NCCL refuses duplicate devices: only the p2p arm runs, and only as a liveness check.
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import paper_conf_sc_yaolhlzz25_b200 as ld  # noqa: E402
from workloads import CONFIGS, gradient, segment_sigmas  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--iters", type=int, default=50)
    ap.add_argument("--arms", default="p2p,nccl")
    a = ap.parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOWDIFF_BENCH_DEVICE", os.environ.get("LOCAL_RANK", "0")))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("gloo")
    barrier = dist.barrier if world > 1 else (lambda: None)
    cfg = CONFIGS[a.config]
    n, k = cfg.n, cfg.k
    lo, hi = ld.shard_bounds(n, world, rank)
    g = gradient(cfg, rank, 0, dev, sigmas=segment_sigmas(cfg, dev))
    r = torch.zeros(n, device=dev)
    pairs = ld.compress(g, r, k, vdt=cfg.vdt)
    del g, r
    cap = min(world * k, hi - lo)
    out = (torch.empty(cap, dtype=torch.int32, device=dev), torch.empty(cap, device=dev),
           torch.zeros(1, dtype=torch.int64, device=dev))
    res = {"metric": "Sync time per iteration (max over ranks)", "config": cfg.name, "P": world, "k": k,
           "pairs_bytes": ld.pairs_bytes(k, cfg.vdt)}
    arms = [x for x in a.arms.split(",") if x]
    if os.environ.get("LOWDIFF_BENCH_DEVICE") is not None and world > 1:
        arms = [x for x in arms if x != "nccl"]        # NCCL refuses several ranks on one device
    for arm in arms:
        if arm == "p2p":
            if world == 1:
                continue                                # P2P needs >= 2 ranks
            h = ld.P2P(world, rank, k, cfg.vdt, device=dev)
            run = lambda: h.allgather_sparse(pairs, lo, hi, True, *out)
        else:
            h = ld.Comm(world, rank) if world > 1 else None
            run = lambda: ld.allgather_sparse(h, pairs, k, cfg.vdt, lo, hi, True, *out)
        for _ in range(5):
            run()
        torch.cuda.synchronize()
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(a.iters):
            run()
        e1.record()
        torch.cuda.synchronize()
        t = torch.tensor([e0.elapsed_time(e1) / a.iters], dtype=torch.float64)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        if arm == "p2p":
            h.status()
        res[f"{arm}_us"] = float(t.item()) * 1e3
        res[f"{arm}_nnz_rank0"] = int(out[2].item())
        barrier()
        if h is not None:
            h.destroy()
    if rank == 0:
        print(json.dumps(res), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
