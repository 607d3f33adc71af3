"""Multi-process (world size 2, gloo, CPU) coverage of the N > 1 host logic of the path.

On a multi-GPU box each rank compresses its own gradient, one fixed-size all-gather moves every
rank's packed pairs, and rank p coalesces / merges / replays only its shard [lo_p, hi_p)
(DESIGN.md §7). Here the GPU pieces are replaced by the CPU oracle (test
infrastructure) and the all-gather by gloo, to check the host-side plumbing:
  * shard bounds from the C ABI tile [0, n) exactly, identically on every rank;
  * the unique-id broadcast used to bootstrap the NCCL communicator delivers rank 0's bytes;
  * per-shard coalesce of the gathered lists, concatenated over ranks, equals the unsharded
    coalesce (the invariant the sharded pipeline relies on), and per-shard SUM records concatenate
    to the unsharded record's index/value sections.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import oracle
        import paper_conf_sc_yaolhlzz25_b200 as ld
        from workloads import CONFIGS, gradient, segment_sigmas

        # 1. shard bounds
        n = 1_000_003
        lo, hi = ld.shard_bounds(n, world, rank)
        allb = [None] * world
        dist.all_gather_object(allb, (lo, hi))
        assert allb[0][0] == 0 and allb[-1][1] == n
        assert all(allb[p][1] == allb[p + 1][0] for p in range(world - 1))

        # 2. id broadcast
        payload = bytes(range(128)) if rank == 0 else None
        got = ld.broadcast_bytes(payload, 128)
        assert got == bytes(range(128))

        # 3. sharded coalesce + merge == unsharded
        cfg = CONFIGS[2]
        n2 = 300_000
        k = max(1, int(cfg.rho * n2))
        sig = segment_sigmas(cfg)[:n2]
        r = np.zeros(n2, np.float32)
        lo2, hi2 = ld.shard_bounds(n2, world, rank)
        my_diffs, full_diffs = [], []
        for t in range(3):
            g = gradient(cfg, rank, t, "cpu", sigmas=sig, n=n2).numpy()
            idx, val, r = oracle.compress(g, r, k)
            mine = torch.from_numpy(oracle.pairs_pack(idx, val))
            gathered = [torch.zeros_like(mine) for _ in range(world)]
            dist.all_gather(gathered, mine)
            pairs = [x.numpy() for x in gathered]
            my_diffs.append(oracle.coalesce(pairs, k, oracle.F32, lo2, hi2, True))
            full_diffs.append(oracle.coalesce(pairs, k, oracle.F32, 0, n2, True))
        shard_parts = [None] * world
        dist.all_gather_object(shard_parts, [(i.tolist(), v.view(np.uint32).tolist()) for i, v in my_diffs])
        for t in range(3):
            cat_i = np.concatenate([np.array(shard_parts[p][t][0], np.uint32) for p in range(world)])
            cat_v = np.concatenate([np.array(shard_parts[p][t][1], np.uint32) for p in range(world)])
            assert np.array_equal(cat_i, full_diffs[t][0])
            assert np.array_equal(cat_v, full_diffs[t][1].view(np.uint32))
        rec = oracle.parse_record(oracle.batch_merge(my_diffs, 0.1, oracle.SUM, n2, lo2, hi2, 0, world))
        full = oracle.parse_record(oracle.batch_merge(full_diffs, 0.1, oracle.SUM, n2, 0, n2, 0, world))
        recs = [None] * world
        dist.all_gather_object(recs, (rec["idx"].tolist(), rec["val"].view(np.uint32).tolist()))
        assert np.array_equal(np.concatenate([np.array(x[0], np.uint32) for x in recs]), full["idx"])
        assert np.array_equal(np.concatenate([np.array(x[1], np.uint32) for x in recs]),
                              full["val"].view(np.uint32))
        # 4. bench.py's multi-rank plumbing: the job's step time is the slowest rank's, and rank 0
        #    gathers every rank's device / shard-record evidence (the driver reads both)
        import bench
        assert bench.max_over_ranks(10.0 + 5.0 * rank, world) == 10.0 + 5.0 * (world - 1)
        table = bench.rank_table(world, rank, rank, 1000 * (rank + 1), 7 * (rank + 1))
        if rank == 0:
            assert [row["rank"] for row in table] == list(range(world))
            assert [row["record_bytes"] for row in table] == [1000 * (p + 1) for p in range(world)]
        else:
            assert table is None
        dist.barrier()
        dist.destroy_process_group()
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, traceback.format_exc()))


def test_two_rank_gloo_host_logic():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert results == {0: "ok", 1: "ok"}, results
