"""GPU parity of the peer-memory Sync (include/lowdiff.h (2'), Alg.1 line 5): the
all-gather fused with the coalesce, each rank's pairs read straight out of its owner's exchange
window. Compared bit for bit with the oracle's coalesce of all P lists (oracle.coalesce).

One GPU is available, so the P ranks run as P processes sharing the device through CUDA IPC (the
real bootstrap: handle export, all_gather_object exchange, cudaIpcOpenMemHandle; each process
has its own context, so a spinning wait of one rank never blocks another rank's stream). Several
epochs reuse both slots; the zero-copy slot and a captured CUDA graph are covered. (Several ranks
on separate streams of ONE process and ONE device are not used: streams can share a hardware
queue, and then a spinning wait blocks a peer's work until it times out.)
"""
import os
import socket

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_yaolhlzz25_b200 as ld

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_sc_yaolhlzz25_b200 import build
    build.build()
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"


def rank_pairs(P, n, k, vdt, seed, clustered=False):
    """P packed pair buffers (oracle layout): ascending unique indices, normal values, some -0."""
    rng = np.random.default_rng(seed)
    o_vdt = oracle.BF16 if vdt == "bf16" else oracle.F32
    out = []
    for _ in range(P):
        if clustered:
            base = int(rng.integers(0, n - 3 * k))
            idx = np.sort(rng.choice(np.arange(base, base + 3 * k), k, replace=False)).astype(np.uint32)
        else:
            idx = np.sort(rng.choice(n, k, replace=False)).astype(np.uint32)
        val = rng.standard_normal(k).astype(np.float32)
        val[rng.random(k) < 0.03] = -0.0
        if vdt == "bf16":
            val = torch.from_numpy(val).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
        out.append(oracle.pairs_pack(idx, val, o_vdt))
    return out


def check(pairs, k, vdt, lo, hi, average, idx, val, d_nnz):
    oi, ov = oracle.coalesce(pairs, k, oracle.BF16 if vdt == "bf16" else oracle.F32, lo, hi, average)
    nnz = int(d_nnz.item())
    assert nnz == oi.size
    assert np.array_equal(idx[:nnz].cpu().numpy().view(np.uint32), oi)
    assert np.array_equal(val[:nnz].cpu().numpy().view(np.uint32), ov.view(np.uint32))


def test_p2p_missing_peer_times_out(monkeypatch):
    monkeypatch.setenv("LOWDIFF_P2P_TIMEOUT_MS", "300")
    n, k = 50_000, 500
    hs = ld.P2P.local(2, k)
    (p0,) = rank_pairs(1, n, k, "f32", seed=5)
    hs[0].allgather_sparse(torch.from_numpy(p0).cuda(), 0, n)     # rank 1 never makes the call
    torch.cuda.synchronize()
    with pytest.raises(ld.LowDiffError) as ei:
        hs[0].status()
    assert ei.value.status == "ETIMEOUT"
    hs[1].status()                                                 # rank 1 itself saw nothing
    for h in hs:
        h.destroy()


def test_p2p_rejects_bad_arguments():
    with pytest.raises(ld.LowDiffError):
        ld.P2P.local(1, 100)                                       # P2P needs >= 2 ranks
    hs = ld.P2P.local(2, 1000)
    pairs = torch.zeros(ld.pairs_bytes(1000), dtype=torch.uint8, device="cuda")
    with pytest.raises(ld.LowDiffError):
        hs[0].allgather_sparse(pairs, 10, 10)                      # empty shard
    small = torch.empty(16, dtype=torch.int32, device="cuda")     # out_cap < min(P*k, hi-lo): C-level check
    code = ld.lib().lowdiff_p2p_allgather_sparse(hs[0]._h, pairs.data_ptr(), 0, 10_000, 1, small.data_ptr(),
                                                 small.data_ptr(), 16, small.data_ptr(), pairs.data_ptr(),
                                                 pairs.numel(), torch.cuda.current_stream().cuda_stream)
    assert ld.STATUS[code] == "EINVAL"
    for h in hs:
        h.destroy()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ipc_worker(rank, world, vdt, port, q):
    """One rank: eager epochs (shard and full-range coalesce, mean and sum, copy and zero-copy slot),
    then two calls captured in a CUDA graph and replayed three times. Every rank draws all ranks'
    lists from the same seeds, so each checks its own output against the oracle."""
    try:
        import torch.distributed as dist
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        n, k = 300_000, 4_000
        h = ld.P2P(world, rank, k, vdt, device="cuda:0")
        for e in range(6):
            pairs = rank_pairs(world, n, k, vdt, seed=7 + e, clustered=e % 2 == 1)
            lo, hi = ld.shard_bounds(n, world, rank) if e != 3 else (0, n)
            average = e != 2
            src = torch.from_numpy(pairs[rank]).cuda()
            if e >= 4:                                  # compress would write straight into the slot
                slot = h.slot()
                slot.copy_(src)
                src = slot
            idx, val, d_nnz = h.allgather_sparse(src, lo, hi, average)
            torch.cuda.synchronize()
            h.status()
            check(pairs, k, vdt, lo, hi, average, idx, val, d_nnz)
        # CUDA graph: the epoch lives on the device, so replays publish fresh flag values
        lo, hi = ld.shard_bounds(n, world, rank)
        cap = min(world * k, hi - lo)
        src = [torch.empty(ld.pairs_bytes(k, vdt), dtype=torch.uint8, device="cuda") for _ in range(2)]
        out = [(torch.empty(cap, dtype=torch.int32, device="cuda"), torch.empty(cap, device="cuda"),
                torch.zeros(1, dtype=torch.int64, device="cuda")) for _ in range(2)]
        ws = torch.empty(ld.coalesce_workspace_size(world, k, vdt, lo, hi), dtype=torch.uint8, device="cuda")
        side = torch.cuda.Stream()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=side):
            for c in range(2):
                h.allgather_sparse(src[c], lo, hi, True, *out[c], ws=ws)
        for rep in range(3):
            pairs = [rank_pairs(world, n, k, vdt, seed=900 + 2 * rep + c) for c in range(2)]
            for c in range(2):
                src[c].copy_(torch.from_numpy(pairs[c][rank]))
            g.replay()
            torch.cuda.synchronize()
            h.status()
            for c in range(2):
                check(pairs[c], k, vdt, lo, hi, True, *out[c])
        dist.barrier()
        del g
        h.destroy()
        dist.destroy_process_group()
        q.put((rank, "ok"))
    except Exception:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, traceback.format_exc()))


@pytest.mark.parametrize("world,vdt", [(2, "f32"), (3, "bf16")])
def test_p2p_processes_ipc(world, vdt):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, world, vdt, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert results == {r: "ok" for r in range(world)}, results


def _loop_worker(rank, world, port, q):
    """One rank of the in-loop driver over the fused peer-memory Sync: per iteration compress into
    the exchange window, the P2P coalesce of this rank's shard, the live update, and LowDiff's
    checkpoint side. Checks: the coalesced G~ equals the oracle's coalesce of every rank's pairs
    (recomputed from the same seeds), and the recovered shard equals the live one bit for bit."""
    try:
        import torch.distributed as dist
        from paper_conf_sc_yaolhlzz25_b200.loop import LowDiffLoop
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        n, T, B = 200_003, 8, 4
        k = ld.k_for_density(n, 0.01)
        h = ld.P2P(world, rank, k, "f32", device="cuda:0")
        w = torch.zeros(n, device="cuda")
        opt = {"kind": "adam", "beta1": 0.9, "beta2": 0.999, "eps": 1e-8}
        loop = LowDiffLoop(w, opt, lr=1e-3, rho=0.01, B=B, full_every=8, world=world, rank=rank,
                           retain_fulls=None, p2p=h)
        r_o = [np.zeros(n, np.float32) for _ in range(world)]
        for t in range(T):
            gs = [(np.random.default_rng(1000 * t + p).standard_normal(n) * 0.1).astype(np.float32)
                  for p in range(world)]
            loop.step(torch.from_numpy(gs[rank]).cuda())
            pairs = []
            for p in range(world):
                oi, ov, r_o[p] = oracle.compress(gs[p], r_o[p], k)
                pairs.append(oracle.pairs_pack(oi, ov))
            torch.cuda.synchronize()
            h.status()
            idx, val, d_nnz = loop.ring[-1][:3] if loop.ring else loop.slots[(len(loop.slots) - 1)]
            check(pairs, k, "f32", loop.lo, loop.hi, True, idx, val, d_nnz)
        live = [loop.state[key].clone() for key in ("x", "m", "v")]
        rec = loop.recover(T)
        for a, b in zip((rec["x"], rec["m"], rec["v"]), live):
            assert torch.equal(a.view(torch.int32), b.view(torch.int32))
        dist.barrier()
        h.destroy()
        dist.destroy_process_group()
        q.put((rank, "ok"))
    except Exception:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, traceback.format_exc()))


def test_in_loop_over_p2p_processes():
    """LowDiffLoop (in-loop LowDiff) with the fused peer-memory Sync at world 2:
    two processes sharing the GPU through CUDA IPC (round 1's P2P loop stalled and was not shipped)."""
    import torch.multiprocessing as mp
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_loop_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert results == {r: "ok" for r in range(world)}, results
