"""In-loop LowDiff (Alg. 1 lines 1-15, and the data
dependency analysis of §3.4): the compressed, synchronized gradient G~_t of every
training iteration both drives the live optimizer update and IS the differential checkpoint.

Per iteration t (one call of `LowDiffLoop.step(grad)`), all on the training stream, no host sync:
  1. G~_t <- Sync(Comp(G_t))        lowdiff_compress (top-k + EF) -> lowdiff_allgather_sparse
  2. live update M_{t+1} = M_t + Opt(G~_t) on this rank's shard: lowdiff_update — the replay
     kernel on G~_t as a one-iteration differential, so recovery reproduces the live trajectory
     bit for bit (Finding 1)
  3. the Reusing Queue: G~_t stays in its own ring slot (no copy of its values); when
     lowdiff_plan_record_due says so — every B iterations, and right before every full checkpoint
     (a short record, reading #25) — the batch is merged into one record on the training
     stream (§4.2) into one of two device record buffers
  4. the checkpoint side (`_service`, run by the host at the start of each step): once a merge has
     finished (event query, never a wait) the record's byte count is read from pinned memory and
     the record is staged D2H on a copy stream into a pinned buffer from a reused pool (the
     paper's offload_to_cpu)
  5. every `full_every` iterations (and at t = 0) a full checkpoint C^F_t: a device snapshot of
     the shard state (D2D on the training stream), then D2H on the copy stream (CheckFreq-style
     snapshot -> persist). Older full checkpoints and the records before them are
     released once a newer full checkpoint is on the host (`retain_fulls`; None keeps all).
     Any full_every works: the record-boundary policy is the C ABI's lowdiff_plan_record_due.

World > 1 (ZeRO-style reading of §8(e)): rank p owns the optimizer state of the shard [lo, hi) of
the flat parameter vector and updates it from the coalesced G~_t of that shard. The shard state
lives in its own (256-byte aligned) buffers; after each update it is copied into x[lo:hi] and, if
a torch.distributed process group is given (`param_group`), the updated shards are all-gathered
into every rank's x (parameter re-replication, plumbing outside the checkpoint path). Without a
group only x[lo:hi] is current on this rank.

`recover(t)` rebuilds the state at iteration t from the latest full checkpoint at or before t
and the staged records after it (Alg. 1 lines 16-24): host -> device loads, then lowdiff_replay.

Marshalling only: every step runs in liblowdiff's kernels (or NCCL); this module owns buffers,
streams and bookkeeping.
"""
from __future__ import annotations

import numpy as np
import torch

from . import (LowDiffError, allgather_sparse, batch_merge, compress, pairs_bytes, pairs_views, plan_init,
               plan_record_due, record_max_bytes, replay, stage_d2h, update)

_STATE_KEYS = ("x", "m", "v")


class LowDiffLoop:
    def __init__(self, x: torch.Tensor, opt: dict, lr: float, rho: float, B: int, full_every: int,
                 comm=None, rank: int = 0, world: int = 1, adam_step: int = 0, checkpoint: bool = True,
                 retain_fulls: int | None = 2, param_group=None, p2p=None):
        assert x.dtype == torch.float32 and x.is_cuda and x.dim() == 1
        assert retain_fulls is None or retain_fulls >= 1
        self.n = x.numel()
        self.plan = plan_init(self.n, rho, B, full_every, "f32", "f32", world, rank)
        self.k, self.lo, self.hi = self.plan.k, self.plan.lo, self.plan.hi
        self.world, self.comm, self.opt = world, comm, dict(opt)
        self.x_full, self.param_group = x, param_group
        # world > 1: the Sync is the fused peer-memory one when a lowdiff P2P handle is given
        # (compress writes straight into this rank's exchange window), else ncclAllGather + coalesce
        self.p2p = p2p
        self.lr = float(np.float32(lr))
        self.B, self.full_every, self.retain_fulls = B, full_every, retain_fulls
        dev = x.device
        self.r = torch.zeros(self.n, device=dev)                      # EF residual
        L = self.hi - self.lo
        kind = opt["kind"]
        # world 1: the state IS x; world > 1: the shard in its own aligned buffer (lo % 4 may be != 0)
        xs = x if world == 1 else x[self.lo:self.hi].clone()
        self.state = {"x": xs, "m": None if kind == "sgd" else torch.zeros(L, device=dev),
                      "v": torch.zeros(L, device=dev) if kind == "adam" else None, "x_bf16": None,
                      "n": self.n, "lo": self.lo, "hi": self.hi, "t": 0, "adam_step": adam_step,
                      "momentum_initialized": 0}
        self.cap = min(world * self.k, L)
        self.checkpoint = checkpoint          # False: the same training step without checkpointing
        self.t = 0
        self.copy_stream = torch.cuda.Stream(device=dev)
        # the Reusing Queue: B ring slots of G~ (the open batch). The batch merge is issued on the
        # training stream right after the batch's last update, so stream order puts it before the
        # next batch's writes into the same slots.
        R = B if checkpoint else 1
        # P = 1: the Sync of one list is the identity, so a slot IS the compressed pairs buffer
        # (compress writes it; the update and the merge read it in place: views + a count of k)
        self.zero_copy = world == 1
        if self.zero_copy:
            d_k = torch.full((1,), self.k, dtype=torch.int64, device=dev)
            self.pair_slots = [torch.empty(pairs_bytes(self.k), dtype=torch.uint8, device=dev) for _ in range(R)]
            self.slots = [pairs_views(p, self.k) + (d_k,) for p in self.pair_slots]
        else:
            self.slots = [(torch.empty(self.cap, dtype=torch.int32, device=dev),
                           torch.empty(self.cap, dtype=torch.float32, device=dev),
                           torch.zeros(1, dtype=torch.int64, device=dev)) for _ in range(R)]
        self.ring = []                                                  # G~ of the open batch
        self.pairs = torch.empty(pairs_bytes(self.k), dtype=torch.uint8, device=dev)
        if not checkpoint:
            return
        self.rec_cap = record_max_bytes("stack", B, max(B * self.cap, 1), self.lo, self.hi)
        # two device record buffers: one being merged while the other is staged
        self.drec = [{"buf": torch.empty(self.rec_cap, dtype=torch.uint8, device=dev),
                      "nb": torch.zeros(1, dtype=torch.int64, device=dev),
                      "h_nb": torch.zeros(1, dtype=torch.int64, pin_memory=True),
                      "merged": None, "staged": None, "t_first": None} for _ in range(2)]
        self.next_drec = 0
        self.pending = []                                               # merged, not yet staged
        self.pool = []                                                  # free pinned record buffers
        self.records = []                                               # (t_first, pinned, nb, copied ev)
        self.snap = None                                                # device snapshot buffers
        self.snap_free = None                                           # event: snapshot D2H done
        self.fulls = []                                                 # (t, {x,m,v pinned,...}, ev)
        self.full_pool = []                                             # free pinned full buffers
        if retain_fulls is not None:                                    # reserve the host memory up front
            L = self.hi - self.lo
            keys = [k for k in _STATE_KEYS if self.state[k] is not None]
            self.full_pool = [{k: torch.empty(L, dtype=torch.float32, pin_memory=True) for k in keys}
                              for _ in range(retain_fulls + 1)]
            self.pool = [torch.empty(self.rec_cap, dtype=torch.uint8, pin_memory=True)
                         for _ in range(min(retain_fulls * (-(-max(full_every, 1) // B)) + 2, 16))]   # more on demand

    # ---- one training iteration ---------------------------------------------------------------
    def step(self, grad: torch.Tensor):
        close, _, full_due = plan_record_due(self.plan, self.t)
        if self.checkpoint:
            self._service()
            if full_due:
                self._full_checkpoint()
        slot = len(self.ring) % len(self.slots)                         # the open record's next slot
        idx, val, nnz = self.slots[slot]
        if self.zero_copy:
            compress(grad, self.r, self.k, pairs=self.pair_slots[slot])
        elif self.p2p is not None:
            pairs = compress(grad, self.r, self.k, pairs=self.p2p.slot())
            self.p2p.allgather_sparse(pairs, self.lo, self.hi, True, out_idx=idx, out_val=val, d_nnz=nnz)
        else:
            pairs = compress(grad, self.r, self.k, pairs=self.pairs)
            allgather_sparse(self.comm, pairs, self.k, "f32", self.lo, self.hi, out_idx=idx, out_val=val,
                             d_nnz=nnz)
        g_t = (idx, val, nnz, self.cap, self.lr)
        update(self.state, self.opt, g_t)                               # live M_{t+1}
        if self.world > 1:
            self._replicate()
        self.t += 1
        if not self.checkpoint:
            return
        self.ring.append(g_t)                                           # Q.put: zero copy
        if close:                                                       # every B, and before a full checkpoint
            self._close_batch()

    def _replicate(self):
        """x[lo:hi] <- the updated shard; with a process group, all-gather every rank's shard."""
        self.x_full[self.lo:self.hi].copy_(self.state["x"])
        if self.param_group is None:
            return
        import torch.distributed as dist
        P = self.world
        S = -(-self.n // P) + 1                                         # shards differ by at most 1
        if not hasattr(self, "_gbuf"):
            self._gbuf = torch.empty(P * S, device=self.x_full.device)
            self._mine = torch.empty(S, device=self.x_full.device)
        self._mine[:self.hi - self.lo].copy_(self.state["x"])
        dist.all_gather_into_tensor(self._gbuf, self._mine, group=self.param_group)
        for p in range(P):
            lo, hi = p * self.n // P, (p + 1) * self.n // P
            if p != self.plan.rank:
                self.x_full[lo:hi].copy_(self._gbuf[p * S:p * S + hi - lo])

    def _close_batch(self):
        d = self.drec[self.next_drec]
        self.next_drec ^= 1
        if d["t_first"] is not None:                                    # buffer still in use
            self._drain(d)
        t_first = self.t - len(self.ring)
        batch_merge(self.ring, "stack", self.n, self.lo, self.hi, t_first, self.world, record=d["buf"],
                    d_record_bytes=d["nb"])
        d["h_nb"].copy_(d["nb"], non_blocking=True)
        d["merged"] = torch.cuda.Event()
        d["merged"].record()
        d["t_first"] = t_first
        self.pending.append(d)
        self.ring = []

    def _stage(self, d):
        """Checkpoint side: the merge of `d` has finished; stage its bytes to a pinned buffer."""
        nb = int(d["h_nb"][0])
        if nb > self.rec_cap:
            raise LowDiffError(4, f"record of {nb} bytes exceeds its buffer ({self.rec_cap})")
        pinned = self.pool.pop() if self.pool else torch.empty(self.rec_cap, dtype=torch.uint8, pin_memory=True)
        self.copy_stream.wait_event(d["merged"])
        stage_d2h(d["buf"], nb, pinned, self.copy_stream)
        ev = torch.cuda.Event()
        ev.record(self.copy_stream)
        d["staged"] = ev
        self.records.append((d["t_first"], pinned, nb, ev))
        self.pending = [p for p in self.pending if p is not d]

    def _drain(self, d):
        if any(p is d for p in self.pending):
            d["merged"].synchronize()
            self._stage(d)
        d["staged"].synchronize()
        d["t_first"] = None

    def _service(self):
        for d in list(self.pending):
            if d["merged"].query():
                self._stage(d)
        self._retire()

    def _retire(self):
        """Release full checkpoints (and the records before them) older than the newest
        `retain_fulls` full checkpoints that are completely on the host."""
        if self.retain_fulls is None:
            return
        done = [f for f in self.fulls if f[2].query()]
        if len(done) < self.retain_fulls:
            return
        t_keep = done[-self.retain_fulls][0]
        for f in self.fulls:
            if f[0] < t_keep:
                self.full_pool.append({k: f[1][k] for k in _STATE_KEYS if k in f[1]})
        self.fulls = [f for f in self.fulls if f[0] >= t_keep]
        keep = []
        for rec in self.records:
            if rec[0] < t_keep and rec[3].query():
                self.pool.append(rec[1])
            else:
                keep.append(rec)
        self.records = keep

    def _full_checkpoint(self):
        st = self.state
        if self.snap is None:
            self.snap = {k: torch.empty_like(st[k]) for k in _STATE_KEYS if st[k] is not None}
        elif self.snap_free is not None:
            self.snap_free.synchronize()                                # previous D2H finished
        for k, buf in self.snap.items():                                # snapshot (training stream)
            buf.copy_(st[k])
        taken = torch.cuda.Event()
        taken.record()
        self.copy_stream.wait_event(taken)
        host = self.full_pool.pop() if self.full_pool else \
            {k: torch.empty(buf.numel(), dtype=buf.dtype, pin_memory=True) for k, buf in self.snap.items()}
        with torch.cuda.stream(self.copy_stream):                       # persist (copy engine)
            for k, buf in self.snap.items():
                host[k].copy_(buf, non_blocking=True)
        ev = torch.cuda.Event()
        ev.record(self.copy_stream)
        self.snap_free = ev
        host.update(adam_step=st["adam_step"], momentum_initialized=st["momentum_initialized"])
        self.fulls.append((self.t, host, ev))

    def flush(self):
        """Wait until every closed batch and full checkpoint is on the host."""
        for d in list(self.pending):
            d["merged"].synchronize()
            self._stage(d)
        self.copy_stream.synchronize()

    # ---- recovery (Alg. 1 lines 16-24) -----------------------------------------------------------
    def recover(self, t: int) -> dict:
        """State of this shard at iteration t (t a record boundary), from the latest full checkpoint
        at or before t and the staged records after it, loaded back from the host."""
        self.flush()
        tf, snap, _ = max((f for f in self.fulls if f[0] <= t), key=lambda f: f[0])
        dev = self.state["x"].device
        load = lambda k: None if k not in snap else snap[k].to(dev, non_blocking=True)
        st = {"x": torch.empty(self.hi - self.lo, device=dev), "x0": load("x"),
              "m": None if "m" not in snap else torch.empty_like(snap["m"], device=dev), "m0": load("m"),
              "v": None if "v" not in snap else torch.empty_like(snap["v"], device=dev), "v0": load("v"),
              "x_bf16": None, "n": self.n, "lo": self.lo, "hi": self.hi, "t": tf,
              "adam_step": snap["adam_step"], "momentum_initialized": snap["momentum_initialized"]}
        chain = sorted((r for r in self.records if tf <= r[0] < t), key=lambda r: r[0])
        if chain:
            replay(st, self.opt, [(p[:nb].to(dev, non_blocking=True), p[:nb]) for _, p, nb, _ in chain])
        else:
            for k in _STATE_KEYS:
                if st[k] is not None:
                    st[k].copy_(st[k + "0"])
        assert st["t"] == t, (st["t"], t)
        return st
