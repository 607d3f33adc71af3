"""In-loop LowDiff (Alg. 1 lines 1-15, and the data
dependency analysis of §3.4): the compressed, synchronized gradient G~_t of every
training iteration both drives the live optimizer update and IS the differential checkpoint.

Per iteration t (one call of `LowDiffLoop.step(grad)`):
  1. G~_t <- Sync(Comp(G_t))        lowdiff_compress (top-k + EF) -> lowdiff_allgather_sparse
  2. live update M_{t+1} = M_t + Opt(G~_t) on this rank's shard: G~_t as a one-iteration record
     (lowdiff_batch_merge, STACK) replayed onto the live state (lowdiff_replay, K = 1) — the
     same kernels and op order recovery uses, so recovery reproduces the live trajectory bit for
     bit (Finding 1)
  3. the Reusing Queue: G~_t is handed to the checkpoint side without a copy of its
     values through the device ring; every B iterations the batch is merged into one record and
     staged to pinned host memory on a copy stream (§4.2)
  4. every `full_every` iterations (and at t = 0) a full checkpoint C^F_t of the shard state.

`recover(t)` rebuilds the state at iteration t from the latest full checkpoint at or before t
and the staged records after it (Alg. 1 lines 16-24), through lowdiff_replay.

Marshalling only: every step runs in liblowdiff's kernels (or NCCL); this module owns buffers,
streams and bookkeeping.
"""
from __future__ import annotations

import numpy as np
import torch

from . import (allgather_sparse, batch_merge, compress, k_for_density, record_bytes, replay,
               shard_bounds, stage_d2h)


class LowDiffLoop:
    def __init__(self, x: torch.Tensor, opt: dict, lr: float, rho: float, B: int, full_every: int,
                 comm=None, rank: int = 0, world: int = 1, adam_step: int = 0, checkpoint: bool = True):
        assert x.dtype == torch.float32 and x.is_cuda and x.dim() == 1
        assert full_every % B == 0, "full checkpoints fall on batch boundaries (records chain from them)"
        self.n = x.numel()
        self.k = k_for_density(self.n, rho)
        self.lo, self.hi = shard_bounds(self.n, world, rank)
        self.world, self.comm, self.opt = world, comm, dict(opt)
        self.lr = float(np.float32(lr))
        self.B, self.full_every = B, full_every
        self.r = torch.zeros(self.n, device=x.device)                 # EF residual
        L = self.hi - self.lo
        kind = opt["kind"]
        self.state = {"x": x[self.lo:self.hi], "m": None if kind == "sgd" else torch.zeros(L, device=x.device),
                      "v": torch.zeros(L, device=x.device) if kind == "adam" else None, "x_bf16": None,
                      "n": self.n, "lo": self.lo, "hi": self.hi, "t": 0, "adam_step": adam_step,
                      "momentum_initialized": 0}
        self.cap = min(world * self.k, L)
        self.ring = []                                                  # G~ of the open batch
        self.records = []                                               # (t_first, device rec, pinned)
        self.fulls = []                                                 # (t, {x, m, v, adam_step, mi})
        self.copy_stream = torch.cuda.Stream(device=x.device)
        self.checkpoint = checkpoint          # False: the same training step without checkpointing
        self.t = 0

    # ---- one training iteration ---------------------------------------------------------------
    def step(self, grad: torch.Tensor):
        if self.checkpoint and self.t % self.full_every == 0:
            self._full_checkpoint()
        pairs = compress(grad, self.r, self.k)
        idx, val, nnz = allgather_sparse(self.comm, pairs, self.k, "f32", self.lo, self.hi)
        g_t = (idx, val, nnz, self.cap, self.lr)
        # live update: G~_t as a one-iteration record, replayed onto the live state (K = 1)
        rec1, d_nb = batch_merge([g_t], "stack", self.n, self.lo, self.hi, self.t, self.world)
        nb = record_bytes(d_nb, rec1.numel())
        head = torch.empty(80 + 4 + 16, dtype=torch.uint8, pin_memory=True)
        stage_d2h(rec1, 84, head)
        torch.cuda.current_stream().synchronize()
        replay(self.state, self.opt, [(rec1[:nb], head)])
        self.t += 1
        if not self.checkpoint:
            return
        # checkpoint side: the ring holds G~_t (its own buffers) until the batch is merged
        self.ring.append(g_t)
        if len(self.ring) == self.B:
            self._close_batch()

    def _close_batch(self):
        t_first = self.t - len(self.ring)
        rec, d_nb = batch_merge(self.ring, "stack", self.n, self.lo, self.hi, t_first, self.world)
        nb = record_bytes(d_nb, rec.numel())
        pinned = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
        self.copy_stream.wait_stream(torch.cuda.current_stream())
        stage_d2h(rec, nb, pinned, self.copy_stream)                  # async persist staging
        self.records.append((t_first, rec, pinned))
        self.ring = []

    def _full_checkpoint(self):
        st = self.state
        snap = {"x": st["x"].clone(), "m": None if st["m"] is None else st["m"].clone(),
                "v": None if st["v"] is None else st["v"].clone(), "adam_step": st["adam_step"],
                "momentum_initialized": st["momentum_initialized"]}
        self.fulls.append((self.t, snap))

    # ---- recovery (Alg. 1 lines 16-24) -----------------------------------------------------------
    def recover(self, t: int) -> dict:
        """State of this shard at iteration t (t a batch boundary), from the latest full checkpoint
        at or before t and the staged records after it."""
        self.copy_stream.synchronize()
        tf, snap = max((f for f in self.fulls if f[0] <= t), key=lambda f: f[0])
        L = self.hi - self.lo
        st = {"x": torch.empty(L, device=snap["x"].device), "x0": snap["x"],
              "m": None if snap["m"] is None else torch.empty_like(snap["m"]), "m0": snap["m"],
              "v": None if snap["v"] is None else torch.empty_like(snap["v"]), "v0": snap["v"],
              "x_bf16": None, "n": self.n, "lo": self.lo, "hi": self.hi, "t": tf,
              "adam_step": snap["adam_step"], "momentum_initialized": snap["momentum_initialized"]}
        chain = [(rec, pinned) for (t0, rec, pinned) in self.records if tf <= t0 < t]
        if chain:
            replay(st, self.opt, [(rec[:p.numel()], p) for rec, p in chain])
        else:
            st["x"].copy_(snap["x"])
            if st["m"] is not None:
                st["m"].copy_(snap["m"])
            if st["v"] is not None:
                st["v"].copy_(snap["v"])
        assert st["t"] == t, (st["t"], t)
        return st
