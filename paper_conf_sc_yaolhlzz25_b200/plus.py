"""LowDiff+ — checkpointing without gradient compression (§5, Algorithm 2, P:353-441;
SURVEY §8(f) NEXT-4).

  * Layer-wise reuse and snapshot (§5.1; Alg. 2 lines 4-5, 9-10, 17-19): every
    parameter's gradient is copied to pinned host memory on a copy stream the moment autograd has
    accumulated it (a post-accumulate-grad hook), so the D2H transfer of layer n overlaps the
    backward of layers n-1, n-2, ... instead of waiting for the whole backward.
  * GPU update (line 7): M^G_{t+1} = M^G_t + Opt(G_t) through lowdiff_dense_update on the flat
    parameter storage the module's parameters are re-pointed into.
  * CPU replica (§5.2-5.3, lines 11-12): a worker thread waits for iteration t's copies and
    applies the same step to the host replica M^C through lowdiff_host_update (native C++, all
    cores, the GIL released) — bit-identical arithmetic, so M^C_t == M^G_t exactly. The replica is
    the in-memory checkpoint; persisting it (line 13) is storage I/O and out of scope.
  * Recovery from a software failure: `recover()` restores the GPU model from the
    replica without touching storage.

Two pinned gradient buffers alternate between iterations; `zero_grad()` (the start of an
iteration) waits until the replica has consumed the buffer it is about to reuse, which is the
only point where training can wait for the checkpoint side.

Multi-GPU: pass a torch.distributed process group as `group` and every gradient is all-reduced
(sum, then divided by the world size) inside its hook before the snapshot (Alg. 2 line 15,
`Sync`); every rank then holds the same G_t, model and replica.
"""
from __future__ import annotations

import os
import queue
import threading

import numpy as np
import torch

from . import dense_update, host_update


class LowDiffPlus:
    def __init__(self, model: torch.nn.Module, opt: dict, lr: float, threads: int = 0, group=None,
                 adam_step: int = 0, checkpoint: bool = True):
        params = [p for p in model.parameters() if p.requires_grad]
        assert params and all(p.dtype == torch.float32 and p.is_cuda for p in params)
        dev = params[0].device
        n = sum(p.numel() for p in params)
        self.n, self.opt, self.lr = n, dict(opt), float(np.float32(lr))
        self.threads = threads or os.cpu_count() or 1
        self.group = group
        self.checkpoint = checkpoint          # False: the same training step with no replica
        # the GPU model M^G: parameters and their gradients become views of two flat buffers
        self.flat = torch.empty(n, device=dev)
        self.gflat = torch.zeros(n, device=dev)
        self.slices = []
        off = 0
        for p in params:
            k = p.numel()
            self.flat[off:off + k].copy_(p.detach().reshape(-1))
            p.data = self.flat[off:off + k].view_as(p)
            p.grad = self.gflat[off:off + k].view_as(p)
            self.slices.append((p, off, k))
            off += k
        kind = opt["kind"]
        zeros = lambda: torch.zeros(n, device=dev)
        self.state = {"x": self.flat, "m": None if kind == "sgd" else zeros(),
                      "v": zeros() if kind == "adam" else None, "x_bf16": None, "n": n, "lo": 0, "hi": n,
                      "t": 0, "adam_step": adam_step, "momentum_initialized": 0}
        torch.cuda.synchronize(dev)
        # the CPU replica M^C (aligned with M^G at t = 0)
        host = lambda t: None if t is None else t.detach().cpu().clone()
        self.replica = {**{k: host(self.state[k]) for k in ("x", "m", "v")}, "x_bf16": None, "n": n, "lo": 0,
                        "hi": n, "t": 0, "adam_step": adam_step, "momentum_initialized": 0}
        self.hbuf = [torch.empty(n, pin_memory=True) for _ in range(2)]
        self.copy_stream = torch.cuda.Stream(device=dev)
        self.free = [threading.Event(), threading.Event()]
        for e in self.free:
            e.set()
        self.q: queue.Queue = queue.Queue()
        self.error = None
        self.worker = threading.Thread(target=self._worker, daemon=True)
        self.worker.start()
        self.t = 0
        for p, off, k in self.slices:
            p.register_post_accumulate_grad_hook(self._hook(off, k))

    # ---- training side ---------------------------------------------------------------------------
    def zero_grad(self):
        """Start of an iteration: wait until the replica released the pinned buffer this
        iteration snapshots into, then zero the gradients in place (they stay views)."""
        if not self.checkpoint:
            self.gflat.zero_()
            return
        self.free[self.t % 2].wait()
        if self.error:
            raise self.error
        self.free[self.t % 2].clear()
        torch.cuda.current_stream().wait_stream(self.copy_stream)   # last snapshot read gflat
        self.gflat.zero_()

    def _hook(self, off: int, k: int):
        def hook(p):
            g = self.gflat[off:off + k]
            if self.group is not None:                         # Sync (Alg. 2 line 15)
                torch.distributed.all_reduce(g, group=self.group)
                g.div_(torch.distributed.get_world_size(self.group))
            if not self.checkpoint:
                return
            ready = torch.cuda.Event()
            ready.record()
            self.copy_stream.wait_event(ready)
            with torch.cuda.stream(self.copy_stream):          # layer-wise snapshot (line 19)
                self.hbuf[self.t % 2][off:off + k].copy_(g, non_blocking=True)
        return hook

    def step(self, lr: float | None = None):
        """After backward: the GPU update (line 7); iteration t's snapshot goes to the replica."""
        lr = self.lr if lr is None else float(np.float32(lr))
        dense_update(self.state, self.opt, self.gflat, lr)
        if not self.checkpoint:
            self.t += 1
            return
        copied = torch.cuda.Event()
        copied.record(self.copy_stream)
        self.q.put((self.t % 2, copied, lr))
        self.t += 1

    # ---- checkpointing side -------------------------------------------------------------------------
    def _worker(self):
        while True:
            item = self.q.get()
            if item is None:
                return
            slot, copied, lr = item
            try:
                copied.synchronize()                                # all layers snapshotted
                host_update(self.replica, self.opt, self.hbuf[slot], lr, self.threads)   # line 12
            except Exception as e:                                  # surfaced on the training side
                self.error = e
            self.free[slot].set()

    def flush(self):
        """Wait until the replica has applied every finished iteration."""
        for e in self.free:
            e.wait()
        if self.error:
            raise self.error

    def recover(self):
        """Software-failure recovery: the GPU model and optimizer state from the
        in-memory replica."""
        self.flush()
        for k in ("x", "m", "v"):
            if self.state[k] is not None:
                self.state[k].copy_(self.replica[k], non_blocking=False)
        for k in ("t", "adam_step", "momentum_initialized"):
            self.state[k] = self.replica[k]
        self.t = self.replica["t"]
        return self.state

    def close(self):
        self.q.put(None)
        self.worker.join()
