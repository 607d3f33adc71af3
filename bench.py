#!/usr/bin/env python
"""LowDiff hot-path benchmark (BASELINE.json metric: "diff-build & replay gradient GB/s at
1/2/4/8 B200, % of HBM roofline").

One STEP = one pass of the whole hot path over one replay chain of
K = R*B iterations (the config's chain length; R = K/B batch records):
  R times: B iterations of compress (top-k + EF) -> sparse all-gather (NCCL for P > 1) + coalesce
  of this rank's shard -> ring slot; then batch merge of the B differentials -> record -> async
  D2H stage into pinned host memory (copy stream);
  then recovery: Load(C^F) + replay of the R-record chain onto this rank's checkpoint shard.
value = gradient bytes all ranks fed through the path per second = P * K * n * sizeof(g) / t_step.

Workload (N = 1 line): config C3 = BASELINE configs[2], the VGG-16-shaped gradient the metric's
1/2/4/8-GPU scaling is quoted on (n = 138,357,544 fp32, rho = 0.001, B = 16, K = 16: one record,
Adam replay of its 16 iterations). Inputs are synthetic (workloads/, seeded), resident in HBM
before timing; every gradient (553 MB) is larger than the 126 MB L2, so no flush is needed.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config 3] [--impl ours|reference]
  torchrun --nproc-per-node N bench.py --gpus N ...
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

REASONS = {  # nvidia-smi clocks_event_reasons bits
    0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
    0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
    0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}


def parse_args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-graph", action="store_true", help="time eager launches (no CUDA graph)")
    ap.add_argument("--exact-replay", action="store_true",
                    help="Adam replay with correctly rounded sqrt/div (bit-exact vs the oracle) in the timed "
                         "step; default approx_math (MUFU sqrt/rcp, x within north_star's fp32 tolerance)")
    ap.add_argument("--sync", default="p2p", choices=["p2p", "nccl"],
                    help="N > 1: all-gather fused with the coalesce over peer memory (p2p, default) or "
                         "ncclAllGather + coalesce (nccl)")
    ap.add_argument("--copy-sync", action="store_true",
                    help="P = 1: run the (identity) coalesce into a separate ring slot instead of the "
                         "zero-copy hand-off")
    ap.add_argument("--grad-pool", type=int, default=0,
                    help="distinct resident gradients cycled through (0 = one per iteration of the batch)")
    return ap.parse_args()


# ---------------------------------------------------------------------------------------------
# CPU oracle arm (cpu_baseline and --impl reference): the oracle as it stands, bounded sample
# ---------------------------------------------------------------------------------------------
def oracle_step_sample(cfg, n_s: int, t0: int = 0, grads=None):
    """Time the oracle on one step of the same workload restricted to the first n_s gradient
    elements (same rho, B, chain length, optimizer): R = K/B batches of B compress + coalesce and
    one merge each, then one replay of the R-record chain. `grads`: host copies of the GPU arm's own
    gradient tensors (same values); else drawn on the CPU. Returns (seconds, gradient bytes)."""
    import numpy as np
    import oracle
    from workloads import gradient, segment_sigmas
    import torch
    k = max(1, int(cfg.rho * n_s))
    R = chain_records(cfg)
    if grads is None:
        sig = segment_sigmas(cfg)[:n_s]
        grads = [gradient(cfg, 0, t0 + t, "cpu", sigmas=sig, n=n_s) for t in range(cfg.B)]
        grads = [g.view(torch.int16).numpy().view(np.uint16) if cfg.gdt == "bf16" else g.numpy() for g in grads]
    r = np.zeros(n_s, np.float32)
    lr = np.float32(cfg.hyper["lr"])
    x = np.zeros(n_s, np.float32); m = np.zeros(n_s, np.float32); v = np.zeros(n_s, np.float32)
    o_vdt = oracle.BF16 if cfg.vdt == "bf16" else oracle.F32
    mode = oracle.STACK if cfg.merge == "stack" else oracle.SUM
    t_start = time.perf_counter()
    recs = []
    for b in range(R):
        diffs = []
        for t in range(cfg.B):
            idx, val, r = oracle.compress(grads[t], r, k, o_vdt)
            diffs.append(oracle.coalesce([oracle.pairs_pack(idx, val, o_vdt)], k, o_vdt, 0, n_s, True))
        recs.append(oracle.batch_merge(diffs, lr, mode, n_s, 0, n_s, t0 + b * cfg.B, 1))
    st = {"x": x, "m": m if cfg.opt != "sgd" else None, "v": v if cfg.opt == "adam" else None,
          "n": n_s, "lo": 0, "hi": n_s, "t": t0, "adam_step": 1000, "momentum_initialized": 1}
    opt = {"kind": cfg.opt, **{k2: v2 for k2, v2 in cfg.hyper.items() if k2 != "lr"}}
    oracle.replay(opt, st, recs)
    dt = time.perf_counter() - t_start
    gbytes = R * cfg.B * n_s * (2 if cfg.gdt == "bf16" else 4)
    return dt, gbytes


def host_description() -> dict:
    """nproc and the CPU model of the host the oracle runs on."""
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    try:
        avail = len(os.sched_getaffinity(0))
    except AttributeError:
        avail = os.cpu_count()
    return {"nproc": avail, "cpu_model": model}


def _oracle_worker(args):
    cfg_id, n_s, grads = args
    from workloads import CONFIGS
    dt, gb = oracle_step_sample(CONFIGS[cfg_id], n_s, grads=grads)
    return dt, gb


def oracle_all_cores(cfg, n_s: int, grads, procs: int) -> dict:
    """The same bounded step as `procs` independent oracle processes at once (independent units, as
    P data-parallel ranks would be): aggregate gradient GB/s over the wall time."""
    import multiprocessing as mp
    ctx = mp.get_context("fork")
    t0 = time.perf_counter()
    with ctx.Pool(procs) as pool:
        res = pool.map(_oracle_worker, [(cfg.cid, n_s, grads)] * procs)
    wall = time.perf_counter() - t0
    return {"value": sum(gb for _, gb in res) / wall / 1e9, "unit": "GB/s", "processes": procs,
            "wall_s": wall}


def max_over_ranks(ms: float, world: int) -> float:
    """The step time of the whole job: the slowest rank's device time (all_reduce MAX over the
    host process group; identity at world 1)."""
    if world <= 1:
        return ms
    import torch
    import torch.distributed as dist
    t = torch.tensor([ms], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def rank_table(world: int, rank: int, local: int, nbytes: int, nnz: int) -> list | None:
    """Per-rank device id, PCI bus id and shard record size, gathered to rank 0 (evidence that
    every rank ran on its own GPU, and the shard skew of SURVEY §8(e))."""
    import torch
    pci = None
    try:
        pci = torch.cuda.get_device_properties(local).pci_bus_id
    except Exception:
        pass
    mine = {"rank": rank, "device": local, "pci_bus_id": pci, "record_bytes": int(nbytes), "nnz": int(nnz)}
    if world <= 1:
        return [mine]
    import torch.distributed as dist
    out = [None] * world
    dist.all_gather_object(out, mine)
    return out if rank == 0 else None


def chain_records(cfg) -> int:
    """Records per step: the config's replay chain of K differentials is K/B batch records."""
    return max(1, cfg.K // cfg.B)


def run_reference(args, cfg):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return  # rank 0 alone runs the CPU oracle arm
    import numpy as np
    import torch
    from workloads import gradient, segment_sigmas
    n_s = max(1 << 16, cfg.n // 16)                    # the same bounded sample as the GPU arm's cpu_baseline
    # the GPU arm's own gradient values: drawn with the CUDA generator when a GPU is present
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    sig = segment_sigmas(cfg, dev)[:n_s]
    grads = [gradient(cfg, 0, t, dev, sigmas=sig, n=n_s) for t in range(cfg.B)]
    grads = [g.view(torch.int16).cpu().numpy().view(np.uint16) if cfg.gdt == "bf16" else g.cpu().numpy()
             for g in grads]
    for w in range(args.warmup):
        oracle_step_sample(cfg, n_s, grads=grads)
    times, gb = [], 0
    for s in range(args.steps):
        dt, gb = oracle_step_sample(cfg, n_s, grads=grads)
        times.append(dt)
    tot = sum(times)
    val = args.steps * gb / tot / 1e9
    sample = (f"oracle (plain C++, 1 thread) full step of {cfg.name} on the first {n_s} of n={cfg.n} "
              f"gradient elements (rho={cfg.rho}, {chain_records(cfg)} batches of B={cfg.B}, {cfg.opt} replay "
              f"of the {cfg.K}-iteration chain; gradients from the {dev.upper()} generator, the GPU arm's values)")
    line = {"impl": "reference", "metric": "diff-build & replay gradient GB/s at 1/2/4/8 B200, % of HBM roofline",
            "value": val, "unit": "GB/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * tot / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32" if cfg.gdt == "f32" else "bf16", "data": "synthetic",
            "config": {"workload": cfg.name, "n": cfg.n, "n_sample": n_s, "rho": cfg.rho, "B": cfg.B,
                       "replay": f"{cfg.opt}, chain of {cfg.K} iterations ({chain_records(cfg)} records)"},
            "cpu_baseline": {"value": val, "unit": "GB/s", "cores": 1, "kind": "oracle", "sample": sample,
                             **host_description()},
            "e2e": {"value": val, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line)


# ---------------------------------------------------------------------------------------------
# GPU arm
# ---------------------------------------------------------------------------------------------
class ClockSampler:
    """SM clock and clock-event (throttle) reasons DURING the timed region: NVML polled every ~5 ms
    from a thread (one sample at start() and one at stop() as well, so even a few-millisecond timed
    region has samples); nvidia-smi -lms 20 only if NVML is unavailable."""

    def __init__(self, index: int):
        self.index, self.proc, self.path, self.thread = index, None, None, None
        self.samples, self.stop_flag = [], False

    def _nvml_sample(self):
        import pynvml
        sm = pynvml.nvmlDeviceGetClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        mx = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        try:
            bits = pynvml.nvmlDeviceGetCurrentClocksEventReasons(self.h)
        except Exception:
            bits = pynvml.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
        self.samples.append((float(sm), float(mx), int(bits)))

    def start(self):
        try:
            import threading
            import pynvml
            pynvml.nvmlInit()
            self.h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self._nvml_sample()

            def run():
                while not self.stop_flag:
                    self._nvml_sample()
                    time.sleep(0.005)
            self.thread = threading.Thread(target=run, daemon=True)
            self.thread.start()
            return
        except Exception:
            self.thread = None
        try:
            self.path = os.path.join("/tmp", f"lowdiff_clocks_{os.getpid()}.csv")
            self.f = open(self.path, "w")
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index),
                 "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active",
                 "--format=csv,noheader,nounits", "-lms", "20"], stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.thread is not None:
            self.stop_flag = True
            self.thread.join()
            self._nvml_sample()
            rows = self.samples
        elif self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
            self.f.close()
            rows = []
            for line in open(self.path):
                parts = [p.strip() for p in line.split(",")]
                try:
                    rows.append((float(parts[0]), float(parts[1]), int(parts[2], 16)))
                except (ValueError, IndexError):
                    continue
        else:
            return None
        sm = [r[0] for r in rows]
        if not sm:
            return None
        reasons = {name for r in rows for b, name in REASONS.items() if r[2] & b and name != "gpu_idle"}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(r[1] for r in rows),
                "reasons": sorted(reasons), "samples": len(sm)}


def run_ours(args, cfg):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_sc_yaolhlzz25_b200 as ld
    from paper_conf_sc_yaolhlzz25_b200 import build
    from workloads import full_checkpoint, gradient, segment_sigmas

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("LOWDIFF_BENCH_DEVICE") is not None:   # tests: several ranks on one GPU
        local = int(os.environ["LOWDIFF_BENCH_DEVICE"])
    assert world == args.gpus or world == 1, "--gpus must match the torchrun world size"
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        # host plumbing only (barriers, the max-over-ranks time, the p2p handle exchange, the NCCL id
        # broadcast): gloo; the data path never goes through torch.distributed
        dist.init_process_group("gloo")
    build.build()
    P = world
    n, k, B = cfg.n, cfg.k, cfg.B
    gsz = 2 if cfg.gdt == "bf16" else 4
    lo, hi = ld.shard_bounds(n, P, rank)
    p2p, sync_note = None, None
    if P > 1 and args.sync == "p2p":
        try:
            p2p = ld.P2P(P, rank, k, cfg.vdt, device=dev)
        except ld.LowDiffError as e:                    # e.g. no IPC / peer access between the GPUs
            sync_note = f"p2p unavailable ({e}); ncclAllGather + coalesce"
            print(sync_note, file=sys.stderr)
    # N > 1: the NCCL communicator always exists (the baseline Sync route; with the fused P2P Sync
    # as the default it is timed as a second arm below), so every multi-GPU run shows NCCL
    comm, nccl_note = None, None
    if P > 1:
        try:
            comm = ld.Comm(P, rank)
        except ld.LowDiffError as e:                    # e.g. several ranks sharing one GPU (liveness runs)
            if p2p is None:
                raise
            nccl_note = f"NCCL communicator unavailable ({e}); P2P Sync only"
            print(nccl_note, file=sys.stderr)
    if P > 1:
        print(f"lowdiff rank {rank}/{P}: cuda:{local} ({torch.cuda.get_device_name(local)}), NCCL communicator "
              f"{'+ P2P exchange windows' if p2p is not None else 'only'}" if comm is not None else
              f"lowdiff rank {rank}/{P}: cuda:{local}, P2P exchange windows", file=sys.stderr, flush=True)

    # ---- resident inputs: B gradients (seeded, per rank), residual, full-checkpoint shard ----
    sig = segment_sigmas(cfg, dev)
    pool = B if args.grad_pool <= 0 else min(B, args.grad_pool)
    grads = [gradient(cfg, rank, t, dev, sigmas=sig) for t in range(pool)]
    del sig
    r = torch.zeros(n, device=dev)
    # Full checkpoint C^F shard (resident) and the recovered state M: every step's replay is one
    # recovery, Load(C^F_t) + replay of the batch's record (Alg.1 l.16-24), read from the checkpoint
    # and written to the state buffers (out of place: same HBM traffic as in place).
    ck = full_checkpoint(cfg, lo, hi, dev)
    # C4 (bf16 gradients, fp32 master): the replay also writes the bf16 copy of x
    xb = torch.empty(hi - lo, dtype=torch.bfloat16, device=dev) if cfg.gdt == "bf16" else None
    state = {"x0": ck["x"], "m0": ck["m"], "v0": ck["v"],
             "x": torch.empty_like(ck["x"]), "m": None if ck["m"] is None else torch.empty_like(ck["m"]),
             "v": None if ck["v"] is None else torch.empty_like(ck["v"]), "x_bf16": xb, "n": n, "lo": lo,
             "hi": hi, "t": 0, "adam_step": ck["adam_step"], "momentum_initialized": ck["momentum_initialized"]}
    opt = {"kind": cfg.opt, **{kk: vv for kk, vv in cfg.hyper.items() if kk != "lr"}}
    if cfg.opt == "adam":                                # DESIGN.md reading #33: x within 1e-6 rel / 1e-7 abs
        opt["approx_math"] = 0 if args.exact_replay else 1
    lr = float(np.float32(cfg.hyper["lr"]))
    cap = min(P * k, hi - lo)
    ring = [(torch.empty(cap, dtype=torch.int32, device=dev), torch.empty(cap, device=dev),
             torch.zeros(1, dtype=torch.int64, device=dev)) for _ in range(B)]
    pairs = torch.empty(ld.pairs_bytes(k, cfg.vdt), dtype=torch.uint8, device=dev)
    # the residual's own compress workspace: it carries the warm threshold state between calls
    cws = torch.empty(ld.compress_workspace_size(n, k), dtype=torch.uint8, device=dev)
    # P = 1: the Sync of one list is the identity (union of one list, fp32(v) / 1 exact), so ring
    # slot j IS iteration j's compressed pairs buffer — the Reusing Queue's
    # zero-copy hand-off: compress writes into the slot, the merge reads it in place.
    zero_copy = P == 1 and not args.copy_sync        # (bf16 values: widened exactly by the merge)
    if zero_copy:
        slots = [torch.empty(ld.pairs_bytes(k, cfg.vdt), dtype=torch.uint8, device=dev) for _ in range(B)]
        d_k = torch.full((1,), k, dtype=torch.int64, device=dev)
        ring = [ld.pairs_views(sl, k, cfg.vdt) + (d_k,) for sl in slots]
    rec_cap = ld.record_max_bytes(cfg.merge, B, B * cap, lo, hi)
    R = chain_records(cfg)                              # batch records per step (replay chain K = R*B)
    records = [torch.empty(rec_cap, dtype=torch.uint8, device=dev) for _ in range(R)]
    d_bytes = [torch.zeros(1, dtype=torch.int64, device=dev) for _ in range(R)]   # one per record
    meta = torch.cuda.Stream(device=dev)             # the checkpoint thread's size queries
    rec_done = [torch.cuda.Event() for _ in range(R)]
    heads = [torch.empty(80 + 4 * B + 16, dtype=torch.uint8, pin_memory=True) for _ in range(R)]
    staged = [torch.empty(rec_cap, dtype=torch.uint8, pin_memory=True) for _ in range(R)]
    main = torch.cuda.current_stream()
    copy_stream = torch.cuda.Stream()
    t_iter = [0]

    h2d_stream = torch.cuda.Stream()
    ev_copy = [torch.cuda.Event() for _ in range(2)]
    ev_free = [torch.cuda.Event() for _ in range(2)]

    use_p2p = [p2p is not None]                       # the Sync route of the build phase

    def build_phase(h2d=None):
        """B iterations of compress -> sparse all-gather + coalesce of this rank's shard -> ring.
        e2e (h2d given): iteration j's gradient is copied from pinned host memory on a copy stream
        into one of two device buffers, overlapping the compute of iteration j-1."""
        cs = torch.cuda.current_stream()              # the graph-capture stream when captured
        for j in range(B):
            if h2d is not None:
                D = len(h2d[0])
                d = j % D
                if j == 0:
                    h2d_stream.wait_stream(cs)        # buffers free: the previous batch is done
                elif j >= D:
                    h2d_stream.wait_event(ev_free[d])
                with torch.cuda.stream(h2d_stream):
                    h2d[0][d].copy_(h2d[1][j % len(h2d[1])], non_blocking=True)
                ev_copy[d].record(h2d_stream)
                cs.wait_event(ev_copy[d])
                g = h2d[0][d]
            else:
                g = grads[j % len(grads)]
            pp = p2p if use_p2p[0] else None
            dst = pp.slot() if pp is not None else pairs     # p2p: compress straight into the window
            if zero_copy:
                dst = slots[j]
            ld.compress(g, r, k, vdt=cfg.vdt, pairs=dst, ws=cws)
            if h2d is not None:
                ev_free[d].record(cs)
            if zero_copy:
                pass                                    # the slot already holds G~_t
            elif pp is not None:
                pp.allgather_sparse(dst, lo, hi, True, *ring[j])
            else:
                ld.allgather_sparse(comm, pairs, k, cfg.vdt, lo, hi, True, *ring[j])
        if h2d is not None:
            cs.wait_stream(h2d_stream)

    rec_nb = [0] * R

    def checkpoint_phase(b):
        """Batch merge -> record b (+ its header D2H for the host-side replay), enqueued on the
        training stream; the size query and the staging follow in finish(b)."""
        diffs = [(ring[j][0], ring[j][1], ring[j][2], cap, lr) for j in range(B)]
        ld.batch_merge(diffs, cfg.merge, n, lo, hi, t_iter[0], P, record=records[b], d_record_bytes=d_bytes[b])
        ld.stage_d2h(records[b], 80 + 4 * B, heads[b], main)   # header + lr[] for the host-side replay
        rec_done[b].record(main)
        t_iter[0] += B

    def finish(b):
        """The checkpoint thread learns record b's size on its own stream (waits for record b only:
        the training stream has already moved on to the next batch's compress), then stages it."""
        meta.wait_event(rec_done[b])
        nb = ld.record_bytes(d_bytes[b], rec_cap, stream=meta)   # syncs `meta` (covers the header)
        rec_nb[b] = nb
        if b < R - 1:                                   # the last record is staged behind the replay launch
            ld.stage_d2h(records[b], nb, staged[b], copy_stream)   # async persist staging (copy engine);
        return nb                                       # the record is complete: the host just synced

    def recovery_phase():
        """Load(C^F) + replay of the step's chain of R records (K = R*B iterations); the headers were
        copied before the last record_bytes synchronization, so the replay launches at once and the
        last record's staging is issued right after it (the copy engine works beside the replay)."""
        if os.environ.get("LOWDIFF_BENCH_SERIAL_STAGE"):  # experiment: staging not overlapped with replay
            ld.stage_d2h(records[R - 1], rec_nb[R - 1], staged[R - 1], copy_stream)
            copy_stream.synchronize()
        state["t"] = t_iter[0] - R * B                  # the checkpoint is stamped at the chain start
        state["adam_step"] = ck["adam_step"]
        state["momentum_initialized"] = ck["momentum_initialized"]
        ld.replay(state, opt, [(records[b], heads[b]) for b in range(R)], check=False)
        if not os.environ.get("LOWDIFF_BENCH_SERIAL_STAGE"):
            ld.stage_d2h(records[R - 1], rec_nb[R - 1], staged[R - 1], copy_stream)
        main.wait_stream(copy_stream)                   # the next step's merge overwrites the records

    def step(graph=None, h2d=None):
        """One pass of the path: R batches built, merged and staged, then the chain replayed."""
        nb = 0
        for b in range(R):
            if graph is not None:
                graph.replay()
            else:
                build_phase(h2d)
            checkpoint_phase(b)
            if b:
                nb += finish(b - 1)                     # record b-1's size while batch b builds
        nb += finish(R - 1)
        recovery_phase()
        return nb

    def timed(nsteps, **kw):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        nb = 0
        for _ in range(nsteps):
            nb = step(**kw)
        e1.record()
        torch.cuda.synchronize()
        ms = max_over_ranks(e0.elapsed_time(e1), world)
        if world > 1:
            dist.barrier()
        return ms, nb

    def capture(h2d=None):
        """The build phase as one CUDA graph (launch-latency removal); None if capture fails."""
        if args.no_graph:
            return None, 0
        try:
            torch.cuda.synchronize()
            g = torch.cuda.CUDAGraph()
            l0 = ld.launch_count()
            with torch.cuda.graph(g):
                build_phase(h2d)
            return g, ld.launch_count() - l0
        except Exception as e:                           # pragma: no cover
            print(f"graph capture failed ({e}); timing eager launches", file=sys.stderr)
            torch.cuda.synchronize()
            return None, 0

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    graph, graph_launches = capture()
    if graph is not None:
        step(graph=graph)                               # warm the graph once
        torch.cuda.synchronize()

    # ---- timed region (value): the whole path, build phase as a graph ----
    clocks = ClockSampler(local)
    clocks.start()
    launches0 = ld.launch_count()
    cc0 = ld.compress_counters(ws=cws)
    ms, rec_bytes = timed(args.steps, graph=graph)
    ld.replay_check()                                   # no record body failed device validation
    cc1 = ld.compress_counters(ws=cws)
    launches = ld.launch_count() - launches0 + (graph_launches * args.steps if graph is not None else 0)
    clk = clocks.stop()
    # ---- profiled pass (same work, eager launches, CUDA events around every kernel) ----
    ld.profile_enable(True)
    pms, _ = timed(args.steps)
    ld.profile_enable(False)
    cc2 = ld.compress_counters(ws=cws)
    # compress paths over both passes: 0 = warm first-pass candidates, 2 = rescan
    # recovery inside the select, 1 = exact full-array select; counted on the device
    paths = {"calls": cc2["calls"] - cc0["calls"], "fast_select": cc2["fast_calls"] - cc0["fast_calls"],
             "rescans": cc2["rescans"] - cc0["rescans"],
             "fallbacks": cc2["fallbacks"] - cc0["fallbacks"],
             "timed": {q: cc1[q] - cc0[q] for q in ("calls", "rescans", "fallbacks")},
             "since_start": {q: cc2[q] for q in ("calls", "rescans", "fallbacks", "nonfinite_calls")},
             "last_candidates_per_k": cc2["last_candidates"] / k, "margin": cc2["delta"]}
    prof = {c: ld.profile_query(c) for c in ("compress_stream", "compress_select",
                                             "coalesce", "starts", "merge", "merge_pack",
                                             "replay_dense", "replay_sparse")}
    ms_step = ms / args.steps
    value = P * R * B * n * gsz / (ms_step * 1e-3) / 1e9
    # ---- N > 1: the same steps with the baseline Sync (ncclAllGather + coalesce) as a second arm ----
    sync_arms = None
    if P > 1:
        sync_arms = {("p2p" if use_p2p[0] else "nccl"): ms_step}
        if p2p is not None and comm is not None:
            use_p2p[0] = False
            g_nccl, _ = capture()
            step(graph=g_nccl) if g_nccl is not None else step()
            ms_n, _ = timed(args.steps, graph=g_nccl) if g_nccl is not None else timed(args.steps)
            sync_arms["nccl"] = ms_n / args.steps
            use_p2p[0] = True
        sync_arms["unit"] = "ms per step (max over ranks)"
        if nccl_note:
            sync_arms["note"] = nccl_note
    nnz_rank = int(np.frombuffer(heads[0].numpy().tobytes()[:80], dtype=np.uint64)[7]) if R else 0
    ranks = rank_table(world, rank, local, sum(rec_nb), nnz_rank)

    # ---- roofline of the dominant kernel (measured live over the timed region) ----
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    peak_note = "MEASURED_PEAKS.json hbm_gbs (measured copy)" if "hbm_gbs" in peaks else "fallback 6.65 TB/s"
    cs_ms, cs_n = prof["compress_stream"]
    alg_bytes = (gsz + 8) * n + (4 + (2 if cfg.vdt == "bf16" else 4) + 4) * k   # read g,r; write r; pairs; r on S
    achieved = alg_bytes / (cs_ms / cs_n * 1e-3) / 1e9 if cs_n else 0.0
    traffic = None
    summ = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if os.path.exists(summ):
        try:
            traffic = json.load(open(summ)).get(cfg.name, {}).get("compress_stream", {}).get("dram_bytes_per_launch")
        except Exception:
            traffic = None
    total_prof = sum(v[0] for v in prof.values()) or 1.0
    kernels = {c: {"ms_per_step": v[0] / args.steps, "launches_per_step": v[1] / args.steps,
                   "share": v[0] / total_prof} for c, v in prof.items() if v[1]}
    roofline = {"bound": "hbm", "kernel": "compress_stream", "achieved": achieved, "peak": hbm_peak,
                "unit": "GB/s", "frac": achieved / hbm_peak, "traffic": traffic,
                "alg_bytes_per_launch": alg_bytes, "launch_ms": cs_ms / cs_n if cs_n else None,
                "peak_source": peak_note}

    # ---- the replay kernel against its own bound (HBM bytes and, for Adam, the MUFU floor) ----
    replay_roof = None
    rp_ms, rp_n = prof.get("replay_dense", (0.0, 0))
    if rp_n:
        nloc = hi - lo
        sb = {"sgd": 8, "momentum": 16, "adam": 24}[cfg.opt]          # read + write of x (m, v)
        sb += 2 if xb is not None else 0                                 # + the bf16 copy of x (C4)
        alg = sb * nloc + int(rec_bytes)                                 # + the chain's records
        t_s = rp_ms / args.steps * 1e-3                                  # per step (one chain)
        replay_roof = {"kernel": "replay_dense", "alg_bytes_per_step": alg,
                       "achieved_gbs": alg / t_s / 1e9, "hbm_frac": alg / t_s / 1e9 / hbm_peak,
                       "ms_per_step": rp_ms / args.steps}
        if cfg.opt == "adam" and opt.get("approx_math"):
            # approx_math: in the zero-gradient loop one MUFU.RSQ every other step
            # (0.5 per parameter-step; the XU pipe issues 16 lanes/clk/SM: 32 parameter-steps/clk/SM)
            # and 6.5 fp32 lane-ops per parameter-step (FFMA2/FMUL2; 128 lanes/clk/SM: 19.7
            # parameter-steps/clk/SM): the fp32 pipe is the floor.
            f_mhz = (clk or {}).get("sm_mhz") or 1965.0
            psteps = nloc * R * B
            floor_s = psteps / (148 * (128 / 6.5) * f_mhz * 1e6)
            replay_roof.update({"bound": "alu", "math": "approx", "alu_floor_ms": floor_s * 1e3,
                                "alu_frac": floor_s / t_s,
                                "alu_peak": f"19.7 parameter-steps/clk/SM x 148 SMs at {f_mhz:.0f} MHz (6.5 fp32 "
                                            "lane-ops at 128 lanes/clk/SM; 0.5 MUFU at 16 lanes/clk/SM)",
                                "param_steps_per_s": psteps / t_s})
        elif cfg.opt == "adam":
            # Per parameter-step the exact Adam step issues 15 fp32 operations (FFMA2 pairs) and 2
            # MUFU ops. Measured on B200 (scripts/micro/adam_mix.cu, profiles/adam_mix_r01.txt):
            # fp32 128 lanes/clk/SM, MUFU 32/clk/SM, so the fp32 pipe is the floor; the same
            # instruction mix with no memory or bookkeeping peaks at 1.96 T parameter-steps/s.
            f_mhz = (clk or {}).get("sm_mhz") or 1965.0
            psteps = nloc * R * B
            floor_s = 15.0 * psteps / (148 * 128 * f_mhz * 1e6)
            mix_s = psteps / 1.96e12
            replay_roof.update({"bound": "alu", "math": "exact", "alu_floor_ms": floor_s * 1e3, "alu_frac": floor_s / t_s,
                                "alu_peak": f"fp32 128 lanes/clk/SM x 148 SMs at {f_mhz:.0f} MHz (15 ops per "
                                            "parameter-step; MUFU 32/clk/SM is not binding)",
                                "mix_ceiling_ms": mix_s * 1e3, "mix_frac": mix_s / t_s,
                                "param_steps_per_s": psteps / t_s})
        else:
            replay_roof["bound"] = "alu" if replay_roof["hbm_frac"] < 0.5 else "hbm"

    # ---- recovery from host memory: the staged records copied H2D, then the replay ----
    def replay_from_host(reps=3):
        torch.cuda.synchronize()
        copy_stream.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            for b in range(R):
                records[b][:rec_nb[b]].copy_(staged[b][:rec_nb[b]], non_blocking=True)
            recovery_phase()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / reps
    replay_h2d_ms = replay_from_host()

    # ---- the same recovery with the correctly rounded Adam (bit-exact vs the oracle), for reference ----
    replay_exact = None
    if opt.get("approx_math"):
        def replay_ms(o, reps=3):
            torch.cuda.synchronize()
            a, z = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            for _ in range(reps):
                state["t"], state["adam_step"] = t_iter[0] - R * B, ck["adam_step"]
                ld.replay(state, o, [(records[b], heads[b]) for b in range(R)], check=False)
            z.record()
            torch.cuda.synchronize()
            return a.elapsed_time(z) / reps
        replay_exact = {"ms_exact": replay_ms({**opt, "approx_math": 0}), "ms_approx": replay_ms(opt),
                        "note": "recovery replay of the step's chain alone, Load(C^F) included; exact = correctly "
                                "rounded sqrt/div, bit-exact vs the oracle; approx = the timed step's"}

    # ---- stage (a5): the D2H copies of the step's records on the copy engine, and the pinned peak ----
    def stage_timing():
        torch.cuda.synchronize()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(R)]
        for b in range(R):
            ev[b][0].record(copy_stream)
            ld.stage_d2h(records[b], rec_nb[b], staged[b], copy_stream)
            ev[b][1].record(copy_stream)
        copy_stream.synchronize()
        st_ms = sum(a.elapsed_time(z) for a, z in ev)
        probe = torch.empty(1 << 28, dtype=torch.uint8, device=dev)
        host = torch.empty(1 << 28, dtype=torch.uint8, pin_memory=True)
        a, z = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        host.copy_(probe, non_blocking=True)
        a.record()
        for _ in range(3):
            host.copy_(probe, non_blocking=True)
        z.record()
        torch.cuda.synchronize()
        peak = 3 * (1 << 28) / (a.elapsed_time(z) * 1e-3) / 1e9
        del probe, host
        nbs = sum(rec_nb)
        return {"bytes_per_step": int(nbs), "ms_per_step": st_ms, "gbs": nbs / (st_ms * 1e-3) / 1e9 if st_ms else None,
                "pcie_d2h_peak_gbs": peak, "engine": "copy stream (cudaMemcpyAsync D2H into pinned memory)",
                "hidden": bool(st_ms < replay_prof_ms),
                "hidden_basis": "the last record's copy overlaps the recovery replay that follows it in the step"}
    build_prof_ms = sum(v[0] for c, v in prof.items() if not c.startswith("replay")) / args.steps
    replay_prof_ms = sum(v[0] for c, v in prof.items() if c.startswith("replay")) / args.steps
    stage = stage_timing()

    # ---- e2e: same metric through the public API with host buffers (pinned H2D of every gradient) ----
    e2e = None
    cpu_grads = grads[:2]                               # kept for the CPU baseline (same values)
    if not args.no_e2e:
        npool = min(B, 2)
        hpool = [torch.empty(n, dtype=grads[0].dtype, pin_memory=True) for _ in range(npool)]
        for i in range(npool):
            hpool[i].copy_(grads[i])
        dpool = [torch.empty_like(grads[0]) for _ in range(npool)]
        del grads
        torch.cuda.empty_cache()
        eg, _ = capture(h2d=(dpool, hpool))
        kw = {"graph": eg} if eg is not None else {"h2d": (dpool, hpool)}
        step(**kw)
        e_steps = max(1, min(args.steps, 3))
        ems, enb = timed(e_steps, **kw)
        e_ms = ems / e_steps
        e2e = {"value": P * R * B * n * gsz / (e_ms * 1e-3) / 1e9, "unit": "GB/s",
               "h2d_bytes_per_step": R * B * n * gsz, "d2h_bytes_per_step": int(enb) + R * (80 + 4 * B + 8),
               "ms_per_step": e_ms, "steps": e_steps}

    # ---- CPU oracle baseline (rank 0, N = 1 only), on the GPU arm's own gradient values ----
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle
        n_s = max(1 << 16, cfg.n // 16)
        hgr = [(gg[:n_s].view(torch.int16).cpu().numpy().view(np.uint16) if cfg.gdt == "bf16"
                else gg[:n_s].cpu().numpy()) for gg in cpu_grads]
        hgr = [hgr[t % len(hgr)] for t in range(B)]
        dts = []
        for _ in range(2):
            dt, gb = oracle_step_sample(cfg, n_s, grads=hgr)
            dts.append(dt)
        dt = min(dts)
        host = host_description()
        cpu = {"value": gb / dt / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle",
               "sample": f"one full step of {cfg.name} on the first {n_s} of n={cfg.n} elements of the GPU "
                         f"arm's own gradient tensors (B={cfg.B} compress+coalesce, merge, {cfg.opt} replay), "
                         f"best of 2: {dt:.1f} s",
               **host}
        try:
            cpu["all_cores"] = oracle_all_cores(cfg, n_s, hgr, max(1, min(host["nproc"] or 1, 16)))
        except Exception as e:                          # pragma: no cover
            cpu["all_cores"] = {"error": str(e)[:200]}
        # one full-n compress step on the GPU's exact inputs (its gradient and current residual):
        # the oracle's time for that step, and the GPU's output for the same inputs compared bytewise
        g_full, r_dev = cpu_grads[0], r.clone()
        g_np = g_full.view(torch.int16).cpu().numpy().view(np.uint16) if cfg.gdt == "bf16" else g_full.cpu().numpy()
        r_np = r_dev.cpu().numpy()
        ovd = oracle.BF16 if cfg.vdt == "bf16" else oracle.F32
        t0 = time.perf_counter()
        oi, ov, ro = oracle.compress(g_np, r_np, k, ovd)
        t_c = time.perf_counter() - t0
        pairs_chk = ld.compress(g_full, r_dev, k, vdt=cfg.vdt)
        same = bool(np.array_equal(pairs_chk.cpu().numpy(), oracle.pairs_pack(oi, ov, ovd)) and
                    np.array_equal(r_dev.cpu().numpy().view(np.uint32), ro.view(np.uint32)))
        cpu["compress_full_n"] = {"value": n * gsz / t_c / 1e9, "unit": "GB/s", "seconds": t_c,
                                  "gpu_equals_oracle": same,
                                  "sample": "one compress of the full gradient at the bench's EF state "
                                            "(D2H copies of the GPU's g and residual)"}

    if p2p is not None:                                 # a timed-out peer wait voids the numbers
        torch.cuda.synchronize()
        p2p.status()
    if rank == 0:
        line = {"metric": "diff-build & replay gradient GB/s at 1/2/4/8 B200, % of HBM roofline",
                "value": value, "unit": "GB/s", "n_gpus": P, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
                "dtype": "f32" if cfg.gdt == "f32" else "bf16", "data": "synthetic",
                "config": {"workload": cfg.name, "n": n, "k": k, "rho": cfg.rho, "B": B, "P": P,
                           "sync": (("local (P = 1): zero-copy ring of compressed pairs" if zero_copy else
                                     "local (P = 1): coalesce into the ring") if P == 1 else sync_note or args.sync),
                           "shard": [lo, hi], "replay": f"{cfg.opt}, chain of {R * B} iterations ({R} {cfg.merge.upper()} record{'s' if R > 1 else ''} of B={B})",
                           "l2": (f"inputs larger than L2 (each gradient {n * gsz / 1e6:.0f} MB > 126 MB), no flush"
                                  if n * gsz > 126e6 else
                                  f"working set {n * (gsz + 8) / 1e6:.1f} MB fits L2 (latency-class config)"),
                           "grad_pool": pool,
                           "batches_per_step": R,
                           "differentials_per_s": P * R * B / (build_prof_ms * 1e-3) if build_prof_ms else None,
                           "replayed_iterations_per_s": R * B / (replay_prof_ms * 1e-3) if replay_prof_ms else None,
                           "replayed_iterations_per_s_from_host": R * B / (replay_h2d_ms * 1e-3),
                           "throughput_basis": "differentials/s = P*K / (build+merge+stage kernel time per "
                                               "step); replayed iterations/s = K / replay kernel time, and "
                                               "with the records copied H2D from pinned memory first "
                                               "(profiled pass, CUDA events)",
                           "record_bytes": int(rec_bytes),
                           "ranks": ranks,
                           "shard_skew": (max(x["record_bytes"] for x in ranks) /
                                          (sum(x["record_bytes"] for x in ranks) / len(ranks))) if ranks else None,
                           "sync_arms": sync_arms,
                           "compress_paths": paths},
                "timing": {"build_phase": "one CUDA graph per step" if graph is not None else "eager launches",
                           "profiled_ms_per_step": pms / args.steps,
                           "profiled": "separate pass, eager launches, CUDA events around every kernel"},
                "roofline": roofline, "replay_roofline": replay_roof, "replay_math": replay_exact, "stage": stage, "kernels": kernels, "cpu_baseline": cpu, "e2e": e2e,
                "gpu_launches": int(launches), "clocks": clk}
        emit(line)
    if comm is not None:
        comm.destroy()
    if p2p is not None:
        dist.barrier()
        p2p.destroy()
    if world > 1:
        dist.destroy_process_group()


_JSON_OUT = None                                     # the real stdout when it is redirected (N > 1)


def emit(line: dict):
    """The one JSON line of this run, on the process's real stdout."""
    if _JSON_OUT is not None:
        _JSON_OUT.write(json.dumps(line) + "\n")
        _JSON_OUT.flush()
    else:
        print(json.dumps(line), flush=True)


def main():
    global _JSON_OUT
    if int(os.environ.get("WORLD_SIZE", "1")) > 1:
        # under torchrun, NCCL / c10d print banners (e.g. "NCCL version ...") on stdout at
        # communicator creation: route fd 1 to stderr for the run and keep the real stdout for the
        # JSON line alone
        sys.stdout.flush()
        _JSON_OUT = os.fdopen(os.dup(1), "w")
        os.dup2(2, 1)
    args = parse_args()
    from workloads import CONFIGS
    cfg = CONFIGS[args.config]
    if args.impl == "reference":
        run_reference(args, cfg)
    else:
        run_ours(args, cfg)


if __name__ == "__main__":
    main()
