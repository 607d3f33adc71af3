"""Device time of the recovery replay alone (GPU): the bench's C3/C4 record chain, replayed from
the full checkpoint back to back with CUDA events, with SM clocks sampled by NVML meanwhile.
python scripts/time_replay.py [--config 3] [--reps 20]"""
import argparse
import json
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sc_yaolhlzz25_b200 as ld  # noqa: E402
from workloads import CONFIGS, full_checkpoint, gradient, segment_sigmas  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=3)
ap.add_argument("--reps", type=int, default=20)
ap.add_argument("--ef-warmup", type=int, default=0, help="EF iterations (gradient cycle of B) before the chain")
ap.add_argument("--grad-pool", type=int, default=0, help="distinct gradients cycled (default B; C5 needs <= 4)")
ap.add_argument("--approx", type=int, default=0, help="lowdiff_opt.approx_math (Adam: MUFU sqrt/rcp)")
a = ap.parse_args()
cfg = CONFIGS[a.config]
dev = torch.device("cuda", 0)
n, k, B, K = cfg.n, cfg.k, cfg.B, cfg.K
sig = segment_sigmas(cfg, dev)
r = torch.zeros(n, device=dev)
ws = torch.zeros(ld.compress_workspace_size(n, k), dtype=torch.uint8, device=dev)
slots = [torch.empty(ld.pairs_bytes(k, cfg.vdt), dtype=torch.uint8, device=dev) for _ in range(B)]
d_k = torch.full((1,), k, dtype=torch.int64, device=dev)
lr = float(np.float32(cfg.hyper["lr"]))
G = a.grad_pool or B
grads = [gradient(cfg, 0, t, dev, sigmas=sig) for t in range(G)]
for t in range(a.ef_warmup):                     # error-feedback steady state, as in the bench
    ld.compress(grads[t % G], r, k, vdt=cfg.vdt, pairs=slots[0], ws=ws)
recs = []
for b in range(K // B):
    ring = []
    for j in range(B):
        ld.compress(grads[j % G], r, k, vdt=cfg.vdt, pairs=slots[j], ws=ws)
        ring.append(ld.pairs_views(slots[j], k, cfg.vdt) + (d_k, k, lr))
    rec, d_bytes = ld.batch_merge(ring, "stack", n, 0, n, b * B, 1)
    nb = ld.record_bytes(d_bytes, rec.numel())
    head = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
    ld.stage_d2h(rec, nb, head)
    torch.cuda.synchronize()
    recs.append((rec, head))
del sig, r, ws, grads
ck = full_checkpoint(cfg, 0, n, dev)
xb = torch.empty(n, dtype=torch.bfloat16, device=dev) if cfg.gdt == "bf16" else None
st = {"x0": ck["x"], "m0": ck["m"], "v0": ck["v"], "x": torch.empty_like(ck["x"]), "m": torch.empty_like(ck["m"]),
      "v": torch.empty_like(ck["v"]) if ck["v"] is not None else None, "x_bf16": xb, "n": n, "lo": 0, "hi": n}
opt = {"kind": cfg.opt, **{k2: v2 for k2, v2 in cfg.hyper.items() if k2 != "lr"}, "approx_math": a.approx}
clocks, stop = [], [False]


def sample():
    import pynvml
    pynvml.nvmlInit()
    h = pynvml.nvmlDeviceGetHandleByIndex(0)
    while not stop[0]:
        clocks.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
        time.sleep(0.002)


def run(reps):
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for i in range(reps):
        st.update(t=0, adam_step=ck["adam_step"], momentum_initialized=ck["momentum_initialized"])
        ev[i][0].record()
        ld.replay(st, opt, recs, check=False)
        ev[i][1].record()
    torch.cuda.synchronize()
    return [x.elapsed_time(y) for x, y in ev]


run(3)
th = threading.Thread(target=sample)
th.start()
ms = run(a.reps)
stop[0] = True
th.join()
print(json.dumps({"config": cfg.name, "ef_warmup": a.ef_warmup, "approx": a.approx, "replay_ms_median": float(np.median(ms)), "replay_ms_min": min(ms),
                  "sm_mhz_median": float(np.median(clocks)) if clocks else None,
                  "sm_mhz_min": min(clocks) if clocks else None, "clock_samples": len(clocks)}))
