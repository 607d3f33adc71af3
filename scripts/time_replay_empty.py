"""Lower bound of the dense Adam replay: the C3-sized chain with NO entries (every step a decay step),
same launch configuration as time_replay.py. python scripts/time_replay_empty.py [--config 3] [--approx 1]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sc_yaolhlzz25_b200 as ld  # noqa: E402
from workloads import CONFIGS, full_checkpoint  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=3)
ap.add_argument("--approx", type=int, default=1)
ap.add_argument("--reps", type=int, default=10)
a = ap.parse_args()
cfg = CONFIGS[a.config]
dev = torch.device("cuda", 0)
n, B, K = cfg.n, cfg.B, cfg.K
lr = float(np.float32(cfg.hyper["lr"]))
recs = []
for b in range(K // B):
    ring = [(torch.zeros(1, dtype=torch.int32, device=dev), torch.zeros(1, device=dev),
             torch.zeros(1, dtype=torch.int64, device=dev), 1, lr) for _ in range(B)]
    rec, d_bytes = ld.batch_merge(ring, "stack", n, 0, n, b * B, 1)
    nb = ld.record_bytes(d_bytes, rec.numel())
    head = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
    ld.stage_d2h(rec, nb, head)
    torch.cuda.synchronize()
    recs.append((rec, head))
ck = full_checkpoint(cfg, 0, n, dev)
st = {"x0": ck["x"], "m0": ck["m"], "v0": ck["v"], "x": torch.empty_like(ck["x"]), "m": torch.empty_like(ck["m"]),
      "v": torch.empty_like(ck["v"]), "x_bf16": None, "n": n, "lo": 0, "hi": n}
opt = {"kind": "adam", **{k2: v2 for k2, v2 in cfg.hyper.items() if k2 != "lr"}, "approx_math": a.approx}
ms = []
for i in range(a.reps + 3):
    st.update(t=0, adam_step=ck["adam_step"], momentum_initialized=0)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    ld.replay(st, opt, recs, check=False)
    e1.record()
    torch.cuda.synchronize()
    if i >= 3:
        ms.append(e0.elapsed_time(e1))
print(json.dumps({"config": cfg.name, "approx": a.approx, "empty_chain_replay_ms_median": float(np.median(ms)),
                  "param_steps": n * K}))
