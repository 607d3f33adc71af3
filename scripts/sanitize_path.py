"""Every kernel of liblowdiff on C1-sized inputs, for compute-sanitizer (memcheck, racecheck,
synccheck, initcheck): python scripts/sanitize_path.py
Compress (warm fast select, general select, rescan and full-array recovery, bf16), coalesce over
P = 3 lists, SUM / STACK merges, D2H stage, replay (sparse SGD, dense SGD+wd, momentum, Adam with the
bf16 copy), the live update, LowDiff+ dense update and parallel recovery. Exits non-zero on a
status error; the sanitizer reports memory / race / sync findings itself."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sc_yaolhlzz25_b200 as ld  # noqa: E402
from workloads import CONFIGS, gradient, segment_sigmas  # noqa: E402

dev = torch.device("cuda", 0)
cfg = CONFIGS[1]
n, k, B = cfg.n, cfg.k, 4
sig = segment_sigmas(cfg, dev)
r = torch.zeros(n, device=dev)
ws = torch.zeros(ld.compress_workspace_size(n, k), dtype=torch.uint8, device=dev)
ring = []
for t in range(6):                                   # cold (rescan), then warm calls
    g = gradient(cfg, 0, t, dev, sigmas=sig)
    pairs = ld.compress(g, r, k, ws=ws)
    di, dv, dn = ld.allgather_sparse(None, pairs, k, "f32", 0, n)
    ring.append((di, dv, dn, k, 0.1))
print("compress paths", ld.compress_counters(ws=ws))
# a larger k so the grid select (fast path) runs instead of the one-CTA select
k2 = 20_000
ws2 = torch.zeros(ld.compress_workspace_size(n, k2), dtype=torch.uint8, device=dev)
r2 = torch.zeros(n, device=dev)
for t in range(4):
    ld.compress(gradient(cfg, 0, t, dev, sigmas=sig), r2, k2, ws=ws2)
print("grid-select warm paths", ld.compress_counters(ws=ws2))
for t1, t2 in ((0x7F000000, None), (0, None), (0x7F000000, 0x7F000000)):   # rescan / full-array paths
    ld.debug_force_threshold(t1)
    ld.debug_force_rescan_threshold(t2)
    ld.compress(gradient(cfg, 0, 9, dev, sigmas=sig), r2, k2, ws=ws2)
ld.debug_force_threshold(None)
ld.debug_force_rescan_threshold(None)
print("grid-select forced paths", ld.compress_counters(ws=ws2))
gb = gradient(cfg, 0, 3, dev, sigmas=sig).to(torch.bfloat16)
ld.compress(gb, r2, k2, vdt="bf16", ws=ws2)
print("bf16 call path", ld.compress_stats(n, k2, ws=ws2)["path"])
# coalesce of P = 3 lists
P = 3
pl = [ld.compress(gradient(cfg, p, 0, dev, sigmas=sig), torch.zeros(n, device=dev), k) for p in range(P)]
gathered = torch.cat(pl)
lo, hi = ld.shard_bounds(n, P, 1)
ld.coalesce(gathered, P, k, "f32", lo, hi, True)
# merges, stage, replay
recs = []
for mode in ("sum", "stack"):
    rec, d_bytes = ld.batch_merge(ring[:B], mode, n, 0, n, 0, 1)
    nb = ld.record_bytes(d_bytes, rec.numel())
    pinned = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
    ld.stage_d2h(rec, nb, pinned)
    torch.cuda.synchronize()
    recs.append((rec, pinned))
x0 = torch.randn(n, device=dev) * 0.05
for kind, opt, rr in (("sgd", {"kind": "sgd"}, recs[0]), ("sgd", {"kind": "sgd", "weight_decay": 1e-4}, recs[1]),
                      ("momentum", {"kind": "momentum", "momentum": 0.9, "dampening": 0.1}, recs[1]),
                      ("adam", {"kind": "adam", "beta1": 0.9, "beta2": 0.999, "eps": 1e-8}, recs[1]),
                      ("adam", {"kind": "adam", "beta1": 0.9, "beta2": 0.999, "eps": 1e-8, "approx_math": 1}, recs[1])):
    st = {"x": x0.clone(), "m": None if kind == "sgd" else torch.zeros(n, device=dev),
          "v": torch.full((n,), 1e-8, device=dev) if kind == "adam" else None,
          "x_bf16": torch.empty(n, dtype=torch.bfloat16, device=dev) if kind == "adam" else None,
          "n": n, "lo": 0, "hi": n, "t": 0, "adam_step": 10, "momentum_initialized": 1}
    ld.replay(st, opt, [rr])
    st["t"] = 0
    ld.update(st, opt, ring[0])
st = {"x": x0.clone(), "m": None, "v": None, "x_bf16": None, "n": n, "lo": 0, "hi": n, "t": 0, "adam_step": 0,
      "momentum_initialized": 0}
ld.replay_parallel(st, {"kind": "sgd"}, [recs[0]])
st = {"x": x0.clone(), "m": torch.zeros(n, device=dev), "v": torch.zeros(n, device=dev), "x_bf16": None,
      "n": n, "lo": 0, "hi": n, "t": 0, "adam_step": 0, "momentum_initialized": 0}
ld.dense_update(st, {"kind": "adam", "beta1": 0.9, "beta2": 0.999, "eps": 1e-8}, torch.randn(n, device=dev), 1e-3)
torch.cuda.synchronize()
print("sanitize_path: done, launches", ld.launch_count())
