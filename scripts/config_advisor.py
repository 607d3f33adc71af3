#!/usr/bin/env python
"""Recommend the full-checkpoint frequency and batching size (§3.5, Eq. 5) from a bench
line and the job's own parameters, through the library's lowdiff_optimal_config.

    python scripts/config_advisor.py bench.json --iter-ms 350 --mtbf-h 24 --write-gbs 2 \
        --gpus 8 --hours 72 --load-full-s 60

R_D is the time to merge (replay) ONE batched differential checkpoint onto the full one: Eq. 3 counts
1/(f b) batched records per chain, so R_D is the bench line's replay time per step
divided by the records per step (a STACK record of B iterations replays B optimizer steps); S is
the full checkpoint the bench replays onto (x, m, v fp32 of the shard, times P ranks). Every time is
converted to training iterations (reading #29).
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("bench_json")
    ap.add_argument("--iter-ms", type=float, required=True, help="training iteration time")
    ap.add_argument("--mtbf-h", type=float, required=True, help="mean time between failures, hours")
    ap.add_argument("--write-gbs", type=float, required=True, help="checkpoint write bandwidth, GB/s")
    ap.add_argument("--gpus", type=int, default=8)
    ap.add_argument("--hours", type=float, default=72.0, help="total run time")
    ap.add_argument("--load-full-s", type=float, default=60.0, help="time to load a full checkpoint")
    a = ap.parse_args()
    import paper_conf_sc_yaolhlzz25_b200 as ld
    d = json.loads(open(a.bench_json).read().strip().splitlines()[-1])
    cfg = d["config"]
    records = cfg.get("batches_per_step", 1)
    rd_ms = d["kernels"].get("replay_dense", d["kernels"].get("replay_sparse"))["ms_per_step"] / records
    state_bytes = {"sgd": 4, "momentum": 8, "adam": 12}[cfg["replay"].split(",")[0]] * cfg["n"]
    it_s = a.iter_ms * 1e-3
    model = {"N": a.gpus, "M": a.mtbf_h * 3600 / it_s, "W": a.write_gbs * 1e9 * it_s, "S": state_bytes,
             "T": a.hours * 3600 / it_s, "R_F": a.load_full_s / it_s, "R_D": rd_ms * 1e-3 / it_s}
    r = ld.optimal_config(model)
    print(json.dumps({"model_in_iterations": model, **r,
                      "wasted_at_optimum_iterations": ld.wasted_time(model, 1.0 / r["fcf"], r["B"])}, indent=1))


if __name__ == "__main__":
    main()
