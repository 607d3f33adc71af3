#!/usr/bin/env python
"""Summarise ncu --set full captures (.ncu-rep) into a small JSON for profiles/.

    python scripts/ncu_summarize.py OUT.json gpurun_out/prof_*_TAG.ncu-rep

Per captured kernel: duration, DRAM bytes read/written (the `traffic` the bench line quotes),
DRAM throughput, achieved occupancy, IPC, registers, the top warp-stall reasons and pipe
utilisations.
"""
import csv
import io
import json
import subprocess
import sys

METRICS = {
    "duration_us": ("gpu__time_duration.sum", 1e-3),          # ncu reports ms for this metric in raw
    "dram_read_bytes": ("dram__bytes_read.sum", 1),
    "dram_write_bytes": ("dram__bytes_write.sum", 1),
    "dram_throughput_pct": ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", 1),
    "achieved_occupancy_pct": ("sm__warps_active.avg.pct_of_peak_sustained_active", 1),
    "ipc_active": ("sm__inst_executed.avg.per_cycle_active", 1),
    "registers_per_thread": ("launch__registers_per_thread", 1),
    "grid_size": ("launch__grid_size", 1),
    "block_size": ("launch__block_size", 1),
    "warp_instructions": ("smsp__inst_executed.sum", 1),
}
UNITS = {"msecond": 1e3, "usecond": 1.0, "nsecond": 1e-3, "second": 1e6, "ms": 1e3, "us": 1.0, "ns": 1e-3, "s": 1e6}
BYTES = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def num(s):
    try:
        return float(str(s).replace(",", ""))
    except ValueError:
        return None


def summarize(rep):
    hdr, units, rows = raw(rep)
    res = []
    for r in rows:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        k = {"kernel": d.get("Kernel Name", "")[:120]}
        for name, (metric, _) in METRICS.items():
            v = num(d.get(metric))
            if v is None:
                continue
            unit = u.get(metric, "")
            if name == "duration_us":
                v *= UNITS.get(unit, 1.0)
            elif name.endswith("_bytes"):
                v *= BYTES.get(unit, 1.0)
            k[name] = v
        stalls = {m.split("stalled_")[1]: num(d[m]) for m in d
                  if m.startswith("smsp__pcsamp_warps_issue_stalled_") and not m.endswith("not_issued")
                  and num(d[m])}
        tot = sum(stalls.values()) or 1.0
        k["top_stalls_pct"] = {s: round(100 * v / tot, 1) for s, v in
                               sorted(stalls.items(), key=lambda kv: -kv[1])[:5]}
        pipes = {m.split("sm__pipe_")[1].split("_cycles")[0]: num(d[m]) for m in d
                 if m.startswith("sm__pipe_") and m.endswith("_cycles_active.avg.pct_of_peak_sustained_active")
                 and num(d[m])}
        k["pipe_util_pct"] = {p: round(v, 1) for p, v in sorted(pipes.items(), key=lambda kv: -kv[1])[:5]}
        if "dram_read_bytes" in k and "dram_write_bytes" in k:
            k["dram_bytes"] = k["dram_read_bytes"] + k["dram_write_bytes"]
        res.append(k)
    return res


def main():
    out, reps = sys.argv[1], sys.argv[2:]
    summary = {}
    for rep in reps:
        summary[rep.split("/")[-1]] = summarize(rep)
    json.dump(summary, open(out, "w"), indent=1)
    for rep, ks in summary.items():
        for k in ks:
            print(rep, k["kernel"][:60], {x: k.get(x) for x in ("duration_us", "dram_bytes", "dram_throughput_pct",
                                                                  "achieved_occupancy_pct", "ipc_active")})


if __name__ == "__main__":
    main()
