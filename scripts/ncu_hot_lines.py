#!/usr/bin/env python
"""Top source lines of an ncu report by warp-stall samples (reads `--page source --print-source
cuda,sass` CSV): python scripts/ncu_hot_lines.py REPORT.ncu-rep [N]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
fname, hdr, agg = None, None, []
for r in rows:
    if r and r[0] == "File Path":
        fname = r[1].split("/")[-1]
    elif r and r[0] == "Line No":
        hdr = r
    elif hdr and len(r) == len(hdr) and r[0].isdigit():
        iS = hdr.index("Warp Stall Sampling (All Samples)")
        iE = hdr.index("Instructions Executed")
        stalls = {c: float(r[k] or 0) for k, c in enumerate(hdr) if c.startswith("stall_") and "Not Issued" not in c}
        agg.append((float(r[iS] or 0), float(r[iE] or 0), fname, r[0], r[1].strip(), stalls))
tot_s = sum(a[0] for a in agg) or 1
tot_e = sum(a[1] for a in agg) or 1
print(f"samples {tot_s:.0f}, warp instructions {tot_e:.0f}")
for s, e, f, ln, src, st in sorted(agg, key=lambda a: -a[0])[:N]:
    top = ", ".join(f"{k[6:]} {100 * v / s:.0f}%" for k, v in sorted(st.items(), key=lambda kv: -kv[1])[:2] if s)
    print(f"{100 * s / tot_s:5.1f}% {100 * e / tot_e:5.1f}%i {f}:{ln:<5} {src[:80]:<80} [{top}]")
