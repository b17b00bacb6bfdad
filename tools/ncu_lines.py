#!/usr/bin/env python
"""Per-source-line instruction counts and stall samples of one kernel in an ncu report:
    python tools/ncu_lines.py REPORT KERNEL_REGEX [UNITS] [MIN_PCT]
UNITS divides the instruction counts (e.g. events per launch)."""
import csv, subprocess, sys
rep, kern = sys.argv[1], sys.argv[2]
units = float(sys.argv[3]) if len(sys.argv) > 3 else 1.0
minp = float(sys.argv[4]) if len(sys.argv) > 4 else 0.5
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", f"regex:{kern}",
                      "--print-source", "cuda,sass"], capture_output=True, text=True).stdout
hdr = fname = None
res = []
for l in out.splitlines():
    if l.startswith('"File Path"'):
        fname = l.split(",", 1)[1].strip('"').split("/")[-1]; continue
    if l.startswith('"Function Name"'):
        continue
    if l.startswith('"Line No"'):
        hdr = next(csv.reader([l])); continue
    d = dict(zip(hdr, next(csv.reader([l]))))
    if d.get("Line No"):
        try:
            res.append((fname, int(d["Line No"]), int(d["Instructions Executed"] or 0),
                        int(d["Warp Stall Sampling (All Samples)"] or 0)))
        except (ValueError, KeyError):
            pass
ti = sum(r[2] for r in res); ts = sum(r[3] for r in res) or 1
print(f"warp-instructions {ti} ({ti/units:.2f} per unit), samples {ts}")
for f, ln, i, s in sorted(res, key=lambda r: (r[0], r[1])):
    if 100 * s / ts >= minp or 100 * i / max(ti, 1) >= minp:
        print(f"{f}:{ln:4d} {i/units:8.3f} ins/unit {100*i/max(ti,1):5.1f}% ins {100*s/ts:5.1f}% smp")
