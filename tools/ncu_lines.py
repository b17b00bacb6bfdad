#!/usr/bin/env python
"""Per-source-line hot spots of one kernel in an ncu report:
    python tools/ncu_lines.py REPORT KERNEL_REGEX [N]"""
import csv, io, subprocess, sys
rep, kern = sys.argv[1], sys.argv[2]
N = int(sys.argv[3]) if len(sys.argv) > 3 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", f"regex:{kern}",
                      "--print-source", "cuda,sass"], capture_output=True, text=True).stdout
rows, fname = [], None
lines = out.splitlines()
i = 0
tot_s = tot_i = 0
while i < len(lines):
    l = lines[i]
    if l.startswith('"File Path"') or l.startswith('"File Name"'):
        fname = l.split(",", 1)[1].strip('"').split("/")[-1]
        i += 1
        continue
    if l.startswith('"Line No"'):
        hdr = next(csv.reader([l]))
        j = i + 1
        block = []
        while j < len(lines) and not lines[j].startswith('"File') and not lines[j].startswith('"Function'):
            block.append(lines[j]); j += 1
        for r in csv.reader(io.StringIO("\n".join(block))):
            d = dict(zip(hdr, r))
            try:
                s = int(d.get("Warp Stall Sampling (All Samples)", "0") or 0)
                ins = int(d.get("Instructions Executed", "0") or 0)
            except ValueError:
                continue
            tot_s += s; tot_i += ins
            if (s or ins) and d.get("Line No"):
                rows.append((s, ins, fname, d["Line No"], d["Source"].strip()[:90]))
        i = j
        continue
    i += 1
rows.sort(key=lambda r: -r[0])
print(f"total samples {tot_s}, warp-instructions {tot_i}")
for s, ins, f, ln, src in rows[:N]:
    print(f"{100*s/max(tot_s,1):5.1f}% smp {100*ins/max(tot_i,1):5.1f}% ins  {f}:{ln}  {src}")
