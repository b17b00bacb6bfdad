#!/usr/bin/env python
"""Summarise a gpurun ncu capture into profiles/ markdown + traffic.json.

    python tools/ncu_summary.py gpurun_out/TAG ROUNDNAME

Reads TAG/launches.csv (the `--metrics gpu__time_duration.sum` launch list of one
bench step) and TAG/full.ncu-rep (`--set full` of k_partition / k_replay), writes
profiles/ROUNDNAME_launches.md, profiles/ROUNDNAME_ncu_full.md and refreshes
profiles/traffic.json (DRAM bytes per launch, used by bench.py's roofline)."""
from __future__ import annotations

import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "smsp__inst_executed.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__shared_mem_per_block_dynamic",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
]


def short(name, keep_template=False):
    n = name.split("(")[0].strip().replace("void ", "")
    if not keep_template and ("k_replay" in n or "k_partition" in n):
        n = n.split("<")[0]             # k_replay<BO>: one row per kernel
    return n


def launches(path):
    rows = []
    with open(path) as fh:
        text = fh.read()
    start = text.find('"ID"')
    for r in csv.DictReader(io.StringIO(text[start:])):
        if r.get("Metric Name") == "gpu__time_duration.sum":
            v = float(r["Metric Value"].replace(",", ""))
            unit = r["Metric Unit"]
            ms = v / 1e6 if unit == "ns" else v / 1e3 if unit == "us" else v if unit == "ms" else v / 1e6
            rows.append((short(r["Kernel Name"]), ms))
    return rows


def full(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    start = out.find('"ID"')
    rdr = list(csv.reader(io.StringIO(out[start:])))
    head, units, data = rdr[0], rdr[1], rdr[2:]
    res = []
    for row in data:
        d = dict(zip(head, row))
        u = dict(zip(head, units))
        res.append((short(d["Kernel Name"]), d, u))
    return res


def to_num(s):
    try:
        return float(s.replace(",", ""))
    except Exception:
        return None


def main():
    tag, name = sys.argv[1], sys.argv[2]
    prof = os.environ.get("OUTDIR", os.path.join(ROOT, "profiles"))
    lpath = os.path.join(tag, "launches.csv")
    lib = [(k, ms) for k, ms in launches(lpath) if k.startswith("arb::")] if os.path.exists(lpath) else []
    agg = defaultdict(lambda: [0, 0.0])
    for k, ms in lib:
        agg[k][0] += 1
        agg[k][1] += ms
    tot = sum(v[1] for v in agg.values()) or 1.0
    what = os.environ.get("WHAT", "the first batch (one flush, ~1.0e9 records) of the whole config-5 trace, N = 1")
    cmd = os.environ.get("CMD", "python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --no-side --max-batches 1")
    lines = [f"# {name} — launch list: {what}", "",
             f"`ncu --metrics gpu__time_duration.sum --clock-control none` over `{cmd}` (cold-cache, serialised; "
             "compare shares, not absolutes).  Generator kernels run before the timed region "
             "and are excluded.", "",
             "| kernel | launches | total ms | share of library time |", "|---|---|---|---|"]
    for k, (c, ms) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        lines.append(f"| {k} | {c} | {ms:.3f} | {100 * ms / tot:.1f}% |")
    lines.append(f"| **total** | {sum(v[0] for v in agg.values())} | {tot:.3f} | 100% |")
    with open(os.path.join(prof, f"{name}_launches.md"), "w") as fh:
        fh.write("\n".join(lines) + "\n")
    rep = os.path.join(tag, "full.ncu-rep")
    if os.path.exists(rep):
        ks = full(rep)
        cols = [k for k, _, _ in ks]
        lines = [f"# {name} — ncu --set full of the hot kernels: {what}", "",
                 f"`ncu --set full --clock-control none --import-source on -k regex:\"k_partition|k_replay\" -c 2 {cmd}`",
                 "",
                 "| metric | " + " | ".join(cols) + " |", "|---|" + "---|" * len(cols)]
        for m in METRICS:
            vals = [d.get(m, "") for _, d, _ in ks]
            unit = ks[0][2].get(m, "")
            lines.append(f"| {m} ({unit}) | " + " | ".join(vals) + " |")
        with open(os.path.join(prof, f"{name}_ncu_full.md"), "w") as fh:
            fh.write("\n".join(lines) + "\n")
        tj_path = os.path.join(prof, "traffic.json")
        try:
            tj = json.load(open(tj_path))
        except Exception:
            tj = {}
        recs = None
        for k, d, u in ks:
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
            rd = to_num(d["dram__bytes_read.sum"]) * scale[u["dram__bytes_read.sum"]]
            wr = to_num(d["dram__bytes_write.sum"]) * scale[u["dram__bytes_write.sum"]]
            kk = k.replace("arb::", "")
            old = tj.get(kk, {})
            recs = old.get("records_in_launch")
            tj[kk] = {"dram_bytes_per_launch": rd + wr, "read": rd, "write": wr,
                      "records_in_launch": int(sys.argv[3]) if len(sys.argv) > 3 else recs,
                      "source": f"profiles/{name}_ncu_full.md ({what})"}
        with open(tj_path, "w") as fh:
            json.dump(tj, fh, indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
