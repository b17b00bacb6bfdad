"""Kernel timeline of a few flushes (CUPTI through torch.profiler; real
concurrency, not ncu's serialised replay): per kernel name the count and total
device time, and the idle gaps of the device between kernels, per flush.

    python tools/timeline.py [--workload config5] [--batches 2] [--out gpurun_out/timeline.json]
"""
import argparse
import collections
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="config5")
    ap.add_argument("--batches", type=int, default=2)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    import torch
    import bench
    from paper_conf_ipps_yuphs21_b200 import Context, ARB_F_TIMING
    prog = bench.make_program(a.workload)
    lo, hi = bench.rank_range(prog, 0, 1)
    batches = bench.time_batches(prog, bench.DEFAULT_BATCHES if a.workload == "config5" else 1)[:a.batches]
    dev = torch.device("cuda", 0)
    src = bench.BatchSource(prog, lo, hi, dev)
    ctx = Context(lo * 8, (hi - lo) * 8, flags=ARB_F_TIMING, report_capacity=1 << 25)
    made = [src.make(g0, g1) for g0, g1 in batches[:1]]
    recs, gidx, flushes = made[0]

    def one():
        for f0, f1 in flushes:
            ctx.submit_events(recs[f0:f1], global_index=None)
            rc, n, _ = ctx.flush()
            assert rc == 0, ctx.last_error()
    one(); one()                       # warm-up (allocations)
    torch.cuda.synchronize()
    from torch.profiler import profile, ProfilerActivity
    with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
        for _ in range(3):
            one()
        torch.cuda.synchronize()
    evs = [e for e in prof.events() if e.device_type.name == "CUDA"]
    ks = sorted(((e.time_range.start, e.time_range.end, e.name) for e in evs), key=lambda t: t[0])
    tot = collections.defaultdict(lambda: [0, 0.0])
    for s, e, n in ks:
        tot[n][0] += 1
        tot[n][1] += (e - s) / 1000.0
    span = (ks[-1][1] - ks[0][0]) / 1000.0
    busy = 0.0
    gaps = []
    cur_end = ks[0][0]
    for s, e, n in ks:
        if s > cur_end:
            gaps.append(((s - cur_end) / 1000.0, n))
        cur_end = max(cur_end, e)
    busy = span - sum(g for g, _ in gaps)
    print(f"3 flushes: span {span:.3f} ms, device busy {busy:.3f} ms, idle {span - busy:.3f} ms")
    for n, (c, t) in sorted(tot.items(), key=lambda kv: -kv[1][1])[:30]:
        print(f"  {t / 3:9.3f} ms/flush {c // 3:5d} launches/flush  {n[:90]}")
    big = sorted(gaps, reverse=True)[:25]
    print("largest idle gaps (ms, next kernel):")
    for g, n in big:
        print(f"  {g:.3f}  {n[:80]}")
    if a.out:
        with open(a.out, "w") as fh:
            json.dump({"kernels": [(s, e, n) for s, e, n in ks]}, fh)


if __name__ == "__main__":
    main()
