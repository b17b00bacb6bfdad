"""Per-flush phase timings of one workload through the C-ABI (ARB_F_TIMING).
usage: python tools/probe.py [workload] [scale]"""
import sys, time, torch
sys.path.insert(0, '.')
from paper_conf_ipps_yuphs21_b200 import Context, ARB_F_TIMING
import bench
wl = sys.argv[1] if len(sys.argv) > 1 else "config5"
scale = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
prog = bench.make_program(wl, scale)
t0 = time.time()
recs, gidx, flushes, (lo, hi) = bench.rank_batches(prog, 0, 1, torch.device('cuda', 0))
print(f"{wl}: {recs.shape[0]} records, {len(flushes)} flushes, generated in {time.time() - t0:.1f} s", flush=True)
ctx = Context(lo * 8, (hi - lo) * 8, flags=ARB_F_TIMING, report_capacity=1 << 25)
keys = ('records', 'buckets', 'max_bucket_events', 'steps_fast', 'steps_sort', 'range_words', 'ms_sample',
        'ms_partition', 'ms_control', 'ms_replay', 'ms_mir', 'ms_reports', 'ms_total')
for it in range(2):
    for a, b in flushes:
        ctx.submit_events(recs[a:b], global_index=gidx[a:b]); ctx.flush()
        st = ctx.stats()
        print({k: (round(st[k], 3) if isinstance(st[k], float) else st[k]) for k in keys}, flush=True)
