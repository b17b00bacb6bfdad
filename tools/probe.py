import sys, torch, numpy as np
sys.path.insert(0, '.')
from gen import native
from paper_conf_ipps_yuphs21_b200 import Context, ARB_F_TIMING
import bench
prog = native.config5()
recs, gidx, flushes, (lo, hi) = bench.rank_batches(prog, 0, 1, torch.device('cuda', 0))
ctx = Context(lo*8, (hi-lo)*8, flags=ARB_F_TIMING, report_capacity=1<<25)
for it in range(2):
    for a, b in flushes:
        ctx.submit_events(recs[a:b], global_index=gidx[a:b]); ctx.flush()
        st = ctx.stats()
        print({k: (round(st[k],3) if isinstance(st[k], float) else st[k]) for k in ('records','buckets','max_bucket_events','steps_sort','ms_sample','ms_partition','ms_control','ms_replay','ms_mir','ms_reports','ms_total')})
