"""Debug: config-5 shard-0 batches of various sizes through one flush (no oracle)."""
import os, sys
import numpy as np
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R); sys.path.insert(0, os.path.join(R, "tests"))
import torch
import bench
from gen import native
from paper_conf_ipps_yuphs21_b200 import Context, ARB_F_TIMING
from paper_conf_ipps_yuphs21_b200.shard import shard_range
tot = int(float(sys.argv[1])); groups = int(sys.argv[2])
prog = native.config5(total_records=tot, groups=groups)
lo, hi = shard_range(native.C5_BASE_WORD, native.C5_WORDS, 0, 8)
src = bench.BatchSource(prog, lo, hi, torch.device("cuda", 0))
recs, gidx, _ = src.make(0, prog.n)
ctx = Context(lo * 8, (hi - lo) * 8, flags=ARB_F_TIMING, report_capacity=1 << 25)
ctx.submit_events(recs, global_index=gidx)
rc, n, _ = ctx.flush(check=False)
st = ctx.stats()
print("records", recs.shape[0], "rc", rc, n, "run steps", st["steps_run"], "fast", st["steps_fast"], "sort", st["steps_sort"],
      "hot", st["hot_buckets"], "items", st["work_items"], ctx.last_error() if rc else "")
