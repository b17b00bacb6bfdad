"""Debug: run form / run steps on the large run program per bucket size."""
import os, sys
import numpy as np
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R); sys.path.insert(0, os.path.join(R, "tests"))
from gen.fuzz import run_program
from gpu_util import run_gpu
rec, base, span = run_program(3000, n_arrays=8, array_words=1 << 16, steps=4000, loop_max=6000)
op = (rec[:, 0] >> np.uint64(48)) & np.uint64(0xFF)
print("records", rec.shape[0], "control", int((op >= 4).sum()))
for bb in (0, 9, 12, 15):
    rc, got, sh, st = run_gpu(rec, base, span, bucket_bits=bb)
    print("bb", bb, "rc", rc, {k: st[k] for k in ("steps_run", "steps_fast", "steps_sort", "segments", "work_items", "hot_buckets", "buckets")})
