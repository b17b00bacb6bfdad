"""Debug: run_program parity per bucket size / flush cuts (with and without the run form)."""
import os, sys
import numpy as np
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R); sys.path.insert(0, os.path.join(R, "tests"))
import oracle
from gen.fuzz import run_program
from gpu_util import run_gpu
seed = int(sys.argv[1]) if len(sys.argv) > 1 else 0
rec, base, span = run_program(2000 + seed)
exp = oracle.replay(rec, base, span)
et = exp.triples()
for bb in (0, 9, 12):
    rc, got, sh, st = run_gpu(rec, base, span, bucket_bits=bb)
    print("bb", bb, "rc", rc, "reports", len(got), len(et), got == et, "shadow", np.array_equal(sh, exp.shadow),
          "run steps", st["steps_run"], "fast", st["steps_fast"], "sort", st["steps_sort"], "items", st["work_items"], "hot", st["hot_buckets"])
    if got != et:
        g, e = set(got), set(et)
        print("  missing", sorted(e - g)[:8], "extra", sorted(g - e)[:8])
cuts = sorted(int(x) for x in np.random.default_rng(seed).choice(rec.shape[0], 3, replace=False))
rc, got, sh, st = run_gpu(rec, base, span, flush_points=cuts)
print("cuts", cuts, rc, got == et, np.array_equal(sh, exp.shadow))
if got != et:
    g, e = set(got), set(et)
    print("  missing", sorted(e - g)[:8], "extra", sorted(g - e)[:8])
