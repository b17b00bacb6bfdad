"""Debug: config 2 shadow mismatches between run steps and the oracle."""
import os, sys
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import oracle
from gen.configs import config2
from gpu_util import run_gpu
rec, base, size = config2()
exp = oracle.replay(rec, base, size)
rc, got, sh, st = run_gpu(rec, base, size)
print("rc", rc, "reports equal", got == exp.triples(), st["steps_run"], st["segments"], st["buckets"])
bad = np.nonzero(sh != exp.shadow)[0]
print("mismatched words", bad.size, bad[:20])
w0 = base // 8
op = (rec[:, 0] >> np.uint64(48)) & np.uint64(0xFF)
addr = rec[:, 0] & np.uint64((1 << 48) - 1)
ln = rec[:, 1] & np.uint64((1 << 48) - 1)
for w in bad[:4]:
    print("word", w, "got", sh[w], "exp", exp.shadow[w])
    wa = (w0 + w) * 8
    acc = np.nonzero((op < 4) & (addr < wa + 8) & (addr + ln > wa))[0]
    ctl = np.nonzero((op >= 8) & (addr < wa + 8) & (addr + ln > wa))[0]
    print("  accesses", [(int(i), int(op[i])) for i in acc[-12:]])
    print("  control", [(int(i), int(op[i]), int(rec[i, 0] >> np.uint64(56))) for i in ctl[-8:]])
