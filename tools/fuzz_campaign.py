#!/usr/bin/env python
"""Randomised parity campaign (GPU vs the oracle) over all modes — not part of the
test suite.  usage: python tools/fuzz_campaign.py N_PROGRAMS [SEED0]"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import oracle                                   # noqa: E402
from gen.fuzz import random_program             # noqa: E402
from gpu_util import run_gpu                    # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 200
seed0 = int(sys.argv[2]) if len(sys.argv) > 2 else 90000
bad = 0
modes = 0
for k in range(n):
    seed = seed0 + k
    rs = np.random.default_rng(seed)
    mode = ["plain", "bo", "um", "md2", "md3"][k % 5]
    nd = {"md2": 2, "md3": 3}.get(mode, 1)
    flags = {"bo": 8, "um": 16, "md2": 1 << 8, "md3": 2 << 8}.get(mode, 0)
    if rs.random() < 0.3:
        flags |= 4                               # word-range parts / time slices
    if rs.random() < 0.2:
        flags |= 1                               # dedup-first
    big = rs.random() < float(os.environ.get("BIG_FRACTION", "0.2"))
    rec, base, span = random_program(seed, n_arrays=int(rs.integers(1, 6)),
                                     array_words=int(rs.choice([16, 64, 512, 4096])) if not big else 8192,
                                     steps=int(rs.integers(20, 200)) if not big else 400,
                                     loop_max=48 if not big else 5000,
                                     p_task=float(rs.uniform(0, 0.5)), p_always=float(rs.uniform(0, 0.5)),
                                     p_depend=float(rs.uniform(0, 0.7)), n_devices=nd)
    exp = oracle.replay(rec, base, span, dedup_first=bool(flags & 1), detect_bo=bool(flags & 8),
                        unified=bool(flags & 16), n_devices=nd)
    cuts = None
    if rs.random() < 0.5 and rec.shape[0] > 10 and not (flags & 1):
        cuts = sorted(set(int(x) for x in rs.integers(1, rec.shape[0], int(rs.integers(1, 6)))))
    words = span // 8
    bb = int(rs.choice([b for b in (0, 0, 2, 5, 11) if b == 0 or -(-words >> b) <= 2048]))
    rc, got, shadow, _ = run_gpu(rec, base, span, flags=flags, bucket_bits=bb, flush_points=cuts)
    if exp.rc == -7 and cuts is not None:
        ok = rc == 0
    else:
        ok = rc == exp.rc and (rc != 0 or (sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)))
    modes += 1
    if not ok:
        bad += 1
        print(f"MISMATCH seed={seed} mode={mode} flags={flags:#x} bb={bb} cuts={cuts} rc={rc}/{exp.rc} "
              f"got={len(got)} exp={len(exp.triples())}", flush=True)
print(f"campaign: {modes} programs, {bad} mismatches")
