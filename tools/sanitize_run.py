"""Small replays for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
config 1, a prefix of config 2, random programs with tasks / depend / flush cuts, and
the forced-parts / time-slice (K5), buffer-overflow, unified-memory and
several-accelerator kernel instances.  Each result is checked against the oracle.

    compute-sanitizer --tool racecheck python tools/sanitize_run.py [quick]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402


def main():
    quick = "quick" in sys.argv
    import oracle
    from gen.configs import config1, config2
    from gen.fuzz import random_program
    from gpu_util import run_gpu
    cases = []
    rec, base, size = config1()
    cases.append(("config1", rec, base, size, 0, {}))
    rec2, base2, size2 = config2()
    op = (rec2[:, 0] >> np.uint64(48)) & np.uint64(0xFF)
    depth = np.cumsum((op == 12).astype(np.int64) - (op == 13).astype(np.int64))
    ok = np.nonzero(depth == 0)[0] + 1
    cut = int(ok[np.searchsorted(ok, 20_000 if quick else 120_000)])
    cases.append(("config2_prefix", rec2[:cut], base2, size2, 0, {}))
    for seed in range(2 if quick else 4):
        r, b, s = random_program(4242 + seed, p_task=0.4, p_depend=0.3, p_always=0.2, steps=60)
        cases.append((f"fuzz{seed}", r, b, s, 0, {}))
        cases.append((f"fuzz{seed}_parts_slices", r, b, s, 4, {}))
        cases.append((f"fuzz{seed}_bo", r, b, s, 8, {"detect_bo": True}))
        cases.append((f"fuzz{seed}_um", r, b, s, 16, {"unified": True}))
        cases.append((f"fuzz{seed}_dedup", r, b, s, 1, {"dedup_first": True}))
        r3, b3, s3 = random_program(4300 + seed, n_devices=3, p_task=0.3, steps=60)
        cases.append((f"fuzz{seed}_3dev", r3, b3, s3, 2 << 8, {"n_devices": 3}))
    bad = 0
    for name, r, b, s, flags, okw in cases:
        exp = oracle.replay(r, b, s, **okw)
        if exp.rc != 0:
            print(f"{name}: oracle rc {exp.rc}, skipped")
            continue
        cuts = [r.shape[0] // 3, 2 * r.shape[0] // 3] if name.startswith("fuzz") else []
        rc, got, shadow, st = run_gpu(r, b, s, flags=flags, flush_points=cuts)
        same = rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)
        bad += not same
        print(f"{name}: {r.shape[0]} records, {len(got)} reports, {st['kernel_launches']} launches, "
              f"{'ok' if same else 'MISMATCH'}", flush=True)
    print("SANITIZE_RUN", "FAILED" if bad else "OK", flush=True)


if __name__ == "__main__":
    main()
