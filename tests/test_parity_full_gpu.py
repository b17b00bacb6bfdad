"""Exact GPU-vs-oracle parity at BASELINE.json's full sizes, in the launch
configuration bench.py times (north_star: "GPU reports must match the oracle
bit-exactly, as the same report set ... on all configs").

* config 5: the whole 9.0e9-record trace over 2^33 words (64 GiB of locations),
  replayed exactly as the N = 1 bench line replays it -- 9 time batches cut at
  quiescent points, each generated on the device and replayed as one flush of at
  most 2^30 records -- compared batch by batch with the oracle (address-sharded over
  the host cores, continuing from the previous batch's final shadow), then the
  whole 8 GiB final shadow byte for byte;
* configs 3 and 4: the whole trace of each (1.0e9 / 0.89e9 records; config 4 with
  2^34 words = 16 GiB of shadow), every report and every shadow byte.

The oracle's inputs are the generator's records (gen/, the seeded input module
both sides share); nothing it reads comes from the CUDA path.
"""
import os

import numpy as np
import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

THREADS = os.cpu_count() or 8


def _reports_np(rep):
    """(n, 2) arb_report array -> oracle REPORT_DTYPE array (word, record, kind)."""
    from oracle.oracle import REPORT_DTYPE
    rep = np.asarray(rep, dtype=np.uint64).reshape(-1, 2)
    out = np.zeros(rep.shape[0], dtype=REPORT_DTYPE)
    out["word"] = rep[:, 0] & np.uint64((1 << 48) - 1)
    out["kind"] = (rep[:, 0] >> np.uint64(48)) & np.uint64(0xFF)
    out["record"] = rep[:, 1]
    return out


def _dedup_first(rep):
    """Z3 applied to a canonical raw report list: the first report per (word, kind)."""
    if rep.size == 0:
        return rep
    key = rep["word"].astype(np.uint64) * np.uint64(8) + rep["kind"].astype(np.uint64)
    order = np.lexsort((rep["record"], key))
    k = key[order]
    first = np.ones(k.size, dtype=bool)
    first[1:] = k[1:] != k[:-1]
    keep = np.sort(order[first])
    return rep[keep]


def _gpu_batch(ctx, recs, gidx, flushes):
    out = []
    for a, b in flushes:
        if b > a:
            ctx.submit_events(recs[a:b], global_index=None if gidx is None else gidx[a:b])
        rc, n, _ = ctx.flush()
        assert rc == 0, ctx.last_error()
        out.append(_reports_np(ctx.get_reports(n)))
    got = np.concatenate(out) if out else _reports_np(np.zeros((0, 2), np.uint64))
    # each flush's list is canonical; the batch's is the canonical order of their union
    return got[np.lexsort((got["kind"], got["record"], got["word"]))]


def _compare_shadow(ctx, lo, n, expected, chunk=1 << 30):
    for a in range(0, n, chunk):
        m = min(chunk, n - a)
        got = ctx.get_shadow(lo + a, m)
        assert np.array_equal(got, expected[a:a + m]), f"shadow differs in words [{lo + a}, {lo + a + m})"


def test_config5_whole_trace_exact(orc):
    """The benchmarked workload, all 9.0e9 records: raw reports per batch and the final shadow."""
    import torch
    import bench
    from paper_conf_ipps_yuphs21_b200 import Context, ARB_F_TIMING
    prog = bench.make_program("config5")
    lo, hi = bench.rank_range(prog, 0, 1)
    batches = bench.time_batches(prog, bench.DEFAULT_BATCHES)
    src = bench.BatchSource(prog, lo, hi, torch.device("cuda", 0))
    ctx = Context(lo * 8, (hi - lo) * 8, flags=ARB_F_TIMING, report_capacity=1 << 25)
    shadow = None
    n_rep = 0
    for g0, g1 in batches:
        recs, gidx, flushes = src.make(g0, g1)
        assert gidx is None and recs.shape[0] == g1 - g0
        got = _gpu_batch(ctx, recs, gidx, flushes)
        host = recs.cpu().numpy().view(np.uint64)
        exp = orc.replay(host, lo * 8, (hi - lo) * 8, global_index=np.arange(g0, g1, dtype=np.uint64),
                         threads=THREADS, shadow_in=shadow)
        del host
        assert exp.rc == 0
        assert np.array_equal(got, exp.reports), f"batch [{g0}, {g1}): reports differ"
        n_rep += got.size
        shadow = exp.shadow
    assert n_rep > 10_000
    _compare_shadow(ctx, lo, hi - lo, shadow)
    ctx.close()


def test_config5_whole_trace_dedup_first(orc):
    """ARB_F_DEDUP_FIRST (the bench's production default) across all batches and flushes
    equals Z3 applied to the whole trace's oracle reports."""
    import torch
    import bench
    from paper_conf_ipps_yuphs21_b200 import Context, ARB_F_TIMING, ARB_F_DEDUP_FIRST
    prog = bench.make_program("config5")
    lo, hi = bench.rank_range(prog, 0, 1)
    batches = bench.time_batches(prog, bench.DEFAULT_BATCHES)[:3]   # the first three batches (the state carries)
    src = bench.BatchSource(prog, lo, hi, torch.device("cuda", 0))
    ctx = Context(lo * 8, (hi - lo) * 8, flags=ARB_F_TIMING | ARB_F_DEDUP_FIRST, report_capacity=1 << 25)
    shadow = None
    got, raw = [], []
    for g0, g1 in batches:
        recs, gidx, flushes = src.make(g0, g1)
        got.append(_gpu_batch(ctx, recs, gidx, flushes))
        host = recs.cpu().numpy().view(np.uint64)
        exp = orc.replay(host, lo * 8, (hi - lo) * 8, global_index=np.arange(g0, g1, dtype=np.uint64),
                         threads=THREADS, shadow_in=shadow)
        del host
        assert exp.rc == 0
        raw.append(exp.reports)
        shadow = exp.shadow
    got = np.concatenate(got)
    got = got[np.lexsort((got["kind"], got["record"], got["word"]))]
    raw = np.concatenate(raw)
    raw = raw[np.lexsort((raw["kind"], raw["record"], raw["word"]))]
    assert np.array_equal(got, _dedup_first(raw))
    ctx.close()


@pytest.mark.parametrize("name", ["config3", "config4"])
def test_whole_trace_exact(orc, name):
    import torch
    import bench
    from paper_conf_ipps_yuphs21_b200 import Context, ARB_F_TIMING
    prog = bench.make_program(name)
    lo, hi = bench.rank_range(prog, 0, 1)
    (g0, g1), = bench.time_batches(prog, 1)
    src = bench.BatchSource(prog, lo, hi, torch.device("cuda", 0))
    ctx = Context(lo * 8, (hi - lo) * 8, flags=ARB_F_TIMING, report_capacity=1 << 25)
    recs, gidx, flushes = src.make(g0, g1)
    got = _gpu_batch(ctx, recs, gidx, flushes)
    host = recs.cpu().numpy().view(np.uint64)
    del recs, src
    torch.cuda.empty_cache()
    exp = orc.replay(host, lo * 8, (hi - lo) * 8, threads=THREADS)
    del host
    assert exp.rc == 0
    assert {int(k) for k in np.unique(exp.reports["kind"])} == ({1, 2, 3} if name == "config3" else {2})
    assert np.array_equal(got, exp.reports)
    _compare_shadow(ctx, lo, hi - lo, exp.shadow)
    ctx.close()
