"""GPU parity on the large configs (3, 4, 5).

* scaled: the same generator programs at sizes the oracle replays in seconds,
  compared element by element (every report, every shadow byte);
* full size: the whole traces of configs 3-5 exactly in test_parity_full_gpu.py;
  here rank 0's config-5 batch (1.0e9 records) in a single flush, exactly.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _gpu_run(prog, lo, hi, flushes=None, recs=None, gidx=None, flags=0):
    import torch
    from paper_conf_ipps_yuphs21_b200 import Context, reports_to_triples
    from gpu_util import to_device
    ctx = Context(lo * 8, (hi - lo) * 8, report_capacity=1 << 25, flags=flags)
    if recs is None:
        rec = prog.fill_host()
        recs = to_device(rec)
        gidx = to_device(np.arange(rec.shape[0], dtype=np.uint64))
        flushes = [(0, rec.shape[0])]
    triples = []
    for a, b in flushes:
        ctx.submit_events(recs[a:b], global_index=gidx[a:b])
        rc, n, _ = ctx.flush()
        triples += reports_to_triples(ctx.get_reports(n))
    torch.cuda.synchronize()
    return ctx, triples


def _check_full(orc, prog, flags=0):
    rec = prog.fill_host()
    lo, hi = prog.addr_base // 8, (prog.addr_base + prog.addr_bytes) // 8
    exp = orc.replay(rec, prog.addr_base, prog.addr_bytes, detect_bo=bool(flags & 8))
    assert exp.rc == 0
    ctx, got = _gpu_run(prog, lo, hi, flags=flags)
    assert sorted(got) == exp.triples()
    assert np.array_equal(ctx.get_shadow(lo, hi - lo), exp.shadow)
    ctx.close()
    return exp


@pytest.mark.parametrize("flags", [0, 4, 8])
def test_config3_scaled(orc, flags):
    """flags=4 (ARB_F_SMALL_PARTS): busy small buckets replayed as time slices (K5);
    flags=8 (ARB_F_BO): the buffer-overflow extension (every kernel access is inside a
    mapped section here, so the report set is the same)."""
    from gen import native
    exp = _check_full(orc, native.config3(scale=0.01), flags=flags)
    kinds = {k for _, _, k in exp.triples()}
    assert kinds == {1, 2, 3}          # alloc-mapped row read, stale `stop`, the missing taskwait


@pytest.mark.parametrize("flags", [0, 4])
def test_config4_scaled(orc, flags):
    """flags=4 (ARB_F_SMALL_PARTS): the range-heavy buckets run as word-range parts."""
    from gen import native
    exp = _check_full(orc, native.config4(scale=1 / 512), flags=flags)
    assert {k for _, _, k in exp.triples()} == {2}   # 503.postencil: stale output reads


def test_config5_scaled_shard(orc):
    """Rank 1 of 8 of a small config-5 trace: a shard with boundary-spanning maps."""
    from gen import native
    from paper_conf_ipps_yuphs21_b200.shard import shard_range
    prog = native.config5(total_records=16_000_000, groups=64, stale_rate=200)
    lo, hi = shard_range(native.C5_BASE_WORD, native.C5_WORDS, 1, 8)
    rec, gi = prog.filter_host(word_lo=lo, word_hi=hi)
    exp = orc.replay(rec, lo * 8, (hi - lo) * 8, global_index=gi)
    assert exp.rc == 0 and len(exp.triples()) > 0
    from gpu_util import to_device
    ctx, got = _gpu_run(prog, lo, hi, flushes=[(0, rec.shape[0])], recs=to_device(rec), gidx=to_device(gi))
    assert sorted(got) == exp.triples()
    assert np.array_equal(ctx.get_shadow(lo, hi - lo), exp.shadow)
    ctx.close()


@pytest.mark.slow
def test_config5_one_flush_near_max_batch(orc):
    """Rank 0 of 8 of the full config-5 trace (1.0e9 records, record positions up to
    2^30) in ONE flush -- the largest batch the ABI accepts -- every report and every
    shadow byte against the address-sharded oracle."""
    import os
    import torch
    import bench
    from gen import native
    from paper_conf_ipps_yuphs21_b200 import Context, ARB_F_TIMING
    from paper_conf_ipps_yuphs21_b200.shard import shard_range
    from test_parity_full_gpu import _gpu_batch, _compare_shadow
    prog = native.config5()
    lo, hi = shard_range(native.C5_BASE_WORD, native.C5_WORDS, 0, 8)
    src = bench.BatchSource(prog, lo, hi, torch.device("cuda", 0))
    recs, gidx, _ = src.make(0, prog.n)
    assert 2 ** 29 < recs.shape[0] <= 2 ** 30
    ctx = Context(lo * 8, (hi - lo) * 8, flags=ARB_F_TIMING, report_capacity=1 << 25)
    got = _gpu_batch(ctx, recs, gidx, [(0, recs.shape[0])])
    host, gi = recs.cpu().numpy().view(np.uint64), gidx.cpu().numpy().view(np.uint64)
    del recs, gidx, src
    torch.cuda.empty_cache()
    exp = orc.replay(host, lo * 8, (hi - lo) * 8, global_index=gi, threads=os.cpu_count() or 8)
    assert exp.rc == 0 and exp.reports.size > 0
    assert np.array_equal(got, exp.reports)
    _compare_shadow(ctx, lo, hi - lo, exp.shadow)
    ctx.close()


def test_batch_limit():
    """More than 2^30 records in one batch is ARB_EINVAL; the context stays usable."""
    import torch
    from paper_conf_ipps_yuphs21_b200 import Context, ArbError, reports_to_triples
    from gen.configs import config1
    ctx = Context(0x1000_0000, 1 << 16)
    big = torch.empty(((1 << 30) + 1, 2), dtype=torch.int64, device="cuda")
    with pytest.raises(ArbError):
        ctx.submit_events(big)
    del big
    torch.cuda.empty_cache()
    rec, base, size = config1()
    ctx.close()
    ctx = Context(base, size)
    from gpu_util import to_device
    d = to_device(rec)
    ctx.submit_events(d)
    rc, n, _ = ctx.flush()
    assert rc == 0 and n == 1024
    ctx.close()
