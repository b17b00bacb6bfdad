"""GPU parity on the large configs (3, 4, 5).

* scaled: the same generator programs at sizes the oracle replays in seconds,
  compared element by element (every report, every shadow byte);
* full size (BASELINE.json sizes, in the launch configuration bench.py times:
  device-generated trace, rank-0 shard, quiescent flushes): compared on a random
  sample of words, for which the oracle replays the filtered trace (control
  records + the accesses touching the sampled words) in sparse mode.  Word
  states are independent, so the sampled comparison is exact for those words.
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


def _sampled_full_size(orc, prog, lo, hi, n_sample=3000, seed=0, one_flush=False, flags=0):
    """Run the bench configuration on the device, then compare sampled words.
    one_flush: the whole batch in a single flush (near the 2^30-record maximum)."""
    import torch
    import bench
    recs, gidx, flushes, (lo2, hi2) = bench.rank_batches(prog, 0, 1, torch.device("cuda", 0))
    assert (lo2, hi2) == (lo, hi)
    if one_flush:
        assert 2 ** 29 < recs.shape[0] <= 2 ** 30
        flushes = [(0, recs.shape[0])]
    ctx, got = _gpu_run(prog, lo, hi, flushes=flushes, recs=recs, gidx=gidx, flags=flags)
    rs = np.random.default_rng(seed)
    # half of the sample from the words the trace touches most densely (mapped sections)
    secs = np.array([(a, b) for a, b, _ in prog.sections if b > lo and a < hi], dtype=np.int64)
    words = set(rs.integers(lo, hi, n_sample // 2).tolist())
    for _ in range(n_sample // 2):
        a, b = secs[rs.integers(len(secs))]
        a, b = max(a, lo), min(b, hi)
        words.add(int(rs.integers(a, b)))
    # plus every word the GPU reported on (sampled to keep the filter small)
    rep_words = sorted({w for w, _, _ in got})
    words.update(rs.choice(rep_words, min(500, len(rep_words)), replace=False).tolist() if rep_words else [])
    words = np.array(sorted(words), dtype=np.uint64)
    del recs, gidx
    torch.cuda.empty_cache()
    frec, fgi = prog.filter_host(words=words, cap=30_000_000)
    exp = orc.replay(frec, lo * 8, (hi - lo) * 8, tracked_words=words, global_index=fgi)
    assert exp.rc == 0
    wset = set(words.tolist())
    assert sorted(t for t in got if t[0] in wset) == exp.triples()
    gpu_shadow = np.array([ctx.get_shadow(int(w), 1)[0] for w in words], dtype=np.uint8)
    assert np.array_equal(gpu_shadow, exp.shadow)
    ctx.close()
    return exp


@pytest.mark.slow
def test_config5_full_size_sampled(orc):
    from gen import native
    from paper_conf_ipps_yuphs21_b200.shard import shard_range
    prog = native.config5()
    lo, hi = shard_range(native.C5_BASE_WORD, native.C5_WORDS, 0, 8)
    exp = _sampled_full_size(orc, prog, lo, hi)
    assert len(exp.triples()) > 0


@pytest.mark.slow
def test_config3_full_size_sampled(orc):
    from gen import native
    prog = native.config3()
    lo, hi = prog.addr_base // 8, (prog.addr_base + prog.addr_bytes) // 8
    _sampled_full_size(orc, prog, lo, hi)


@pytest.mark.slow
def test_config4_full_size_sampled(orc):
    from gen import native
    prog = native.config4()
    lo, hi = prog.addr_base // 8, (prog.addr_base + prog.addr_bytes) // 8
    _sampled_full_size(orc, prog, lo, hi)


@pytest.mark.slow
def test_config5_one_flush_near_max_batch(orc):
    """Rank 0's whole config-5 batch (1.0e9 records, record positions up to 2^30)
    in one flush: the largest batch the ABI accepts, sampled against the oracle."""
    from gen import native
    from paper_conf_ipps_yuphs21_b200.shard import shard_range
    prog = native.config5()
    lo, hi = shard_range(native.C5_BASE_WORD, native.C5_WORDS, 0, 8)
    exp = _sampled_full_size(orc, prog, lo, hi, one_flush=True, seed=3)
    assert len(exp.triples()) > 0


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
