"""The oracle's address-sharded mode (the same sequential replay on
all host cores, one thread per contiguous word range) returns exactly what the
single-threaded replay returns: reports, final shadow and counters.  Pinned
against orc_replay itself, which the other oracle tests pin to the paper."""
import numpy as np
import pytest


def _same(a, b):
    assert a.rc == b.rc
    if a.rc != 0:
        return
    assert np.array_equal(a.reports, b.reports)
    if a.shadow is not None:
        assert np.array_equal(a.shadow, b.shadow)
    for k in ("records", "word_events", "transitions", "control_records", "ignored_word_events", "tasks"):
        assert a.stats[k] == b.stats[k], k


@pytest.mark.parametrize("seed", range(8))
@pytest.mark.parametrize("threads", [2, 3, 8])
def test_sharded_equals_sequential_fuzz(orc, seed, threads):
    from gen.fuzz import random_program
    rec, base, span = random_program(900 + seed, p_task=0.4, p_depend=0.3, p_always=0.2)
    for kw in ({}, {"dedup_first": True}, {"detect_bo": True}):
        one = orc.replay(rec, base, span, **kw)
        many = orc.replay(rec, base, span, threads=threads, **kw)
        _same(one, many)


@pytest.mark.parametrize("n_dev", [2, 3])
def test_sharded_devices(orc, n_dev):
    from gen.fuzz import random_program
    rec, base, span = random_program(950 + n_dev, n_devices=n_dev, p_task=0.3)
    _same(orc.replay(rec, base, span, n_devices=n_dev), orc.replay(rec, base, span, n_devices=n_dev, threads=5))


def test_sharded_config5_with_global_index(orc):
    """A shard of the config-5 shape (global record indices, boundary-spanning maps)."""
    from gen import native
    from paper_conf_ipps_yuphs21_b200.shard import shard_range
    prog = native.config5(total_records=400_000, groups=24, stale_rate=20)
    lo, hi = shard_range(native.C5_BASE_WORD, native.C5_WORDS, 3, 8)
    rec, gi = prog.filter_host(word_lo=lo, word_hi=hi)
    one = orc.replay(rec, lo * 8, (hi - lo) * 8, global_index=gi)
    assert len(one.reports) > 0
    _same(one, orc.replay(rec, lo * 8, (hi - lo) * 8, global_index=gi, threads=7))


def test_sharded_sparse_mode(orc):
    from gen.fuzz import random_program
    rec, base, span = random_program(977, p_task=0.4)
    rs = np.random.default_rng(1)
    words = np.unique(rs.integers(base // 8, (base + span) // 8, 300)).astype(np.uint64)
    one = orc.replay(rec, base, span, tracked_words=words)
    _same(one, orc.replay(rec, base, span, tracked_words=words, threads=4))


def test_sharded_error_codes(orc):
    from gen.fuzz import random_program
    rec, base, span = random_program(978, p_task=0.4)
    bad = rec.copy()
    bad[len(bad) // 2, 1] = (bad[len(bad) // 2, 1] & ~np.uint64((1 << 48) - 1)) | np.uint64(0)
    one = orc.replay(bad, base, span)
    many = orc.replay(bad, base, span, threads=4)
    assert one.rc == many.rc and one.stats["error_record"] == many.stats["error_record"]


def test_continuation_equals_whole_trace(orc):
    """shadow_in: replaying a trace in quiescent pieces, each starting from the
    previous piece's final shadow, gives the whole trace's reports and shadow."""
    from gen import native
    prog = native.config5(total_records=300_000, groups=12, stale_rate=10)
    lo, n_words = native.C5_BASE_WORD, native.C5_SHARD_WORDS // 64     # a slice of shard 0
    rec, gi = prog.filter_host(word_lo=lo, word_hi=lo + n_words)
    whole = orc.replay(rec, lo * 8, n_words * 8, global_index=gi)
    assert whole.rc == 0
    q = sorted(set(np.searchsorted(gi, np.array(prog.quiescent, dtype=np.uint64)).tolist()) | {0, len(gi)})
    cuts = [q[0], q[len(q) // 3], q[2 * len(q) // 3], q[-1]]
    sh, reps = None, []
    for a, b in zip(cuts[:-1], cuts[1:]):
        r = orc.replay(rec[a:b], lo * 8, n_words * 8, global_index=gi[a:b], shadow_in=sh, threads=3)
        assert r.rc == 0
        reps.append(r.reports)
        sh = r.shadow
    got = np.concatenate(reps)
    got = got[np.lexsort((got["kind"], got["record"], got["word"]))]
    assert np.array_equal(got, whole.reports)
    assert np.array_equal(sh, whole.shadow)
