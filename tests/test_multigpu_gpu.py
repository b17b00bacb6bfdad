"""The multi-GPU path on one GPU.

Two NCCL ranks cannot share a device, so the collective is exercised through a
1-rank communicator (arb_config.world == 1 with an NCCL id): every arb_flush then
runs the same two ncclAllGather exchanges (validation status, then status and
report count) that a sharded job runs.  The sharding itself is checked with the
SURVEY §4.5 fake: 8 contexts on one GPU, each fed its address shard (all control
records + the accesses touching its words, with global record indices); their
report lists concatenated in rank order and their shadows must equal the
unsharded oracle, including map ranges that span shard boundaries.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _uid():
    from paper_conf_ipps_yuphs21_b200.shard import nccl_unique_id
    return nccl_unique_id()


def test_one_rank_communicator_exchange(orc):
    from gen.configs import config1
    from gpu_util import to_device
    from paper_conf_ipps_yuphs21_b200 import Context, reports_to_triples
    rec, base, size = config1()
    exp = orc.replay(rec, base, size)
    ctx = Context(base, size, world=1, rank=0, nccl_unique_id=_uid())
    st = ctx.stats()
    assert st["nccl_ranks"] == 1
    for _ in range(2):                      # the communicator survives across flushes
        ctx.submit_events(to_device(rec))
        rc, n, off = ctx.flush()
        assert rc == 0 and off == 0 and n == len(exp.triples())
        st = ctx.stats()
        assert st["exchanges"] == 2         # validation status + {status, count}
    ctx.close()
    # the first pass alone equals the oracle
    ctx = Context(base, size, world=1, rank=0, nccl_unique_id=_uid())
    ctx.submit_events(to_device(rec))
    rc, n, off = ctx.flush()
    assert reports_to_triples(ctx.get_reports(n)) == exp.triples()
    ctx.close()


def test_one_rank_communicator_error_is_collective_safe(orc):
    """A malformed record fails the validation exchange: the batch is discarded,
    no second collective runs, and the context (and its communicator) stay usable."""
    from gen.configs import config1
    from gpu_util import to_device
    from paper_conf_ipps_yuphs21_b200 import Context, ARB_ETRACE, reports_to_triples
    rec, base, size = config1()
    bad = rec.copy()
    bad[5, 1] = (bad[5, 1] & ~np.uint64((1 << 48) - 1)) | np.uint64(9)   # access of 9 bytes (Z18)
    ctx = Context(base, size, world=1, rank=0, nccl_unique_id=_uid())
    ctx.submit_events(to_device(bad))
    rc, _, _ = ctx.flush(check=False)
    assert rc == ARB_ETRACE
    assert ctx.stats()["exchanges"] == 1
    ctx.submit_events(to_device(rec))
    rc, n, off = ctx.flush()
    assert rc == 0 and off == 0
    exp = orc.replay(rec, base, size)
    assert reports_to_triples(ctx.get_reports(n)) == exp.triples()
    ctx.close()


def test_unknown_flag_bits_rejected():
    from paper_conf_ipps_yuphs21_b200 import Context, ArbError
    for flags in (1 << 5, 1 << 10, 1 << 31, 3 << 8):
        with pytest.raises(ArbError):
            Context(0x1000, 4096, flags=flags)


@pytest.mark.parametrize("with_comm", [False, True])
def test_eight_shard_contexts_equal_unsharded(orc, with_comm):
    """SURVEY §4.5 CI fake: config-5 shape over all 8 shards (2^33 words) with map
    sections centred on the shard boundaries; one context per shard on one GPU."""
    import torch
    from gen import native
    from gpu_util import to_device
    from paper_conf_ipps_yuphs21_b200 import Context, reports_to_triples
    from paper_conf_ipps_yuphs21_b200.shard import shard_range
    prog = native.config5(total_records=4_000_000, groups=48, stale_rate=40, seed=0xA4BA1E57 + 105)
    lo_all, n_all = native.C5_BASE_WORD, native.C5_WORDS
    rec = prog.fill_host()
    whole = orc.replay(rec, lo_all * 8, n_all * 8, threads=8)
    assert whole.rc == 0 and len(whole.triples()) > 0
    merged, offs = [], []
    for r in range(8):
        lo, hi = shard_range(lo_all, n_all, r, 8)
        srec, gi = prog.filter_host(word_lo=lo, word_hi=hi)
        ctx = Context(lo * 8, (hi - lo) * 8, world=1, rank=0, nccl_unique_id=_uid() if with_comm else None)
        ctx.submit_events(to_device(srec), global_index=to_device(gi))
        rc, n, off = ctx.flush()
        assert rc == 0
        offs.append(len(merged))
        merged += reports_to_triples(ctx.get_reports(n))
        sh = ctx.get_shadow(lo, hi - lo)
        assert np.array_equal(sh, whole.shadow[lo - lo_all:hi - lo_all]), f"shard {r} shadow"
        ctx.close()
        torch.cuda.synchronize()
    assert merged == whole.triples()         # rank order is canonical (word-major)
    assert len({bisect_rank(w, lo_all, n_all) for w, _, _ in merged}) >= 2


def bisect_rank(word, lo_all, n_all):
    return (word - lo_all) * 8 // n_all
