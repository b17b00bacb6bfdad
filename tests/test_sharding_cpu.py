"""Multi-process (gloo, world_size 2, CPU) checks of the address-sharded path.

The library's collective (ncclAllGather of report counts inside arb_flush)
needs GPUs; here the host-side logic around it is checked with the CPU oracle
standing in for each rank's replay: shard ranges, order-preserving selection of
a shard's records (all control records + the accesses touching its words, with
global record indices), the count exchange and offsets, and the rank-order
concatenation that must equal the unsharded result.
"""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, rec, base_word, n_words, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import torch
    import oracle
    from paper_conf_ipps_yuphs21_b200.shard import shard_range, shard_records
    lo, hi = shard_range(base_word, n_words, rank, world)
    srec, gidx = shard_records(rec, lo, hi)
    res = oracle.replay(srec, lo * 8, (hi - lo) * 8, global_index=gidx)
    assert res.rc == 0
    mine = torch.tensor([len(res.reports)], dtype=torch.int64)
    counts = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
    dist.all_gather(counts, mine)
    offset = int(sum(c.item() for c in counts[:rank]))
    triples = res.triples()
    import hashlib
    digest = hashlib.sha1(res.shadow.tobytes()).hexdigest()
    gathered = [None] * world
    dist.all_gather_object(gathered, (offset, triples, digest, int(lo), int(hi)))
    if rank == 0:
        out.put(gathered)
    dist.barrier()
    dist.destroy_process_group()


def _run_world(rec, base_word, n_words, world=2):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, rec, base_word, n_words, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return got


@pytest.mark.parametrize("case", ["config5", "fuzz"])
def test_two_rank_sharding_equals_unsharded(orc, case):
    if case == "config5":
        from gen import native
        prog = native.config5(total_records=2_000_000, groups=32, stale_rate=50)
        base_word, n_words = native.C5_BASE_WORD, native.C5_SHARD_WORDS * 2   # shards 0-1 of 8
        lo_all, hi_all = base_word, base_word + n_words
        rec, _ = prog.filter_host(word_lo=lo_all, word_hi=hi_all)
    else:
        from gen.fuzz import random_program
        rec, base, span = random_program(5, n_arrays=6, array_words=512, steps=300)
        base_word, n_words = base // 8, span // 8
    whole = orc.replay(rec, base_word * 8, n_words * 8)
    assert whole.rc == 0
    gathered = _run_world(rec, base_word, n_words)
    # counts exchanged -> offsets are the exclusive prefix
    offs = [g[0] for g in gathered]
    lens = [len(g[1]) for g in gathered]
    assert offs == [sum(lens[:r]) for r in range(len(lens))]
    merged = []
    for g in gathered:
        merged.extend(tuple(t) for t in g[1])
    assert merged == whole.triples()            # rank order is already canonical
    import hashlib
    for g in gathered:                          # each shard's final shadow = the unsharded slice
        lo, hi = g[3] - base_word, g[4] - base_word
        assert g[2] == hashlib.sha1(whole.shadow[lo:hi].tobytes()).hexdigest()


def test_boundary_straddling_access_goes_to_both_owners():
    from paper_conf_ipps_yuphs21_b200.shard import shard_range, shard_records
    from gen.trace import TraceBuilder
    lo0, hi0 = shard_range(0x100, 64, 0, 2)
    tb = TraceBuilder()
    tb.rh(hi0 * 8 - 4, 8)          # words hi0-1 and hi0
    tb.enter(0, 0x100 * 8, 64 * 8)
    tb.wt((hi0 + 3) * 8)
    rec = tb.array()
    r0, g0 = shard_records(rec, lo0, hi0)
    lo1, hi1 = shard_range(0x100, 64, 1, 2)
    r1, g1 = shard_records(rec, lo1, hi1)
    assert g0.tolist() == [0, 1] and g1.tolist() == [0, 1, 2]
