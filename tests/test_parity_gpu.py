"""GPU parity: libarbalest (through the C ABI) vs the CPU oracle, element by element.

Report sets must be identical triples (word, record, kind) — bit-exact, this is
integer work — and the final shadow must be identical byte for byte.
"""
import numpy as np
import pytest

from golden_io import load
from gpu_util import run_gpu

pytestmark = pytest.mark.gpu


def check(orc, rec, base, size, **kw):
    okw = {k: kw.pop(k) for k in ("dedup_first",) if k in kw}
    flags = (1 if okw.get("dedup_first") else 0) | kw.pop("flags", 0)
    okw["detect_bo"] = bool(flags & 8)                    # ARB_F_BO <-> the oracle's extension (Z20)
    okw["unified"] = bool(flags & 16)                     # ARB_F_UNIFIED <-> unified memory (Z23)
    okw["n_devices"] = 1 + ((flags >> 8) & 3)             # ARB_F_DEVICES(n) <-> accelerators (Z24)
    exp = orc.replay(rec, base, size, **okw)
    rc, got, shadow, st = run_gpu(rec, base, size, flags=flags, **kw)
    assert rc == exp.rc
    if rc == 0:
        assert got == exp.triples()
        assert np.array_equal(shadow, exp.shadow)
        assert st["access_words"] + st["range_words"] == exp.stats["word_events"]
    return exp, st


@pytest.mark.parametrize("name", ["fig1_n3.trace", "fig2_no_sync.trace", "fig2_sync.trace"])
@pytest.mark.parametrize("bb", [0, 3])
def test_golden(orc, name, bb):
    rec, base, size, expect = load(name)
    exp, _ = check(orc, rec, base, size, bucket_bits=bb)
    assert exp.triples() == expect


def test_config1(orc):
    from gen.configs import config1
    rec, base, size = config1()
    exp, st = check(orc, rec, base, size)
    assert len(exp.triples()) == 1024
    assert st["reports"] == 1024 and st["reports_by_kind"][2] == 1024


@pytest.mark.parametrize("bb", [0, 14])
def test_config2(orc, bb):
    from gen.configs import config2
    rec, base, size = config2()
    check(orc, rec, base, size, bucket_bits=bb)


@pytest.mark.parametrize("seed", range(60))
def test_fuzz_small(orc, seed):
    from gen.fuzz import random_program
    rec, base, span = random_program(seed)
    for bb in (0, 2, 5):
        check(orc, rec, base, span, bucket_bits=bb)


@pytest.mark.parametrize("seed", range(8))
def test_fuzz_large_steps(orc, seed):
    """Buckets with many steps (> 4096 events), range ops cutting steps, ragged tails."""
    from gen.fuzz import random_program
    rec, base, span = random_program(1000 + seed, n_arrays=6, array_words=8192, steps=500,
                                     loop_max=20000)
    for bb in (0, 11):
        check(orc, rec, base, span, bucket_bits=bb)


@pytest.mark.parametrize("seed", range(12))
def test_split_parts(orc, seed):
    """Range-heavy buckets replayed as word-range parts by separate CTAs
    (ARB_F_SMALL_PARTS forces the split at 1024-word parts)."""
    from gen.fuzz import random_program
    rec, base, span = random_program(2000 + seed, n_arrays=4, array_words=8192, steps=200)
    for bb in (0, 13):
        _, st = check(orc, rec, base, span, bucket_bits=bb, flags=4)


def test_config2_split_parts(orc):
    from gen.configs import config2
    rec, base, size = config2()
    check(orc, rec, base, size, flags=4)


@pytest.mark.parametrize("n,flags", [(100000, 0), (100000, 4), (400000, 0)])
def test_hot_word(orc, n, flags):
    """One word with 10^5..4x10^5 events spanning many steps (the bfs `stop` flag
    shape).  400000 events make the bucket hot (K5: replayed as time slices across
    CTAs); flags=4 (ARB_F_SMALL_PARTS) forces 3 slices at 10^5."""
    from gen.trace import MAP, OP, TraceBuilder
    tb = TraceBuilder()
    A = 0x8000
    tb.wh(A)
    tb.enter(MAP.TO, A, 64)
    rs = np.random.default_rng(5)
    ops = rs.choice([OP.RT, OP.WT, OP.RH, OP.WH], size=n, p=[.4, .2, .3, .1])
    for chunk in np.array_split(ops, 10):
        arr = np.zeros((chunk.size, 2), dtype=np.uint64)
        arr[:, 0] = np.uint64(A) | (chunk.astype(np.uint64) << np.uint64(48))
        arr[:, 1] = 8
        tb.add_array(arr)
        tb.update(0, A, 64)
    tb.exit(MAP.TOFROM, A, 64)
    _, st = check(orc, tb.array(), A, 64, flags=flags)
    if n > 300000 or flags:
        assert st["hot_buckets"] >= 1


def test_multi_flush_quiescent(orc):
    """Flushes cut where no task is open or unjoined give the oracle's whole-trace result."""
    from gen.configs import config2
    rec, base, size, inst, spans = config2(reps=2, with_index=True)
    exp = orc.replay(rec, base, size)
    cuts = [s[2] for s in spans[1:]][::7]          # pattern boundaries are quiescent
    rc, got, shadow, st = run_gpu(rec, base, size, flush_points=cuts)
    # each flush is in canonical order; the union over flushes is the oracle's set
    assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)
    assert st["flushes"] == len(cuts) + 1


def test_host_submit_and_global_index(orc):
    from gen.fuzz import random_program
    rec, base, span = random_program(77)
    gi = np.arange(rec.shape[0], dtype=np.uint64) * 3 + 1000
    exp = orc.replay(rec, base, span, global_index=gi)
    for host in (True, False):
        rc, got, shadow, _ = run_gpu(rec, base, span, host=host, global_index=gi)
        assert rc == 0 and got == exp.triples() and np.array_equal(shadow, exp.shadow)


def test_several_submits_one_flush(orc):
    import torch
    from gpu_util import to_device
    from paper_conf_ipps_yuphs21_b200 import Context, reports_to_triples
    from gen.fuzz import random_program
    rec, base, span = random_program(78)
    exp = orc.replay(rec, base, span)
    ctx = Context(base, span)
    k = rec.shape[0] // 3
    d0, d2 = to_device(rec[:k]), to_device(rec[2 * k:])   # device buffers stay alive until flush
    ctx.submit_events(d0)
    ctx.submit_events(np.ascontiguousarray(rec[k:2 * k]))
    ctx.submit_events(d2)
    rc, n, _ = ctx.flush()
    assert reports_to_triples(ctx.get_reports(n)) == exp.triples()
    assert np.array_equal(ctx.get_shadow(base // 8, span // 8), exp.shadow)
    ctx.close()
    torch.cuda.synchronize()


def test_dedup_first(orc):
    from gen.configs import config2
    rec, base, size = config2(reps=2)
    check(orc, rec, base, size, dedup_first=True)


@pytest.mark.parametrize("bad", ["op", "len", "emap", "present", "nested"])
def test_errors_leave_state_unchanged(orc, bad):
    from gen.trace import MAP, TraceBuilder
    from paper_conf_ipps_yuphs21_b200 import Context, reports_to_triples
    from gpu_util import to_device
    A = 0x4000
    good = TraceBuilder()
    good.wh(A); good.enter(MAP.TO, A, 64); good.wt(A + 8)
    tb = TraceBuilder()
    tb.rt(A)
    if bad == "op":
        tb._add(7, A, 8)
    elif bad == "len":
        tb.rh(A, 0)
    elif bad == "emap":
        tb.enter(MAP.TO, A + 32, 64)
    elif bad == "present":
        tb.enter(MAP.TO | MAP.PRESENT, A + 128, 64)       # not mapped: ARB_EMAP (Z21)
    elif bad == "nested":
        tb.task_begin(3); tb.task_begin(4)
    ctx = Context(A, 256)
    dg = to_device(good.array())
    ctx.submit_events(dg)
    ctx.flush()
    before = ctx.get_shadow(A // 8, 32).copy()
    db = to_device(tb.array())
    ctx.submit_events(db)
    rc, _, _ = ctx.flush(check=False)
    whole = np.concatenate([good.array(), tb.array()])
    assert rc == orc.replay(whole, A, 256).rc
    assert rc in (-4, -5)
    assert np.array_equal(ctx.get_shadow(A // 8, 32), before)
    # the context stays usable: the same good continuation works
    nxt = TraceBuilder(); nxt.rt(A + 8); nxt.rh(A)
    dn = to_device(nxt.array())
    ctx.submit_events(dn)
    rc, n, _ = ctx.flush()
    exp = orc.replay(np.concatenate([good.array(), nxt.array()]), A, 256)
    assert reports_to_triples(ctx.get_reports(n)) == [t for t in exp.triples() if t[1] >= 3]
    ctx.close()


def test_truncation_count_exact(orc):
    from gen.configs import config1
    from paper_conf_ipps_yuphs21_b200 import Context, reports_to_triples, ARB_TRUNCATED
    from gpu_util import to_device
    rec, base, size = config1()
    exp = orc.replay(rec, base, size)
    ctx = Context(base, size, report_capacity=100)
    dr = to_device(rec)
    ctx.submit_events(dr)
    rc, n, _ = ctx.flush()
    assert rc == ARB_TRUNCATED and n == len(exp.triples()) == 1024
    got = reports_to_triples(ctx.get_reports(100))
    assert len(got) == 100 and set(got) <= set(exp.triples())
    ctx.close()


def test_untracked_words_ignored(orc):
    """Z12: words outside the tracked range are ignored by both sides."""
    from gen.fuzz import random_program
    rec, base, span = random_program(91)
    check(orc, rec, base + 256, span // 2)


# ---- buffer-overflow extension (ARB_F_BO = 8, Z20) ---------------
@pytest.mark.parametrize("write", [False, True])
def test_bo_half_mapped_array(orc, write):
    """only the first half of the array is mapped, the kernel loops over all of it."""
    from gen.trace import MAP, OP, TraceBuilder
    A, n = 0x40000, 4096
    tb = TraceBuilder()
    tb.loop([(OP.WH, A)], n, 8)
    tb.enter(MAP.TOFROM, A, 8 * (n // 2))
    k0 = len(tb)
    tb.loop([(OP.WT if write else OP.RT, A)], n, 8)
    tb.exit(MAP.TOFROM, A, 8 * (n // 2))
    exp, st = check(orc, tb.array(), A, 8 * n, flags=8)
    assert exp.triples() == [(A // 8 + i, k0 + i, 4) for i in range(n // 2, n)]
    assert st["reports_bo"] == n // 2


@pytest.mark.parametrize("seed", range(24))
def test_bo_fuzz_small(orc, seed):
    from gen.fuzz import random_program
    rec, base, span = random_program(3000 + seed)
    for bb in (0, 2, 5):
        check(orc, rec, base, span, bucket_bits=bb, flags=8)


@pytest.mark.parametrize("seed", range(4))
def test_bo_fuzz_large_steps(orc, seed):
    """Many steps per bucket, sort steps, range ops cutting steps; with parts (flags 4)."""
    from gen.fuzz import random_program
    rec, base, span = random_program(1000 + seed, n_arrays=6, array_words=8192, steps=500,
                                     loop_max=20000)
    for bb in (0, 11):
        check(orc, rec, base, span, bucket_bits=bb, flags=8)
    check(orc, rec, base, span, flags=8 | 4)


def test_bo_config2_and_hot_word(orc):
    """The DRACC-style suite and a hot word under ARB_F_BO: the hot bucket is replayed
    as K5 time slices whose per-word functions are selector pairs keyed by the CV
    present bit (the CV is deleted and re-created between the slices' events)."""
    from gen.configs import config2
    from gen.trace import MAP, OP, TraceBuilder
    rec, base, size = config2()
    check(orc, rec, base, size, flags=8)
    tb = TraceBuilder()
    A = 0x8000
    tb.wh(A)
    rs = np.random.default_rng(6)
    ops = rs.choice([OP.RT, OP.WT, OP.RH, OP.WH], size=400000, p=[.4, .2, .3, .1])
    for j, chunk in enumerate(np.array_split(ops, 10)):
        if j % 2 == 0:
            tb.enter(MAP.TO, A, 64)       # odd chunks run with the CV deleted: their target accesses are BO
        arr = np.zeros((chunk.size, 2), dtype=np.uint64)
        arr[:, 0] = np.uint64(A) | (chunk.astype(np.uint64) << np.uint64(48))
        arr[:, 1] = 8
        tb.add_array(arr)
        if j % 2 == 0:
            tb.exit(MAP.DELETE, A, 64)
    exp, st = check(orc, tb.array(), A, 64, flags=8)
    assert st["hot_buckets"] >= 1 and st["reports_bo"] > 0
    check(orc, tb.array(), A, 64, flags=8 | 4)         # forced slices of every busy bucket


def test_bo_patterns(orc):
    """The buffer-overflow patterns (DRACC 23/25/28-31 analogues), buggy and fixed,
    concatenated on separate regions: GPU = oracle with the extension on."""
    from gen.patterns import BO_PATTERNS
    from gen.trace import TraceBuilder
    tb = TraceBuilder()
    region, base, k = 1 << 16, 0x100000, 0
    for esz in (4, 8):
        for name in sorted(BO_PATTERNS):
            for buggy in (True, False):
                BO_PATTERNS[name][0](tb, base + k * region, 2048, esz, buggy, 5)
                k += 1
    exp, st = check(orc, tb.array(), base, k * region, flags=8)
    assert {t[2] for t in exp.triples()} == {4} and st["reports_bo"] == len(exp.triples())


# ---- N2: flushes between a nowait block's end and its join ------------
def _cuts(rec, k, seed, inside=None):
    """k random flush points; inside=True/False restricts them to positions inside
    / outside TASK_BEGIN..TASK_END blocks (None: anywhere).  Open blocks and
    unjoined instances then cross flushes (N2)."""
    op = (rec[:, 0] >> np.uint64(48)) & np.uint64(0xFF)
    depth = np.cumsum((op == 12).astype(np.int64) - (op == 13).astype(np.int64))
    ok = np.arange(1, rec.shape[0])                        # cut after record i - 1
    if inside is not None:
        ok = ok[(depth[ok - 1] > 0) == inside]
    rs = np.random.default_rng(seed)
    return sorted(set(int(x) for x in rs.choice(ok, size=min(k, ok.size), replace=False)))


def _unjoined_across(rec, cuts):
    """How many cuts separate a TASK_END from its join."""
    op = (rec[:, 0] >> np.uint64(48)) & np.uint64(0xFF)
    ends = np.nonzero(op == 13)[0]
    syncs = np.nonzero(op == 14)[0]
    n = 0
    for e in ends:
        j = syncs[syncs > e]
        j = j[0] if j.size else rec.shape[0]
        n += sum(1 for c in cuts if e < c <= j)
    return n


@pytest.mark.parametrize("seed", range(24))
def test_flush_cuts_unjoined_tasks_fuzz(orc, seed):
    """The union of the flushes' reports equals the whole-trace oracle for any
    flush points (N2: open blocks and unjoined instances are carried across)."""
    from gen.fuzz import random_program
    rec, base, span = random_program(4000 + seed, p_task=0.4)
    exp = orc.replay(rec, base, span)
    cuts = _cuts(rec, 6, seed, inside=None if seed % 3 == 0 else seed % 3 == 1)
    rc, got, shadow, st = run_gpu(rec, base, span, flush_points=cuts)
    if exp.rc == -7:                             # the trace ends inside a block: the oracle's end-of-trace
        assert rc == 0                           # ARB_EOPEN; a flush just carries the open block
        return
    assert rc == exp.rc                          # a malformed program fails in the flush holding the error
    if rc == 0:
        assert sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


def test_flush_cuts_unjoined_tasks_config2(orc):
    from gen.configs import config2
    rec, base, size = config2(reps=2)
    exp = orc.replay(rec, base, size)
    cuts = _cuts(rec, 40, 7, inside=False) + _cuts(rec, 20, 8, inside=True)
    cuts = sorted(set(cuts))
    assert _unjoined_across(rec, cuts) > 0
    rc, got, shadow, st = run_gpu(rec, base, size, flush_points=cuts)
    assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


def test_flush_between_end_and_join(orc):
    """Fig. 2 shape across three flushes: the nowait write (flush 1), the racy host
    read (flush 2), the taskwait (flush 3): the MIR at the host read is reported."""
    from gen.trace import MAP, TraceBuilder
    A = 0x4000
    tb = TraceBuilder()
    tb.wh(A); tb.enter(MAP.TOFROM, A, 64)
    tb.task_begin(7); tb.wt(A); tb.task_end(7)
    c1 = len(tb)
    i_race = tb.rh(A + 0)
    tb.wh(A + 8)
    c2 = len(tb)
    tb.sync(7)
    tb.exit(MAP.TOFROM, A, 64)
    rec = tb.array()
    exp = orc.replay(rec, A, 64)
    assert (A // 8, i_race, 3) in exp.triples()
    rc, got, shadow, st = run_gpu(rec, A, 64, flush_points=[c1, c2])
    assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


@pytest.mark.parametrize("seed", range(16))
def test_always_modifier_fuzz(orc, seed):
    """The `always` map-type modifier (N4, Z21) on random programs, with and
    without flush cuts."""
    from gen.fuzz import random_program
    rec, base, span = random_program(5000 + seed, p_always=0.5, p_task=0.3)
    check(orc, rec, base, span)
    exp = orc.replay(rec, base, span)
    if exp.rc == 0:
        rc, got, shadow, _ = run_gpu(rec, base, span, flush_points=_cuts(rec, 4, seed))
        assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


@pytest.mark.parametrize("seed", range(16))
def test_depend_fuzz(orc, seed):
    """Task dependencies (N4, Z22) on random programs, with and without flush cuts
    (dependencies between instances carried across flushes)."""
    from gen.fuzz import random_program
    rec, base, span = random_program(6000 + seed, p_task=0.45, p_depend=0.6)
    exp, _ = check(orc, rec, base, span)
    if exp.rc == 0:
        rc, got, shadow, _ = run_gpu(rec, base, span, flush_points=_cuts(rec, 5, seed))
        assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


# ---- unified memory (ARB_F_UNIFIED = 16, Z23) ---------------------
@pytest.mark.parametrize("name", ["fig1_n3.trace", "fig2_no_sync.trace", "fig2_sync.trace"])
def test_unified_golden(orc, name):
    rec, base, size, _ = load(name)
    check(orc, rec, base, size, flags=16)


@pytest.mark.parametrize("seed", range(12))
def test_unified_fuzz(orc, seed):
    """Random programs (tasks, depend, modifiers) under unified memory, several bucket
    sizes, forced parts / time slices (flags 4), and flush cuts."""
    from gen.fuzz import random_program
    rec, base, span = random_program(7000 + seed, p_task=0.3, p_always=0.3, p_depend=0.3, steps=120)
    exp, _ = check(orc, rec, base, span, flags=16)
    for bb in (2, 5):
        check(orc, rec, base, span, bucket_bits=bb, flags=16)
    check(orc, rec, base, span, flags=16 | 4)
    if exp.rc == 0:
        rc, got, shadow, _ = run_gpu(rec, base, span, flags=16, flush_points=_cuts(rec, 4, seed))
        ex2 = orc.replay(rec, base, span, unified=True)
        assert rc == 0 and sorted(got) == ex2.triples() and np.array_equal(shadow, ex2.shadow)


def test_unified_config2_and_hot_word(orc):
    from gen.configs import config2
    from gen.trace import MAP, OP, TraceBuilder
    rec, base, size = config2()
    check(orc, rec, base, size, flags=16)
    tb = TraceBuilder()
    A = 0x8000
    tb.wh(A)
    tb.enter(MAP.TO, A, 64)
    rs = np.random.default_rng(8)
    ops = rs.choice([OP.RT, OP.WT, OP.RH, OP.WH], size=400000, p=[.4, .2, .3, .1])
    arr = np.zeros((ops.size, 2), dtype=np.uint64)
    arr[:, 0] = np.uint64(A) | (ops.astype(np.uint64) << np.uint64(48))
    arr[:, 1] = 8
    tb.add_array(arr)
    tb.exit(MAP.TOFROM, A, 64)
    _, st = check(orc, tb.array(), A, 64, flags=16)
    assert st["hot_buckets"] >= 1                      # K5 time slices compose the shared-value writes


def test_unified_excludes_bo():
    from paper_conf_ipps_yuphs21_b200 import Context, ArbError
    with pytest.raises(ArbError):
        Context(0x1000, 4096, flags=8 | 16)


def test_empty_flushes(orc):
    """An empty batch flushes cleanly (multi-GPU runs pad their flush schedules with
    them so that every rank joins every count exchange) and changes nothing."""
    from gen.configs import config1
    rec, base, size = config1()
    exp = orc.replay(rec, base, size)
    rc, got, shadow, st = run_gpu(rec, base, size, flush_points=[0, 0, rec.shape[0], rec.shape[0]])
    assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)
    assert st["flushes"] == 5



# ---- several accelerators (ARB_F_DEVICES(n), Z24) ----------------------
def test_devices_example(orc):
    from gen.trace import encode, OP, MAP
    A = 0x1000
    recs = [encode(OP.WH, A, 8), encode(OP.MAP_ENTER, A, 8, arg=MAP.TO | (1 << 6)),
            encode(OP.RT, A, 8, arg=0), encode(OP.RT, A, 8, arg=1), encode(OP.WT, A, 8, arg=1),
            encode(OP.RH, A, 8), encode(OP.MAP_EXIT, A, 8, arg=MAP.FROM | (1 << 6)), encode(OP.RH, A, 8)]
    exp, _ = check(orc, np.array(recs, dtype=np.uint64).reshape(-1, 2), A, 64, flags=1 << 8)
    assert exp.triples() == [(A // 8, 2, 1), (A // 8, 5, 2)]   # RT on device 0: no CV there; stale host read


@pytest.mark.parametrize("seed", range(12))
def test_devices_fuzz(orc, seed):
    """Random programs on 2 and 3 accelerators: several bucket sizes, word-range
    parts (flags 4) and flush cuts."""
    from gen.fuzz import random_program
    nd = 2 + seed % 2
    fl = (nd - 1) << 8
    rec, base, span = random_program(8000 + seed, n_devices=nd, p_task=0.3, p_always=0.2, steps=120)
    exp, _ = check(orc, rec, base, span, flags=fl)
    for bb in (2, 5):
        check(orc, rec, base, span, bucket_bits=bb, flags=fl)
    check(orc, rec, base, span, flags=fl | 4)
    if exp.rc == 0:
        rc, got, shadow, _ = run_gpu(rec, base, span, flags=fl, flush_points=_cuts(rec, 4, seed))
        assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


@pytest.mark.parametrize("seed", range(4))
def test_devices_large_steps(orc, seed):
    """Many steps per bucket with sort steps and range ops cutting steps, 3 devices."""
    from gen.fuzz import random_program
    rec, base, span = random_program(8100 + seed, n_arrays=6, array_words=8192, steps=500,
                                     loop_max=20000, n_devices=3)
    for bb in (0, 11):
        check(orc, rec, base, span, bucket_bits=bb, flags=2 << 8)


def test_depend_binds_to_joined_instance_across_flush(orc):
    """a TASK_DEPEND(k) after a flush cut binds to the last ended
    instance of task id k even when that instance was joined in the earlier flush
    (Z22).  X(1) and Y(1) end, Z(2) depends on Y, SYNC(2) joins Z and, through the
    dependency, Y; X stays unjoined and is carried.  After the cut W(3) depends on
    task 1 = Y (joined: no constraint), so W's read of the word X wrote races with X."""
    from gen.trace import TraceBuilder, MAP
    base = 0x1000_0000
    tb = TraceBuilder()
    tb.wh(base)
    tb.enter(MAP.TOFROM, base, 64)
    tb.task_begin(1); tb.wt(base); tb.task_end(1)          # X
    tb.task_begin(1); tb.wt(base + 8); tb.task_end(1)      # Y
    tb.task_begin(2); tb.depend(1); tb.rt(base + 8); tb.task_end(2)   # Z after Y
    tb.sync(2)                                              # joins Z and Y
    cut = len(tb)
    tb.task_begin(3); tb.depend(1); tb.rt(base); tb.task_end(3)        # W
    w_read = len(tb) - 2
    tb.sync()
    tb.exit(MAP.TOFROM, base, 64)
    rec = tb.array()
    exp = orc.replay(rec, base, 64)
    assert exp.rc == 0
    assert (base // 8, w_read, 3) in exp.triples()           # W races with X
    for cuts in ([], [cut]):
        rc, got, shadow, _ = run_gpu(rec, base, 64, flush_points=cuts)
        assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


@pytest.mark.parametrize("seed", range(10))
def test_dedup_first_across_flush_cuts(orc, seed):
    """ARB_F_DEDUP_FIRST with random flush cuts (also inside task blocks) equals the
    whole-trace oracle in dedup-first mode (Z3 over the whole trace)."""
    from gen.fuzz import random_program
    rec, base, span = random_program(8100 + seed, p_task=0.35, p_depend=0.2, steps=90)
    exp = orc.replay(rec, base, span, dedup_first=True)
    if exp.rc != 0:
        pytest.skip("program rejected by the oracle")
    for k in (3, 9):
        rc, got, shadow, _ = run_gpu(rec, base, span, flags=1, flush_points=_cuts(rec, k, seed))
        assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


def test_dedup_first_set_grows(orc):
    """Many flushes, many distinct (word, kind) pairs: the persistent set is rehashed."""
    from gen.configs import config2
    rec, base, size = config2()
    exp = orc.replay(rec, base, size, dedup_first=True)
    assert exp.rc == 0 and len(exp.triples()) > 1000
    op = (rec[:, 0] >> np.uint64(48)) & np.uint64(0xFF)
    depth = np.cumsum((op == 12).astype(np.int64) - (op == 13).astype(np.int64))
    ok = np.nonzero(depth == 0)[0] + 1
    cuts = sorted(set(ok[np.linspace(0, ok.size - 1, 40).astype(int)].tolist()) - {rec.shape[0]})
    rc, got, shadow, _ = run_gpu(rec, base, size, flags=1, flush_points=cuts)
    assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


@pytest.mark.parametrize("split", [1, 3])
def test_host_submit_host_global_index(orc, split):
    """Host records with host global indices (a shard of config 5): the indices are not
    copied to the device; the report path translates positions on the host (§8(b))."""
    from gen import native
    from paper_conf_ipps_yuphs21_b200 import Context, reports_to_triples
    from paper_conf_ipps_yuphs21_b200.shard import shard_range
    prog = native.config5(total_records=2_000_000, groups=24, stale_rate=10)
    lo, hi = shard_range(native.C5_BASE_WORD, native.C5_WORDS, 2, 8)
    rec, gi = prog.filter_host(word_lo=lo, word_hi=hi)
    exp = orc.replay(rec, lo * 8, (hi - lo) * 8, global_index=gi)
    assert exp.rc == 0 and len(exp.triples()) > 0
    ctx = Context(lo * 8, (hi - lo) * 8)
    cuts = np.linspace(0, rec.shape[0], split + 1).astype(int)
    for a, b in zip(cuts[:-1], cuts[1:]):          # several host submits, one flush
        ctx.submit_events(np.ascontiguousarray(rec[a:b]), global_index=np.ascontiguousarray(gi[a:b]))
    rc, n, _ = ctx.flush()
    assert rc == 0
    assert reports_to_triples(ctx.get_reports(n)) == exp.triples()
    import torch
    dev_out = torch.zeros((max(n, 1), 2), dtype=torch.int64, device="cuda")
    ctx.get_reports(n, out=dev_out)                 # device output of host-translated reports
    assert reports_to_triples(dev_out[:n].cpu().numpy().view(np.uint64)) == exp.triples()
    ctx.close()


# ---- N1: buffer overflow through a tagged pointer (ARB_BASE, Z25) -------------
def test_bo_overflow_into_adjacent_cv_gpu(orc):
    """The P:279 case the present-bit form misses: the kernel's pointer to A runs into
    B's (mapped) CV; every such access is BO and still reads B's CV."""
    from gen.trace import TraceBuilder, MAP, OP, encode
    A, n = 0x4000, 64
    B = A + 8 * (n // 2)
    tb = TraceBuilder()
    tb.loop([(OP.WH, A)], n, 8)
    tb.enter(MAP.TO, A, 8 * (n // 2))
    tb.enter(MAP.TO, B, 8 * (n // 2))
    tb.add_array(np.array([encode(OP.BASE, A, 0, task=1)], dtype=np.uint64))
    for i in range(n):
        tb.add_array(np.array([encode(OP.RT, A + 8 * i, 8, task=1)], dtype=np.uint64))
    tb.exit(MAP.TO, B, 8 * (n // 2))
    tb.exit(MAP.TO, A, 8 * (n // 2))
    rec = tb.array()
    exp, st = check(orc, rec, A, 8 * n, flags=8)
    assert len(exp.triples()) == n // 2 and {t[2] for t in exp.triples()} == {4}
    assert st["reports_bo"] == n // 2


@pytest.mark.parametrize("seed", range(10))
def test_bo_tags_fuzz(orc, seed):
    """Random programs with pointer tags, re-based tags, tasks and flush cuts (the tag
    bases and entries carried across flushes), several bucket sizes."""
    from gen.fuzz import random_program
    rec, base, span = random_program(9100 + seed, p_tag=0.6, p_task=0.3, steps=120)
    exp, _ = check(orc, rec, base, span, flags=8)
    check(orc, rec, base, span, flags=8, bucket_bits=4)
    if exp.rc == 0:
        rc, got, shadow, _ = run_gpu(rec, base, span, flags=8, flush_points=_cuts(rec, 5, seed))
        assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


# ---- N1: CV -> OV translation (ARB_CV_BASE, CV-addressed target accesses, Z26) -----
@pytest.mark.parametrize("seed", range(8))
def test_cv_addressed_fuzz(orc, seed):
    """Random programs whose target accesses to mapped words use CV (device) addresses:
    the batch is partitioned, the CV placements resolved, the accesses translated and
    the batch partitioned again; with flush cuts (placements carried across flushes),
    with the buffer-overflow extension, and with only half of the accesses rewritten."""
    from gen.fuzz import random_program, to_cv_addressing
    rec, base, span = random_program(9400 + seed, p_task=0.3, steps=100)
    cv = to_cv_addressing(rec, frac=1.0 if seed % 2 else 0.5, seed=seed)
    exp, _ = check(orc, cv, base, span)
    check(orc, cv, base, span, flags=8)
    if exp.rc == 0:
        rc, got, shadow, _ = run_gpu(cv, base, span, flush_points=_cuts(cv, 4, seed))
        assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


def test_devices_hot_word(orc):
    """A hot word on 3 accelerators: K5 time slices with 8-output selector functions
    (writes on different devices, transfers to and from each device between them)."""
    from gen.trace import MAP, OP, TraceBuilder, encode_np
    A = 0x8000
    tb = TraceBuilder()
    tb.wh(A)
    rs = np.random.default_rng(8)
    for j in range(12):
        d = j % 3
        tb.enter(MAP.TO | (d << 6), A, 64)
        ops = rs.choice([OP.RT, OP.WT, OP.RH, OP.WH], size=40000, p=[.4, .2, .3, .1])
        dev = np.where((ops == OP.RT) | (ops == OP.WT), rs.integers(0, 3, ops.size), 0)
        tb.add_array(encode_np(0, np.full(ops.size, A, dtype=np.uint64), 8) |
                     np.stack([(ops.astype(np.uint64) << np.uint64(48)) | (dev.astype(np.uint64) << np.uint64(56)),
                               np.zeros(ops.size, np.uint64)], axis=1))
        tb.exit(MAP.FROM | (d << 6), A, 64)
    rec = tb.array()
    exp, st = check(orc, rec, A, 64, flags=2 << 8)
    assert st["hot_buckets"] >= 1
    check(orc, rec, A, 64, flags=(2 << 8) | 4)


@pytest.mark.parametrize("seed", range(12))
def test_runs_fuzz(orc, seed):
    """Run-form chunks and run steps: loops mostly over consecutive
    words, bucket sizes that put bucket boundaries inside runs, the BO and UM
    instances, flush cuts (tasks included)."""
    from gen.fuzz import run_program
    rec, base, span = run_program(2000 + seed)
    flags = [0, 8, 16][seed % 3]
    runs = 0
    for bb in (0, 9, 12):
        exp, st = check(orc, rec, base, span, bucket_bits=bb, flags=flags)
        runs += st["steps_run"]
    assert runs > 0
    cuts = sorted(int(x) for x in np.random.default_rng(seed).choice(rec.shape[0], 3, replace=False))
    rc, got, shadow, st = run_gpu(rec, base, span, flags=flags, bucket_bits=9, flush_points=cuts)
    assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


@pytest.mark.parametrize("seed", [3000, 3001, 3002, 3004, 3005, 3006])   # well-formed programs (rc 0)
def test_runs_fuzz_large(orc, seed):
    """Traces of more chunks than the partition has warps, so that runs continue
    from a warp's chunk into its next one (one entry per run), with
    range ops, tasks and flush cuts; the BO and UM instances."""
    from gen.fuzz import run_program
    rec, base, span = run_program(seed, n_arrays=8, array_words=1 << 16, steps=500, loop_max=40000)
    assert rec.shape[0] > 2 * 148 * 16 * 256 and orc.replay(rec, base, span).rc == 0
    flags = [0, 8, 16][seed % 3]
    for bb in (0, 12, 15):
        exp, st = check(orc, rec, base, span, bucket_bits=bb, flags=flags)
        # automatic buckets are narrower than the runs here; 2^15-word buckets are few
        # and heavy, so they are replayed as K5 time slices (event steps)
        assert st["steps_run"] > 0 or bb != 12
    cuts = sorted(int(x) for x in np.random.default_rng(seed).choice(rec.shape[0], 4, replace=False))
    rc, got, shadow, st = run_gpu(rec, base, span, flags=flags, flush_points=cuts)
    assert rc == 0 and sorted(got) == exp.triples() and np.array_equal(shadow, exp.shadow)


@pytest.mark.parametrize("bb", [0, 9, 12])
def test_runs_across_4gib_address_blocks(orc, bb):
    """Runs whose words straddle a 2^32-byte address boundary (the partition's fast
    decode takes word differences from the low 32 address bits of record 0's block or
    a neighbouring one), with map / update range ops and sub-word accesses mixed in."""
    from gen.trace import MAP, OP, UPD, TraceBuilder, encode_np
    base = (1 << 32) - 3000 * 8                       # 3000 words below the boundary
    n_words = 8192
    tb = TraceBuilder()
    rs = np.random.default_rng(bb)
    tb.enter(MAP.TOFROM, base, n_words * 8)
    for k in range(40):
        lo = int(rs.integers(0, n_words - 1200))
        ln = int(rs.integers(1, 1200))
        op = int(rs.choice([OP.RH, OP.WH, OP.RT, OP.WT]))
        size = 8 if k % 5 else 4
        tb.add_array(encode_np(op, base + 8 * (lo + np.arange(ln, dtype=np.uint64)), size))
        if k % 7 == 3:
            tb.update(int(rs.choice([UPD.TO, UPD.FROM])), base, n_words * 8)
    tb.exit(MAP.TOFROM, base, n_words * 8)
    rec = tb.array()
    check(orc, rec, base, n_words * 8, bucket_bits=bb)
