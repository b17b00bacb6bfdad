"""Pins of the oracle against the paper's worked examples and special cases.

Each test names the passage it follows.  None of the expected values comes
from the CUDA path; they are the paper's (cited) or derived by hand from
Definition 1 / Table I and cross-checked with the independent value simulator.
"""
import numpy as np
import pytest

from gen.trace import MAP, OP, UPD, TraceBuilder
from golden_io import load
from valuesim import ValueSim

UUM, USD, MIR = 1, 2, 3


def run(orc, rec, base, size, **kw):
    res = orc.replay(rec, base, size, **kw)
    assert res.rc == 0, res.rc
    return res


@pytest.mark.parametrize("name", ["fig1_n3.trace", "fig2_no_sync.trace", "fig2_sync.trace"])
def test_golden_trace(orc, name):
    rec, base, size, expect = load(name)
    res = run(orc, rec, base, size)
    assert res.triples() == expect
    # the UUM/USD part must agree with Definition 1 evaluated on values
    vs = ValueSim().run(rec)
    assert sorted(vs) == sorted(t for t in expect if t[2] != MIR)
    assert res.stats["transitions"] == res.stats["word_events"]


def test_fig2_paper_lines(orc):
    """'There are two data mapping issues residing in lines 5 and 16'; line 5 is USD."""
    rec, base, size, _ = load("fig2_no_sync.trace")
    res = run(orc, rec, base, size)
    by_rec = {}
    for w, r, k in res.triples():
        by_rec.setdefault(r, set()).add(k)
    assert by_rec[5] == {USD}            # line 5: use of stale data
    assert MIR in by_rec[13]             # line 16: nondeterministic (race with the nowait region)
    assert MIR in by_rec[12]             # line 14 exit transfer "may conflict"
    # the fix of P:163 removes every race
    rec2, base2, size2, _ = load("fig2_sync.trace")
    assert all(k != MIR for _, _, k in run(orc, rec2, base2, size2).triples())


def test_config1_tiny(orc):
    """BASELINE config 1 (Fig. 2 lines 1-5 scaled): exactly 1,024 USD at the host reads."""
    from gen.configs import config1
    rec, base, size = config1()
    assert rec.shape[0] == 4098
    res = run(orc, rec, base, size)
    t = res.triples()
    assert len(t) == 1024
    assert all(k == USD for _, _, k in t)
    assert [r for _, r, _ in t] == list(range(3074, 4098))
    assert [w for w, _, _ in t] == list(range(base // 8, base // 8 + 1024))
    assert res.stats["word_events"] == 7168 == res.stats["transitions"]
    # final state: OV invalid but initialised, CV released (Table II bits: OVi only)
    assert set(res.shadow.tolist()) == {0b0100}


def test_initial_state_invalid(orc):
    """tuples start invalid; a read of a never-written word is a UUM."""
    tb = TraceBuilder()
    tb.rh(0x100)
    tb.rt(0x108)
    res = run(orc, tb.array(), 0x100, 16)
    assert res.triples() == [(0x20, 0, UUM), (0x21, 1, UUM)]


def test_prose_edges(orc):
    """Every edge the prose states, observed through reads of each side."""
    A = 0x1000

    def state_after(build):
        tb = TraceBuilder()
        build(tb)
        return run(orc, tb.array(), A, 8).shadow[0] & 3  # (OVv, CVv)

    H, T, C, I = 1, 2, 3, 0
    # invalid --write_host--> host ; invalid --write_target--> target
    assert state_after(lambda t: t.wh(A)) == H
    assert state_after(lambda t: (t.enter(MAP.ALLOC, A, 8), t.wt(A))) == T
    # host --update_target--> consistent ; host --write_target--> target
    assert state_after(lambda t: (t.wh(A), t.enter(MAP.TO, A, 8))) == C
    assert state_after(lambda t: (t.wh(A), t.enter(MAP.ALLOC, A, 8), t.wt(A))) == T
    # host --update_host--> invalid (OV overwritten by the invalid CV value)
    assert state_after(lambda t: (t.wh(A), t.enter(MAP.ALLOC, A, 8), t.update(UPD.FROM, A, 8))) == I
    # target --update_host--> consistent ; target --update_target--> invalid ; target --release--> invalid
    base_t = lambda t: (t.enter(MAP.ALLOC, A, 8), t.wt(A))
    assert state_after(lambda t: (base_t(t), t.update(UPD.FROM, A, 8))) == C
    assert state_after(lambda t: (base_t(t), t.update(UPD.TO, A, 8))) == I
    assert state_after(lambda t: (base_t(t), t.exit(MAP.RELEASE, A, 8))) == I
    # consistent --write_host--> host ; consistent --write_target--> target
    assert state_after(lambda t: (t.wh(A), t.enter(MAP.TO, A, 8), t.wh(A))) == H
    assert state_after(lambda t: (t.wh(A), t.enter(MAP.TO, A, 8), t.wt(A))) == T
    # faults: read_target in host, read_host in target, no fault in consistent
    tb = TraceBuilder(); tb.wh(A); tb.enter(MAP.ALLOC, A, 8); tb.rt(A); tb.rh(A)
    assert run(orc, tb.array(), A, 8).triples() == [(A // 8, 2, UUM)]
    tb = TraceBuilder(); tb.wh(A); tb.enter(MAP.TO, A, 8); tb.wt(A); tb.rh(A); tb.rt(A)
    assert run(orc, tb.array(), A, 8).triples() == [(A // 8, 3, USD)]


def test_granularity_8_bytes(orc):
    """8-byte granularity; an unaligned access touches two words (Z4)."""
    tb = TraceBuilder()
    tb.rh(0x1004, 8)      # words 0x200 and 0x201
    tb.wh(0x1000, 2)      # validates all of word 0x200
    tb.rh(0x1006, 2)
    res = run(orc, tb.array(), 0x1000, 16)
    assert res.triples() == [(0x200, 0, UUM), (0x201, 0, UUM)]
    assert res.stats["word_events"] == 4


def test_table1_nested_refcount(orc):
    """Table I: inner `from` at ref_count 2 copies nothing; the outer exit copies (tofrom)."""
    A = 0x2000
    tb = TraceBuilder()
    tb.wh(A)
    tb.enter(MAP.TOFROM, A, 8)      # rc 1: new + memcpy(CV, OV)
    tb.enter(MAP.FROM, A, 8)        # rc 2: no transfer
    tb.wt(A)
    tb.exit(MAP.FROM, A, 8)         # rc 1: no transfer
    tb.rh(A)                        # 5: stale
    tb.exit(MAP.TOFROM, A, 8)       # rc 0: memcpy(OV, CV), delete
    tb.rh(A)                        # 7: fine
    res = run(orc, tb.array(), A, 8)
    assert res.triples() == [(A // 8, 5, USD)]


def test_table1_release_vs_delete(orc):
    """Table I: `release` decrements (no delete at rc>0); `delete` forces rc=0 and deletes."""
    A = 0x2000
    for mt, expect in ((MAP.RELEASE, []), (MAP.DELETE, [(A // 8, 5, USD)])):
        tb = TraceBuilder()
        tb.wh(A)
        tb.enter(MAP.TO, A, 8)
        tb.enter(MAP.TO, A, 8)       # rc 2
        tb.exit(mt, A, 8)            # release: rc 1 ; delete: rc 0 -> CV deleted
        tb.wt(A)                     # release: present CV written; delete: a write to an unmapped CV
        tb.rt(A)                     # 5: release -> valid ; delete -> still valid (written by WT)
        res = run(orc, tb.array(), A, 8)
        assert res.triples() == [], mt
        # after delete a fresh map(alloc) gives an uninitialised CV
        tb.enter(MAP.ALLOC, A, 8)
        tb.rt(A)
        res = run(orc, tb.array(), A, 8)
        if mt == MAP.DELETE:
            assert res.triples() == [(A // 8, 7, UUM)]
        else:
            assert res.triples() == []   # still present (rc 2): no new CV, no transfer


def test_update_not_present_is_noop(orc):
    """Z7 (OpenMP 5.1): target update / exit of a non-present item does nothing."""
    A = 0x2000
    tb = TraceBuilder()
    tb.wh(A)
    tb.update(UPD.FROM, A, 8)
    tb.exit(MAP.FROM, A, 8)
    tb.rh(A)
    res = run(orc, tb.array(), A, 8)
    assert res.triples() == []
    assert res.stats["word_events"] == 2


def test_section_subset_reuses_entry(orc):
    """Z6: a subset section reuses the containing entry (rc+1, no transfer)."""
    A = 0x3000
    tb = TraceBuilder()
    tb.wh(A); tb.wh(A + 8)
    tb.enter(MAP.ALLOC, A, 16)       # entry [A, A+16), uninitialised CV
    tb.enter(MAP.TO, A + 8, 8)       # present: rc 2, no memcpy
    tb.rt(A + 8)                     # 4: UUM — the `to` did not transfer
    tb.exit(MAP.FROM, A + 8, 8)      # rc 1
    tb.exit(MAP.RELEASE, A, 16)      # rc 0: delete
    res = run(orc, tb.array(), A, 16)
    assert res.triples() == [((A + 8) // 8, 4, UUM)]


def test_partial_overlap_is_emap(orc):
    A = 0x3000
    tb = TraceBuilder()
    tb.enter(MAP.TO, A, 16)
    tb.enter(MAP.TO, A + 8, 16)
    assert orc.replay(tb.array(), A, 64).rc == -4


@pytest.mark.parametrize("bad", ["nested_task", "end_mismatch", "access_len", "bad_op",
                                 "sync_in_task", "bad_enter_type"])
def test_etrace(orc, bad):
    tb = TraceBuilder()
    if bad == "nested_task":
        tb.task_begin(1); tb.task_begin(2)
    elif bad == "end_mismatch":
        tb.task_begin(1); tb.task_end(2)
    elif bad == "access_len":
        tb.rh(0x1000, 9)
    elif bad == "bad_op":
        tb._add(5, 0x1000, 8)
    elif bad == "sync_in_task":
        tb.task_begin(1); tb.sync(1)
    elif bad == "bad_enter_type":
        tb.enter(MAP.DELETE, 0x1000, 8)
    assert orc.replay(tb.array(), 0x1000, 64).rc == -5


def test_eopen(orc):
    tb = TraceBuilder()
    tb.task_begin(1); tb.wt(0x1000)
    assert orc.replay(tb.array(), 0x1000, 64).rc == -7


def test_postencil_pointer_swap(orc):
    """503.postencil: pointer swap with a `to`-mapped partner and an odd
    iteration count (3) leaves the output stale (USD at the host reads); an even count
    or `tofrom` on both is clean."""
    from gen.patterns import p10
    n, esz = 64, 4
    for buggy, expect_usd in ((True, True), (False, False)):
        tb = TraceBuilder()
        p10(tb, 0x10000, n, esz, buggy, 1)
        res = run(orc, tb.array(), 0x10000, 2 * n * esz)
        kinds = {k for _, _, k in res.triples()}
        assert kinds == ({USD} if expect_usd else set())
        if expect_usd:
            # every host read of the output array is stale (size-4 reads)
            assert len(res.triples()) == n  # one report per read record (two per word)
    # tofrom on both arrays: clean for any count
    tb = TraceBuilder()
    x, y = 0x10000, 0x10000 + n * esz
    tb.loop([(OP.WH, x)], n, esz); tb.loop([(OP.WH, y)], n, esz)
    tb.enter(MAP.TOFROM, x, n * esz); tb.enter(MAP.TOFROM, y, n * esz)
    src, dst = x, y
    for _ in range(3):
        tb.loop([(OP.RT, src), (OP.WT, dst)], n, esz)
        src, dst = dst, src
    tb.exit(MAP.TOFROM, x, n * esz); tb.exit(MAP.TOFROM, y, n * esz)
    tb.loop([(OP.RH, src)], n, esz)
    assert run(orc, tb.array(), 0x10000, 2 * n * esz).triples() == []


def test_dedup_first_mode(orc):
    """Z3 option: first report per (word, kind) only."""
    rec, base, size, expect = load("fig2_no_sync.trace")
    res = run(orc, rec, base, size, dedup_first=True)
    assert res.triples() == [(0x200, 5, USD), (0x200, 10, MIR)]


def test_sparse_mode_matches_dense(orc):
    """Tracking a subset of words gives the dense result restricted to those words."""
    from gen.configs import config2
    rec, base, size = config2(reps=1)
    dense = run(orc, rec, base, size)
    rs = np.random.default_rng(7)
    words = np.unique(rs.integers(base // 8, (base + size) // 8, 4000)).astype(np.uint64)
    sparse = run(orc, rec, base, size, tracked_words=words)
    keep = set(words.tolist())
    assert sparse.triples() == [t for t in dense.triples() if t[0] in keep]
    assert np.array_equal(sparse.shadow, dense.shadow[(words - base // 8).astype(np.int64)])


def test_global_index(orc):
    rec, base, size, expect = load("fig2_sync.trace")
    gi = np.arange(rec.shape[0], dtype=np.uint64) * 10 + 7
    res = run(orc, rec, base, size, global_index=gi)
    assert res.triples() == [(w, r * 10 + 7, k) for w, r, k in expect]


# ---- buffer-overflow extension (reading Z20) -----------------------
BO = 4


def _half_mapped(n, write):
    """"the host program only maps the first half of an array to the
    accelerator, while the compute kernel loops through the whole array"."""
    A = 0x4000
    tb = TraceBuilder()
    tb.loop([(OP.WH, A)], n, 8)                       # host initialises a[0:n]
    tb.enter(MAP.TOFROM, A, 8 * (n // 2))             # map(tofrom: a[0:n/2])
    k0 = len(tb)
    tb.loop([(OP.WT if write else OP.RT, A)], n, 8)   # kernel: for i < n: a[i] (= or read)
    tb.exit(MAP.TOFROM, A, 8 * (n // 2))
    return tb.array(), A, k0


@pytest.mark.parametrize("write", [False, True])
def test_bo_half_mapped_array(orc, write):
    n = 64
    rec, A, k0 = _half_mapped(n, write)
    res = run(orc, rec, A, 8 * n, detect_bo=True)
    # exactly the kernel accesses of the unmapped half, nothing else
    assert res.triples() == [(A // 8 + i, k0 + i, BO) for i in range(n // 2, n)]
    assert res.stats["transitions"] == res.stats["word_events"]
    # the overflowing accesses had no effect: the unmapped half's OV still holds
    # the host values (OVv, OVi) and it never had a CV; the mapped half was copied
    # back at the tofrom exit and its CV released (CVp clear): OVv | OVi everywhere
    assert set(res.shadow.tolist()) == {0b0101}
    # without the extension the reads of the unmapped half are UUM (no CV value) and the
    # writes are silent (P:263 only checks reads)
    plain = run(orc, rec, A, 8 * n).triples()
    assert plain == ([] if write else [(A // 8 + i, k0 + i, UUM) for i in range(n // 2, n)])


def test_bo_fixed_mapping_is_clean(orc):
    """The fixed program maps the whole array: no report with or without the extension."""
    A, n = 0x4000, 64
    tb = TraceBuilder()
    tb.loop([(OP.WH, A)], n, 8)
    tb.enter(MAP.TOFROM, A, 8 * n)
    tb.loop([(OP.RT, A), (OP.WT, A)], n, 8)
    tb.exit(MAP.TOFROM, A, 8 * n)
    tb.loop([(OP.RH, A)], n, 8)
    res = run(orc, tb.array(), A, 8 * n, detect_bo=True)
    assert res.triples() == []


def test_bo_after_release_and_host_unaffected(orc):
    """A kernel access after the CV was deleted is BO; host accesses never are."""
    A = 0x4000
    tb = TraceBuilder()
    tb.wh(A)
    tb.enter(MAP.TO, A, 8)
    i_ok = tb.rt(A)
    tb.exit(MAP.DELETE, A, 8)
    i_bo = tb.rt(A)
    i_h = tb.rh(A)
    res = run(orc, tb.array(), A, 8, detect_bo=True)
    assert res.triples() == [(A // 8, i_bo, BO)]
    assert i_ok < i_bo < i_h


def test_always_modifier_nested_region(orc):
    """OpenMP 5.1 `always` (N4, Z21): inside an outer `target data map(tofrom)`, an
    inner `map(always, tofrom)` refreshes the CV on entry and the OV on exit, so the
    host read after the inner region is clean; without `always` it is stale (the
    nested-refcount case of Table I)."""
    A = 0x4000
    for always, expect_usd in ((False, True), (True, False)):
        tb = TraceBuilder()
        tb.wh(A)
        tb.enter(MAP.TOFROM, A, 8)                          # outer region: rc = 1
        tb.wh(A)                                            # host update inside the outer region
        mt = MAP.TOFROM | (MAP.ALWAYS if always else 0)
        tb.enter(mt, A, 8)                                  # inner: rc = 2 (+ copy with always)
        i_rt = tb.rt(A)
        tb.wt(A)
        tb.exit(mt, A, 8)                                   # rc = 1 (+ copy back with always)
        i_rh = tb.rh(A)
        tb.exit(MAP.TOFROM, A, 8)
        res = run(orc, tb.array(), A, 8)
        kinds = {(r, k) for _, r, k in res.triples()}
        assert ((i_rt, USD) in kinds) == expect_usd          # the kernel read sees the old CV
        assert ((i_rh, USD) in kinds) == expect_usd          # the host read misses the kernel write
        assert sorted(ValueSim().run(tb.array())) == res.triples()


def test_unified_memory_paper(orc):
    """Unified memory (reading Z23): "on-demand page migration helps
    resolve data mapping issues in a data-race-free OpenMP application" — Fig. 1's
    UUMs and Fig. 2's stale reads disappear, the synchronized Fig. 2 is clean — but
    "data mapping issues may arise when updates on the host and reads on the GPU
    occur concurrently without proper synchronization": the host accesses of lines
    13 and 16 still race with the nowait region (the exit transfer of line 14 no
    longer exists, so it no longer races)."""
    for name, expect in (("fig1_n3.trace", set()), ("fig2_sync.trace", set()),
                         ("fig2_no_sync.trace", {(10, MIR), (11, MIR), (13, MIR)})):
        rec, base, size, _ = load(name)
        res = run(orc, rec, base, size, unified=True)
        assert {(r, k) for _, r, k in res.triples()} == expect, name


def test_bo_overflow_into_adjacent_cv(orc):
    """"the host program only maps the first half of an array ... the compute
    kernel loops through the whole array ... It may retrieve a valid value from an
    adjacent memory location which happens to be another variable's CV."  Here the
    adjacent location IS mapped (variable B right after A's first half), so the
    present-bit form (Z20) sees nothing; through the kernel's pointer to A (tag 1,
    base A) every access to B's words is BO (Z25), and the accesses still
    read B's CV."""
    from gen.trace import encode
    A, n = 0x4000, 64
    B = A + 8 * (n // 2)                 # B occupies the second half of A's extent
    tb = TraceBuilder()
    tb.loop([(OP.WH, A)], n, 8)          # host initialises A's first half and B
    tb.enter(MAP.TO, A, 8 * (n // 2))    # map(to: a[0:n/2])
    tb.enter(MAP.TO, B, 8 * (n // 2))    # map(to: b[0:n/2]) -- B's CV, adjacent
    tb.add_array(np.array([encode(11, A, 0, task=1)], dtype=np.uint64))   # pointer tag 1 -> base A
    k0 = len(tb)
    for i in range(n):
        tb.add_array(np.array([encode(OP.RT, A + 8 * i, 8, task=1)], dtype=np.uint64))
    tb.exit(MAP.TO, B, 8 * (n // 2))
    tb.exit(MAP.TO, A, 8 * (n // 2))
    rec = tb.array()
    res = run(orc, rec, A, 8 * n, detect_bo=True)
    assert res.triples() == [(A // 8 + i, k0 + i, BO) for i in range(n // 2, n)]
    # the present-bit form alone (no tag) reports nothing: B's words have a CV
    untagged = rec.copy()
    untagged[k0:k0 + n, 1] &= np.uint64((1 << 48) - 1)
    assert run(orc, untagged, A, 8 * n, detect_bo=True).triples() == []
    # a correctly mapped array (one section for the whole extent) is clean
    tb2 = TraceBuilder()
    tb2.loop([(OP.WH, A)], n, 8)
    tb2.enter(MAP.TO, A, 8 * n)
    tb2.add_array(np.array([encode(11, A, 0, task=1)], dtype=np.uint64))
    for i in range(n):
        tb2.add_array(np.array([encode(OP.RT, A + 8 * i, 8, task=1)], dtype=np.uint64))
    tb2.exit(MAP.TO, A, 8 * n)
    assert run(orc, tb2.array(), A, 8 * n, detect_bo=True).triples() == []


@pytest.mark.parametrize("seed", range(6))
def test_dedup_first_is_first_per_word_kind(orc, seed):
    """Z3: dedup-first mode returns exactly the earliest raw report of every
    (word, kind) pair -- checked against the raw report list on random programs
    with tasks (MIR), unaligned accesses and map errors avoided by the generator."""
    from gen.fuzz import random_program
    rec, base, span = random_program(7700 + seed, p_task=0.4, p_depend=0.2)
    raw = run(orc, rec, base, span)
    if raw.rc != 0:
        pytest.skip("program rejected")
    first = {}
    for w, r, k in raw.triples():                    # canonical order: word, record, kind
        first.setdefault((w, k), (w, r, k))
    assert run(orc, rec, base, span, dedup_first=True).triples() == sorted(first.values())
