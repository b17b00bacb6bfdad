"""Brute-force pins: oracle vs the Definition-1 value simulator (tests/valuesim.py).

SURVEY §4 / §8(c): every record sequence of bounded length over the access +
map + update alphabet, on 1-word and 2-word arrays (sections [0,1), [1,2),
[0,2)), must give the same UUM/USD reports and the same final per-word state
(Table II bits P:330-333) as the value-level simulator, which knows nothing
about the state machine and implements Table I's reference counting on its own.
"""
import itertools

import numpy as np
import pytest

from gen.trace import MAP, OP, UPD, encode
from valuesim import MapError, ValueSim

ACC = [OP.RH, OP.WH, OP.RT, OP.WT]
ENTER_T = [MAP.TO, MAP.FROM, MAP.TOFROM, MAP.ALLOC]
EXIT_T = [MAP.TO, MAP.FROM, MAP.TOFROM, MAP.ALLOC, MAP.RELEASE, MAP.DELETE]


def alphabet(nwords):
    sections = [(0, 1)] if nwords == 1 else [(0, 1), (1, 2), (0, 2)]
    sym = []
    for op in ACC:
        for w in range(nwords):
            sym.append(("acc", op, w * 8, 8))
    for lo, hi in sections:
        for t in ENTER_T:
            sym.append(("ctl", OP.MAP_ENTER, lo * 8, (hi - lo) * 8, t))
        for t in EXIT_T:
            sym.append(("ctl", OP.MAP_EXIT, lo * 8, (hi - lo) * 8, t))
        for d in (UPD.TO, UPD.FROM):
            sym.append(("ctl", OP.UPDATE, lo * 8, (hi - lo) * 8, d))
    return sym


def encode_seq(seq, base):
    out = []
    for s in seq:
        if s[0] == "acc":
            out.append(encode(s[1], base + s[2], s[3]))
        else:
            out.append(encode(s[1], base + s[2], s[3], arg=s[4]))
    return out


def check_batch(orc, seqs, nwords, bo=False, unified=False):
    """Concatenate the sequences on disjoint arrays, run the oracle once, compare per array.
    bo: the buffer-overflow extension on both sides (reading Z20)."""
    stride = 8 * nwords
    recs, expect, states, offsets = [], [], [], []
    for j, seq in enumerate(seqs):
        base = stride * j
        enc = encode_seq(seq, base)
        vs = ValueSim(bo=bo, unified=unified)
        try:
            issues = vs.run(enc)
        except MapError:
            continue
        off = len(recs)
        offsets.append(off)
        recs.extend(enc)
        expect.extend((w, i + off, k) for (w, i, k) in issues)
        states.extend(vs.state_bits(base // 8 + w) for w in range(nwords))
    arr = np.array(recs, dtype=np.uint64).reshape(-1, 2)
    nseq = len(offsets)
    res = orc.replay(arr, 0, stride * (len(seqs)), detect_bo=bo, unified=unified)
    assert res.rc == 0
    assert res.triples() == sorted(expect)
    # final states: only the arrays that were kept
    got = []
    kept = 0
    for j, seq in enumerate(seqs):
        try:
            ValueSim().run(encode_seq(seq, stride * j))
        except MapError:
            continue
        got.extend(int(res.shadow[(stride * j) // 8 + w]) for w in range(nwords))
        kept += 1
    assert got == states
    assert res.stats["transitions"] == res.stats["word_events"]
    return nseq


def test_one_word_exhaustive(orc):
    sym = alphabet(1)
    seqs = [s for L in range(1, 5) for s in itertools.product(sym, repeat=L)]
    assert check_batch(orc, seqs, 1) > 60000


def test_one_word_random_long(orc):
    sym = alphabet(1)
    rs = np.random.default_rng(11)
    seqs = [tuple(sym[i] for i in rs.integers(0, len(sym), rs.integers(5, 9))) for _ in range(40000)]
    check_batch(orc, seqs, 1)


def test_two_words_exhaustive(orc):
    sym = alphabet(2)
    seqs = [s for L in range(1, 4) for s in itertools.product(sym, repeat=L)]
    assert check_batch(orc, seqs, 2) > 50000


def test_two_words_random_long(orc):
    sym = alphabet(2)
    rs = np.random.default_rng(12)
    seqs = [tuple(sym[i] for i in rs.integers(0, len(sym), rs.integers(4, 8))) for _ in range(40000)]
    check_batch(orc, seqs, 2)


@pytest.mark.parametrize("alpha", ["plain", "modifiers"])
def test_emap_agrees(orc, alpha):
    """Sequences the independent refcount model rejects (partial overlaps; with the
    modifiers also `present` on an unmapped section) are rejected by the oracle (ARB_EMAP)."""
    sym = alphabet(2) if alpha == "plain" else alphabet_always(2)
    n_bad = 0
    for seq in itertools.product(sym, repeat=2):
        enc = encode_seq(seq, 0)
        try:
            ValueSim().run(enc)
            bad = False
        except MapError:
            bad = True
        rc = orc.replay(np.array(enc, dtype=np.uint64).reshape(-1, 2), 0, 16).rc
        assert (rc == -4) == bad
        n_bad += bad
    assert n_bad > 0


def test_one_word_len6_reduced(orc):
    """Length <= 6 (north_star) over a 10-symbol alphabet: accesses, enter to/alloc,
    exit from/release, update to/from."""
    full = alphabet(1)
    keep = [s for s in full if s[0] == "acc" or
            (s[1] == OP.MAP_ENTER and s[4] in (MAP.TO, MAP.ALLOC)) or
            (s[1] == OP.MAP_EXIT and s[4] in (MAP.FROM, MAP.RELEASE)) or s[1] == OP.UPDATE]
    assert len(keep) == 10
    seqs = list(itertools.product(keep, repeat=6))
    for k in range(0, len(seqs), 250000):
        check_batch(orc, seqs[k:k + 250000], 1)


@pytest.mark.parametrize("nwords,length", [(1, 4), (2, 3)])
def test_bo_exhaustive(orc, nwords, length):
    """Buffer-overflow extension (Z20): the oracle's CVp bit and BO
    reports equal the value simulator's CV existence on every sequence (target
    accesses before any map, after release/delete, outside a 1-word section of
    a 2-word array), together with the UUM/USD reports and final states."""
    sym = alphabet(nwords)
    seqs = [s for L in range(1, length + 1) for s in itertools.product(sym, repeat=L)]
    assert check_batch(orc, seqs, nwords, bo=True) > 50000


def test_bo_random_long(orc):
    sym = alphabet(2)
    rs = np.random.default_rng(13)
    seqs = [tuple(sym[i] for i in rs.integers(0, len(sym), rs.integers(4, 9))) for _ in range(40000)]
    check_batch(orc, seqs, 2, bo=True)


def alphabet_always(nwords):
    """alphabet() plus the `always` map-type modifier on to/tofrom entries and
    from/tofrom exits (OpenMP 5.1, reading Z21)."""
    sym = alphabet(nwords)
    sections = [(0, 1)] if nwords == 1 else [(0, 1), (1, 2), (0, 2)]
    for lo, hi in sections:
        for t in (MAP.TO, MAP.TOFROM):
            sym.append(("ctl", OP.MAP_ENTER, lo * 8, (hi - lo) * 8, t | MAP.ALWAYS))
        for t in (MAP.FROM, MAP.TOFROM):
            sym.append(("ctl", OP.MAP_EXIT, lo * 8, (hi - lo) * 8, t | MAP.ALWAYS))
        sym.append(("ctl", OP.MAP_ENTER, lo * 8, (hi - lo) * 8, MAP.TO | MAP.PRESENT))
    return sym


@pytest.mark.parametrize("nwords,length", [(1, 4), (2, 3)])
def test_always_exhaustive(orc, nwords, length):
    """The `always` modifier: the oracle's reports and final states equal the value
    simulator's (its own Table I + `always` reference-count model) on every sequence."""
    sym = alphabet_always(nwords)
    seqs = [s for L in range(1, length + 1) for s in itertools.product(sym, repeat=L)]
    assert check_batch(orc, seqs, nwords) > 50000


def test_always_random_long(orc):
    sym = alphabet_always(2)
    rs = np.random.default_rng(14)
    seqs = [tuple(sym[i] for i in rs.integers(0, len(sym), rs.integers(4, 9))) for _ in range(40000)]
    check_batch(orc, seqs, 2)


@pytest.mark.parametrize("nwords,length", [(1, 4), (2, 3)])
def test_unified_exhaustive(orc, nwords, length):
    """Unified memory (reading Z23): the oracle's reports and final
    states equal the value simulator's with OV and CV aliased (one storage; only
    never-written words can be read wrongly — no stale copies exist)."""
    sym = alphabet_always(nwords)
    seqs = [s for L in range(1, length + 1) for s in itertools.product(sym, repeat=L)]
    assert check_batch(orc, seqs, nwords, unified=True) > 50000


def alphabet_devices(ndev):
    """One word, several accelerators (reading Z24): host accesses, target
    accesses and map / update clauses on every device (device in the access arg,
    in bits 6-7 of a map / update arg)."""
    sym = [("acc", OP.RH, 0, 8), ("acc", OP.WH, 0, 8)]
    for d in range(ndev):
        sym += [("accd", OP.RT, d), ("accd", OP.WT, d)]
        for t in (MAP.TO, MAP.FROM, MAP.TOFROM, MAP.ALLOC):
            sym.append(("ctl", OP.MAP_ENTER, 0, 8, t | (d << 6)))
        for t in (MAP.FROM, MAP.TOFROM, MAP.RELEASE):
            sym.append(("ctl", OP.MAP_EXIT, 0, 8, t | (d << 6)))
        for u in (UPD.TO, UPD.FROM):
            sym.append(("ctl", OP.UPDATE, 0, 8, u | (d << 6)))
    return sym


def _enc_dev(seq, base):
    out = []
    for s in seq:
        if s[0] == "accd":
            out.append(encode(s[1], base, 8, arg=s[2]))
        elif s[0] == "acc":
            out.append(encode(s[1], base + s[2], s[3]))
        else:
            out.append(encode(s[1], base + s[2], s[3], arg=s[4]))
    return out


@pytest.mark.parametrize("ndev,length", [(2, 4), (3, 3)])
def test_devices_exhaustive(orc, ndev, length):
    """Several accelerators: the oracle's (n+1)-tuple states and reports equal the
    value simulator's with one CV and one mapping table per device."""
    sym = alphabet_devices(ndev)
    recs, expect, states, n = [], [], [], 0
    for L in range(1, length + 1):
        for j, seq in enumerate(itertools.product(sym, repeat=L)):
            base = 8 * n
            enc = _enc_dev(seq, base)
            vs = ValueSim(devices=ndev)
            try:
                issues = vs.run(enc)
            except MapError:
                continue
            off = len(recs)
            recs.extend(enc)
            expect.extend((w, i + off, k) for (w, i, k) in issues)
            states.append(vs.state_bits(base // 8))
            n += 1
    res = orc.replay(np.array(recs, dtype=np.uint64).reshape(-1, 2), 0, 8 * n, n_devices=ndev)
    assert res.rc == 0
    assert res.triples() == sorted(expect)
    assert res.shadow.tolist() == states
    assert n > 20000
    # a single-device run of device-0-only sequences is the plain oracle
    one = [s for s in sym if not (s[0] == "accd" and s[2]) and not (s[0] == "ctl" and s[4] >> 6)]
    enc = _enc_dev(one, 0)
    assert orc.replay(np.array(enc, dtype=np.uint64).reshape(-1, 2), 0, 8, n_devices=ndev).triples() == \
        orc.replay(np.array(enc, dtype=np.uint64).reshape(-1, 2), 0, 8).triples()


# ---- buffer overflow through a tagged pointer (reading Z25) ---------------------
BASE_OP = 11     # ORC_BASE / ARB_BASE: pointer tag (task-id field) -> base byte address


def alphabet_tags():
    """Two adjacent 1-word variables A (word 0) and B (word 1) of one 2-word region:
    target accesses through pointer tag a (0), b (1) or none (None), host accesses,
    entering / exiting either variable, and defining the tags' bases (also the
    wrong one: tag a -> B)."""
    sym = []
    for op in (OP.RT, OP.WT):
        for w in (0, 1):
            for t in (None, 0, 1):
                sym.append(("acc", op, w * 8, 8, t))
    for op in (OP.RH, OP.WH):
        for w in (0, 1):
            sym.append(("acc", op, w * 8, 8, None))
    for w in (0, 1):
        for t in (MAP.TO, MAP.ALLOC):
            sym.append(("ctl", OP.MAP_ENTER, w * 8, 8, t))
        for t in (MAP.FROM, MAP.RELEASE):
            sym.append(("ctl", OP.MAP_EXIT, w * 8, 8, t))
    sym += [("base", 0, 0), ("base", 1, 8), ("base", 0, 8)]
    return sym


def encode_tagged(seq, base, tag0):
    """Sequence j uses the pointer tags tag0 + 0 / + 1 (tags are global to the trace)."""
    out = []
    for s in seq:
        if s[0] == "acc":
            t = 0 if s[4] is None else tag0 + s[4]
            out.append(encode(s[1], base + s[2], s[3], task=t))
        elif s[0] == "base":
            out.append(encode(BASE_OP, base + s[2], 0, task=tag0 + s[1]))
        else:
            out.append(encode(s[1], base + s[2], s[3], arg=s[4]))
    return out


def check_tagged(orc, seqs):
    recs, expect, states = [], [], []
    for j, seq in enumerate(seqs):
        base = 16 * j
        enc = encode_tagged(seq, base, 1 + 2 * j)
        vs = ValueSim(bo=True)
        issues = vs.run(enc)
        off = len(recs)
        recs.extend(enc)
        expect.extend((w, i + off, k) for (w, i, k) in issues)
        states.extend(vs.state_bits(base // 8 + w) for w in range(2))
    arr = np.array(recs, dtype=np.uint64).reshape(-1, 2)
    res = orc.replay(arr, 0, 16 * len(seqs), detect_bo=True)
    assert res.rc == 0
    assert res.triples() == sorted(expect)
    assert [int(x) for x in res.shadow[:2 * len(seqs)]] == states
    return len(seqs)


def test_bo_base_tags_exhaustive(orc):
    """Z25 against the value simulator, which gives every mapping entry its own CV
    and asks whether a tagged access reached the CV of its pointer's base: every
    sequence of length <= 3 over the alphabet above (in chunks: tags are 16-bit)."""
    sym = alphabet_tags()
    seqs = [s for L in range(1, 4) for s in itertools.product(sym, repeat=L)]
    n = 0
    for k in range(0, len(seqs), 30000):
        n += check_tagged(orc, seqs[k:k + 30000])
    assert n > 20000


def test_bo_base_tags_random_long(orc):
    sym = alphabet_tags()
    rs = np.random.default_rng(14)
    seqs = [tuple(sym[i] for i in rs.integers(0, len(sym), rs.integers(4, 10))) for _ in range(30000)]
    check_tagged(orc, seqs)


def test_bo_base_tags_off_without_extension(orc):
    """Without detect_bo the tags and ARB_BASE records change nothing (plain VSM)."""
    sym = alphabet_tags()
    rs = np.random.default_rng(15)
    for _ in range(300):
        seq = tuple(sym[i] for i in rs.integers(0, len(sym), 8))
        tagged = np.array(encode_tagged(seq, 0, 1), dtype=np.uint64).reshape(-1, 2)
        plain_seq = [s[:4] + (None,) if s[0] == "acc" else s for s in seq if s[0] != "base"]
        plain = np.array(encode_tagged(plain_seq, 0, 1), dtype=np.uint64).reshape(-1, 2)
        a, b = orc.replay(tagged, 0, 16), orc.replay(plain, 0, 16)
        assert a.rc == b.rc == 0
        # same reports up to the index shift of the removed ARB_BASE records
        keep = [i for i, s in enumerate(seq) if s[0] != "base"]
        assert [(w, keep[r], k) for w, r, k in b.triples()] == a.triples()
        assert np.array_equal(a.shadow, b.shadow)


@pytest.mark.parametrize("seed", range(12))
def test_bo_base_tags_fuzz_programs(orc, seed):
    """Random offload programs with pointer tags (gen/fuzz.py p_tag): the oracle's
    UUM/USD/BO reports equal the value simulator's (MIR is not a value-level issue)."""
    from gen.fuzz import random_program
    rec, base, span = random_program(9000 + seed, p_tag=0.6, p_task=0.2)
    try:
        expect = sorted(ValueSim(bo=True).run(rec))
    except MapError:
        pytest.skip("program rejected by the refcount model")
    res = orc.replay(rec, base, span, detect_bo=True)
    assert res.rc == 0
    assert [t for t in res.triples() if t[2] != 3] == expect


# ---- CV -> OV translation (P:269 interval tree, reading Z26) --------------------------------
CV_BASE_OP, CV_ADDR = 16, 0x80


def alphabet_cv():
    """Two words A (0) and B (1): target accesses by OV address or by CV address
    (the CV of the entry holding the word, or a stray one), host accesses, entering
    / exiting A, B or both, and the runtime's CV placement records (CV_BASE) --
    including a wrong one (B's CV placed where A's is)."""
    sym = []
    for op in (OP.RT, OP.WT):
        for w in (0, 1):
            sym.append(("acc", op, w * 8, 8, 0))
        for c in (0, 8, 16):                              # CV byte offsets (16: past both)
            sym.append(("cva", op, c, 8, CV_ADDR))
    for op in (OP.RH, OP.WH):
        for w in (0, 1):
            sym.append(("acc", op, w * 8, 8, 0))
    for lo, hi in ((0, 1), (1, 2), (0, 2)):
        for t in (MAP.TO, MAP.ALLOC):
            sym.append(("ctl", OP.MAP_ENTER, lo * 8, (hi - lo) * 8, t))
        for t in (MAP.FROM, MAP.RELEASE):
            sym.append(("ctl", OP.MAP_EXIT, lo * 8, (hi - lo) * 8, t))
    sym += [("cvb", 0, 0), ("cvb", 8, 8), ("cvb", 8, 0)]  # OV byte -> CV offset
    return sym


def encode_cv(seq, base, cvbase):
    out = []
    for s in seq:
        if s[0] == "acc":
            out.append(encode(s[1], base + s[2], s[3]))
        elif s[0] == "cva":
            out.append(encode(s[1], cvbase + s[2], s[3], arg=s[4]))
        elif s[0] == "cvb":
            out.append(encode(CV_BASE_OP, base + s[1], cvbase + s[2]))
        else:
            out.append(encode(s[1], base + s[2], s[3], arg=s[4]))
    return out


def check_cv(orc, seqs, bo):
    recs, expect, states = [], [], []
    for j, seq in enumerate(seqs):
        base, cvbase = 16 * j, (1 << 40) + 64 * j
        enc = encode_cv(seq, base, cvbase)
        vs = ValueSim(bo=bo)
        try:
            issues = vs.run(enc)
        except MapError:
            continue
        off = len(recs)
        recs.extend(enc)
        expect.extend((w, i + off, k) for (w, i, k) in issues)
        states.extend(vs.state_bits(base // 8 + w) for w in range(2))
    arr = np.array(recs, dtype=np.uint64).reshape(-1, 2)
    res = orc.replay(arr, 0, 16 * len(seqs), detect_bo=bo)
    assert res.rc == 0
    assert res.triples() == sorted(expect)
    return len(states) // 2


@pytest.mark.parametrize("bo", [False, True])
def test_cv_translation_exhaustive(orc, bo):
    """Z26 against the value simulator, which keeps its own CV-address table per entry
    and translates a device address through it: every sequence of length <= 3."""
    sym = alphabet_cv()
    seqs = [s for L in range(1, 4) for s in itertools.product(sym, repeat=L)]
    n = 0
    for k in range(0, len(seqs), 40000):
        n += check_cv(orc, seqs[k:k + 40000], bo)
    assert n > 20000


@pytest.mark.parametrize("bo", [False, True])
def test_cv_translation_random_long(orc, bo):
    sym = alphabet_cv()
    rs = np.random.default_rng(16 + bo)
    seqs = [tuple(sym[i] for i in rs.integers(0, len(sym), rs.integers(4, 10))) for _ in range(30000)]
    check_cv(orc, seqs, bo)


def test_cv_translation_equals_ov_addressing(orc):
    """A trace whose target accesses to mapped words use CV addresses, with every CV
    placed by a CV_BASE record, replays exactly like the same trace with OV
    addresses (a target access to an unmapped word keeps its OV address: its CV
    address would be in no CV, Z26)."""
    from gen.fuzz import random_program
    for seed in range(6):
        rec, base, span = random_program(9300 + seed, p_task=0.3)
        op = (rec[:, 0] >> np.uint64(48)) & np.uint64(0xFF)
        addr = rec[:, 0] & np.uint64((1 << 48) - 1)
        cv_off = np.uint64(1 << 44)                      # every CV at OV + 2^44
        tracker = ValueSim()                             # which words are mapped, record by record
        out = []
        for i in range(rec.shape[0]):
            w0, w1 = int(rec[i, 0]), int(rec[i, 1])
            mapped = op[i] in (OP.RT, OP.WT) and tracker._entry_of(int(addr[i])) is not None
            try:
                tracker.record(int(op[i]), int(addr[i]), w1 & ((1 << 48) - 1), w0 >> 56, i)
            except MapError:
                pass
            if mapped:
                w0 = (w0 & ~((1 << 48) - 1) & ~(0xFF << 56)) | int(addr[i] + cv_off) | ((CV_ADDR | (w0 >> 56)) << 56)
            out.append((w0, w1))
            if op[i] == OP.MAP_ENTER:                    # the runtime reports where the CV went
                out.append(encode(CV_BASE_OP, int(addr[i]), int(addr[i] + cv_off)))
        cv = np.array(out, dtype=np.uint64)
        a = orc.replay(rec, base, span)
        b = orc.replay(cv, base, span)
        assert a.rc == b.rc
        if a.rc != 0:
            continue
        # same reports, record indices shifted by the inserted CV_BASE records
        keep = [j for j, (w0, _) in enumerate(out) if ((w0 >> 48) & 0xFF) != CV_BASE_OP]
        assert [(w, keep[r], k) for w, r, k in a.triples()] == b.triples()
        assert np.array_equal(a.shadow, b.shadow)
