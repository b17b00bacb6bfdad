"""Metamorphic pins of the sub-word reading (Z4, "8-byte granularity";
Table II P:337 access sizes 1..8 bytes).

Reading Z4 says the detector tracks 8-byte words: an access of 1..8 bytes acts on
every word its byte range touches, as a whole-word access of the same op with the
same record index.  Two consequences that do not mention the state machine at
all, checked on random programs (gen/fuzz.py: tasks, modifiers, unaligned
strides) so that a mistake in the oracle's byte-range -> word expansion (a wrong
last word, a dropped second word, an off-by-one at a word edge) fails one:

1. sub-word invariance: replacing every one-word access by a random (offset,
   length) inside the same word, or by the aligned 8-byte access, changes
   neither the reports nor the final states;
2. split equivalence: an access straddling words w, w + 1 equals the aligned
   access to w followed by the aligned access to w + 1 (an inserted record),
   once the report record indices of the second trace are mapped back.
"""
import numpy as np
import pytest

from gen.fuzz import random_program

M48 = (1 << 48) - 1


def _fields(r):
    w0, w1 = int(r[0]), int(r[1])
    return w0 & M48, (w0 >> 48) & 0xFF, w1 & M48


def _with(r, addr, length):
    w0, w1 = int(r[0]), int(r[1])
    return [(w0 & ~M48) | addr, (w1 & ~M48) | length]


def _words(addr, length):
    return list(range(addr // 8, (addr + length - 1) // 8 + 1))


def _program(seed):
    rec, base, span = random_program(seed, p_task=0.3, p_depend=0.1, p_always=0.1)
    return np.asarray(rec, dtype=np.uint64), base, span


@pytest.mark.parametrize("seed", range(8))
def test_subword_invariance(orc, seed):
    rec, base, span = _program(9100 + seed)
    ref = orc.replay(rec, base, span)
    if ref.rc != 0:
        pytest.skip("program rejected")
    rs = np.random.default_rng(seed)
    aligned, jittered = [], []
    n_sub = 0
    for r in rec:
        addr, op, length = _fields(r)
        if op < 4 and len(_words(addr, length)) == 1:
            w = addr // 8
            aligned.append(_with(r, w * 8, 8))
            off = int(rs.integers(0, 8))
            ln = int(rs.integers(1, 9 - off))
            jittered.append(_with(r, w * 8 + off, ln))
            n_sub += (addr, length) != (w * 8, 8)
        else:
            aligned.append([int(r[0]), int(r[1])])
            jittered.append([int(r[0]), int(r[1])])
    for t in (aligned, jittered):
        got = orc.replay(np.array(t, dtype=np.uint64), base, span)
        assert got.rc == 0
        assert got.triples() == ref.triples()
        assert np.array_equal(got.shadow, ref.shadow)


@pytest.mark.parametrize("seed", range(8))
def test_straddling_access_is_two_word_accesses(orc, seed):
    rec, base, span = _program(9200 + seed)
    ref = orc.replay(rec, base, span)
    if ref.rc != 0:
        pytest.skip("program rejected")
    out, back = [], []          # back[j'] = record index in the original trace
    n_split = 0
    for i, r in enumerate(rec):
        addr, op, length = _fields(r)
        ws = _words(addr, length) if op < 4 else []
        if len(ws) == 2:
            n_split += 1
            out.append(_with(r, ws[0] * 8, 8)); back.append(i)
            out.append(_with(r, ws[1] * 8, 8)); back.append(i)
        else:
            out.append([int(r[0]), int(r[1])]); back.append(i)
    got = orc.replay(np.array(out, dtype=np.uint64), base, span)
    assert got.rc == 0
    mapped = sorted((w, back[j], k) for w, j, k in got.triples())
    assert mapped == ref.triples()
    assert np.array_equal(got.shadow, ref.shadow)


def test_programs_exercise_both_cases(orc):
    """The fixtures above are not vacuous: the generator's strides produce both
    sub-word one-word accesses and straddling accesses."""
    sub = straddle = 0
    for seed in range(8):
        rec, _, _ = _program(9100 + seed)
        for r in rec:
            addr, op, length = _fields(r)
            if op < 4:
                nw = len(_words(addr, length))
                straddle += nw == 2
                sub += nw == 1 and (addr % 8 != 0 or length != 8)
    assert sub > 50 and straddle > 50
