"""DRACC-style pattern catalogue (config 2; Table III).

Buggy variants must show exactly their labelled kinds; fixed variants must be
clean (no false positives on the issue-free DRACC programs).  The UUM /
USD part is cross-checked with the Definition-1 value simulator.
"""
import pytest

from gen.patterns import PATTERNS
from gen.trace import TraceBuilder
from valuesim import ValueSim

BASE = 0x100000


@pytest.mark.parametrize("name", sorted(PATTERNS))
@pytest.mark.parametrize("esz", [4, 8])
def test_pattern(orc, name, esz):
    fn, label = PATTERNS[name]
    n = 64
    for buggy in ((True, False) if label is not None else (False,)):
        tb = TraceBuilder()
        fn(tb, BASE, n, esz, buggy, 5)
        rec = tb.array()
        res = orc.replay(rec, BASE, 4 * n * esz)
        assert res.rc == 0
        kinds = {k for _, _, k in res.triples()}
        assert kinds == (label if buggy else set()), (name, buggy, kinds)
        vs = ValueSim().run(rec)
        assert sorted(vs) == [t for t in res.triples() if t[2] != 3]
        assert res.stats["transitions"] == res.stats["word_events"]


def test_config2_suite(orc):
    from gen.configs import config2
    rec, base, size, inst, spans = config2(reps=2, with_index=True)
    res = orc.replay(rec, base, size)
    assert res.rc == 0
    from gen.configs import REGION
    per = {}
    for w, r, k in res.triples():
        j = (w * 8 - base) // REGION
        per.setdefault(j, set()).add(k)
    for j, d in enumerate(inst):
        assert per.get(j, set()) == d["label"], (d["name"], d["buggy"])


@pytest.mark.parametrize("name", sorted(__import__("gen.patterns", fromlist=["BO_PATTERNS"]).BO_PATTERNS))
@pytest.mark.parametrize("esz", [4, 8])
def test_bo_pattern(orc, name, esz):
    """Buffer-overflow patterns (Table III row BO) with the extension of
    P:277-281: buggy -> BO only, fixed -> clean; the value simulator (CV
    existence as a set) agrees on every report."""
    from gen.patterns import BO_PATTERNS
    fn, label = BO_PATTERNS[name]
    n = 64
    for buggy in (True, False):
        tb = TraceBuilder()
        fn(tb, BASE, n, esz, buggy, 5)
        rec = tb.array()
        res = orc.replay(rec, BASE, 4 * n * esz, detect_bo=True)
        assert res.rc == 0
        kinds = {k for _, _, k in res.triples()}
        assert kinds == (label if buggy else set()), (name, buggy, kinds)
        vs = ValueSim(bo=True).run(rec)
        assert sorted(vs) == [t for t in res.triples() if t[2] != 3]
