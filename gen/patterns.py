"""DRACC-style micro offload kernels as trace writers.

Each pattern writes the serialized trace (Theorem 1(2)) of a small
OpenMP offload program on one array ``a`` of ``n`` elements of ``esz`` bytes
starting at ``base``, in a *buggy* or a *fixed* variant.  ``LABELS`` holds
the kinds the pattern's author expects in the buggy variant (DRACC classes of
Table III); the fixed variant is expected to be clean.
These labels are claims of the generator, checked by tests against the oracle
and the Definition-1 value simulator — never used as expected values for the
CUDA path (those come from the oracle).
"""
from __future__ import annotations

from .trace import MAP, OP, UPD, SYNC_ALL, TraceBuilder

UUM, USD, MIR = 1, 2, 3


def _init(tb, a, n, esz):
    tb.loop([(OP.WH, a)], n, esz)


def _kread(tb, a, n, esz):
    tb.loop([(OP.RT, a)], n, esz)


def _kwrite(tb, a, n, esz):
    tb.loop([(OP.WT, a)], n, esz)


def _kupdate(tb, a, n, esz):          # a[i] = a[i] + 1 on the device
    tb.loop([(OP.RT, a), (OP.WT, a)], n, esz)


def _hread(tb, a, n, esz):
    tb.loop([(OP.RH, a)], n, esz)


def _hwrite(tb, a, n, esz):
    tb.loop([(OP.WH, a)], n, esz)


def p01(tb, a, n, esz, buggy, task):   # map(alloc) + kernel read (Fig. 1, DRACC 22)
    _init(tb, a, n, esz)
    mt = MAP.ALLOC if buggy else MAP.TO
    tb.enter(mt, a, n * esz); _kread(tb, a, n, esz); tb.exit(mt, a, n * esz)


def p02(tb, a, n, esz, buggy, task):   # map(from) + kernel read before write
    _init(tb, a, n, esz)
    mt = MAP.FROM if buggy else MAP.TOFROM
    tb.enter(mt, a, n * esz); _kupdate(tb, a, n, esz); tb.exit(mt, a, n * esz)
    _hread(tb, a, n, esz)


def p03(tb, a, n, esz, buggy, task):   # enter data map(alloc) + kernel read
    _init(tb, a, n, esz)
    tb.enter(MAP.ALLOC if buggy else MAP.TO, a, n * esz)
    tb.enter(MAP.TOFROM, a, n * esz); _kread(tb, a, n, esz); tb.exit(MAP.TOFROM, a, n * esz)
    tb.exit(MAP.DELETE, a, n * esz)


def p04(tb, a, n, esz, buggy, task):   # uninitialised host array map(to) + kernel read
    if not buggy:
        _init(tb, a, n, esz)
    tb.enter(MAP.TO, a, n * esz); _kread(tb, a, n, esz); tb.exit(MAP.TO, a, n * esz)


def p05(tb, a, n, esz, buggy, task):   # map(from), kernel writes half, host reads other half
    _init(tb, a, n, esz)
    mt = MAP.FROM if buggy else MAP.TOFROM
    h = n // 2
    tb.enter(mt, a, n * esz); _kwrite(tb, a, h, esz); tb.exit(mt, a, n * esz)
    _hread(tb, a + h * esz, n - h, esz)


def p06(tb, a, n, esz, buggy, task):   # release, re-map(alloc), kernel read
    _init(tb, a, n, esz)
    tb.enter(MAP.TO, a, n * esz); _kread(tb, a, n, esz); tb.exit(MAP.RELEASE, a, n * esz)
    mt = MAP.ALLOC if buggy else MAP.TO
    tb.enter(mt, a, n * esz); _kread(tb, a, n, esz); tb.exit(MAP.DELETE, a, n * esz)


def p07(tb, a, n, esz, buggy, task):   # map(to) + kernel write + host read (Fig. 2 l.1-5)
    _init(tb, a, n, esz)
    mt = MAP.TO if buggy else MAP.TOFROM
    tb.enter(mt, a, n * esz); _kupdate(tb, a, n, esz); tb.exit(mt, a, n * esz)
    _hread(tb, a, n, esz)


def p08(tb, a, n, esz, buggy, task):   # missing `target update from` inside target data
    _init(tb, a, n, esz)
    tb.enter(MAP.TOFROM, a, n * esz); _kupdate(tb, a, n, esz)
    if not buggy:
        tb.update(UPD.FROM, a, n * esz)
    _hread(tb, a, n, esz)
    tb.exit(MAP.TOFROM, a, n * esz)


def p09(tb, a, n, esz, buggy, task):   # missing `target update to` after a host write
    _init(tb, a, n, esz)
    tb.enter(MAP.TO, a, n * esz); _hwrite(tb, a, n, esz)
    if not buggy:
        tb.update(UPD.TO, a, n * esz)
    _kread(tb, a, n, esz)
    tb.exit(MAP.TO, a, n * esz)


def p10(tb, a, n, esz, buggy, task):   # 503.postencil pointer swap
    x = a                              # mapped tofrom
    y = a + n * esz                    # mapped to
    _init(tb, x, n, esz); _init(tb, y, n, esz)
    tb.enter(MAP.TOFROM, x, n * esz); tb.enter(MAP.TO, y, n * esz)
    iters = 3 if buggy else 2
    src, dst = x, y
    for _ in range(iters):
        tb.loop([(OP.RT, src), (OP.WT, dst)], n, esz)
        src, dst = dst, src            # host swaps the two pointers
    tb.exit(MAP.TOFROM, x, n * esz); tb.exit(MAP.TO, y, n * esz)
    _hread(tb, src, n, esz)            # output of the last iteration (now `src`)


def p11(tb, a, n, esz, buggy, task):   # nested target data: inner from at rc=2 copies nothing
    _init(tb, a, n, esz)
    tb.enter(MAP.TO, a, n * esz)
    tb.enter(MAP.FROM, a, n * esz); _kupdate(tb, a, n, esz); tb.exit(MAP.FROM, a, n * esz)
    if not buggy:
        tb.update(UPD.FROM, a, n * esz)
    _hread(tb, a, n, esz)
    tb.exit(MAP.TO, a, n * esz)


def p12(tb, a, n, esz, buggy, task):   # enter data to + host modify + kernel read
    _init(tb, a, n, esz)
    tb.enter(MAP.TO, a, n * esz); _hwrite(tb, a, n, esz)
    if not buggy:
        tb.update(UPD.TO, a, n * esz)
    _kread(tb, a, n, esz)
    tb.exit(MAP.DELETE, a, n * esz)


def p13(tb, a, n, esz, buggy, task):   # exit data delete after a kernel write + host read
    _init(tb, a, n, esz)
    tb.enter(MAP.TO, a, n * esz); _kupdate(tb, a, n, esz)
    tb.exit(MAP.DELETE if buggy else MAP.FROM, a, n * esz)
    _hread(tb, a, n, esz)


def p14(tb, a, n, esz, buggy, task):   # exit data release at rc>1 + host read
    _init(tb, a, n, esz)
    tb.enter(MAP.TO, a, n * esz); tb.enter(MAP.TO, a, n * esz)
    _kupdate(tb, a, n, esz)
    tb.exit(MAP.RELEASE, a, n * esz)
    if not buggy:
        tb.update(UPD.FROM, a, n * esz)
    _hread(tb, a, n, esz)
    tb.exit(MAP.DELETE, a, n * esz)


def p15(tb, a, n, esz, buggy, task):   # host write inside the region + kernel read
    _init(tb, a, n, esz)
    tb.enter(MAP.TOFROM, a, n * esz); _kread(tb, a, n, esz)
    _hwrite(tb, a, n, esz)
    if not buggy:
        tb.update(UPD.TO, a, n * esz)
    _kupdate(tb, a, n, esz)
    tb.exit(MAP.TOFROM, a, n * esz)


def p23(tb, a, n, esz, buggy, task):   # section map a[0:n/2] + kernel write + host read
    _init(tb, a, n, esz)
    h = n // 2
    mt = MAP.TO if buggy else MAP.TOFROM
    tb.enter(mt, a, h * esz); _kupdate(tb, a, h, esz); tb.exit(mt, a, h * esz)
    _hread(tb, a, h, esz)


def p25(tb, a, n, esz, buggy, task):   # outer target data to, inner target map(from)
    _init(tb, a, n, esz)
    tb.enter(MAP.TO, a, n * esz)
    tb.enter(MAP.FROM, a, n * esz); _kupdate(tb, a, n, esz); tb.exit(MAP.FROM, a, n * esz)
    if not buggy:
        tb.update(UPD.FROM, a, n * esz)
    tb.exit(MAP.TO, a, n * esz)
    _hread(tb, a, n, esz)


def p16(tb, a, n, esz, buggy, task):   # target nowait write + host read without taskwait
    _init(tb, a, n, esz)
    tb.enter(MAP.TOFROM, a, n * esz)
    tb.task_begin(task); _kupdate(tb, a, n, esz); tb.task_end(task)
    if buggy:
        _hread(tb, a, n, esz)
        tb.sync(task)
    else:
        tb.sync(task)
        tb.update(UPD.FROM, a, n * esz)
        _hread(tb, a, n, esz)
    tb.exit(MAP.TOFROM, a, n * esz)


def p17(tb, a, n, esz, buggy, task):   # nowait + target data exit before taskwait
    _init(tb, a, n, esz)
    tb.enter(MAP.TOFROM, a, n * esz)
    tb.task_begin(task); _kupdate(tb, a, n, esz); tb.task_end(task)
    if buggy:
        tb.exit(MAP.TOFROM, a, n * esz); tb.sync(task)
    else:
        tb.sync(task); tb.exit(MAP.TOFROM, a, n * esz)
    _hread(tb, a, n, esz)


def p18(tb, a, n, esz, buggy, task):   # two nowait kernels writing the same array
    _init(tb, a, n, esz)
    tb.enter(MAP.TOFROM, a, n * esz)
    tb.task_begin(task); _kupdate(tb, a, n, esz); tb.task_end(task)
    if not buggy:
        tb.sync(task)
    tb.task_begin(task + 1); _kupdate(tb, a, n, esz); tb.task_end(task + 1)
    tb.sync(SYNC_ALL)
    tb.exit(MAP.TOFROM, a, n * esz)
    _hread(tb, a, n, esz)


def p19(tb, a, n, esz, buggy, task):   # nowait kernel reads while the host writes
    _init(tb, a, n, esz)
    tb.enter(MAP.TO, a, n * esz)
    tb.task_begin(task); _kread(tb, a, n, esz); tb.task_end(task)
    if not buggy:
        tb.sync(task)
    _hwrite(tb, a, n, esz)
    tb.sync(SYNC_ALL)
    tb.exit(MAP.TO, a, n * esz)
    _hread(tb, a, n, esz)


def p20(tb, a, n, esz, buggy, task):   # target update from nowait + host read
    _init(tb, a, n, esz)
    tb.enter(MAP.TOFROM, a, n * esz); _kupdate(tb, a, n, esz)
    tb.task_begin(task); tb.update(UPD.FROM, a, n * esz); tb.task_end(task)
    if not buggy:
        tb.sync(task)
    _hread(tb, a, n, esz)
    tb.sync(SYNC_ALL)
    tb.exit(MAP.TOFROM, a, n * esz)


def p21(tb, a, n, esz, buggy, task):   # enter data nowait map(to) + host write
    _init(tb, a, n, esz)
    tb.task_begin(task); tb.enter(MAP.TO, a, n * esz); tb.task_end(task)
    if not buggy:
        tb.sync(task)
    _hwrite(tb, a, n, esz)
    tb.sync(SYNC_ALL)
    tb.update(UPD.TO, a, n * esz)
    _kread(tb, a, n, esz)
    tb.exit(MAP.DELETE, a, n * esz)


def p22(tb, a, n, esz, buggy, task):   # clean: nowait on A while the host touches B
    b = a + n * esz
    _init(tb, a, n, esz)
    tb.enter(MAP.TOFROM, a, n * esz)
    tb.task_begin(task); _kupdate(tb, a, n, esz); tb.task_end(task)
    _hwrite(tb, b, n, esz); _hread(tb, b, n, esz)
    tb.sync(task)
    tb.exit(MAP.TOFROM, a, n * esz)
    _hread(tb, a, n, esz)


def p24(tb, a, n, esz, buggy, task):   # clean: read-only scalar map(to)
    tb.wh(a, esz)
    tb.enter(MAP.TO, a, esz)
    tb.loop([(OP.RT, a)], 1, esz)
    for _ in range(3):
        tb.rt(a, esz)
    tb.exit(MAP.TO, a, esz)
    tb.rh(a, esz)


PATTERNS = {
    "P01": (p01, {UUM}), "P02": (p02, {UUM}), "P03": (p03, {UUM}), "P04": (p04, {UUM}),
    "P05": (p05, {UUM}), "P06": (p06, {UUM}),
    "P07": (p07, {USD}), "P08": (p08, {USD}), "P09": (p09, {USD}), "P10": (p10, {USD}),
    "P11": (p11, {USD}), "P12": (p12, {USD}), "P13": (p13, {USD}), "P14": (p14, {USD}),
    "P15": (p15, {USD}), "P23": (p23, {USD}), "P25": (p25, {USD}),
    "P16": (p16, {MIR, USD}), "P17": (p17, {MIR}), "P18": (p18, {MIR}), "P19": (p19, {MIR}),
    "P20": (p20, {MIR}), "P21": (p21, {MIR}),
    "P22": (p22, None), "P24": (p24, None),   # clean-only
}
# bytes a pattern touches beyond ``n*esz`` from its base (P10 and P22 use two arrays)
FOOTPRINT_ARRAYS = {"P10": 2, "P22": 2}


# ---- buffer-overflow patterns (DRACC 23, 25, 28-31 analogues; Table III row BO,
# P:376; detected with the extension of P:277-281, ARB_F_BO / detect_bo) ----------
BO = 4


def b23(tb, a, n, esz, buggy, task):   # map(tofrom: a[0:n/2]) but the kernel updates a[0:n]
    _init(tb, a, n, esz)
    sec = (n // 2 if buggy else n) * esz
    tb.enter(MAP.TOFROM, a, sec); _kupdate(tb, a, n, esz); tb.exit(MAP.TOFROM, a, sec)
    _hread(tb, a, n, esz)


def b25(tb, a, n, esz, buggy, task):   # enter data map(to: a[0:n/2]), kernel reads a[0:n]
    _init(tb, a, n, esz)
    sec = (n // 2 if buggy else n) * esz
    tb.enter(MAP.TO, a, sec); _kread(tb, a, n, esz); tb.exit(MAP.DELETE, a, sec)


def b28(tb, a, n, esz, buggy, task):   # section one 8-B word short (P:267 granularity), kernel writes a[0:n]
    _init(tb, a, n, esz)
    sec = n * esz - (8 if buggy else 0)
    tb.enter(MAP.FROM, a, sec); _kwrite(tb, a, n, esz); tb.exit(MAP.FROM, a, sec)
    _hread(tb, a, sec // esz, esz)


def b29(tb, a, n, esz, buggy, task):   # the kernel runs after `exit data delete`
    _init(tb, a, n, esz)
    tb.enter(MAP.TO, a, n * esz)
    if buggy:
        tb.exit(MAP.DELETE, a, n * esz); _kread(tb, a, n, esz)
    else:
        _kread(tb, a, n, esz); tb.exit(MAP.DELETE, a, n * esz)


def b30(tb, a, n, esz, buggy, task):   # the kernel indexes past the mapped section's start
    _init(tb, a, n, esz)
    lo = n // 4 if buggy else 0
    tb.enter(MAP.TOFROM, a + lo * esz, (n - lo) * esz)
    _kupdate(tb, a, n, esz)
    tb.exit(MAP.TOFROM, a + lo * esz, (n - lo) * esz)


BO_PATTERNS = {"B23": (b23, {BO}), "B25": (b25, {BO}), "B28": (b28, {BO}), "B29": (b29, {BO}),
               "B30": (b30, {BO})}
