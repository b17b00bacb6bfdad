"""Seeded random offload programs for parity fuzzing (structure only).

A program works on a few arrays; it opens and closes data regions on whole
arrays or halves, runs host and device loops with random unaligned 1..8-byte
accesses, target updates, nowait blocks (some joined late or never) and
taskwaits.  The generator keeps a little bookkeeping so that most programs
stay well-formed; it computes nothing the replay computes.
"""
from __future__ import annotations

import numpy as np

from .trace import MAP, OP, UPD, SYNC_ALL, TraceBuilder, encode_np


def random_program(seed: int, n_arrays: int = 4, array_words: int = 64, steps: int = 60,
                   base: int = 0x10000, loop_max: int = 48, p_task: float = 0.15, p_always: float = 0.0,
                   p_depend: float = 0.0, n_devices: int = 1, p_tag: float = 0.0,
                   strides=(1, 4, 8, 8, 8, 12), sizes=(1, 2, 4, 8, 8, 8)):
    """p_always > 0: map clauses carry the `always` modifier with that probability;
    p_depend > 0: a new nowait block depends on an earlier task with that
    probability; n_devices > 1: target accesses and map / update clauses on a
    random accelerator (the device in the access arg and in bits 6-7 of a
    map / update arg); p_tag > 0: pointer tags (ARB_BASE records, reading Z25): tag
    i + 1 has array i's base, target accesses carry a tag with that probability
    (mostly their own array's, sometimes another's), and tags are sometimes
    redefined (the RNG streams of the defaults are unchanged).  strides / sizes: the
    loop access strides and sizes are drawn from them (8 / 8: runs over consecutive
    words)."""
    rs = np.random.default_rng(seed)
    tb = TraceBuilder()
    arrays = [base + i * array_words * 8 * 2 for i in range(n_arrays)]   # gap between arrays
    # list of (lo, hi) byte sections entered, per array (and device with n_devices > 1)
    present = {(i, d): [] for i in range(n_arrays) for d in range(n_devices)}

    def pdev():
        return int(rs.integers(n_devices)) if n_devices > 1 else 0
    if p_tag:
        for i in range(n_arrays):
            tb._add(OP.BASE, arrays[i], 0, task=i + 1)
    in_task = 0
    next_task = 1
    unjoined = []
    ended_ids = []

    def section(i):
        a = arrays[i]
        n = array_words * 8
        kind = rs.integers(0, 4)
        if kind == 0:
            return a, n
        if kind == 1:
            return a, n // 2
        if kind == 2:
            return a + n // 2, n - n // 2
        lo = int(rs.integers(0, array_words - 1)) * 8
        return a + lo, int(rs.integers(1, array_words - lo // 8)) * 8

    def loop(op):
        i = int(rs.integers(n_arrays))
        cnt = int(rs.integers(1, loop_max))
        start = int(rs.integers(0, array_words * 8 - 8))
        stride = int(rs.choice(list(strides)))
        size = int(rs.choice(list(sizes)))
        addr = arrays[i] + start + stride * np.arange(cnt, dtype=np.uint64)
        addr = addr[addr + size <= arrays[i] + array_words * 8 + 8]
        if addr.size:
            arg = pdev() if op in (OP.RT, OP.WT) else 0
            tag = 0
            if p_tag and op in (OP.RT, OP.WT) and rs.random() < p_tag:
                tag = i + 1 if rs.random() < 0.7 else int(rs.integers(1, n_arrays + 2))
            tb.add_array(encode_np(op, addr, size, arg=arg, task=tag))

    for _ in range(steps):
        if p_tag and rs.random() < 0.04:         # a pointer re-based into some array
            j = int(rs.integers(n_arrays))
            tb._add(OP.BASE, arrays[j] + 8 * int(rs.integers(array_words)), 0, task=int(rs.integers(1, n_arrays + 2)))
        r = rs.random()
        if r < 0.35:
            loop(int(rs.choice([OP.RH, OP.WH, OP.RT, OP.WT])))
        elif r < 0.5:
            i = int(rs.integers(n_arrays))
            lo, n = section(i)
            hi = lo + n
            dv = pdev()
            pr = present[(i, dv)]
            ok = all(hi <= a or lo >= b or (a <= lo and hi <= b) for a, b in pr)
            if ok:
                mt = int(rs.choice([MAP.TO, MAP.FROM, MAP.TOFROM, MAP.ALLOC]))
                if p_always and rs.random() < p_always:
                    mt |= MAP.ALWAYS
                if p_always and any(a <= lo and hi <= b for a, b in pr) and rs.random() < p_always:
                    mt |= MAP.PRESENT            # a mapped section: `present` holds
                tb.enter(mt | (dv << 6), lo, n)
                pr.append((lo, hi))
        elif r < 0.65:
            i = int(rs.integers(n_arrays))
            dv = pdev()
            pr = present[(i, dv)]
            if pr:
                k = int(rs.integers(len(pr)))
                lo, hi = pr[k]
                # exit only sections that contain no other present section
                if all(not (lo <= a and b <= hi and (a, b) != (lo, hi)) for a, b in pr):
                    mt = int(rs.choice([MAP.TO, MAP.FROM, MAP.TOFROM, MAP.ALLOC, MAP.RELEASE, MAP.DELETE]))
                    if p_always and rs.random() < p_always:
                        mt |= MAP.ALWAYS
                    tb.exit(mt | (dv << 6), lo, hi - lo)
                    pr.pop(k)
        elif r < 0.72:
            i = int(rs.integers(n_arrays))
            dv = pdev()
            pr = present[(i, dv)]
            if pr:
                lo, hi = pr[int(rs.integers(len(pr)))]
                tb.update(int(rs.choice([UPD.TO, UPD.FROM])) | (dv << 6), lo, hi - lo)
            elif rs.random() < 0.3:
                tb.update(int(rs.choice([UPD.TO, UPD.FROM])) | (dv << 6), arrays[i], array_words * 8)
        elif r < 0.72 + p_task and not in_task:
            k = next_task
            next_task = next_task + 1 if next_task < 60000 else 1
            tb.task_begin(k)
            in_task = k
            if p_depend and ended_ids and rs.random() < p_depend:
                tb.depend(int(ended_ids[int(rs.integers(len(ended_ids)))]))
        elif in_task and r < 0.95:
            tb.task_end(in_task)
            unjoined.append(in_task)
            ended_ids.append(in_task)
            in_task = 0
        elif not in_task and unjoined and r >= 0.95:
            if rs.random() < 0.5:
                tb.sync(SYNC_ALL)
                unjoined = []
            else:
                k = unjoined.pop(int(rs.integers(len(unjoined))))
                tb.sync(k)
    if in_task:
        tb.task_end(in_task)
    span = n_arrays * array_words * 8 * 2
    return tb.array(), base, span


def to_cv_addressing(rec, cv_off=1 << 44, frac=1.0, seed=0):
    """The same program with its target accesses to mapped words addressed by CV
    (device) address (arg bit 0x80, reading Z26): every entry's CV sits at its OV
    address + cv_off, reported by an ARB_CV_BASE record (op 16) after each map entry.
    frac < 1: only that fraction of the eligible accesses is rewritten.  Mapped-ness
    is tracked with a plain interval list (structure only, no replay)."""
    rs = np.random.default_rng(seed)
    op = ((rec[:, 0] >> np.uint64(48)) & np.uint64(0xFF)).astype(np.int64)
    addr = (rec[:, 0] & np.uint64((1 << 48) - 1)).astype(np.int64)
    ln = (rec[:, 1] & np.uint64((1 << 48) - 1)).astype(np.int64)
    arg = (rec[:, 0] >> np.uint64(56)).astype(np.int64)
    entries = []                                  # [lo, hi, rc]
    out = []
    for i in range(rec.shape[0]):
        w0, w1 = int(rec[i, 0]), int(rec[i, 1])
        o, a, n = int(op[i]), int(addr[i]), int(ln[i])
        if o in (OP.RT, OP.WT) and any(e[0] <= a < e[1] for e in entries) and rs.random() < frac:
            w0 = (w0 & ~((1 << 48) - 1) & ~(0xFF << 56)) | (a + cv_off) | ((0x80 | int(arg[i])) << 56)
        out.append((w0, w1))
        if o == OP.MAP_ENTER:
            hit = [e for e in entries if e[0] <= a and a + n <= e[1]]
            if hit:
                hit[0][2] += 1
            elif not any(a < e[1] and e[0] < a + n for e in entries):
                entries.append([a, a + n, 1])
                out.append(tuple(int(x) for x in encode_np(16, [a], [a + cv_off])[0]))
        elif o == OP.MAP_EXIT:
            hit = [e for e in entries if e[0] <= a and a + n <= e[1]]
            if hit:
                e = hit[0]
                e[2] = 0 if (int(arg[i]) & 0xF) == MAP.DELETE else e[2] - 1
                if e[2] == 0:
                    entries.remove(e)
    return np.array(out, dtype=np.uint64).reshape(-1, 2)


def run_program(seed: int, n_arrays: int = 6, array_words: int = 4096, steps: int = 400, loop_max: int = 1500):
    """Programs whose loops are mostly runs (stride 8, size 8: consecutive records
    on consecutive words with one op), so that most chunks take the partition's run
    form, with some stride-4 / stride-16 loops mixed in."""
    return random_program(seed, n_arrays=n_arrays, array_words=array_words, steps=steps, loop_max=loop_max,
                          strides=(8, 8, 8, 8, 8, 8, 8, 4, 16), sizes=(8, 8, 8, 8, 8, 8, 8, 4, 8))
