"""Counter-based generator programs for the large configs (3, 4, 5).

A *program* is a small table of segments (``gen/arbgen.cuh``): literal records
(control records), loops over array bodies (streams, stencils, 2-D blocks,
random / skewed gathers) and random-run bodies.  Record i of the trace is a
pure function of (table, i), so ``fill_host`` (C, OpenMP) and ``fill_device``
(CUDA) produce identical bytes and any slice can be generated independently.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from .configs import BASE_SEED, rng
from .trace import MAP, OP, SYNC_ALL, encode

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "arbgen.cu")
_HDR = os.path.join(_HERE, "arbgen.cuh")
_LIB = os.path.join(_HERE, "libarbgen.so")

SEG_LIT, SEG_LOOP, SEG_RUNS = 0, 1, 2
M_LINEAR, M_2D, M_RANDOM, M_SKEW = 0, 1, 2, 3

ENTRY_DT = np.dtype([("op", "<u4"), ("size", "<u4"), ("mode", "<u4"), ("pad", "<u4"),
                     ("base", "<u8"), ("stride", "<u8"), ("range", "<u8")])
SEG_DT = np.dtype([("start", "<u8"), ("count", "<u8"), ("type", "<u4"), ("body_len", "<u4"),
                   ("body_off", "<u4"), ("width", "<u4"), ("t0", "<u8"), ("seed", "<u8")] +
                  [(f"p{i}", "<u8") for i in range(8)])
assert ENTRY_DT.itemsize == 40 and SEG_DT.itemsize == 112


def build(force: bool = False) -> str:
    newest = max(os.path.getmtime(_SRC), os.path.getmtime(_HDR))
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < newest:
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-O3", "-std=c++17", "-shared",
                               "-gencode", "arch=compute_100a,code=sm_100a",
                               "-Xcompiler", "-fPIC,-fopenmp", "-o", tmp, _SRC, "-lgomp"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        vp, u64, u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32
        lib.arbgen_fill_host.argtypes = [vp, u32, vp, vp, u64, u64, vp]
        lib.arbgen_fill_host.restype = ctypes.c_int
        lib.arbgen_filter_host.argtypes = [vp, u32, vp, vp, u64, u64, vp, u64, u64, u64, vp, vp, u64]
        lib.arbgen_filter_host.restype = u64
        lib.arbgen_fill_device.argtypes = [vp, u32, vp, vp, u64, u64, vp, vp]
        lib.arbgen_fill_device.restype = ctypes.c_int
        lib.arbgen_filter_device.argtypes = [vp, u64, u64, u64, u64, vp, vp, vp, ctypes.POINTER(u64), vp]
        lib.arbgen_filter_device.restype = ctypes.c_int
        _lib = lib
    return _lib


class Program:
    """Segment table of one synthetic trace plus metadata."""

    def __init__(self, name, addr_base, addr_bytes):
        self.name = name
        self.addr_base, self.addr_bytes = addr_base, addr_bytes
        self._segs, self._ents, self._lits = [], [], []
        self.n = 0
        self.quiescent = [0]          # record indices where a flush may cut
        self.sections = []            # (word_lo, word_hi) of mapped sections, for W accounting
        self.meta = {}
        self._dev = None

    # -- construction ---------------------------------------------------------
    def lit(self, *recs):
        s = np.zeros(1, SEG_DT)[0]
        s["start"], s["count"], s["type"], s["body_off"] = self.n, len(recs), SEG_LIT, len(self._lits)
        self._lits.extend(recs)
        self._segs.append(s)
        self.n += len(recs)

    def loop(self, body, iters, t0=0, width=1, seed=0):
        """body: list of (op, size, mode, base, stride, range)."""
        if iters <= 0:
            return
        s = np.zeros(1, SEG_DT)[0]
        s["start"], s["count"], s["type"] = self.n, iters * len(body), SEG_LOOP
        s["body_len"], s["body_off"], s["width"], s["t0"], s["seed"] = len(body), len(self._ents), width, t0, seed
        for (op, size, mode, base, stride, rng_) in body:
            e = np.zeros(1, ENTRY_DT)[0]
            e["op"], e["size"], e["mode"], e["base"], e["stride"], e["range"] = op, size, mode, base, stride, rng_
            self._ents.append(e)
        self._segs.append(s)
        self.n += iters * len(body)

    def runs(self, count, seed, word_lo, span, L, kind, dev_seed=0, overlap=0, stale=0):
        if count <= 0:
            return
        s = np.zeros(1, SEG_DT)[0]
        s["start"], s["count"], s["type"], s["seed"] = self.n, count, SEG_RUNS, seed
        s["p0"], s["p1"], s["p2"], s["p3"], s["p4"], s["p5"], s["p6"] = word_lo, span, L, kind, dev_seed, overlap, stale
        self._segs.append(s)
        self.n += count

    def finish(self):
        self.segs = np.array(self._segs, dtype=SEG_DT) if self._segs else np.zeros(0, SEG_DT)
        self.ents = np.array(self._ents, dtype=ENTRY_DT) if self._ents else np.zeros(1, ENTRY_DT)
        self.lits = np.array(self._lits, dtype=np.uint64).reshape(-1, 2) if self._lits else np.zeros((1, 2), np.uint64)
        if self.quiescent[-1] != self.n:
            self.quiescent.append(self.n)
        return self

    def distinct_words(self, lo, hi, ranges, sector_words=1):
        """W of B_alg for each global record range: the union of the mapped sections
        entered in the range, clipped to the tracked words [lo, hi).  Every access
        of these programs lies inside a section of its own region.  sector_words > 1:
        whole shadow sectors of that many words (1 B of shadow per word) counted as
        touched words (the sector-granular variant of SURVEY §8(d))."""
        secs = np.array(self.sections, dtype=np.uint64).reshape(-1, 3)
        out = []
        g = np.int64(sector_words)
        for g0, g1 in ranges:
            m = (secs[:, 2] >= g0) & (secs[:, 2] < g1)
            a = np.maximum(secs[m, 0], np.uint64(lo)).astype(np.int64)
            b = np.minimum(secs[m, 1], np.uint64(hi)).astype(np.int64)
            if sector_words > 1:
                keep = a < b
                a, b = (a[keep] // g) * g, ((b[keep] + g - 1) // g) * g
            keep = a < b
            a, b = a[keep], b[keep]
            order = np.argsort(a)
            w, cur_a, cur_b = 0, None, None
            for x, y in zip(a[order], b[order]):
                if cur_b is None or x > cur_b:
                    if cur_b is not None:
                        w += cur_b - cur_a
                    cur_a, cur_b = x, y
                else:
                    cur_b = max(cur_b, y)
            if cur_b is not None:
                w += cur_b - cur_a
            out.append(int(w))
        return out

    # -- generation ----------------------------------------------------------------
    def fill_host(self, start=0, count=None) -> np.ndarray:
        count = self.n - start if count is None else count
        out = np.empty((count, 2), dtype=np.uint64)
        _load().arbgen_fill_host(self.segs.ctypes.data, len(self.segs), self.ents.ctypes.data,
                                 self.lits.ctypes.data, start, count, out.ctypes.data)
        return out

    def filter_host(self, words=None, word_lo=0, word_hi=0, start=0, count=None, cap=None):
        """Records touching `words` (sorted u64 array) or [word_lo, word_hi), plus control
        records, with their global indices.  Returns (records, gidx)."""
        count = self.n - start if count is None else count
        cap = count if cap is None else cap
        out = np.empty((max(cap, 1), 2), dtype=np.uint64)
        gi = np.empty(max(cap, 1), dtype=np.uint64)
        w = None if words is None else np.ascontiguousarray(words, dtype=np.uint64)
        k = _load().arbgen_filter_host(self.segs.ctypes.data, len(self.segs), self.ents.ctypes.data,
                                       self.lits.ctypes.data, start, count,
                                       None if w is None else w.ctypes.data, 0 if w is None else w.size,
                                       word_lo, word_hi, out.ctypes.data, gi.ctypes.data, cap)
        assert k <= cap, "filter capacity exceeded"
        return out[:k], gi[:k]

    def device_tables(self):
        import torch
        if self._dev is None:
            t = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.uint8).reshape(-1)).cuda()
            self._dev = (t(self.segs), t(self.ents), t(self.lits))
        return self._dev

    def fill_device(self, out, start=0, count=None, stream=None):
        """Generate records [start, start+count) into the device tensor `out` (>= count*16 B)."""
        count = self.n - start if count is None else count
        segs, ents, lits = self.device_tables()
        rc = _load().arbgen_fill_device(segs.data_ptr(), len(self.segs), ents.data_ptr(), lits.data_ptr(),
                                        start, count, out.data_ptr(),
                                        None if stream is None else stream.cuda_stream)
        assert rc == 0, rc


def filter_device(src, n, word_lo, word_hi, first_index, out, gidx, stream=None):
    """Order-preserving compaction on the device; returns the kept count."""
    import torch
    scratch = torch.empty(((n + 4095) // 4096) * 12 + 64, dtype=torch.uint8, device=src.device)
    k = ctypes.c_uint64()
    rc = _load().arbgen_filter_device(src.data_ptr(), n, word_lo, word_hi, first_index, out.data_ptr(),
                                      None if gidx is None else gidx.data_ptr(), scratch.data_ptr(),
                                      ctypes.byref(k), None if stream is None else stream.cuda_stream)
    assert rc == 0, rc
    return k.value


# ---------------------------------------------------------------------------
# config 5: "synthetic 8-GPU address-sharded trace, 10^10 events over 64 GB of
# locations with boundary-spanning map ranges"
# ---------------------------------------------------------------------------
C5_BASE_WORD = 1 << 37            # byte address 2^40
C5_WORDS = 1 << 33                # 64 GiB of locations = 2^33 8-byte words
C5_SHARDS = 8
C5_SHARD_WORDS = C5_WORDS // C5_SHARDS


def config5(total_records: int = 9 * 10**9, groups: int = 4096, seed: int = BASE_SEED + 5,
            stale_rate: int = 20000) -> Program:
    """Target regions (groups) over map(alloc) sections of 2^19..2^21 words, 25 %
    centred on shard boundaries; device runs (WT, RT, RT) then host runs (WH, RH, RH)
    of geometric length (64..2048 words, mean ~512) at uniform random starts in the
    section (op mix 40 % RT, 20 % WT, ~27 % RH, ~13 % WH); 1 % of regions are nowait,
    10 % of those lack the taskwait before the host runs (MIR); 1 in `stale_rate`
    host runs reads words a device run wrote without a transfer (USD)."""
    p = Program("config5", C5_BASE_WORD * 8, C5_WORDS * 8)
    per = total_records // groups
    task = 1
    for g in range(groups):
        r = rng(seed, 3 * g)
        sec = 1 << (19 + r % 3)
        if (r >> 8) % 4 == 0:
            centre = ((r >> 16) % (C5_SHARDS - 1) + 1) * C5_SHARD_WORDS
        else:
            centre = (r >> 20) % C5_WORDS
        lo = min(max(centre - sec // 2, 0), C5_WORDS - sec)
        r2 = rng(seed, 3 * g + 1)
        L = 64 << bin(r2 & 0x1F).count("1")
        dev_runs = max(1, round(0.6 * per / (3 * L)))
        host_runs = max(1, round(0.4 * per / (3 * L)))
        nowait = (r2 >> 8) % 100 == 0
        missing = nowait and (r2 >> 16) % 10 == 0
        sd, sh = rng(seed, 3 * g + 2), rng(seed + 1, 3 * g + 2)
        wlo = C5_BASE_WORD + lo
        p.sections.append((wlo, wlo + sec, p.n))
        p.lit(encode(OP.MAP_ENTER, wlo * 8, sec * 8, arg=MAP.ALLOC))
        if nowait:
            p.lit(encode(OP.TASK_BEGIN, task=task))
        p.runs(dev_runs * 3 * L, sd, wlo, sec - L, L, 0)
        if nowait:
            p.lit(encode(OP.TASK_END, task=task))
            if not missing:
                p.lit(encode(OP.SYNC, task=task))
        p.runs(host_runs * 3 * L, sh, wlo, sec - L, L, 1, dev_seed=sd, overlap=4 if missing else 0,
               stale=stale_rate)
        if missing:
            p.lit(encode(OP.SYNC, task=SYNC_ALL))
        if nowait:
            task = task + 1 if task < 60000 else 1
        p.lit(encode(OP.MAP_EXIT, wlo * 8, sec * 8, arg=MAP.ALLOC))
        p.quiescent.append(p.n)
    p.meta = dict(groups=groups, total_records=total_records)
    return p.finish()


# ---------------------------------------------------------------------------
# config 3: "Rodinia-like offload loops (hotspot/lud/bfs shapes) with target
# data regions and nowait, ~10^9 events"
# ---------------------------------------------------------------------------
C3_BASE = 0x2000_0000_0000        # byte address of the first array


def _arrays(base, sizes, gap=1 << 20):
    out, a = [], base
    for s in sizes:
        out.append(a)
        a += (s + gap + 4095) & ~4095
    return out, a - base


def config3(scale: float = 1.0, seed: int = BASE_SEED + 3, hotspot_iters: int = 6) -> Program:
    """hotspot: 4096^2 float temp/power/result, 5-point stencil, target data
    map(to:power) map(tofrom:temp) map(alloc:result), per iteration a nowait
    kernel + taskwait; one iteration reads a result row on the host before the
    taskwait (MIR).  lud: 1024^2 doubles in 64x64 blocks (diagonal, perimeter,
    internal kernels), tofrom.  bfs: R-MAT-like (skewed) graph, V=2^22, E=2^25,
    CSR mapped to, mask/visited/cost tofrom, per level kernel + target update
    from(stop) + host read of `stop` (a hot word); one level omits the update
    (USD).  `scale` shrinks the grids / graph for tests."""
    N = max(64, int(4096 * scale ** 0.5)) & ~63
    LN = max(128, int(1024 * scale ** 0.5)) & ~63
    V = max(1 << 10, int((1 << 22) * scale))
    E = 8 * V
    F4, F8 = 4, 8
    sizes = [N * N * F4] * 3 + [LN * LN * F8] + [(V + 1) * F4, E * F4, V * F4, V * F4, V * F4, 64]
    (temp, power, result, lud, rowp, col, mask, visited, cost, stop), span = _arrays(C3_BASE, sizes)
    p = Program("config3", C3_BASE, span)
    L, S = OP, MAP
    # ---------------- hotspot ----------------
    p.loop([(L.WH, F4, M_LINEAR, temp, F4, 0), (L.WH, F4, M_LINEAR, power, F4, 0)], N * N)
    for a, mt in ((power, S.TO), (temp, S.TOFROM), (result, S.ALLOC)):
        p.sections.append((a // 8, (a + N * N * F4 + 7) // 8, p.n))
        p.lit(encode(OP.MAP_ENTER, a, N * N * F4, arg=mt))
    src, dst = temp, result
    task = 1
    for it in range(hotspot_iters):
        p.lit(encode(OP.TASK_BEGIN, task=task))
        c0 = N                                           # interior rows 1 .. N-2
        p.loop([(L.RT, F4, M_LINEAR, src + c0 * F4, F4, 0), (L.RT, F4, M_LINEAR, src + (c0 - 1) * F4, F4, 0),
                (L.RT, F4, M_LINEAR, src + (c0 + 1) * F4, F4, 0), (L.RT, F4, M_LINEAR, src + (c0 - N) * F4, F4, 0),
                (L.RT, F4, M_LINEAR, src + (c0 + N) * F4, F4, 0), (L.RT, F4, M_LINEAR, power + c0 * F4, F4, 0),
                (L.WT, F4, M_LINEAR, dst + c0 * F4, F4, 0)], N * (N - 2))
        # boundary rows: copied through (clamped stencil)
        p.loop([(L.RT, F4, M_LINEAR, src, F4, 0), (L.WT, F4, M_LINEAR, dst, F4, 0),
                (L.RT, F4, M_LINEAR, src + (N - 1) * N * F4, F4, 0),
                (L.WT, F4, M_LINEAR, dst + (N - 1) * N * F4, F4, 0)], N)
        p.lit(encode(OP.TASK_END, task=task))
        if it == 2:   # host reads a boundary row of the result before the taskwait (MIR + stale)
            p.loop([(L.RH, F4, M_LINEAR, dst + N * F4, F4, 0)], N)
        p.lit(encode(OP.SYNC, task=task))
        p.quiescent.append(p.n)
        task += 1
        src, dst = dst, src
    for a, mt in ((power, S.TO), (temp, S.TOFROM), (result, S.ALLOC)):
        p.lit(encode(OP.MAP_EXIT, a, N * N * F4, arg=mt))
    p.loop([(L.RH, F4, M_LINEAR, temp + (N // 2) * N * F4, F4, 0)], N)   # host prints a row
    p.quiescent.append(p.n)
    # ---------------- lud ----------------
    B = 64
    nb = LN // B
    p.loop([(L.WH, F8, M_LINEAR, lud, F8, 0)], LN * LN)
    p.sections.append((lud // 8, lud // 8 + LN * LN, p.n))
    p.lit(encode(OP.MAP_ENTER, lud, LN * LN * F8, arg=S.TOFROM))
    blk = lambda bi, bj: lud + (bi * B * LN + bj * B) * F8
    for k in range(nb):
        p.loop([(L.RT, F8, M_2D, blk(k, k), F8, LN * F8), (L.WT, F8, M_2D, blk(k, k), F8, LN * F8)], B * B, width=B)
        for j in range(k + 1, nb):
            p.loop([(L.RT, F8, M_2D, blk(k, k), F8, LN * F8), (L.RT, F8, M_2D, blk(k, j), F8, LN * F8),
                    (L.WT, F8, M_2D, blk(k, j), F8, LN * F8)], B * B, width=B)
            p.loop([(L.RT, F8, M_2D, blk(k, k), F8, LN * F8), (L.RT, F8, M_2D, blk(j, k), F8, LN * F8),
                    (L.WT, F8, M_2D, blk(j, k), F8, LN * F8)], B * B, width=B)
        for i in range(k + 1, nb):
            for j in range(k + 1, nb):
                p.loop([(L.RT, F8, M_2D, blk(i, k), F8, LN * F8), (L.RT, F8, M_2D, blk(k, j), F8, LN * F8),
                        (L.RT, F8, M_2D, blk(i, j), F8, LN * F8), (L.WT, F8, M_2D, blk(i, j), F8, LN * F8)],
                       B * B, width=B)
    p.lit(encode(OP.MAP_EXIT, lud, LN * LN * F8, arg=S.TOFROM))
    p.loop([(L.RH, F8, M_LINEAR, lud, F8, 0)], LN)
    p.quiescent.append(p.n)
    # ---------------- bfs ----------------
    p.loop([(L.WH, F4, M_LINEAR, rowp, F4, 0)], V + 1)
    p.loop([(L.WH, F4, M_LINEAR, col, F4, 0)], E)
    p.loop([(L.WH, F4, M_LINEAR, mask, F4, 0), (L.WH, F4, M_LINEAR, visited, F4, 0),
            (L.WH, F4, M_LINEAR, cost, F4, 0)], V)
    p.wh_stop = stop
    p.lit(encode(OP.WH, stop, 4))
    for a, n, mt in ((rowp, V + 1, S.TO), (col, E, S.TO), (mask, V, S.TOFROM), (visited, V, S.TOFROM),
                     (cost, V, S.TOFROM), (stop, 1, S.TOFROM)):
        p.sections.append((a // 8, (a + n * F4 + 7) // 8, p.n))
        p.lit(encode(OP.MAP_ENTER, a, n * F4, arg=mt))
    frac = [0.001, 0.01, 0.05, 0.15, 0.25, 0.25, 0.15, 0.08, 0.04, 0.015, 0.004, 0.001]
    e0 = 0
    for lvl, f in enumerate(frac):
        ne = min(E, max(8, int(E * f))) & ~7
        e0 = min(e0, E - ne)
        p.lit(encode(OP.WH, stop, 4), encode(OP.UPDATE, stop, 4, arg=0))       # stop = false; update to
        p.loop([(L.RT, F4, M_LINEAR, mask, F4, 0)], V)                          # scan the frontier mask
        body = [(L.RT, F4, M_SKEW, rowp, F4, V)]                               # frontier vertex's row_ptr
        for k in range(8):   # 8 edges per iteration: col[e], visited[u], cost[u], mask[u]
            body += [(L.RT, F4, M_LINEAR, col + (e0 + k) * F4, 8 * F4, 0),
                     (L.RT, F4, M_SKEW, visited, F4, V), (L.WT, F4, M_SKEW, cost, F4, V),
                     (L.WT, F4, M_SKEW, mask, F4, V)]
        body.append((L.WT, F4, M_LINEAR, stop, 0, 0))                          # the hot `stop` flag
        p.loop(body, ne // 8, seed=rng(seed, lvl))
        e0 = e0 + ne
        if lvl != 5:
            p.lit(encode(OP.UPDATE, stop, 4, arg=1))                            # update from(stop)
        p.lit(encode(OP.RH, stop, 4))                                           # host reads stop
        p.quiescent.append(p.n)
    for a, n, mt in ((rowp, V + 1, S.TO), (col, E, S.TO), (mask, V, S.TOFROM), (visited, V, S.TOFROM),
                     (cost, V, S.TOFROM), (stop, 1, S.TOFROM)):
        p.lit(encode(OP.MAP_EXIT, a, n * F4, arg=mt))
    p.meta = dict(N=N, LN=LN, V=V, E=E)
    return p.finish()


# ---------------------------------------------------------------------------
# config 4: "SPEC-ACCEL-like multi-array stencil with repeated target update
# and array-section maps, 16 GB shadow" (503.postencil P:386)
# ---------------------------------------------------------------------------
C4_BASE = 0x4000_0000_0000


def config4(scale: float = 1.0, iters: int = 3) -> Program:
    """8 arrays of NX*NY*NZ doubles (2048x2048x512 = 2^31 at scale 1 -> 2^34
    words of shadow).  X (mapped tofrom) and Y (mapped to) by target data; six
    more arrays by target enter/exit data.  Each of `iters` (3)
    iterations runs a 7-point stencil over a 1/64 z-slab, src -> dst with a host
    pointer swap (503.postencil), then `target update from` the slab's
    top halo plane of dst and `target update to` its bottom halo plane of src.
    With an odd count the result stays in the `to`-mapped Y: the host's final
    reads (a sample of the output) are stale (USD)."""
    NX = NY = max(64, int(2048 * scale ** (1 / 3))) & ~15
    NZ = max(64, int(512 * scale ** (1 / 3))) & ~63
    plane = NX * NY
    n = plane * NZ
    F8 = 8
    arrs, span = _arrays(C4_BASE, [n * F8] * 8, gap=0)
    X, Y = arrs[0], arrs[1]
    p = Program("config4", C4_BASE, span)
    L, S = OP, MAP
    z0, nz = NZ // 2, max(2, NZ // 64)
    c0, cells = (z0 * plane), nz * plane
    # host initialises the slab (and its halo planes) of X and Y
    p.loop([(L.WH, F8, M_LINEAR, X + (c0 - plane) * F8, F8, 0),
            (L.WH, F8, M_LINEAR, Y + (c0 - plane) * F8, F8, 0)], cells + 2 * plane)
    for a, mt in zip(arrs, [S.TOFROM, S.TO] + [S.TO] * 6):
        p.sections.append((a // 8, a // 8 + n, p.n))
        p.lit(encode(OP.MAP_ENTER, a, n * F8, arg=mt))
    src, dst = X, Y
    for it in range(iters):
        offs = [0, -1, 1, -NX, NX, -plane, plane]
        body = [(L.RT, F8, M_LINEAR, src + (c0 + o) * F8, F8, 0) for o in offs]
        body.append((L.WT, F8, M_LINEAR, dst + c0 * F8, F8, 0))
        p.loop(body, cells)
        p.lit(encode(OP.UPDATE, dst + (c0 + cells - plane) * F8, plane * F8, arg=1),   # update from: top halo
              encode(OP.UPDATE, src + (c0 - plane) * F8, plane * F8, arg=0))           # update to: bottom halo
        src, dst = dst, src
    for a, mt in zip(arrs, [S.TOFROM, S.TO] + [S.TO] * 6):
        p.lit(encode(OP.MAP_EXIT, a, n * F8, arg=mt))
    p.loop([(L.RH, F8, M_LINEAR, src + c0 * F8, 64 * F8, 0)], min(65536, cells // 64))  # sampled output reads
    p.meta = dict(NX=NX, NY=NY, NZ=NZ, words=8 * n)
    return p.finish()


def from_records(name, rec, addr_base, addr_bytes) -> Program:
    """Wrap a host-built trace (configs 1-2) as a literal program."""
    p = Program(name, addr_base, addr_bytes)
    for k in range(0, rec.shape[0], 1 << 16):
        p.lit(*[(int(a), int(b)) for a, b in rec[k:k + (1 << 16)]])
    p.sections.append((addr_base // 8, (addr_base + addr_bytes) // 8, 0))
    return p.finish()
