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

    def distinct_words(self, lo, hi, ranges):
        """W of B_alg for each global record range: the union of the mapped sections
        entered in the range, clipped to the tracked words [lo, hi).  Every access
        of these programs lies inside a section of its own region."""
        secs = np.array(self.sections, dtype=np.uint64).reshape(-1, 3)
        out = []
        for g0, g1 in ranges:
            m = (secs[:, 2] >= g0) & (secs[:, 2] < g1)
            a = np.maximum(secs[m, 0], np.uint64(lo)).astype(np.int64)
            b = np.minimum(secs[m, 1], np.uint64(hi)).astype(np.int64)
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
