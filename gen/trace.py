"""Trace record encoding and a small builder for hand-written traces.

Record layout, two little-endian u64 words:
  w0: [0,48) byte address | [48,56) op | [56,64) arg (map-type / update direction)
  w1: [0,48) length in bytes | [48,64) task id (TASK_BEGIN / TASK_END / SYNC)
"""
from __future__ import annotations

import numpy as np


class OP:
    RH, WH, RT, WT = 0, 1, 2, 3
    MAP_ENTER, MAP_EXIT, UPDATE = 8, 9, 10
    TASK_BEGIN, TASK_END, SYNC = 12, 13, 14
    TASK_DEPEND = 15       # inside a block: depends on the last ended instance of task id k (Z22)
    BASE = 11              # pointer tag k (task field) -> base address (N1, Z25)


class MAP:
    TO, FROM, TOFROM, ALLOC, RELEASE, DELETE = 0, 1, 2, 3, 4, 5
    ALWAYS = 0x10          # map-type modifier bit, or-ed into the map-type (N4, Z21)
    PRESENT = 0x20         # map-type modifier bit: the section must already be mapped (Z21)


class UPD:
    TO, FROM = 0, 1


SYNC_ALL = 0xFFFF
MASK48 = (1 << 48) - 1


def encode(op: int, addr: int = 0, length: int = 0, arg: int = 0, task: int = 0):
    w0 = (addr & MASK48) | ((op & 0xFF) << 48) | ((arg & 0xFF) << 56)
    w1 = (length & MASK48) | ((task & 0xFFFF) << 48)
    return w0, w1


def encode_np(op, addr, length, arg=0, task=0) -> np.ndarray:
    """Vectorised encode; returns an (n, 2) uint64 array."""
    addr = np.asarray(addr, dtype=np.uint64)
    n = addr.size
    out = np.empty((n, 2), dtype=np.uint64)
    out[:, 0] = (addr & np.uint64(MASK48)) | (np.uint64(op & 0xFF) << np.uint64(48)) | \
        (np.asarray(arg, dtype=np.uint64) << np.uint64(56))
    out[:, 1] = (np.asarray(length, dtype=np.uint64) & np.uint64(MASK48)) | \
        (np.asarray(task, dtype=np.uint64) << np.uint64(48))
    return out


class TraceBuilder:
    """Append records; ``array()`` returns an (n, 2) uint64 array.

    Single records are buffered as tuples, vectorised loops as numpy chunks,
    so that traces of ~10^7 records build in well under a second.
    """

    def __init__(self):
        self._chunks: list[np.ndarray] = []
        self._pending: list[tuple[int, int]] = []
        self._n = 0
        self.notes: dict[str, int] = {}

    def __len__(self):
        return self._n

    def _flush_pending(self):
        if self._pending:
            self._chunks.append(np.array(self._pending, dtype=np.uint64).reshape(-1, 2))
            self._pending = []

    def mark(self, name: str) -> int:
        self.notes[name] = self._n
        return self._n

    def _add(self, *a, **k) -> int:
        self._pending.append(encode(*a, **k))
        self._n += 1
        return self._n - 1

    def add_array(self, arr: np.ndarray) -> int:
        self._flush_pending()
        arr = np.asarray(arr, dtype=np.uint64).reshape(-1, 2)
        self._chunks.append(arr)
        start = self._n
        self._n += arr.shape[0]
        return start

    # accesses
    def rh(self, addr, size=8):
        return self._add(OP.RH, addr, size)

    def wh(self, addr, size=8):
        return self._add(OP.WH, addr, size)

    def rt(self, addr, size=8):
        return self._add(OP.RT, addr, size)

    def wt(self, addr, size=8):
        return self._add(OP.WT, addr, size)

    def loop(self, body, n, esz):
        """for i in range(n): for (op, base) in body: op(base + i*esz, esz).

        ``body`` is a list of (op, base_address) pairs; returns the index of
        the first record."""
        k = len(body)
        i = np.arange(n, dtype=np.uint64)
        out = np.empty((n, k, 2), dtype=np.uint64)
        for j, (op, base) in enumerate(body):
            out[:, j, :] = encode_np(op, np.uint64(base) + i * np.uint64(esz), esz)
        return self.add_array(out.reshape(-1, 2))

    # device directives
    def enter(self, maptype, addr, length):
        return self._add(OP.MAP_ENTER, addr, length, arg=maptype)

    def exit(self, maptype, addr, length):
        return self._add(OP.MAP_EXIT, addr, length, arg=maptype)

    def update(self, direction, addr, length):
        return self._add(OP.UPDATE, addr, length, arg=direction)

    def task_begin(self, k):
        return self._add(OP.TASK_BEGIN, task=k)

    def task_end(self, k):
        return self._add(OP.TASK_END, task=k)

    def sync(self, k=SYNC_ALL):
        return self._add(OP.SYNC, task=k)

    def depend(self, k):
        return self._add(OP.TASK_DEPEND, task=k)

    def extend(self, other: "TraceBuilder"):
        base = self._n
        arr = other.array()
        if arr.shape[0]:
            self.add_array(arr)
        for k, v in other.notes.items():
            self.notes[k] = v + base

    def array(self) -> np.ndarray:
        self._flush_pending()
        if not self._chunks:
            return np.zeros((0, 2), dtype=np.uint64)
        if len(self._chunks) > 1:
            self._chunks = [np.concatenate(self._chunks, axis=0)]
        return self._chunks[0]
