"""ctypes wrapper of the plain C oracle (TEST INFRASTRUCTURE ONLY).

``replay(records, addr_base, addr_bytes, ...)`` runs ``orc_replay`` from
``arb_oracle.c`` and returns the canonical report triples and the final
shadow.  See ``arb_oracle.h`` for what each field means and which passage of
PAPER.md each step follows.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "arb_oracle.c")
_HDR = os.path.join(_HERE, "arb_oracle.h")
_LIB = os.path.join(_HERE, "liboracle.so")

KIND_NAMES = {1: "UUM", 2: "USD", 3: "MIR", 4: "BO"}


class _Config(ctypes.Structure):
    _fields_ = [("addr_base", ctypes.c_uint64), ("addr_bytes", ctypes.c_uint64),
                ("dedup_first", ctypes.c_int),
                ("tracked_words", ctypes.POINTER(ctypes.c_uint64)),
                ("n_tracked", ctypes.c_uint64), ("detect_bo", ctypes.c_int), ("unified", ctypes.c_int),
                ("n_devices", ctypes.c_int), ("shadow_in", ctypes.c_void_p)]


class _Stats(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in (
        "records", "word_events", "transitions", "control_records",
        "ignored_word_events", "tasks", "error_record")]


REPORT_DTYPE = np.dtype([("word", "<u8"), ("record", "<u8"), ("kind", "<u4"), ("pad", "<u4")])


def build(force: bool = False) -> str:
    """Compile liboracle.so with plain gcc (no CUDA, no shared code)."""
    newest = max(os.path.getmtime(_SRC), os.path.getmtime(_HDR))
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < newest:
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-Wall", "-shared", "-fPIC",
                               "-o", tmp, _SRC, "-lpthread"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        lib.orc_replay.restype = ctypes.c_int
        lib.orc_replay.argtypes = [ctypes.POINTER(_Config), ctypes.c_void_p, ctypes.c_uint64,
                                   ctypes.c_void_p, ctypes.POINTER(ctypes.c_void_p),
                                   ctypes.POINTER(ctypes.c_uint64), ctypes.c_void_p,
                                   ctypes.POINTER(_Stats)]
        lib.orc_replay_sharded.restype = ctypes.c_int
        lib.orc_replay_sharded.argtypes = [ctypes.POINTER(_Config), ctypes.c_void_p, ctypes.c_uint64,
                                           ctypes.c_void_p, ctypes.c_int, ctypes.POINTER(ctypes.c_void_p),
                                           ctypes.POINTER(ctypes.c_uint64), ctypes.c_void_p,
                                           ctypes.POINTER(_Stats)]
        lib.orc_free.argtypes = [ctypes.c_void_p]
        lib.orc_free.restype = None
        _lib = lib
    return _lib


@dataclass
class OracleResult:
    rc: int
    reports: np.ndarray        # structured REPORT_DTYPE, canonical order
    shadow: np.ndarray | None  # uint8 final states (dense range or tracked words)
    stats: dict

    def triples(self):
        return [(int(r["word"]), int(r["record"]), int(r["kind"])) for r in self.reports]


def replay(records: np.ndarray, addr_base: int, addr_bytes: int, *, dedup_first: bool = False,
           tracked_words: np.ndarray | None = None, global_index: np.ndarray | None = None,
           want_shadow: bool = True, detect_bo: bool = False, unified: bool = False,
           n_devices: int = 1, threads: int = 1, shadow_in: np.ndarray | None = None) -> OracleResult:
    """Replay ``records`` (uint64 array of shape (n, 2): w0, w1) through the oracle.
    ``detect_bo``: the buffer-overflow extension (reading Z20).
    ``threads`` > 1: the address-sharded mode (``orc_replay_sharded``: the same
    sequential replay, one thread per contiguous range of tracked words).
    ``shadow_in``: continuation state (the final shadow of a replay of the preceding
    records, cut at a quiescent point); None = every word starts invalid."""
    lib = _load()
    rec = np.ascontiguousarray(records, dtype=np.uint64).reshape(-1, 2)
    n = rec.shape[0]
    cfg = _Config()
    cfg.addr_base = addr_base
    cfg.addr_bytes = addr_bytes
    cfg.dedup_first = 1 if dedup_first else 0
    cfg.detect_bo = 1 if detect_bo else 0
    cfg.unified = 1 if unified else 0
    cfg.n_devices = n_devices
    tw = None
    if tracked_words is not None:
        tw = np.ascontiguousarray(tracked_words, dtype=np.uint64)
        cfg.tracked_words = tw.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))
        cfg.n_tracked = tw.size
        nslots = tw.size
    else:
        nslots = addr_bytes // 8
    sin = None
    if shadow_in is not None:
        sin = np.ascontiguousarray(shadow_in, dtype=np.uint8)
        assert sin.size >= nslots
        cfg.shadow_in = sin.ctypes.data
    gi = None
    if global_index is not None:
        gi = np.ascontiguousarray(global_index, dtype=np.uint64)
        assert gi.size == n
    shadow = np.zeros(max(nslots, 1), dtype=np.uint8) if want_shadow else None
    out = ctypes.c_void_p()
    nout = ctypes.c_uint64()
    st = _Stats()
    args = (ctypes.byref(cfg), rec.ctypes.data if n else None, n, gi.ctypes.data if gi is not None else None)
    tail = (ctypes.byref(out), ctypes.byref(nout), shadow.ctypes.data if shadow is not None else None,
            ctypes.byref(st))
    if threads > 1:
        rc = lib.orc_replay_sharded(*args, threads, *tail)
    else:
        rc = lib.orc_replay(*args, *tail)
    reps = np.zeros(0, dtype=REPORT_DTYPE)
    if rc == 0 and nout.value:
        buf = (ctypes.c_char * (nout.value * REPORT_DTYPE.itemsize)).from_address(out.value)
        reps = np.frombuffer(buf, dtype=REPORT_DTYPE).copy()
    if out.value:
        lib.orc_free(out)
    stats = {name: int(getattr(st, name)) for name, _ in _Stats._fields_}
    if shadow is not None:
        shadow = shadow[:nslots]
    return OracleResult(rc=rc, reports=reps, shadow=shadow, stats=stats)
