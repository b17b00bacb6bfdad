"""ctypes binding of libarbalest.so — argument marshalling only.

Every step of the replay runs inside the library (include/arbalest.h).  There
is no CPU fallback: if the shared library is missing or cannot be loaded,
``load()`` raises.  torch is used only for device memory and streams.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(PKG, "libarbalest.so")

ARB_OK, ARB_TRUNCATED = 0, 1
ARB_EINVAL, ARB_ENOMEM, ARB_ECUDA, ARB_EMAP, ARB_ETRACE, ARB_ESTATE, ARB_EOPEN = -1, -2, -3, -4, -5, -6, -7
ARB_EPEER = -8
ARB_F_DEDUP_FIRST, ARB_F_TIMING = 0x1, 0x2
ARB_F_SMALL_PARTS = 0x4
ARB_F_BO = 0x8          # buffer-overflow extension (Z20)
ARB_BO = 4
ARB_F_UNIFIED = 0x10    # unified memory (Z23)


def ARB_F_DEVICES(n):
    """n accelerators (Z24), n <= 3."""
    return (n - 1) << 8
STATUS = {0: "ARB_OK", 1: "ARB_TRUNCATED", -1: "ARB_EINVAL", -2: "ARB_ENOMEM", -3: "ARB_ECUDA",
          -4: "ARB_EMAP", -5: "ARB_ETRACE", -6: "ARB_ESTATE", -7: "ARB_EOPEN", -8: "ARB_EPEER"}
EXPORTS = ("arb_init", "arb_submit_events", "arb_flush", "arb_get_reports", "arb_get_shadow",
           "arb_get_stats", "arb_last_error", "arb_destroy")


class arb_config(ctypes.Structure):
    _fields_ = [("addr_base", ctypes.c_uint64), ("addr_bytes", ctypes.c_uint64),
                ("device", ctypes.c_int), ("rank", ctypes.c_int), ("world", ctypes.c_int),
                ("nccl_unique_id", ctypes.c_void_p), ("report_capacity", ctypes.c_uint64),
                ("flags", ctypes.c_uint32), ("bucket_bits", ctypes.c_uint32)]


class arb_stats(ctypes.Structure):
    _fields_ = [("records", ctypes.c_uint64), ("access_words", ctypes.c_uint64),
                ("range_words", ctypes.c_uint64), ("control_records", ctypes.c_uint64),
                ("range_ops", ctypes.c_uint64), ("tasks", ctypes.c_uint64),
                ("reports", ctypes.c_uint64), ("reports_by_kind", ctypes.c_uint64 * 4),
                ("ignored_words", ctypes.c_uint64), ("buckets", ctypes.c_uint64),
                ("bucket_bits", ctypes.c_uint64), ("max_bucket_events", ctypes.c_uint64),
                ("total_records", ctypes.c_uint64), ("total_word_events", ctypes.c_uint64),
                ("total_reports", ctypes.c_uint64), ("flushes", ctypes.c_uint64),
                ("ms_partition", ctypes.c_double), ("ms_control", ctypes.c_double),
                ("ms_replay", ctypes.c_double), ("ms_mir", ctypes.c_double),
                ("ms_reports", ctypes.c_double), ("ms_total", ctypes.c_double),
                ("kernel_launches", ctypes.c_uint64), ("ms_sample", ctypes.c_double),
                ("steps_fast", ctypes.c_uint64), ("steps_sort", ctypes.c_uint64),
                ("ms_segsort", ctypes.c_double), ("ms_host_control", ctypes.c_double),
                ("work_items", ctypes.c_uint64), ("hot_buckets", ctypes.c_uint64),
                ("reports_bo", ctypes.c_uint64), ("nccl_ranks", ctypes.c_uint64),
                ("exchanges", ctypes.c_uint64), ("steps_run", ctypes.c_uint64),
                ("segments", ctypes.c_uint64), ("chunks", ctypes.c_uint64),
                ("chunks_fast", ctypes.c_uint64), ("chunks_run", ctypes.c_uint64),
                ("run_merges", ctypes.c_uint64)]

    def as_dict(self):
        d = {}
        for name, _ in self._fields_:
            v = getattr(self, name)
            d[name] = list(v) if name == "reports_by_kind" else v
        return d


_lib = None


def load():
    """Load libarbalest.so (build it first with paper_conf_ipps_yuphs21_b200.build)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
    lib = ctypes.CDLL(LIB_PATH)
    vp, u64, i32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int
    sig = {
        "arb_init": ([ctypes.POINTER(arb_config), ctypes.POINTER(vp)], i32),
        "arb_submit_events": ([vp, vp, u64, vp, i32, vp], i32),
        "arb_flush": ([vp, vp, ctypes.POINTER(u64), ctypes.POINTER(u64)], i32),
        "arb_get_reports": ([vp, vp, u64, ctypes.POINTER(u64), i32], i32),
        "arb_get_shadow": ([vp, u64, u64, vp, i32], i32),
        "arb_get_stats": ([vp, ctypes.POINTER(arb_stats)], i32),
        "arb_last_error": ([vp], ctypes.c_char_p),
        "arb_destroy": ([vp], i32),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    _lib = lib
    return lib


class ArbError(RuntimeError):
    def __init__(self, rc, msg):
        super().__init__(f"{STATUS.get(rc, rc)}: {msg}")
        self.rc = rc


def _ptr(x):
    """Device/host pointer of a torch tensor or numpy array (or an int)."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    return x.data_ptr()  # torch.Tensor


def _on_device(x):
    return 0 if isinstance(x, np.ndarray) else int(getattr(x, "is_cuda", False))


class Context:
    """One arb_ctx.  Methods mirror the C ABI one to one."""

    def __init__(self, addr_base, addr_bytes, device=0, rank=0, world=1, nccl_unique_id=None,
                 report_capacity=0, flags=0, bucket_bits=0):
        self.lib = load()
        self._nccl_id = nccl_unique_id  # keep the bytes alive
        cfg = arb_config(addr_base, addr_bytes, device, rank, world,
                         ctypes.cast(ctypes.c_char_p(nccl_unique_id), ctypes.c_void_p) if nccl_unique_id else None,
                         report_capacity, flags, bucket_bits)
        h = ctypes.c_void_p()
        rc = self.lib.arb_init(ctypes.byref(cfg), ctypes.byref(h))
        if rc != ARB_OK:
            raise ArbError(rc, "arb_init failed")
        self.h = h
        self.addr_base, self.addr_bytes = addr_base, addr_bytes

    def _check(self, rc, allow=(ARB_OK,)):
        if rc not in allow:
            raise ArbError(rc, self.lib.arb_last_error(self.h).decode())
        return rc

    def submit_events(self, ev, n=None, global_index=None, stream=None, check=True):
        n = (ev.shape[0] if n is None else n)
        rc = self.lib.arb_submit_events(self.h, _ptr(ev), n, _ptr(global_index), _on_device(ev),
                                        _ptr_stream(stream))
        return self._check(rc) if check else rc

    def flush(self, stream=None, check=True):
        nloc, off = ctypes.c_uint64(), ctypes.c_uint64()
        rc = self.lib.arb_flush(self.h, _ptr_stream(stream), ctypes.byref(nloc), ctypes.byref(off))
        if check:
            self._check(rc, (ARB_OK, ARB_TRUNCATED))
        return rc, nloc.value, off.value

    def get_reports(self, cap=None, out=None):
        """Returns an (n, 2) uint64 array [w0, w1] (host) unless `out` is given."""
        if cap is None:
            cap = self.stats()["reports"]
        if out is None:
            out = np.zeros((max(cap, 1), 2), dtype=np.uint64)
        nw = ctypes.c_uint64()
        rc = self.lib.arb_get_reports(self.h, _ptr(out), cap, ctypes.byref(nw), _on_device(out))
        self._check(rc, (ARB_OK, ARB_TRUNCATED))
        return out[:nw.value]

    def get_shadow(self, word_lo, n):
        out = np.zeros(max(n, 1), dtype=np.uint8)
        self._check(self.lib.arb_get_shadow(self.h, word_lo, n, out.ctypes.data, 0))
        return out[:n]

    def stats(self):
        st = arb_stats()
        self._check(self.lib.arb_get_stats(self.h, ctypes.byref(st)))
        return st.as_dict()

    def last_error(self):
        return self.lib.arb_last_error(self.h).decode()

    def close(self):
        if getattr(self, "h", None):
            self.lib.arb_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _ptr_stream(stream):
    if stream is None:
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream  # torch.cuda.Stream


def reports_to_triples(rep: np.ndarray):
    """(n, 2) arb_report array -> list of (word, record, kind)."""
    rep = np.asarray(rep, dtype=np.uint64).reshape(-1, 2)
    w = rep[:, 0] & np.uint64((1 << 48) - 1)
    k = (rep[:, 0] >> np.uint64(48)) & np.uint64(0xFF)
    return list(zip(w.tolist(), rep[:, 1].tolist(), k.tolist()))
