"""Host-side address sharding for multi-GPU replay.

A word's VSM state and its race predicate depend only on that word's events
plus the replicated control stream, so the tracked address range splits into
contiguous shards, one per rank: rank r owns words [lo + r*W/P, lo + (r+1)*W/P).
Each rank receives every control record and the access records that touch its
words (a record straddling a shard edge goes to both owners, each updates only
its own word), in global order, with their global record indices.  The only
data exchanged between ranks is the per-rank report count (ncclAllGather inside
arb_flush); the global report set is the concatenation of the rank slices in
rank order, which is already canonical (word-major).
"""
from __future__ import annotations

import ctypes

import numpy as np

MASK48 = (1 << 48) - 1


def shard_range(word_lo: int, n_words: int, rank: int, world: int):
    """Word range [lo, hi) owned by `rank` (8-byte aligned byte range = 8*lo, 8*hi)."""
    per = -(-n_words // world)
    lo = word_lo + rank * per
    hi = min(word_lo + n_words, lo + per)
    return lo, max(lo, hi)


def shard_records(records: np.ndarray, word_lo: int, word_hi: int, first_index: int = 0):
    """Order-preserving selection of the records a shard needs (host numpy version).
    Returns (records, global_index)."""
    rec = np.asarray(records, dtype=np.uint64).reshape(-1, 2)
    op = (rec[:, 0] >> np.uint64(48)) & np.uint64(0xFF)
    addr = rec[:, 0] & np.uint64(MASK48)
    ln = rec[:, 1] & np.uint64(MASK48)
    x0 = addr >> np.uint64(3)
    x1 = (addr + np.maximum(ln, np.uint64(1)) - np.uint64(1)) >> np.uint64(3)
    keep = (op >= 4) | ((x1 >= np.uint64(word_lo)) & (x0 < np.uint64(word_hi)))
    idx = np.nonzero(keep)[0].astype(np.uint64)
    return rec[keep], idx + np.uint64(first_index)


def merge_rank_reports(per_rank: list) -> list:
    """Global report list = rank slices concatenated in rank order."""
    out = []
    for r in per_rank:
        out.extend(r)
    return out


def nccl_unique_id() -> bytes:
    """ncclGetUniqueId() from the NCCL runtime torch ships (128 bytes)."""
    import os
    import torch
    cands = ["libnccl.so.2"]
    try:
        import nvidia.nccl
        d = os.path.join(os.path.dirname(nvidia.nccl.__file__), "lib", "libnccl.so.2")
        cands.insert(0, d)
    except Exception:
        pass
    lib = None
    for c in cands:
        try:
            lib = ctypes.CDLL(c, mode=ctypes.RTLD_GLOBAL)
            break
        except OSError:
            continue
    if lib is None:
        raise RuntimeError("libnccl.so.2 not found")
    buf = ctypes.create_string_buffer(128)
    rc = lib.ncclGetUniqueId(buf)
    if rc != 0:
        raise RuntimeError(f"ncclGetUniqueId failed: {rc}")
    del torch
    return buf.raw
