"""B200-native ARBALEST replay: libarbalest.so (sm_100a kernels + C ABI) and its binding.

The package holds only the hot path: ``csrc/`` (CUDA kernels, host control
plane, C ABI), ``binding.py`` (ctypes marshalling), ``build.py`` (nvcc build)
and ``shard.py`` (host-side address sharding of traces for multi-GPU runs).
"""
from .binding import (Context, ArbError, load, reports_to_triples, EXPORTS,  # noqa: F401
                      ARB_OK, ARB_TRUNCATED, ARB_EINVAL, ARB_ENOMEM, ARB_ECUDA, ARB_EMAP,
                      ARB_ETRACE, ARB_ESTATE, ARB_EOPEN, ARB_EPEER, ARB_F_DEDUP_FIRST, ARB_F_TIMING,
                      ARB_F_SMALL_PARTS, ARB_F_BO, ARB_BO, ARB_F_UNIFIED, ARB_F_DEVICES)
