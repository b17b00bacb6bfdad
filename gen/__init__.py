"""Seeded synthetic trace generators (shared by tests, bench and both sides).

This package only *writes trace records* in the format of DESIGN.md §3; it
holds none of the method's arithmetic (no state machine, no reference
counting, no race predicate).  Random numbers come from a counter-based
splitmix64 keyed by (seed, counter) so that host (numpy / C) and device
(CUDA, ``gen/arbgen.cuh``) produce identical bytes.
"""
from .trace import TraceBuilder, OP, MAP, UPD, SYNC_ALL, encode  # noqa: F401
