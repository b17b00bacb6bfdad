"""ARBALEST CPU oracle — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  The product path
(``paper_conf_ipps_yuphs21_b200``) never imports it and shares no code with it.

The oracle is plain sequential C (``arb_oracle.c``) following the paper
(Definition 1, Table I, P:255-263 VSM, P:289-292
Theorem 1, Table II) one record and one word-op at a time.
"""
from .oracle import build, replay, OracleResult, KIND_NAMES  # noqa: F401
