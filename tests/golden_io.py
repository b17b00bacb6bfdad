"""Reader for the hand-written golden trace fixtures in tests/golden/*.trace."""
from __future__ import annotations

import os

import numpy as np

from gen.trace import OP, MAP, UPD, encode

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
KINDS = {"UUM": 1, "USD": 2, "MIR": 3}


def load(name):
    path = os.path.join(GOLDEN, name)
    recs, expect = [], []
    base = size = None
    mode = None
    with open(path) as fh:
        for raw in fh:
            line = raw.split("#", 1)[0].strip()
            if not line:
                continue
            tok = line.split()
            if tok[0] == "addr_base":
                base = int(tok[1], 0)
            elif tok[0] == "addr_bytes":
                size = int(tok[1], 0)
            elif tok[0] in ("records", "expect"):
                mode = tok[0]
            elif mode == "records":
                op = tok[0]
                if op in ("RH", "WH", "RT", "WT"):
                    recs.append(encode(getattr(OP, op), int(tok[1], 0), int(tok[2], 0)))
                elif op in ("MAP_ENTER", "MAP_EXIT"):
                    recs.append(encode(getattr(OP, op), int(tok[2], 0), int(tok[3], 0),
                                       arg=getattr(MAP, tok[1])))
                elif op == "UPDATE":
                    recs.append(encode(OP.UPDATE, int(tok[2], 0), int(tok[3], 0),
                                       arg=getattr(UPD, tok[1])))
                elif op in ("TASK_BEGIN", "TASK_END", "SYNC"):
                    recs.append(encode(getattr(OP, op), task=int(tok[1], 0)))
                else:
                    raise ValueError(line)
            elif mode == "expect":
                expect.append((int(tok[0], 0), int(tok[1], 0), KINDS[tok[2]]))
    arr = np.array(recs, dtype=np.uint64).reshape(-1, 2)
    return arr, base, size, sorted(expect)
