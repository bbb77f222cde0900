"""Warp-size simulation input transform ("in future we could
simulate the behavior of smaller/larger warps to find additional latent bugs").

A trace recorded with 32-lane warps is re-split into virtual warps of `ws` lanes (4, 8 or 16): the
physical record (warp w, mask m) becomes, in trace order, one record per virtual warp j of w whose
lanes it touches -- warp (block, (w_in_block * 32 + j * ws) / ws), mask (m >> j*ws) & (2^ws - 1),
addresses addr[j*ws ...].  The virtual warps of one physical instruction run one after the other,
with no lock-step (endi) join between them, so accesses that warp-synchronous code orders only by
executing in one 32-wide warp become concurrent.

Control flow per virtual warp follows its own SIMT stack: an IF whose mask has none of the virtual
warp's lanes is not executed by it, and neither are the matching ELSE / FI nor anything nested.
A BAR that a virtual warp does not reach (mask without its lanes) makes the simulated trace
infeasible -- that is itself a warp-size assumption (barrier inside warp-divergent code).

This is input preparation only (no race arithmetic); both the oracle and the CUDA path consume the
transformed trace with geometry warp_size = ws.  `origin[i]` maps record i of the result back to
(original record, first lane) so a race can be reported against the recorded trace.
"""
from __future__ import annotations

import numpy as np

from .format import RECORD_DTYPE

OP_IF, OP_ELSE, OP_FI = 11, 12, 13


def split_warps(records: np.ndarray, geom: dict, ws: int):
    """Return (records, geometry, origin[n, 2] = (source record, lane offset))."""
    if ws not in (4, 8, 16, 32):
        raise ValueError("warp size must be 4, 8, 16 or 32")
    g2 = dict(geom)
    g2["warp_size"] = ws
    if ws == 32:
        org = np.stack([np.arange(len(records)), np.zeros(len(records), dtype=np.int64)], axis=1)
        return records.copy(), g2, org
    tpb = int(np.prod(geom["block"]))
    wpb32 = (tpb + 31) // 32
    wpb = (tpb + ws - 1) // ws
    k = 32 // ws
    lm = (1 << ws) - 1
    live = {}  # (physical warp, j) -> stack of "this virtual warp executes the construct"
    out, org = [], []
    for i, r in enumerate(records):
        w, m, op, aux = int(r["warp"]), int(r["mask"]), int(r["op"]), int(r["aux"])
        b, wib = divmod(w, wpb32)
        for j in range(k):
            first = wib * 32 + j * ws
            if first >= tpb:
                break
            st = live.setdefault((w, j), [True])
            sm = (m >> (j * ws)) & lm
            if op == OP_IF:
                run = st[-1] and sm != 0
                st.append(run)
            elif op == OP_ELSE:
                run = st[-1]
            elif op == OP_FI:
                run = st.pop()
            else:
                run = sm != 0
            if not run:
                continue
            n = np.zeros(1, dtype=RECORD_DTYPE)[0]
            n["warp"] = b * wpb + first // ws
            n["mask"] = sm
            n["op"], n["space"], n["size_log2"], n["flags"] = r["op"], r["space"], r["size_log2"], r["flags"]
            n["aux"] = (aux >> (j * ws)) & lm if op == OP_IF else 0
            n["addr"][:ws] = r["addr"][j * ws:(j + 1) * ws]
            out.append(n)
            org.append((i, j * ws))
    recs = np.array(out, dtype=RECORD_DTYPE) if out else np.zeros(0, dtype=RECORD_DTYPE)
    return recs, g2, np.array(org, dtype=np.int64).reshape(-1, 2)
