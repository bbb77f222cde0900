"""TraceBuilder: hand-author feasible traces in the paper's record format.

Records are appended in global trace order (the order of the calls).  The
builder keeps a per-warp stack of active masks only so that it can fill in
the ``mask`` field of each record the way the hardware would (feasibility,
PAPER.md L360-366: a warp instruction is logged with exactly its active lanes;
branches are logged as if/else/fi).  It performs no race analysis.
"""
from __future__ import annotations

from typing import Callable, Dict, Iterable, Optional, Union

import numpy as np

from .format import (FLAG_SAME_VALUE, GLOBAL_BASE, OP_ACQ_BLK, OP_ACQ_GLB, OP_AR_BLK,
                     OP_AR_GLB, OP_ATOM, OP_BAR, OP_ELSE, OP_FENCE, OP_FI, OP_IF, OP_LD,
                     OP_REL_BLK, OP_REL_GLB, OP_ST, RECORD_DTYPE, SPACE_GLOBAL,
                     SPACE_SHARED, Geometry)

Addrs = Union[Callable[[int], int], Dict[int, int], Iterable[Optional[int]], int]

_SIZE_LOG2 = {1: 0, 2: 1, 4: 2, 8: 3, 16: 4}


class TraceBuilder:
    def __init__(self, grid=(1, 1, 1), block=(32, 1, 1), smem_bytes=16384, granule_log2=2):
        self.geom = Geometry(grid, block, smem_bytes, granule_log2)
        self._stacks = {}
        self._rows = []

    # ---------------------------------------------------------------- helpers
    def top(self, w: int) -> int:
        st = self._stacks.setdefault(w, [self.geom.init_mask(w)])
        return st[-1]

    def warp(self, block: int, wib: int = 0) -> int:
        return self.geom.warp_id(block, wib)

    def _addr_list(self, mask: int, addrs: Addrs):
        out = [0] * 32
        for lane in range(32):
            if not (mask >> lane) & 1:
                continue
            if callable(addrs):
                a = addrs(lane)
            elif isinstance(addrs, dict):
                a = addrs[lane]
            elif isinstance(addrs, int):
                a = addrs
            else:
                a = list(addrs)[lane]
            assert a is not None, f"lane {lane} active but no address"
            out[lane] = int(a)
        return out

    def raw(self, warp: int, mask: int, op: int, space: int = 0, size_log2: int = 2,
            flags: int = 0, aux: int = 0, addrs=None):
        """Append a record verbatim (no stack bookkeeping): used to author
        infeasible traces in tests."""
        addr = [0] * 32 if addrs is None else self._addr_list(mask, addrs)
        self._rows.append((warp, mask & 0xFFFFFFFF, op, space, size_log2, flags, aux & 0xFFFFFFFF, addr))

    def _emit(self, w, op, space=0, size=4, flags=0, aux=0, addrs=None, mask=None):
        m = self.top(w) if mask is None else mask
        addr = [0] * 32 if addrs is None else self._addr_list(m, addrs)
        self._rows.append((w, m, op, space, _SIZE_LOG2[size], flags, aux & 0xFFFFFFFF, addr))
        return len(self._rows) - 1

    # ------------------------------------------------------------ memory ops
    def ld(self, w, addrs: Addrs, space=SPACE_GLOBAL, size=4):
        return self._emit(w, OP_LD, space, size, 0, 0, addrs)

    def st(self, w, addrs: Addrs, space=SPACE_GLOBAL, size=4, same_value=False):
        return self._emit(w, OP_ST, space, size, FLAG_SAME_VALUE if same_value else 0, 0, addrs)

    def atom(self, w, addrs: Addrs, space=SPACE_GLOBAL, size=4):
        return self._emit(w, OP_ATOM, space, size, 0, 0, addrs)

    # -------------------------------------------------------------- sync ops
    def acq(self, w, addrs: Addrs, scope="glb", space=SPACE_GLOBAL):
        return self._emit(w, OP_ACQ_GLB if scope == "glb" else OP_ACQ_BLK, space, 4, 0, 0, addrs)

    def rel(self, w, addrs: Addrs, scope="glb", space=SPACE_GLOBAL):
        return self._emit(w, OP_REL_GLB if scope == "glb" else OP_REL_BLK, space, 4, 0, 0, addrs)

    def ar(self, w, addrs: Addrs, scope="glb", space=SPACE_GLOBAL):
        return self._emit(w, OP_AR_GLB if scope == "glb" else OP_AR_BLK, space, 4, 0, 0, addrs)

    def fence(self, w):
        return self._emit(w, OP_FENCE)

    def bar(self, w):
        return self._emit(w, OP_BAR)

    # --------------------------------------------------------------- branches
    def if_(self, w, then_lanes):
        """then_lanes: bit mask or iterable of lanes taking the then path."""
        if not isinstance(then_lanes, int):
            m = 0
            for l in then_lanes:
                m |= 1 << l
            then_lanes = m
        top = self.top(w)
        then = top & then_lanes
        idx = self._emit(w, OP_IF, aux=then)
        st = self._stacks[w]
        st.append(top & ~then & 0xFFFFFFFF)  # else entry pushed first
        st.append(then)
        return idx

    def else_(self, w):
        idx = self._emit(w, OP_ELSE)
        self._stacks[w].pop()
        return idx

    def fi(self, w):
        idx = self._emit(w, OP_FI)
        self._stacks[w].pop()
        return idx

    # ------------------------------------------------------------------ output
    def __len__(self):
        return len(self._rows)

    def records(self) -> np.ndarray:
        a = np.zeros(len(self._rows), dtype=RECORD_DTYPE)
        for i, (w, m, op, sp, sl, fl, aux, addr) in enumerate(self._rows):
            a[i]["warp"], a[i]["mask"], a[i]["op"], a[i]["space"] = w, m, op, sp
            a[i]["size_log2"], a[i]["flags"], a[i]["aux"] = sl, fl, aux
            a[i]["addr"] = addr
        return a


def gaddr(i: int, elem: int = 4) -> int:
    """Address of element i of a synthetic global array."""
    return GLOBAL_BASE + i * elem
