"""Trace record format shared by every producer of synthetic input.

This module holds the *input format only* (the paper's queue record,
PAPER.md L1064-1070, §4.2: "Each record contains fields identifying the
warp, the operation, a 32-bit mask of active threads, and 32 entries for the
addresses accessed by each thread in the warp ... a fixed 16 + 8 x 32 = 272
bytes") plus geometry helpers.  It contains none of the race-detection
arithmetic: it is consumed by both the oracle (test infrastructure) and the
CUDA path, which never share code with each other.

Layout (little endian, 272 B, 8-B aligned):

    off  size  field
      0     4  warp        global warp id = block_linear * warps_per_block + warp_in_block
      4     4  mask        bit i = lane i active
      8     1  op          BC_OP_* below
      9     1  space       0 = GLOBAL, 1 = SHARED (offset within the block's smem)
     10     1  size_log2   access width 2^k bytes, k in 0..4
     11     1  flags       bit0 SAME_VALUE (all active lanes store one value)
     12     4  aux         IF: then-lane mask; otherwise 0
     16   256  addr[32]    per-lane byte address (unused lanes 0)
"""
from __future__ import annotations

import numpy as np

RECORD_BYTES = 272
WARP = 32

# operations (paper §3.1); FENCE is a standalone fence
# (no trace op); BAR is one warp's arrival at bar.sync.
OP_LD, OP_ST, OP_ATOM = 0, 1, 2
OP_ACQ_BLK, OP_ACQ_GLB, OP_REL_BLK, OP_REL_GLB, OP_AR_BLK, OP_AR_GLB = 3, 4, 5, 6, 7, 8
OP_FENCE, OP_BAR, OP_IF, OP_ELSE, OP_FI = 9, 10, 11, 12, 13
OP_NAMES = ["LD", "ST", "ATOM", "ACQ_BLK", "ACQ_GLB", "REL_BLK", "REL_GLB",
            "AR_BLK", "AR_GLB", "FENCE", "BAR", "IF", "ELSE", "FI"]
MEM_OPS = (OP_LD, OP_ST, OP_ATOM)
SYNC_OPS = (OP_ACQ_BLK, OP_ACQ_GLB, OP_REL_BLK, OP_REL_GLB, OP_AR_BLK, OP_AR_GLB)
CTRL_OPS = (OP_FENCE, OP_BAR, OP_IF, OP_ELSE, OP_FI)

SPACE_GLOBAL, SPACE_SHARED, SPACE_NONE = 0, 1, 2
FLAG_SAME_VALUE = 1

# race record (32 B), see include/bc.h
KIND_NAMES = ["WW", "WR", "RW", "WA", "AW", "RA", "AR"]
CLS_NAMES = ["SAME_INSN", "BRANCH", "INTRA_BLOCK", "INTER_BLOCK", "BARRIER_DIVERGENCE"]
KIND_NONE = 0xFF

RECORD_DTYPE = np.dtype([
    ("warp", "<u4"), ("mask", "<u4"), ("op", "u1"), ("space", "u1"),
    ("size_log2", "u1"), ("flags", "u1"), ("aux", "<u4"), ("addr", "<u8", (32,)),
])
assert RECORD_DTYPE.itemsize == RECORD_BYTES

RACE_DTYPE = np.dtype([
    ("addr", "<u8"), ("prior_event", "<u8"), ("cur_event", "<u8"),
    ("kind", "u1"), ("cls", "u1"), ("space", "u1"), ("pad", "u1"), ("block", "<u4"),
])
assert RACE_DTYPE.itemsize == 32

GLOBAL_BASE = 0x7F00_0000_0000


class Geometry:
    """Launch geometry (grid of blocks, blocks of warps of
    up to 32 threads; x fastest).  The last warp of a block may be partial
    (P:L451-456)."""

    def __init__(self, grid=(1, 1, 1), block=(32, 1, 1), smem_bytes=0, granule_log2=2):
        grid = tuple(grid) + (1,) * (3 - len(grid))
        block = tuple(block) + (1,) * (3 - len(block))
        self.grid, self.block = grid, block
        self.n_blocks = grid[0] * grid[1] * grid[2]
        self.tpb = block[0] * block[1] * block[2]
        assert 1 <= self.tpb <= 1024
        self.wpb = (self.tpb + WARP - 1) // WARP
        self.n_warps = self.n_blocks * self.wpb
        self.n_threads = self.n_blocks * self.tpb
        self.smem_bytes = smem_bytes
        self.granule_log2 = granule_log2

    def init_mask(self, w: int) -> int:
        wib = w % self.wpb
        lanes = min(WARP, self.tpb - wib * WARP)
        return (1 << lanes) - 1 if lanes < 32 else 0xFFFFFFFF

    def block_of_warp(self, w: int) -> int:
        return w // self.wpb

    def warp_id(self, block: int, wib: int) -> int:
        return block * self.wpb + wib

    def tid(self, w: int, lane: int) -> int:
        return (w // self.wpb) * self.tpb + (w % self.wpb) * WARP + lane

    def as_dict(self):
        return dict(grid=self.grid, block=self.block, smem_bytes=self.smem_bytes,
                    granule_log2=self.granule_log2)


def popc(x: int) -> int:
    return bin(x & 0xFFFFFFFF).count("1")


def count_events(recs: np.ndarray):
    """(lane_events, control_events) per SURVEY §8(d.1): a lane event is one
    active lane of a LD/ST/ATOM/ACQ*/REL*/AR* record; a control event is one
    IF/ELSE/FI/BAR/FENCE record."""
    ops = recs["op"]
    masks = recs["mask"].astype(np.uint64)
    pc = np.zeros(len(recs), dtype=np.int64)
    m = masks.copy()
    # popcount via bit tricks on uint64
    for _ in range(32):
        pc += (m & 1).astype(np.int64)
        m >>= np.uint64(1)
    lane_sel = ops <= OP_AR_GLB
    return int(pc[lane_sel].sum()), int((~lane_sel).sum())
