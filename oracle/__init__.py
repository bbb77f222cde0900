"""oracle — TEST INFRASTRUCTURE ONLY.

Plain CPU reference for the BARRACUDA race check (§3, Fig. 2/3) on
uncompressed per-thread vector clocks (oracle.cpp), plus a brute-force
transitive-closure checker of the §3.2 definition (bf.py).  Only tests/,
__graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
may import this package; the product path never does.

Pinned by tests/test_oracle_*.py.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")

RACE_DTYPE = np.dtype([
    ("addr", "<u8"), ("prior_event", "<u8"), ("cur_event", "<u8"),
    ("kind", "u1"), ("cls", "u1"), ("space", "u1"), ("pad", "u1"), ("block", "<u4"),
])

F_RELEASE_OVERWRITE = 1
F_NO_SAME_VALUE_FILTER = 2
F_CHECK_INVARIANT = 0x100

OK, INVALID_ARG, INFEASIBLE, INVARIANT_VIOLATED = 0, -1, -2, -100


class _Geom(ctypes.Structure):
    _fields_ = [("grid", ctypes.c_uint32 * 3), ("block", ctypes.c_uint32 * 3),
                ("warp_size", ctypes.c_uint32), ("granule_log2", ctypes.c_uint32),
                ("smem_bytes", ctypes.c_uint32), ("flags", ctypes.c_uint32)]


class _Result(ctypes.Structure):
    _fields_ = [("races", ctypes.c_void_p), ("n_races", ctypes.c_uint64),
                ("lane_events", ctypes.c_uint64), ("control_events", ctypes.c_uint64)]


_lib = None


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run __graft_entry__.build()")
        lib = ctypes.CDLL(LIB_PATH)
        lib.oracle_detect.restype = ctypes.c_int
        lib.oracle_detect.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.POINTER(_Geom),
                                      ctypes.POINTER(_Result)]
        lib.oracle_detect_values.restype = ctypes.c_int
        lib.oracle_detect_values.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.POINTER(_Geom),
                                             ctypes.c_void_p, ctypes.POINTER(_Result)]
        lib.oracle_free.argtypes = [ctypes.c_void_p]
        _lib = lib
    return _lib


def detect(records: np.ndarray, grid=(1, 1, 1), block=(32, 1, 1), smem_bytes=0, granule_log2=2,
           flags=0, warp_size=32, values=None):
    """Run the oracle.  Returns (status, races[RACE_DTYPE], stats dict).  values: optional uint64
    array [n_records, 32] of per-lane store values (reading R6b)."""
    lib = _load()
    g = _Geom()
    grid = tuple(grid) + (1,) * (3 - len(grid))
    block = tuple(block) + (1,) * (3 - len(block))
    for i in range(3):
        g.grid[i], g.block[i] = grid[i], block[i]
    g.warp_size, g.granule_log2, g.smem_bytes, g.flags = warp_size, granule_log2, smem_bytes, flags
    recs = np.ascontiguousarray(records)
    res = _Result()
    vals = None if values is None else np.ascontiguousarray(values, dtype=np.uint64).reshape(-1)
    if vals is not None and len(vals) != 32 * len(recs):
        raise ValueError("values must hold 32 entries per record")
    st = lib.oracle_detect_values(recs.ctypes.data if len(recs) else None, len(recs), ctypes.byref(g),
                                  vals.ctypes.data if vals is not None and len(vals) else None, ctypes.byref(res))
    races = np.zeros(res.n_races, dtype=RACE_DTYPE)
    if res.n_races:
        ctypes.memmove(races.ctypes.data, res.races, res.n_races * 32)
        lib.oracle_free(res.races)
    return st, races, dict(lane_events=res.lane_events, control_events=res.control_events)


def detect_geom(records, geom: dict, flags=0, values=None):
    return detect(records, grid=geom["grid"], block=geom["block"], smem_bytes=geom["smem_bytes"],
                  granule_log2=geom.get("granule_log2", 2), flags=flags, values=values,
                  warp_size=geom.get("warp_size", 32))
