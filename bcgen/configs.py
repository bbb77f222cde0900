"""The five synthetic workloads of BASELINE.json `configs`.

C1 is authored directly with TraceBuilder (it is ~140 records).  C2-C5 are
produced by the C++ generator in gen.cpp (libbcgen.so, built by
__graft_entry__.build()).  Every config is a deterministic function of
(config, seed, overrides).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from .builder import TraceBuilder
from .format import GLOBAL_BASE, RACE_DTYPE, RECORD_DTYPE, SPACE_GLOBAL, SPACE_SHARED

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libbcgen.so")

CONFIGS = {
    "c1": "single litmus trace: 2 blocks x 32 threads, shared array with __syncthreads plus one "
          "atomic-flag/threadfence handoff and one unsynchronized write (~2K events)",
    "c2": "shared-memory stencil trace: 256 blocks x 256 threads, __syncthreads-heavy, ~10M events, race-free",
    "c3": "threadFenceReduction-style trace: 4096 blocks x 256 threads, global atomics + __threadfence, ~50M events",
    "c4": "irregular BFS-like trace: 1M threads, random global addresses, atomics and injected races, ~200M events",
    "c5": "scale trace: 4M threads, ~1B events",
    "c6": "lock-heavy hashtable trace (SURVEY row f2, P:L1522-1535): 256 blocks x 128 threads, 2 inserts "
          "per thread under per-bucket locks, with both section-6.3 bugs (CAS without fence, unlock by plain "
          "store); bug=0 is the fixed program",
    "c6f": "lock-heavy hashtable trace, fixed program (every lock an atomicCAS + fence acquire and a fence + "
           "atomicExch release; race-free): 256 blocks x 128 threads, 2 inserts per thread",
}


def make_c1(with_sync: bool = True, rounds: int = 16):
    """C1 litmus: per block 16 rounds of {st.shared s[lane];
    BAR; ld.shared s[(lane+1)%32]; BAR}.  Block 0 then st.global data[lane];
    IF(lane==0){REL_GLB flag}; IF(lane==5){st.global g[0]}.  Block 1 (after
    block 0's release in trace order) IF(lane==0){ACQ_GLB flag}; ld.global
    data[lane]; IF(lane==5){st.global g[0]}.  Expected: exactly one race on
    g[0] (WW, INTER_BLOCK, GLOBAL); without the flag handoff +32 WR races on
    data[].  Returns (records, TraceBuilder)."""
    tb = TraceBuilder(grid=(2, 1, 1), block=(32, 1, 1), smem_bytes=128)
    w0, w1 = tb.warp(0), tb.warp(1)
    data = GLOBAL_BASE
    flag = GLOBAL_BASE + 0x100000
    g0 = GLOBAL_BASE + 0x200000
    for _ in range(rounds):
        for w in (w0, w1):
            tb.st(w, lambda l: 4 * l, space=SPACE_SHARED)
        for w in (w0, w1):
            tb.bar(w)
        for w in (w0, w1):
            tb.ld(w, lambda l: 4 * ((l + 1) % 32), space=SPACE_SHARED)
        for w in (w0, w1):
            tb.bar(w)
    tb.st(w0, lambda l: data + 4 * l)
    tb.if_(w0, [0])
    if with_sync:
        tb.rel(w0, flag, scope="glb")
    tb.else_(w0)
    tb.fi(w0)
    tb.if_(w0, [5])
    tb.st(w0, g0)
    tb.else_(w0)
    tb.fi(w0)
    tb.if_(w1, [0])
    if with_sync:
        tb.acq(w1, flag, scope="glb")
    tb.else_(w1)
    tb.fi(w1)
    tb.ld(w1, lambda l: data + 4 * l)
    tb.if_(w1, [5])
    tb.st(w1, g0)
    tb.else_(w1)
    tb.fi(w1)
    return tb.records(), tb


class _Params(ctypes.Structure):
    _fields_ = [("config", ctypes.c_int32), ("n_blocks", ctypes.c_uint32), ("tpb", ctypes.c_uint32),
                ("iters", ctypes.c_uint32), ("log2_nodes", ctypes.c_uint32),
                ("nodes_per_thread", ctypes.c_uint32), ("max_resident", ctypes.c_uint32),
                ("inject", ctypes.c_uint32), ("inj_scale", ctypes.c_uint32),
                ("deg_lo", ctypes.c_uint32), ("deg_hi", ctypes.c_uint32),
                ("bar_per_node", ctypes.c_uint32), ("seed", ctypes.c_uint64),
                ("bug", ctypes.c_uint32), ("log2_buckets", ctypes.c_uint32)]


class _Info(ctypes.Structure):
    _fields_ = [("n_records", ctypes.c_uint64), ("grid_x", ctypes.c_uint32), ("tpb", ctypes.c_uint32),
                ("smem_bytes", ctypes.c_uint32), ("n_truth", ctypes.c_uint32)]


_lib = None


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run __graft_entry__.build()")
        lib = ctypes.CDLL(LIB_PATH)
        lib.bcgen_plan.restype = ctypes.c_void_p
        lib.bcgen_plan.argtypes = [ctypes.POINTER(_Params), ctypes.POINTER(_Info)]
        lib.bcgen_fill.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int]
        lib.bcgen_truth_list.restype = ctypes.c_uint64
        lib.bcgen_truth_list.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32]
        lib.bcgen_free.argtypes = [ctypes.c_void_p]
        lib.bcgen_fill_shard.restype = ctypes.c_uint64
        lib.bcgen_fill_shard.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32,
                                         ctypes.c_uint32, ctypes.c_int]
        _lib = lib
    return _lib


class ConfigPlan:
    """A scheduled C2-C5 trace.  `fill(buf)` writes the 272-B records into any
    writable buffer (numpy array, pinned torch tensor...)."""

    def __init__(self, config: int, seed: int = None, **kw):
        lib = _load()
        p = _Params()
        p.config = config
        p.seed = config if seed is None else seed
        p.inject = kw.pop("inject", 1 if config in (4, 5) else 0)  # C2 / C3: injected variants on request
        if config == 6:
            p.bug = kw.pop("bug", 3)  # the benchmark as published has both section-6.3 bugs
        for k, v in kw.items():
            setattr(p, k, v)
        info = _Info()
        self._h = lib.bcgen_plan(ctypes.byref(p), ctypes.byref(info))
        self.config = config
        self.n_records = int(info.n_records)
        self.geometry = dict(grid=(int(info.grid_x), 1, 1), block=(int(info.tpb), 1, 1),
                             smem_bytes=int(info.smem_bytes), granule_log2=2)

    def fill(self, buf, begin=0, end=None, threads=None):
        end = self.n_records if end is None else end
        if isinstance(buf, np.ndarray):
            ptr = buf.ctypes.data
        else:  # torch tensor
            ptr = buf.data_ptr()
        threads = threads or min(16, os.cpu_count() or 1)
        _load().bcgen_fill(self._h, ctypes.c_void_p(ptr), begin, end, threads)

    def shard_count(self, rank, world):
        """records in the block shard of `rank`"""
        return int(_load().bcgen_fill_shard(self._h, None, None, rank, world, min(16, os.cpu_count() or 1)))

    def shard(self, rank, world, out=None):
        """The block shard (blocks b % world == rank): (records, global indices uint32).  `out`: an
        optional writable uint8 buffer (e.g. pinned torch tensor) of >= count * 272 bytes."""
        lib = _load()
        threads = min(16, os.cpu_count() or 1)
        n = int(lib.bcgen_fill_shard(self._h, None, None, rank, world, threads))
        idx = np.empty(n, dtype=np.uint32)
        if out is None:
            recs = np.empty(n, dtype=RECORD_DTYPE)
            ptr = recs.ctypes.data
        else:
            recs = out
            ptr = out.ctypes.data if isinstance(out, np.ndarray) else out.data_ptr()
        if n:
            lib.bcgen_fill_shard(self._h, ctypes.c_void_p(ptr), idx.ctypes.data, rank, world, threads)
        return recs, idx

    def records(self) -> np.ndarray:
        a = np.empty(self.n_records, dtype=RECORD_DTYPE)
        self.fill(a)
        return a

    def truth(self, granule_log2=2) -> np.ndarray:
        lib = _load()
        n = lib.bcgen_truth_list(self._h, None, 0, granule_log2)
        a = np.zeros(n, dtype=RACE_DTYPE)
        if n:
            lib.bcgen_truth_list(self._h, a.ctypes.data, n, granule_log2)
        return a

    def close(self):
        if self._h:
            _load().bcgen_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


_CIDX = {"c1": 1, "c2": 2, "c3": 3, "c4": 4, "c5": 5, "c6": 6}


def make_config(name, seed=None, **kw):
    """Return (records ndarray, geometry dict, truth ndarray or None)."""
    idx = _CIDX[name] if isinstance(name, str) else int(name)
    if idx == 1:
        recs, tb = make_c1(**kw)
        return recs, tb.geom.as_dict(), None
    plan = ConfigPlan(idx, seed, **kw)
    recs = plan.records()
    truth = plan.truth() if (idx in (4, 5) or kw.get("inject")) else None
    geom = plan.geometry
    plan.close()
    return recs, geom, truth
