"""paper_conf_pldi_eizenbergppmd17_b200 — B200-native BARRACUDA race check (PLDI'17).

Thin Python binding over the C ABI in include/bc.h (lib/libbc.so, sm_100a kernels).
Argument marshalling only: every step of the race check runs in the CUDA kernels of
csrc/.  There is no CPU fallback: if the extension is missing, importing the binding
functions raises.  PyTorch provides device memory (borrowed device traces, device race
buffers) and streams.

Calls mirror the boundary:

    ctx = Context(geometry, device=0)      # bc_init
    ctx.load_trace(records)                # bc_load_trace  (numpy host array or torch CUDA uint8 tensor)
    stats = ctx.detect()                   # bc_detect
    races = ctx.races()                    # bc_races  -> numpy array of RACE_DTYPE
    ctx.close()                            # bc_destroy
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "libbc.so")

RECORD_BYTES = 272
RACE_DTYPE = np.dtype([
    ("addr", "<u8"), ("prior_event", "<u8"), ("cur_event", "<u8"),
    ("kind", "u1"), ("cls", "u1"), ("space", "u1"), ("pad", "u1"), ("block", "<u4"),
])

OK = 0
STATUS = {0: "OK", -1: "INVALID_ARG", -2: "INFEASIBLE_TRACE", -3: "OOM", -4: "CUDA", -5: "NCCL",
          -6: "STATE", -7: "TRUNCATED", -8: "OVERFLOW"}
F_RELEASE_OVERWRITE = 1
F_NO_SAME_VALUE_FILTER = 2
F_COUNT_GATHERS = 4  # statistics: fill stats["clock_gathers"] (one extra pass)

EXPORTS = sorted(["bc_init", "bc_load_trace", "bc_load_values", "bc_detect", "bc_races", "bc_races_device",
                  "bc_destroy", "bc_status_string", "bc_last_error", "bc_phase_name", "bc_load_trace_shard",
                  "bc_nccl_unique_id", "bc_group_create_local", "bc_group_destroy", "bc_split_warps",
                  "bc_stream_open", "bc_stream_poll", "bc_queue_push"])


class BcError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
_FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)


class _Config(ctypes.Structure):
    _fields_ = [("grid_dim", ctypes.c_uint32 * 3), ("block_dim", ctypes.c_uint32 * 3),
                ("warp_size", ctypes.c_uint32), ("granule_log2", ctypes.c_uint32),
                ("smem_bytes_per_block", ctypes.c_uint32), ("flags", ctypes.c_uint32),
                ("device", ctypes.c_int32), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("stream", ctypes.c_void_p), ("window_events", ctypes.c_uint64),
                ("dev_alloc", _ALLOC_FN), ("dev_free", _FREE_FN), ("alloc_user", ctypes.c_void_p),
                ("nccl_unique_id", ctypes.c_void_p), ("group", ctypes.c_void_p),
                ("global_ranges", ctypes.c_uint64 * 128), ("n_global_ranges", ctypes.c_uint32)]


class _Stats(ctypes.Structure):
    _fields_ = [("records", ctypes.c_uint64), ("lane_events", ctypes.c_uint64),
                ("control_events", ctypes.c_uint64), ("items", ctypes.c_uint64),
                ("segments", ctypes.c_uint64), ("races", ctypes.c_uint64), ("findings", ctypes.c_uint64),
                ("sync_ops", ctypes.c_uint64), ("written_pages", ctypes.c_uint64),
                ("kernel_launches", ctypes.c_uint64), ("clock_gathers", ctypes.c_uint64),
                ("windows", ctypes.c_uint64), ("vc_pool_entries", ctypes.c_uint64),
                ("ms_total", ctypes.c_float), ("ms_kernel", ctypes.c_float * 12)]


_lib = None


def lib():
    """Load lib/libbc.so (fails loudly when the CUDA extension has not been built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: build it with `python __graft_entry__.py` "
                              "(there is no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        L.bc_init.restype = ctypes.c_int
        L.bc_init.argtypes = [ctypes.POINTER(_Config), ctypes.POINTER(ctypes.c_void_p)]
        L.bc_load_trace.restype = ctypes.c_int
        L.bc_load_trace.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int]
        L.bc_load_values.restype = ctypes.c_int
        L.bc_load_values.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int]
        L.bc_detect.restype = ctypes.c_int
        L.bc_detect.argtypes = [ctypes.c_void_p, ctypes.POINTER(_Stats)]
        L.bc_races.restype = ctypes.c_int
        L.bc_races.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64)]
        L.bc_races_device.restype = ctypes.c_int
        L.bc_races_device.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                      ctypes.POINTER(ctypes.c_uint64)]
        L.bc_destroy.argtypes = [ctypes.c_void_p]
        L.bc_status_string.restype = ctypes.c_char_p
        L.bc_status_string.argtypes = [ctypes.c_int]
        L.bc_last_error.restype = ctypes.c_char_p
        L.bc_last_error.argtypes = [ctypes.c_void_p]
        L.bc_phase_name.restype = ctypes.c_char_p
        L.bc_phase_name.argtypes = [ctypes.c_int]
        L.bc_load_trace_shard.restype = ctypes.c_int
        L.bc_load_trace_shard.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                          ctypes.c_uint64, ctypes.c_int]
        L.bc_nccl_unique_id.restype = ctypes.c_int
        L.bc_nccl_unique_id.argtypes = [ctypes.c_void_p]
        L.bc_group_create_local.restype = ctypes.c_int
        L.bc_group_create_local.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_void_p)]
        L.bc_group_destroy.argtypes = [ctypes.c_void_p]
        L.bc_stream_open.restype = ctypes.c_int
        L.bc_stream_open.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                                     ctypes.POINTER(ctypes.c_void_p)]
        L.bc_stream_poll.restype = ctypes.c_int
        L.bc_stream_poll.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.POINTER(_Stats)]
        L.bc_queue_push.restype = ctypes.c_int
        L.bc_queue_push.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p]
        L.bc_split_warps.restype = ctypes.c_int
        L.bc_split_warps.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32,
                                     ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                     ctypes.POINTER(ctypes.c_uint64)]
        _lib = L
    return _lib


def phase_names():
    L = lib()
    out, i = [], 0
    while True:
        p = L.bc_phase_name(i)
        if not p:
            return out
        out.append(p.decode())
        i += 1


def _stats_dict(s: _Stats):
    d = {k: getattr(s, k) for k, _ in _Stats._fields_ if k != "ms_kernel"}
    d["ms_kernel"] = dict(zip(phase_names(), list(s.ms_kernel)))
    return d


def torch_allocator():
    """(dev_alloc, dev_free) callbacks over torch's CUDA caching allocator (bc_config.dev_alloc /
    dev_free: PyTorch supplies the device memory).  Marshalling only."""
    import torch

    def _alloc(nbytes, stream, user):
        try:
            return torch.cuda.caching_allocator_alloc(int(nbytes), torch.cuda.current_device(), stream or 0)
        except Exception:
            return None

    def _free(ptr, nbytes, stream, user):
        torch.cuda.caching_allocator_delete(ptr)

    return _ALLOC_FN(_alloc), _FREE_FN(_free)


class Context:
    """One traced launch geometry on one GPU (bc_init ... bc_destroy)."""

    def __init__(self, geometry: dict, device: int = 0, flags: int = 0, stream=None, rank: int = 0, world: int = 1,
                 window_events: int = 0, allocator=None, nccl_id: bytes = None, group: "LocalGroup" = None,
                 global_ranges=None):
        """rank / world > 1: address-sharded check (bc.h bc_config.rank/world): every rank loads
        the same trace and reports the races of the shadow granules it owns; merge the per-rank
        lists with merge_races() or gather_races().  window_events: bc_config.window_events (0 =
        auto).  allocator: None (cudaMalloc), "torch" (torch's caching allocator) or a
        (dev_alloc, dev_free) pair of ctypes callbacks.  nccl_id (128 bytes of nccl_unique_id() from
        rank 0) or group (LocalGroup): the block-sharded multi-GPU check (load_trace_shard).
        global_ranges: [(base, size), ...] declared global allocations (required for streaming)."""
        L = lib()
        grid = tuple(geometry["grid"]) + (1,) * (3 - len(geometry["grid"]))
        block = tuple(geometry["block"]) + (1,) * (3 - len(geometry["block"]))
        c = _Config()
        for i in range(3):
            c.grid_dim[i], c.block_dim[i] = grid[i], block[i]
        c.warp_size = geometry.get("warp_size", 32)  # 4 / 8 / 16: warp-size simulation (row f4)
        c.granule_log2 = geometry.get("granule_log2", 2)
        c.smem_bytes_per_block = geometry.get("smem_bytes", 0)
        c.flags = flags
        c.device = device
        c.rank, c.world = rank, world
        c.stream = stream
        c.window_events = window_events
        self._nccl_id = None
        if nccl_id is not None:
            self._nccl_id = ctypes.create_string_buffer(bytes(nccl_id), 128)
            c.nccl_unique_id = ctypes.cast(self._nccl_id, ctypes.c_void_p)
        if group is not None:
            c.group = group.handle
        if global_ranges:
            if len(global_ranges) > 64:
                raise ValueError("at most 64 global ranges")
            for i, (base, size) in enumerate(global_ranges):
                c.global_ranges[2 * i], c.global_ranges[2 * i + 1] = int(base), int(size)
            c.n_global_ranges = len(global_ranges)
        self._alloc = None
        if allocator is not None:
            self._alloc = torch_allocator() if allocator == "torch" else tuple(allocator)
            c.dev_alloc, c.dev_free = self._alloc
        h = ctypes.c_void_p()
        st = L.bc_init(ctypes.byref(c), ctypes.byref(h))
        if st != OK:
            raise BcError(st, L.bc_status_string(st).decode())
        self._h = h
        self._keep = None
        self.device = device

    def _check(self, st, allow=()):
        if st != OK and st not in allow:
            L = lib()
            raise BcError(st, f"{L.bc_status_string(st).decode()} ({L.bc_last_error(self._h).decode()})")
        return st

    def load_trace(self, records):
        """records: numpy RECORD_DTYPE array / bytes-like on the host (copied), or a CUDA tensor
        of n*272 bytes (borrowed until the next load_trace / close)."""
        L = lib()
        if hasattr(records, "is_cuda") and records.is_cuda:
            n = records.numel() * records.element_size() // RECORD_BYTES
            self._keep = records
            return self._check(L.bc_load_trace(self._h, ctypes.c_void_p(records.data_ptr()), n, 1))
        if hasattr(records, "data_ptr"):  # pinned / host torch tensor
            n = records.numel() * records.element_size() // RECORD_BYTES
            self._keep = records
            return self._check(L.bc_load_trace(self._h, ctypes.c_void_p(records.data_ptr()), n, 0))
        a = np.ascontiguousarray(records)
        n = a.nbytes // RECORD_BYTES
        self._keep = a
        return self._check(L.bc_load_trace(self._h, ctypes.c_void_p(a.ctypes.data if n else 0), n, 0))

    def load_trace_shard(self, records, rec_index, n_global: int):
        """bc_load_trace_shard: this rank's records (those of blocks b % world == rank, trace order) and
        their global record indices (uint32, increasing); host arrays (copied) or CUDA tensors (borrowed)."""
        L = lib()
        if hasattr(records, "is_cuda") and records.is_cuda:
            n = records.numel() * records.element_size() // RECORD_BYTES
            self._keep, self._keep_idx = records, rec_index
            return self._check(L.bc_load_trace_shard(self._h, ctypes.c_void_p(records.data_ptr()),
                                                      ctypes.c_void_p(rec_index.data_ptr()), n, n_global, 1))
        a = np.ascontiguousarray(records)
        idx = np.ascontiguousarray(rec_index, dtype=np.uint32)
        n = a.nbytes // RECORD_BYTES
        assert len(idx) == n
        self._keep, self._keep_idx = a, idx
        return self._check(L.bc_load_trace_shard(self._h, ctypes.c_void_p(a.ctypes.data if n else 0),
                                                  ctypes.c_void_p(idx.ctypes.data if n else 0), n, n_global, 0))

    def stream_open(self, queue_records: int, max_records: int, min_window: int = 1):
        """bc_stream_open: returns the device address of the record queue (bc.h layout)."""
        q = ctypes.c_void_p()
        self._check(lib().bc_stream_open(self._h, queue_records, max_records, min_window, ctypes.byref(q)))
        return q.value

    def stream_poll(self, finish: bool = False, allow=()):
        """bc_stream_poll: consume committed records, check a window when enough are new; finish=True
        drains the queue and finalises the race list.  Returns (status, stats)."""
        s = _Stats()
        st = self._check(lib().bc_stream_poll(self._h, 1 if finish else 0, ctypes.byref(s)), allow)
        return st, _stats_dict(s)

    def load_values(self, values):
        """bc_load_values: per-lane store values [n_records, 32] (uint64) as a host
        numpy array (copied) or a CUDA tensor (borrowed); None clears them."""
        L = lib()
        if values is None:
            return self._check(L.bc_load_values(self._h, None, 0, 0))
        if hasattr(values, "is_cuda") and values.is_cuda:
            n = values.numel() // 32
            self._keep_values = values
            return self._check(L.bc_load_values(self._h, ctypes.c_void_p(values.data_ptr()), n, 1))
        a = np.ascontiguousarray(values, dtype=np.uint64).reshape(-1)
        self._keep_values = a
        n = len(a) // 32
        return self._check(L.bc_load_values(self._h, ctypes.c_void_p(a.ctypes.data if n else 0), n, 0))

    def detect(self, allow=()):
        """bc_detect; returns (status, stats dict)."""
        s = _Stats()
        st = self._check(lib().bc_detect(self._h, ctypes.byref(s)), allow)
        return st, _stats_dict(s)

    def num_races(self):
        n = ctypes.c_uint64()
        self._check(lib().bc_races(self._h, None, 0, ctypes.byref(n)))
        return int(n.value)

    def races(self):
        n = self.num_races()
        out = np.zeros(n, dtype=RACE_DTYPE)
        if n:
            tot = ctypes.c_uint64()
            self._check(lib().bc_races(self._h, ctypes.c_void_p(out.ctypes.data), n, ctypes.byref(tot)))
        return out

    def races_device(self, out_tensor):
        """Copy races into a CUDA uint8 tensor of >= n*32 bytes; returns n."""
        n = self.num_races()
        tot = ctypes.c_uint64()
        cap = out_tensor.numel() * out_tensor.element_size() // 32
        self._check(lib().bc_races_device(self._h, ctypes.c_void_p(out_tensor.data_ptr()), cap,
                                          ctypes.byref(tot)), allow=(-7,))
        return n

    def close(self):
        if getattr(self, "_h", None):
            lib().bc_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def split_warps(records, geometry: dict, ws: int, device: int = 0):
    """bc_split_warps (reading R17): the trace re-split into virtual warps of ws lanes,
    on the GPU.  records: host array or CUDA uint8 tensor of the 32-lane trace.  Returns (CUDA uint8
    tensor of the split records, geometry with warp_size = ws, CUDA int64 tensor of origins =
    (source record << 5) | first lane).  Marshalling only."""
    import torch
    dev = torch.device("cuda", device)
    if hasattr(records, "is_cuda") and records.is_cuda:
        d_in = records
    else:
        d_in = torch.from_numpy(np.ascontiguousarray(records).view(np.uint8)).to(dev)
    n = d_in.numel() // RECORD_BYTES
    g32 = dict(geometry)
    g32["warp_size"] = 32
    with Context(g32, device=device) as ctx:
        L = lib()
        cnt = ctypes.c_uint64()
        ctx._check(L.bc_split_warps(ctx._h, ctypes.c_void_p(d_in.data_ptr()), n, ws, None, None, 0,
                                    ctypes.byref(cnt)))
        m = int(cnt.value)
        out = torch.empty(max(m, 1) * RECORD_BYTES, dtype=torch.uint8, device=dev)
        org = torch.empty(max(m, 1), dtype=torch.int64, device=dev)
        ctx._check(L.bc_split_warps(ctx._h, ctypes.c_void_p(d_in.data_ptr()), n, ws, ctypes.c_void_p(out.data_ptr()),
                                    ctypes.c_void_p(org.data_ptr()), m, ctypes.byref(cnt)))
    g2 = dict(geometry)
    g2["warp_size"] = ws
    return out[:m * RECORD_BYTES], g2, org[:m]


def queue_push(queue: int, records, stream=None):
    """bc_queue_push: the stand-in producer pushes a CUDA uint8 tensor of records through the queue on
    `stream` (a torch.cuda.Stream or raw handle), asynchronously.  Marshalling only."""
    n = records.numel() // RECORD_BYTES
    h = stream.cuda_stream if hasattr(stream, "cuda_stream") else (stream or 0)
    st = lib().bc_queue_push(ctypes.c_void_p(queue), ctypes.c_void_p(records.data_ptr()), n, ctypes.c_void_p(h))
    if st != OK:
        raise BcError(st, "queue push")


def nccl_unique_id() -> bytes:
    """bc_nccl_unique_id: 128 bytes for Context(nccl_id=...) (rank 0 makes it, the caller broadcasts it)."""
    buf = ctypes.create_string_buffer(128)
    st = lib().bc_nccl_unique_id(buf)
    if st != OK:
        raise BcError(st, "no NCCL library")
    return buf.raw


class LocalGroup:
    """bc_group_create_local: `world` ranks as contexts of this process, one host thread each."""

    def __init__(self, world: int):
        h = ctypes.c_void_p()
        st = lib().bc_group_create_local(world, ctypes.byref(h))
        if st != OK:
            raise BcError(st, "group")
        self.handle, self.world = h, world

    def close(self):
        if self.handle:
            lib().bc_group_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def shard_trace(records, geometry: dict, rank: int, world: int):
    """The block shard of rank `rank`: the records of the traced blocks b with
    b % world == rank, in trace order, and their global record indices (marshalling only)."""
    grid = tuple(geometry["grid"]) + (1,) * (3 - len(geometry["grid"]))
    block = tuple(geometry["block"]) + (1,) * (3 - len(geometry["block"]))
    tpb = block[0] * block[1] * block[2]
    ws = geometry.get("warp_size", 32)
    wpb = (tpb + ws - 1) // ws
    recs = np.asarray(records)
    blocks = recs["warp"].astype(np.int64) // wpb
    idx = np.nonzero(blocks % world == rank)[0].astype(np.uint32)
    return recs[idx], idx


def merge_races(parts) -> np.ndarray:
    """Canonical merge of disjoint per-rank race lists (bc.h bc_race order): findings first by
    (block, record), then global races by address, then shared races by (block, offset); ties by
    (cur_event, prior_event).  Host-side argument marshalling only (no race arithmetic)."""
    parts = [np.asarray(p, dtype=RACE_DTYPE) for p in parts]
    r = np.concatenate(parts) if parts else np.zeros(0, dtype=RACE_DTYPE)
    if len(r) == 0:
        return r
    finding = r["cls"] == 4
    shared = r["space"] == 1
    k1 = np.where(finding, 0, 1)
    k2 = np.where(finding, 0, r["space"].astype(np.int64))
    k3 = np.where(finding | shared, r["block"].astype(np.int64), 0)
    k4 = np.where(finding, 0, r["addr"]).astype(np.uint64)
    order = np.lexsort((r["prior_event"], r["cur_event"], k4, k3, k2, k1))
    return r[order]


def gather_races(local: np.ndarray, group=None, dst: int = 0):
    """Gather every rank's race list over torch.distributed (any backend) and return the canonical
    merge on rank `dst` (None elsewhere)."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    objs = [None] * world if dist.get_rank(group) == dst else None
    dist.gather_object(np.asarray(local, dtype=RACE_DTYPE).tobytes(), objs, dst=dst, group=group)
    if objs is None:
        return None
    return merge_races([np.frombuffer(b, dtype=RACE_DTYPE) for b in objs])


@dataclass
class Result:
    status: int
    races: np.ndarray
    stats: dict


def detect(records, geometry: dict, device="cuda:0", flags: int = 0, stream=None, rank: int = 0,
           world: int = 1, values=None, window_events: int = 0, allocator=None) -> Result:
    """One-shot bc_init/bc_load_trace/bc_detect/bc_races.  Infeasible traces return
    status -2 with no races (as the oracle does)."""
    dev = int(str(device).split(":")[-1]) if str(device).startswith("cuda") else int(device)
    with Context(geometry, device=dev, flags=flags, stream=stream, rank=rank, world=world,
                 window_events=window_events, allocator=allocator) as ctx:
        ctx.load_trace(records)
        if values is not None:
            ctx.load_values(values)
        st, stats = ctx.detect(allow=(-2,))
        races = ctx.races() if st == OK else np.zeros(0, dtype=RACE_DTYPE)
        return Result(st, races, stats)
