"""Multi-GPU modes (bc.h bc_config.rank/world).

Block-sharded (bc_load_trace_shard + a transport): rank r holds the records of the blocks
b % world == r, replays only those, exchanges clock snapshots / branch nodes / sync records, routes
every (granule, event) item to the granule's owner per window, and rank 0 finalizes the gathered
races; its list must equal the oracle's.  The GPU tests run the ranks as threads over the
in-process transport (bc_group_create_local) on one B200 -- the same data plane as NCCL, whose
calls are only the transport.

Replicated-trace address sharding (bc_load_trace with world > 1, no transport): each rank gets the
same trace, derives the same clocks, and checks only the shadow granules it owns; the per-rank race
lists are disjoint and their canonical merge must equal the single-GPU list.

* CPU (`-m "not gpu"`): the host-side merge (merge_races) restores the canonical order from
  any disjoint split of an oracle race list, and gather_races does it across a world-size-2
  gloo process group.
* GPU: every rank of world W in {2, 3, 8} is run as its own context on cuda:0 (the kernels do
  not care which GPU a rank runs on); the merged result is compared with the oracle
  element by element.
"""
import os

import numpy as np
import pytest

import bcgen
import oracle
import paper_conf_pldi_eizenbergppmd17_b200 as bc
from bcgen.configs import ConfigPlan
from bcgen.fuzz import random_trace

import litmus


def _oracle_races(recs, geom):
    st, races, _ = oracle.detect_geom(recs, geom)
    assert st == 0
    return races


def _c4_small():
    plan = ConfigPlan(4, n_blocks=12, log2_nodes=14, nodes_per_thread=2, inj_scale=4)
    return plan.records(), plan.geometry


# ----------------------------------------------------------------------------- CPU
@pytest.mark.parametrize("parts", [1, 2, 5])
def test_merge_restores_canonical_order(parts):
    recs, geom = _c4_small()
    want = _oracle_races(recs, geom)
    assert len(want) > 100
    rng = np.random.default_rng(parts)
    owner = rng.integers(0, parts, size=len(want))
    split = [want[owner == p] for p in range(parts)]
    got = bc.merge_races(split[::-1])
    assert np.array_equal(got.view(np.uint8), want.view(np.uint8))


def test_merge_with_findings_and_shared():
    # a litmus trace with barrier-divergence findings and shared-memory races
    for name, build, _exp, _opts in litmus.SUITE:
        tb = build()
        recs, geom = tb.records(), tb.geom.as_dict()
        st, want, _ = oracle.detect_geom(recs, geom)
        if st != 0 or len(want) < 2:
            continue
        rng = np.random.default_rng(len(want))
        owner = rng.integers(0, 3, size=len(want))
        got = bc.merge_races([want[owner == p] for p in range(3)])
        assert np.array_equal(got.view(np.uint8), want.view(np.uint8)), name


def _gather_worker(rank, world, port, path):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    want = np.load(path)
    mine = want[(np.arange(len(want)) * 7 + 3) % world == rank]
    got = bc.gather_races(mine)
    if rank == 0:
        np.save(path + ".out.npy", got)
    else:
        assert got is None
    dist.destroy_process_group()


def test_gather_over_gloo(tmp_path):
    import socket

    import torch.multiprocessing as mp
    recs, geom = _c4_small()
    want = _oracle_races(recs, geom)
    path = str(tmp_path / "races.npy")
    np.save(path, want)
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    mp.spawn(_gather_worker, args=(2, port, path), nprocs=2, join=True)
    got = np.load(path + ".out.npy")
    assert np.array_equal(got.view(np.uint8), want.view(np.uint8))


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_shard_trace_partitions_blocks(world):
    """bc.shard_trace: the shards are disjoint, cover every record, keep trace order, and hold whole
    blocks (every record of block b on rank b % world)."""
    recs, geom = _c4_small()
    seen = np.zeros(len(recs), dtype=np.int64)
    wpb = (geom["block"][0] + 31) // 32
    for r in range(world):
        loc, idx = bc.shard_trace(recs, geom, r, world)
        assert np.all(np.diff(idx.astype(np.int64)) > 0)
        assert np.array_equal(loc.view(np.uint8), recs[idx].view(np.uint8))
        assert np.all((loc["warp"] // wpb) % world == r)
        seen[idx] += 1
    assert np.all(seen == 1)


def _shard_worker(rank, world, port, path):
    """one rank of a world-size-2 gloo group: shard the trace, all-gather the record indices, and
    check that every global record is on exactly one rank (the loader side of the sharded path)"""
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    recs = np.load(path)
    geom = dict(grid=(12, 1, 1), block=(256, 1, 1), smem_bytes=16)
    loc, idx = bc.shard_trace(recs, geom, rank, world)
    sizes = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
    dist.all_gather(sizes, torch.tensor([len(idx)]))
    mx = int(max(s.item() for s in sizes))
    buf = torch.full((mx,), -1, dtype=torch.int64)
    buf[:len(idx)] = torch.from_numpy(idx.astype(np.int64))
    parts = [torch.zeros(mx, dtype=torch.int64) for _ in range(world)]
    dist.all_gather(parts, buf)
    allidx = torch.cat([p[p >= 0] for p in parts]).numpy()
    assert sorted(allidx.tolist()) == list(range(len(recs)))
    assert int(sum(s.item() for s in sizes)) == len(recs)
    dist.destroy_process_group()


def test_shard_loader_over_gloo(tmp_path):
    import socket

    import torch.multiprocessing as mp
    recs, geom = _c4_small()
    assert geom["grid"][0] == 12
    path = str(tmp_path / "recs.npy")
    np.save(path, recs)
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    mp.spawn(_shard_worker, args=(2, port, path), nprocs=2, join=True)


# ----------------------------------------------------------------------------- GPU
def sharded_detect(recs, geom, world, window_events=0, timeout=300):
    """Block-sharded detect: `world` ranks = threads over one in-process group on cuda:0.  Returns
    rank 0's (status, races, stats) and every rank's status."""
    import threading
    grp = bc.LocalGroup(world)
    out, errs = [None] * world, [None] * world

    def run(r):
        try:
            with bc.Context(geom, device=0, rank=r, world=world, group=grp, window_events=window_events) as ctx:
                loc, idx = bc.shard_trace(recs, geom, r, world)
                ctx.load_trace_shard(loc, idx, len(recs))
                st, stats = ctx.detect(allow=(-2, -8))
                out[r] = (st, ctx.races() if st == 0 else None, stats)
        except Exception as e:  # pragma: no cover - reported below
            errs[r] = e

    ts = [threading.Thread(target=run, args=(r,), daemon=True) for r in range(world)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(timeout)
    assert not any(t.is_alive() for t in ts), "a rank hung"
    grp.close()
    for e in errs:
        if e is not None:
            raise e
    sts = [o[0] for o in out]
    assert len(set(sts)) == 1, sts  # every rank agrees on the status
    for o in out[1:]:
        assert o[0] != 0 or len(o[1]) == 0  # races come back on rank 0 only
    return out[0]


def assert_sharded(recs, geom, world, window_events=0):
    st, want, stats_o = oracle.detect_geom(recs, geom)
    st2, got, stats = sharded_detect(recs, geom, world, window_events)
    assert st2 == st, (st2, st)
    if st != 0:
        return want, stats
    assert len(got) == len(want), (len(got), len(want), got[:3], want[:3])
    assert np.array_equal(got.view(np.uint8), want.view(np.uint8))
    assert stats["lane_events"] == stats_o["lane_events"]
    return want, stats


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("case", range(11), ids=lambda i: f"case{i}")
def test_block_sharded_equals_oracle(case, world):
    name, recs, geom = _cases()[case]
    assert_sharded(recs, geom, world)


@pytest.mark.gpu
def test_block_sharded_litmus_and_random():
    for name, build, _exp, _opts in litmus.SUITE:
        tb = build()
        assert_sharded(tb.records(), tb.geom.as_dict(), 2)
    for seed in range(6000, 6040):
        recs, tb = random_trace(seed)
        assert_sharded(recs, tb.geom.as_dict(), 1 + seed % 4)


@pytest.mark.gpu
@pytest.mark.parametrize("we", [64, 3000])
def test_block_sharded_windows(we):
    """Sharded and windowed: per window the items go to their owners, whose 32-B shadow entries
    carry the state to the next window."""
    for seed in range(6100, 6120):
        recs, tb = random_trace(seed)
        assert_sharded(recs, tb.geom.as_dict(), 2, window_events=we)
    plan = ConfigPlan(4, n_blocks=40, log2_nodes=16, nodes_per_thread=3, inj_scale=8)
    want, stats = assert_sharded(plan.records(), plan.geometry, 3, window_events=we * 20)
    assert stats["windows"] > 1


def _replicated(recs, geom, world):
    parts, items = [], 0
    for r in range(world):
        res = bc.detect(recs, geom, device="cuda:0", rank=r, world=world)
        assert res.status == 0
        parts.append(res.races)
        items += res.stats["items"]
    return bc.merge_races(parts), items


def _cases():
    out = [("c1", *(lambda r, tb: (r, tb.geom.as_dict()))(*bcgen.configs.make_c1())),
           ("c1_nosync", *(lambda r, tb: (r, tb.geom.as_dict()))(*bcgen.configs.make_c1(with_sync=False))),
           ("c4_small", *_c4_small())]
    plan = ConfigPlan(2, n_blocks=8, iters=6)
    out.append(("c2_small", plan.records(), plan.geometry))
    plan = ConfigPlan(3, n_blocks=16, iters=2, tpb=64)
    out.append(("c3_small", plan.records(), plan.geometry))
    for seed in range(6):
        recs, tb = random_trace(seed=1000 + seed)
        out.append((f"random{seed}", recs, tb.geom.as_dict()))
    return out


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 3, 8])
@pytest.mark.parametrize("case", _cases(), ids=lambda c: c[0])
def test_sharded_equals_oracle(case, world):
    name, recs, geom = case
    st, want, _ = oracle.detect_geom(recs, geom)
    if st != 0:
        pytest.skip("infeasible trace")
    got, items = _replicated(recs, geom, world)
    assert len(got) == len(want), (len(got), len(want))
    assert np.array_equal(got.view(np.uint8), want.view(np.uint8))
    single = bc.detect(recs, geom, device="cuda:0")
    assert items == single.stats["items"]  # the shards partition the checked items


@pytest.mark.gpu
def test_sharded_litmus_suite():
    for name, build, _exp, _opts in litmus.SUITE:
        tb = build()
        recs, geom = tb.records(), tb.geom.as_dict()
        st, want, _ = oracle.detect_geom(recs, geom)
        if st != 0:
            continue
        got, _ = _replicated(recs, geom, 4)
        assert np.array_equal(got.view(np.uint8), want.view(np.uint8)), name


# ----------------------------------------------------------------------------- item exchange (row e)
def _mix_owner(g: np.ndarray, world: int) -> np.ndarray:
    """Test model of the owner rule of the sharded data plane (shard.cu k_dest / common.cuh shard_of):
    a murmur3 finaliser of the granule, then a multiply-shift to [0, world)."""
    k = g.astype(np.uint64) & np.uint64(0xFFFFFFFF)
    k ^= k >> np.uint64(16)
    k = (k * np.uint64(0x85EBCA6B)) & np.uint64(0xFFFFFFFF)
    k ^= k >> np.uint64(13)
    k = (k * np.uint64(0xC2B2AE35)) & np.uint64(0xFFFFFFFF)
    k ^= k >> np.uint64(16)
    return ((k * np.uint64(world)) >> np.uint64(32)).astype(np.int64)


def _items(recs, idx, geom):
    """(granule id, global event) of every memory lane op of the records, in trace order (a model of
    K4 for the exchange test: global granules by address, shared granules tagged by block)"""
    G = geom.get("granule_log2", 2)
    wpb = (geom["block"][0] + 31) // 32
    out_g, out_e = [], []
    for rec, gi in zip(recs, idx):
        if rec["op"] > 2:  # LD / ST / ATOM only
            continue
        for l in range(32):
            if (int(rec["mask"]) >> l) & 1:
                a = int(rec["addr"][l])
                if rec["space"] == 1:  # shared: (block, offset), never leaves its block's rank
                    g = (1 << 62) | ((int(rec["warp"]) // wpb) << 32) | (a >> G)
                else:
                    g = a >> G
                out_g.append(g)
                out_e.append((int(gi) << 5) | l)
    return np.array(out_g, dtype=np.uint64), np.array(out_e, dtype=np.int64)


def _exchange_worker(rank, world, port, path):
    """One rank of the per-window item exchange over gloo: expand the rank's block shard, route each
    item to its granule's owner (shared granules stay; global ones by the owner rule) with a stable
    partition, all-to-all the (granule, event) pairs, then sort by event and stably by granule."""
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    recs = np.load(path)
    geom = dict(grid=(12, 1, 1), block=(256, 1, 1), smem_bytes=16, granule_log2=2)
    loc, idx = bc.shard_trace(recs, geom, rank, world)
    g, e = _items(loc, idx, geom)
    shared = (g >> np.uint64(62)) == 1
    dest = np.where(shared, rank, _mix_owner(g, world))
    order = np.argsort(dest, kind="stable")
    counts = np.bincount(dest, minlength=world).astype(np.int64)
    rc = torch.zeros(world, dtype=torch.int64)
    dist.all_to_all_single(rc, torch.from_numpy(counts))
    rc = rc.numpy()
    payload = torch.from_numpy(np.stack([g[order].astype(np.int64), e[order]], axis=1).reshape(-1))
    recv = torch.zeros(int(rc.sum()) * 2, dtype=torch.int64)
    dist.all_to_all_single(recv, payload, [int(c) * 2 for c in rc], [int(c) * 2 for c in counts])
    got = recv.numpy().reshape(-1, 2)
    got = got[np.argsort(got[:, 1], kind="stable")]        # trace order
    got = got[np.argsort(got[:, 0], kind="stable")]        # then grouped by granule
    np.save(f"{path}.{rank}.npy", got)
    dist.destroy_process_group()


def test_item_exchange_over_gloo(tmp_path):
    """Row e's per-window data plane over a world-size-2 gloo group: after the all-to-all every granule
    lives on exactly one rank, each rank's items are grouped by granule in global trace order, and the
    union equals the single-rank expansion of the whole trace."""
    import socket

    import torch.multiprocessing as mp
    recs, geom = _c4_small()
    path = str(tmp_path / "trace.npy")
    np.save(path, recs)
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    mp.spawn(_exchange_worker, args=(2, port, path), nprocs=2, join=True)
    parts = [np.load(f"{path}.{r}.npy") for r in range(2)]
    g_all, e_all = _items(recs, np.arange(len(recs)), dict(geom, granule_log2=2))
    want = np.stack([g_all.astype(np.int64), e_all], axis=1)
    want = want[np.argsort(want[:, 0], kind="stable")]
    assert sum(len(p) for p in parts) == len(want)
    owners = {}
    for r, p in enumerate(parts):
        assert np.all(np.diff(p[:, 0]) >= 0)
        same = p[1:, 0] == p[:-1, 0]
        assert np.all(np.diff(p[:, 1])[same] > 0)  # trace order inside a granule
        for gk in np.unique(p[:, 0]):
            assert owners.setdefault(int(gk), r) == r  # one owner per granule
    merged = np.concatenate(parts)
    merged = merged[np.lexsort((merged[:, 1], merged[:, 0]))]
    assert np.array_equal(merged, want)
