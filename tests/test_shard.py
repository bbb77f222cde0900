"""Address-sharded multi-GPU mode (bc.h bc_config.rank/world).

Each rank gets the same trace, derives the same clocks, and checks only the shadow granules
it owns; the per-rank race lists are disjoint and their canonical merge must equal the
single-GPU list (and hence the oracle's).

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


# ----------------------------------------------------------------------------- GPU
def _sharded(recs, geom, world):
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
    got, items = _sharded(recs, geom, world)
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
        got, _ = _sharded(recs, geom, 4)
        assert np.array_equal(got.view(np.uint8), want.view(np.uint8)), name
