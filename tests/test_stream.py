"""Streaming ingest (the device queue of Fig. 6).

A stand-in producer kernel pushes the records through the lock-free queue (write / commit / read
heads, a small ring so it must wrap and wait for the consumer) while the host polls the context,
which checks each committed range as a trace window with the 32-B shadow entries carried between
windows.  The final race list must be bit-identical to the oracle on the whole trace.
"""
import numpy as np
import pytest

import bcgen
import bcgen.configs
import oracle
import paper_conf_pldi_eizenbergppmd17_b200 as bc
from bcgen.configs import ConfigPlan
from bcgen.format import OP_AR_GLB, SPACE_GLOBAL
from bcgen.fuzz import random_trace

import litmus


def declared_ranges(recs):
    """The 1-MB pages the trace's global accesses touch, as (base, size) runs (test-side input
    preparation: an instrumented program would declare its cudaMalloc'ed buffers)."""
    sel = (recs["op"] <= OP_AR_GLB) & (recs["space"] == SPACE_GLOBAL)
    r = recs[sel]
    pages = set()
    for lane in range(32):
        act = (r["mask"] >> np.uint32(lane)) & np.uint32(1)
        a = r["addr"][:, lane][act.astype(bool)]
        pages.update((a >> np.uint64(20)).tolist())
    out, run = [], None
    for p in sorted(pages):
        if run and p == run[1]:
            run[1] = p + 1
        else:
            if run:
                out.append(run)
            run = [p, p + 1]
    if run:
        out.append(run)
    assert len(out) <= 64
    return [(p0 << 20, (p1 - p0) << 20) for p0, p1 in out]


def streamed(recs, geom, queue_records=256, min_window=64, ranges=None):
    import torch
    d = torch.from_numpy(recs.view(np.uint8).copy()).cuda()
    prod = torch.cuda.Stream()
    prod.wait_stream(torch.cuda.current_stream())  # the records' H2D copy
    with bc.Context(geom, device=0, global_ranges=ranges if ranges is not None else declared_ranges(recs)) as ctx:
        q = ctx.stream_open(queue_records, max(len(recs), 1), min_window)
        done = torch.cuda.Event()
        bc.queue_push(q, d, prod)
        done.record(prod)
        try:
            while not done.query():
                ctx.stream_poll(False)
            st, stats = ctx.stream_poll(True, allow=(-2,))
        finally:
            prod.synchronize()  # never free the queue under a running producer
        races = ctx.races() if st == 0 else None
        return st, races, stats


def assert_streamed(recs, geom, **kw):
    st_o, want, _ = oracle.detect_geom(recs, geom)
    st, got, stats = streamed(recs, geom, **kw)
    assert st == st_o, (st, st_o)
    if st_o == 0:
        assert len(got) == len(want), (len(got), len(want))
        assert np.array_equal(got.view(np.uint8), want.view(np.uint8))
    return stats


@pytest.mark.gpu
def test_stream_c1_and_litmus():
    recs, tb = bcgen.configs.make_c1()
    assert_streamed(recs, tb.geom.as_dict(), queue_records=32, min_window=8)
    for name, build, _exp, _opts in litmus.SUITE:
        tb = build()
        assert_streamed(tb.records(), tb.geom.as_dict(), queue_records=16, min_window=2)


@pytest.mark.gpu
@pytest.mark.parametrize("mw", [3, 40, 1000])
def test_stream_random_traces(mw):
    """Window boundaries anywhere: inside read runs, between a writer and its readers, while a barrier
    is pending (some warps of a block have arrived)."""
    for seed in range(7000, 7030):
        recs, tb = random_trace(seed)
        if oracle.detect_geom(recs, tb.geom.as_dict())[0] != 0:
            continue  # an infeasible trace may fail in any poll; the batch tests cover the status
        assert_streamed(recs, tb.geom.as_dict(), queue_records=64, min_window=mw)


@pytest.mark.gpu
@pytest.mark.parametrize("cfg,kw", [(2, dict(n_blocks=8, iters=6)), (3, dict(n_blocks=9, iters=3, tpb=256)),
                                    (4, dict(n_blocks=40, log2_nodes=16, nodes_per_thread=3, inj_scale=8))])
def test_stream_configs(cfg, kw):
    plan = ConfigPlan(cfg, **kw)
    recs = plan.records()
    stats = assert_streamed(recs, plan.geometry, queue_records=4096, min_window=max(1, len(recs) // 6))
    assert stats["windows"] > 1


@pytest.mark.gpu
def test_stream_undeclared_access_fails():
    """A global access outside the declared allocations cannot be checked: the session fails loudly."""
    recs, tb = random_trace(7100, n_glob=3)
    ranges = declared_ranges(recs)
    with pytest.raises(bc.BcError) as e:
        streamed(recs, tb.geom.as_dict(), queue_records=len(recs) + 1, ranges=ranges[:-1] if len(ranges) > 1 else [(0, 1 << 20)])
    assert e.value.status == -1
