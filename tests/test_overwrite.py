"""GPU parity under BC_F_RELEASE_OVERWRITE (the printed release S_x := C_t, Fig. 3 P:L754-786;
reading R1's alternative).  K3 links each acquire to the window of its slot's latest writer
(DESIGN.md §3.1); the race lists must be bit-identical to the oracle run with F_RELEASE_OVERWRITE."""
import numpy as np
import pytest

import bcgen
import bcgen.configs
import oracle
import paper_conf_pldi_eizenbergppmd17_b200 as bc
from bcgen.configs import ConfigPlan
from bcgen.fuzz import random_trace

import litmus

pytestmark = pytest.mark.gpu
OW = oracle.F_RELEASE_OVERWRITE


def assert_parity(recs, geom, flags=OW, window_events=0):
    st_o, want, _ = oracle.detect_geom(recs, geom, flags)
    res = bc.detect(recs, geom, device="cuda:0", flags=flags, window_events=window_events)
    assert res.status == st_o, (res.status, st_o)
    if st_o == 0:
        got = res.races
        assert len(got) == len(want), (len(got), len(want))
        assert np.array_equal(got.view(np.uint8), want.view(np.uint8))
    return want


def triples(races):
    return sorted((int(r["kind"]), int(r["cls"]), int(r["space"])) for r in races)


@pytest.mark.parametrize("entry", litmus.OVERWRITE_SUITE, ids=[e[0] for e in litmus.OVERWRITE_SUITE])
def test_release_readings(entry):
    name, fn, want_join, want_ow = entry
    tb = fn()
    recs, geom = tb.records(), tb.geom.as_dict()
    assert triples(assert_parity(recs, geom, 0)) == want_join
    assert triples(assert_parity(recs, geom, OW)) == want_ow


@pytest.mark.parametrize("entry", litmus.SUITE, ids=[e[0] for e in litmus.SUITE])
def test_litmus_overwrite(entry):
    name, fn, expected, opts = entry
    tb = fn()
    want = assert_parity(tb.records(), tb.geom.as_dict())
    if "overwrite_expected" in opts:
        assert triples(want) == sorted(opts["overwrite_expected"])


@pytest.mark.parametrize("chunk", range(4))
def test_random_traces_overwrite(chunk):
    for seed in range(20000 + chunk * 60, 20000 + chunk * 60 + 60):
        recs, tb = random_trace(seed, p_sync=0.3, n_sync=2)
        assert_parity(recs, tb.geom.as_dict())


def test_random_traces_overwrite_big_blocks():
    for seed in range(21000, 21030):
        recs, tb = random_trace(seed, max_blocks=6, tpb=256, ops_per_warp=(10, 40), n_glob=6, n_sync=3, p_sync=0.25)
        assert_parity(recs, tb.geom.as_dict())


@pytest.mark.parametrize("we", [300, 5000])
def test_random_traces_overwrite_windows(we):
    for seed in range(22000, 22040):
        recs, tb = random_trace(seed, p_sync=0.3)
        assert_parity(recs, tb.geom.as_dict(), window_events=we)


@pytest.mark.parametrize("bug", [0, 1, 2, 3])
def test_c6_hashtable_overwrite(bug):
    """The lock-heavy hashtable (row f2): every critical section acquires the lock its predecessor
    released, so the two readings agree on the fixed program; the buggy ones race either way."""
    for kw in (dict(n_blocks=2, tpb=32, iters=1, log2_buckets=3), dict(n_blocks=6, tpb=64, iters=2, log2_buckets=5),
               dict(n_blocks=24, tpb=128, iters=2, log2_buckets=7)):
        plan = ConfigPlan(6, bug=bug, **kw)
        assert_parity(plan.records(), plan.geometry)


def test_c3_overwrite():
    plan = ConfigPlan(3, n_blocks=9, iters=3, tpb=256)
    assert_parity(plan.records(), plan.geometry)
