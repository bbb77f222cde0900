"""Parity of the CUDA path (through the C ABI) with the CPU oracle — element by element.

Bar (BASELINE.json north_star): the race set is bit-identical — same granule
addresses, same (prior, current) event pairs, same kind / class / space / block, same
canonical order — and the status (OK / INFEASIBLE) is the same.  All values are integers.
Cases: the paper's worked examples (Fig. 1, Fig. 4), the C1 litmus config, the 66-trace
suite, seeded random feasible traces (nested branches, barrier divergence, block / global
acquire-release, vector accesses, several granule sizes), an exhaustive tiny family,
infeasible traces, and C2-C5 at sizes the oracle finishes in seconds (several tiles and a
ragged tail) plus C2 at full size.
"""
import itertools

import numpy as np
import pytest

import bcgen
import oracle
import paper_conf_pldi_eizenbergppmd17_b200 as bc
from bcgen import GLOBAL_BASE, TraceBuilder
from bcgen.configs import ConfigPlan
from bcgen.fuzz import random_trace

import litmus

pytestmark = pytest.mark.gpu


def _gpu(recs, geom, flags=0, window_events=0):
    return bc.detect(recs, geom, device="cuda:0", flags=flags, window_events=window_events)


def assert_parity(recs, geom, flags=0, expect_status=None, window_events=0):
    st_o, want, stats_o = oracle.detect_geom(recs, geom, flags)
    res = _gpu(recs, geom, flags, window_events)
    assert res.status == st_o, (res.status, st_o)
    if expect_status is not None:
        assert st_o == expect_status
    if st_o != 0:
        return want, res
    got = res.races
    assert len(got) == len(want), (len(got), len(want), got[:4], want[:4])
    assert np.array_equal(got.view(np.uint8), want.view(np.uint8)), _first_diff(got, want)
    assert res.stats["lane_events"] == stats_o["lane_events"]
    assert res.stats["control_events"] == stats_o["control_events"]
    return want, res


def _first_diff(got, want):
    for i, (a, b) in enumerate(zip(got, want)):
        if a.tobytes() != b.tobytes():
            return i, a, b
    return None


# ------------------------------------------------------------------ paper examples
def test_c1_litmus():
    recs, tb = bcgen.configs.make_c1()
    want, res = assert_parity(recs, tb.geom.as_dict())
    assert len(want) == 1
    recs, tb = bcgen.configs.make_c1(with_sync=False)
    want, res = assert_parity(recs, tb.geom.as_dict())
    assert len(want) == 33


def test_fig4_message_passing():
    x, y = GLOBAL_BASE, GLOBAL_BASE + 0x100000
    for rel, acq in itertools.product(("blk", "glb"), repeat=2):
        tb = TraceBuilder(grid=(2,), block=(1,))
        tb.st(0, x)
        tb.rel(0, y, scope=rel)
        tb.acq(1, y, scope=acq)
        tb.ld(1, x)
        want, _ = assert_parity(tb.records(), tb.geom.as_dict())
        assert len(want) == (1 if (rel, acq) == ("blk", "blk") else 0)


def test_fig1_translation():
    a, b, d = GLOBAL_BASE, GLOBAL_BASE + 0x100, GLOBAL_BASE + 0x200
    tb = TraceBuilder(block=(2,))
    tb.ld(0, a); tb.if_(0, [0]); tb.st(0, b); tb.else_(0); tb.fi(0); tb.rel(0, d, scope="blk")
    assert_parity(tb.records(), tb.geom.as_dict())


@pytest.mark.parametrize("entry", litmus.SUITE, ids=[e[0] for e in litmus.SUITE])
def test_litmus_suite(entry):
    name, fn, expected, opts = entry
    tb = fn()
    want, res = assert_parity(tb.records(), tb.geom.as_dict())
    got = sorted((int(r["kind"]), int(r["cls"]), int(r["space"])) for r in res.races)
    assert got == expected


def test_same_value_flag():
    tb = TraceBuilder(block=(32,))
    tb.st(0, lambda l: GLOBAL_BASE if l < 3 else GLOBAL_BASE + 4 * l, same_value=True)
    assert_parity(tb.records(), tb.geom.as_dict())
    want, _ = assert_parity(tb.records(), tb.geom.as_dict(), flags=oracle.F_NO_SAME_VALUE_FILTER)
    assert len(want) == 2


# ------------------------------------------------------------------ random traces
@pytest.mark.parametrize("chunk", range(6))
def test_random_traces(chunk):
    for seed in range(chunk * 50, chunk * 50 + 50):
        recs, tb = random_trace(seed)
        assert_parity(recs, tb.geom.as_dict())


@pytest.mark.parametrize("G", [0, 1, 3, 4])
def test_random_traces_granules(G):
    for seed in range(2000, 2030):
        recs, tb = random_trace(seed, granule_log2=G)
        assert_parity(recs, tb.geom.as_dict())


def test_random_traces_big_blocks():
    for seed in range(3000, 3012):
        recs, tb = random_trace(seed, max_blocks=6, tpb=256, ops_per_warp=(10, 40), n_glob=6, n_sync=3)
        assert_parity(recs, tb.geom.as_dict())


def test_random_traces_same_value():
    for seed in range(4000, 4030):
        recs, tb = random_trace(seed, same_value=True)
        assert_parity(recs, tb.geom.as_dict())
        assert_parity(recs, tb.geom.as_dict(), flags=oracle.F_NO_SAME_VALUE_FILTER)


def test_exhaustive_sample():
    """Every 5th program of the exhaustive 2-warp x 2-lane family of test_oracle_pins."""
    from test_oracle_pins import _alphabet
    ops, addr, s = _alphabet()
    orders = [o for o in itertools.product([0, 1], repeat=4) if sum(o) == 2]
    k = 0
    for p0 in itertools.product(range(len(ops)), repeat=2):
        for p1 in itertools.product(range(len(ops)), repeat=2):
            for order in orders:
                k += 1
                if k % 5:
                    continue
                tb = TraceBuilder(grid=(2,), block=(2,))
                pcs = [0, 0]
                progs = [p0, p1]
                for w in order:
                    kind, pat = ops[progs[w][pcs[w]]]
                    pcs[w] += 1
                    if kind == "rel":
                        tb.rel(w, s)
                    elif kind == "acq":
                        tb.acq(w, s)
                    elif kind == "br":
                        tb.if_(w, [0]); tb.st(w, addr(0)); tb.else_(w); tb.ld(w, addr(0)); tb.fi(w)
                    else:
                        getattr(tb, kind)(w, addr(pat))
                assert_parity(tb.records(), tb.geom.as_dict())


# ------------------------------------------------------------------ infeasible / edge
def _infeasible():
    from test_oracle_pins import _infeasible_traces
    return _infeasible_traces()


@pytest.mark.parametrize("case", _infeasible(), ids=lambda c: c[0])
def test_infeasible(case):
    name, tb = case
    assert_parity(tb.records(), tb.geom.as_dict(), expect_status=oracle.INFEASIBLE)


def test_empty_trace():
    recs = np.zeros(0, dtype=bcgen.RECORD_DTYPE)
    res = _gpu(recs, dict(grid=(1,), block=(32,), smem_bytes=0))
    assert res.status == 0 and len(res.races) == 0


def test_control_only_trace():
    tb = TraceBuilder(block=(64,))
    tb.fence(0); tb.bar(0); tb.bar(1); tb.if_(1, 0); tb.else_(1); tb.fi(1)
    assert_parity(tb.records(), tb.geom.as_dict())


def test_depth_32():
    tb = TraceBuilder(block=(32,))
    for _ in range(32):
        tb.if_(0, 0xFFFFFFFF)
    tb.st(0, lambda l: GLOBAL_BASE + 4 * (l // 2))
    for _ in range(32):
        tb.else_(0); tb.fi(0)
    tb.ld(0, lambda l: GLOBAL_BASE + 4 * ((l + 1) % 16))
    assert_parity(tb.records(), tb.geom.as_dict())


def test_hot_granule_long_segment():
    """One granule touched by thousands of reads and writes from many warps / blocks: the
    segment spans many K7 tiles (range-scan carries), with inflated read vectors."""
    _hot_granule()


def _hot_granule(window_events=0):
    tb = TraceBuilder(grid=(4,), block=(256,))
    hot = GLOBAL_BASE + 0x40
    import random
    rng = random.Random(7)
    for it in range(60):
        for b in range(4):
            for wib in range(8):
                w = tb.warp(b, wib)
                r = rng.random()
                if r < 0.7:
                    tb.ld(w, hot)
                elif r < 0.85:
                    tb.atom(w, hot)
                else:
                    tb.st(w, lambda l: hot if l == rng.randrange(32) else GLOBAL_BASE + 0x1000 + 4 * l)
    want, _ = assert_parity(tb.records(), tb.geom.as_dict(), window_events=window_events)
    assert len(want) > 100


# ------------------------------------------------------------------ configs
@pytest.mark.parametrize("cfg,kw", [
    (2, dict(n_blocks=8, iters=6)),
    (2, dict(n_blocks=5, iters=3, tpb=96)),
    (3, dict(n_blocks=16, iters=2, tpb=64)),
    (3, dict(n_blocks=9, iters=3, tpb=256)),
    (4, dict(n_blocks=12, log2_nodes=14, nodes_per_thread=2, inj_scale=4)),
    (4, dict(n_blocks=40, log2_nodes=16, nodes_per_thread=3, inj_scale=8)),
    (5, dict(n_blocks=8, log2_nodes=15, nodes_per_thread=3, inj_scale=4)),
])
def test_configs_reduced(cfg, kw):
    plan = ConfigPlan(cfg, **kw)
    recs = plan.records()
    want, res = assert_parity(recs, plan.geometry)
    if cfg in (4, 5):
        truth = plan.truth()
        assert np.array_equal(np.sort(want.view("V32")), np.sort(truth.view("V32")))


def test_c3_64_blocks():
    plan = ConfigPlan(3, n_blocks=64)
    assert_parity(plan.records(), plan.geometry)


def test_c4_64_blocks():
    plan = ConfigPlan(4, n_blocks=64)
    assert_parity(plan.records(), plan.geometry)


@pytest.mark.slow
def test_c2_full_size():
    plan = ConfigPlan(2)
    want, res = assert_parity(plan.records(), plan.geometry)
    assert len(want) == 0 and res.stats["lane_events"] > 9_000_000


# ------------------------------------------------------------------ API behaviour
def test_device_borrowed_trace_and_idempotent():
    import torch
    recs, tb = bcgen.configs.make_c1(with_sync=False)
    geom = tb.geom.as_dict()
    st, want, _ = oracle.detect_geom(recs, geom)
    dev = torch.from_numpy(recs.view(np.uint8).copy()).cuda()
    with bc.Context(geom, device=0) as ctx:
        ctx.load_trace(dev)
        for _ in range(3):
            st2, stats = ctx.detect()
            assert st2 == 0
            got = ctx.races()
            assert np.array_equal(got.view(np.uint8), want.view(np.uint8))
        out = torch.zeros(len(want) * 32, dtype=torch.uint8, device="cuda")
        assert ctx.races_device(out) == len(want)
        assert np.array_equal(out.cpu().numpy(), want.view(np.uint8))


# ------------------------------------------------------------------ windows (row a5)
@pytest.mark.parametrize("we", [64, 700, 9000])
def test_windows(we):
    """The trace checked in windows of at most `we` weight (bc_config.window_events): every granule's
    state (last writer, read epoch or read vector, atomic bit: the 32-B shadow entry of Fig. 8,
    P:L1247-1268) is carried from window to window; the race set must not change.  Tiny windows
    put window boundaries inside read runs, after inflations, between a writer and its readers."""
    for seed in range(5000, 5040):
        recs, tb = random_trace(seed)
        _, res = assert_parity(recs, tb.geom.as_dict(), window_events=we)
        assert res.stats["windows"] >= 1
    _hot_granule(window_events=we)
    for cfg, kw in [(2, dict(n_blocks=8, iters=6)), (3, dict(n_blocks=9, iters=3, tpb=256)),
                    (4, dict(n_blocks=40, log2_nodes=16, nodes_per_thread=3, inj_scale=8))]:
        plan = ConfigPlan(cfg, **kw)
        _, res = assert_parity(plan.records(), plan.geometry, window_events={64: 3000, 700: 12000}.get(we, 30000))
        assert res.stats["windows"] > 1


def test_windows_litmus_and_vectors():
    """The 66 litmus traces and random traces with many readers (read vectors carried across windows)
    in windows of one or two records."""
    for name, build, _exp, _opts in litmus.SUITE:
        tb = build()
        assert_parity(tb.records(), tb.geom.as_dict(), window_events=16)
    for seed in range(5100, 5130):
        recs, tb = random_trace(seed, n_glob=2, tpb=128, ops_per_warp=(10, 30))
        _, res = assert_parity(recs, tb.geom.as_dict(), window_events=40)
        assert res.stats["windows"] > 5


def test_long_read_run_after_write():
    """One write, then ~20 K reads of one granule by ~20 K threads and few other items (the
    reads span many K7 warp ranges: the state entering each comes from the range-tail scan, there is
    no walk cap and no wait on another warp), then a plain write that races with every reader."""
    tb = TraceBuilder(grid=(80,), block=(256,))
    flag = GLOBAL_BASE + 0x80
    tb.st(tb.warp(0, 0), lambda l: flag if l == 0 else GLOBAL_BASE + 0x1000 + 4 * l)
    for b in range(80):
        for wib in range(8):
            tb.ld(tb.warp(b, wib), flag)
    tb.st(tb.warp(79, 7), lambda l: flag if l == 3 else GLOBAL_BASE + 0x2000 + 4 * l)
    want, res = assert_parity(tb.records(), tb.geom.as_dict())
    assert len(want) > 20_000
    assert_parity(tb.records(), tb.geom.as_dict(), window_events=2000)


def test_torch_allocator():
    """bc_config.dev_alloc / dev_free over torch's caching allocator."""
    import torch
    recs, tb = random_trace(77)
    geom = tb.geom.as_dict()
    st, want, _ = oracle.detect_geom(recs, geom)
    before = torch.cuda.memory_allocated()
    with bc.Context(geom, device=0, allocator="torch") as ctx:
        ctx.load_trace(recs)
        assert ctx.detect()[0] == 0
        assert torch.cuda.memory_allocated() > before
        assert np.array_equal(ctx.races().view(np.uint8), want.view(np.uint8))
    assert torch.cuda.memory_allocated() == before


# ------------------------------------------------- lock-heavy hashtable
@pytest.mark.parametrize("bug", [0, 1, 2, 3])
def test_c6_hashtable(bug):
    """Per-bucket locks: K3 with thousands of single-lane acquire / release
    records and SPARSEVC-style foreign knowledge; the fixed program and both section-6.3 bugs.
    The fixed program (acquire AND release on every lock) chains every critical section of a
    bucket to the next; its foreign-knowledge queries find the ordering in the view of the newest
    acquire the thread knows, at every size."""
    sizes = (dict(n_blocks=1, tpb=32, iters=1, log2_buckets=1),
             dict(n_blocks=2, tpb=32, iters=1, log2_buckets=3),
             dict(n_blocks=6, tpb=64, iters=2, log2_buckets=5),
             dict(n_blocks=24, tpb=128, iters=2, log2_buckets=7))
    for i, kw in enumerate(sizes):
        plan = ConfigPlan(6, bug=bug, **kw)
        recs = plan.records()
        want, _ = assert_parity(recs, plan.geometry)
        if i > 0:  # (one warp alone: its lanes' turns are ordered by the FI joins anyway)
            assert (len(want) == 0) == (bug == 0)


@pytest.mark.slow
def test_c6_fixed_program_sizes():
    """The fixed hashtable (bug = 0) against the oracle at 64 blocks (131 K records, ~3 min of oracle
    time: its uncompressed vector clocks grow along the lock chains), and at the bench size (256 x 128
    threads, 526 K records; beyond the oracle's memory) race-free as the program is by construction."""
    plan = ConfigPlan(6, bug=0, n_blocks=64)
    want, res = assert_parity(plan.records(), plan.geometry)
    assert len(want) == 0 and res.stats["sync_ops"] > 10_000
    plan = ConfigPlan(6, bug=0)
    res = _gpu(plan.records(), plan.geometry)
    assert res.status == 0 and len(res.races) == 0 and res.stats["sync_ops"] > 60_000


def test_c6_hashtable_bench_shape():
    """The bench workload's shape (128-thread blocks, 2 inserts per thread, 4096 buckets, both
    bugs) at 32 of its 256 blocks."""
    plan = ConfigPlan(6, n_blocks=32)
    want, res = assert_parity(plan.records(), plan.geometry)
    assert len(want) > 0


def test_c6_full_size():
    """The c6 bench workload at full size (526 K records, ~184 K races) against the oracle."""
    plan = ConfigPlan(6)
    want, res = assert_parity(plan.records(), plan.geometry)
    assert len(want) > 100_000


# ------------------------------------------- per-lane store values (reading R6b)
def test_values_random_traces():
    """bc_load_values: the same-value filter compares per-lane store values; parity with the
    oracle on random traces (values partly uniform, partly colliding), host and device values."""
    import torch
    from bcgen.fuzz import random_values
    for seed in range(8000, 8060):
        recs, tb = random_trace(seed, same_value=True, n_glob=2)
        geom = tb.geom.as_dict()
        vals = random_values(recs, seed)
        st_o, want, _ = oracle.detect_geom(recs, geom, values=vals)
        res = bc.detect(recs, geom, device="cuda:0", values=vals)
        assert res.status == st_o
        if st_o == 0:
            assert np.array_equal(res.races.view(np.uint8), want.view(np.uint8)), seed
    recs, tb = random_trace(8100, same_value=True, n_glob=2)
    geom = tb.geom.as_dict()
    vals = random_values(recs, 8100)
    st_o, want, _ = oracle.detect_geom(recs, geom, values=vals)
    with bc.Context(geom, device=0) as ctx:
        ctx.load_trace(recs)
        ctx.load_values(torch.from_numpy(vals).cuda())
        assert ctx.detect()[0] == 0
        assert np.array_equal(ctx.races().view(np.uint8), want.view(np.uint8))
        ctx.load_values(None)  # cleared: back to the record flags
        assert ctx.detect()[0] == 0
        st_f, want_f, _ = oracle.detect_geom(recs, geom)
        assert np.array_equal(ctx.races().view(np.uint8), want_f.view(np.uint8))


@pytest.mark.parametrize("we", [0, 100])
def test_values_byte_granules(we):
    """Values with byte granules (G = 0, the paper's default) and mixed access
    sizes, in one window and in many."""
    from bcgen.fuzz import random_values
    for seed in range(8200, 8240):
        recs, tb = random_trace(seed, same_value=True, n_glob=2, granule_log2=0)
        geom = tb.geom.as_dict()
        vals = random_values(recs, seed)
        st_o, want, _ = oracle.detect_geom(recs, geom, values=vals)
        res = bc.detect(recs, geom, device="cuda:0", values=vals, window_events=we)
        assert res.status == st_o
        if st_o == 0:
            assert np.array_equal(res.races.view(np.uint8), want.view(np.uint8)), seed


# ------------------------------------------------ warp-size simulation
@pytest.mark.parametrize("ws", [16, 8, 4])
def test_warpsim_random_traces(ws):
    """Traces re-split into virtual warps of ws lanes (bcgen.warpsim): bc_config.warp_size = ws;
    bit-exact with the oracle (infeasible splits -- a BAR inside warp-divergent code -- must be
    rejected by both)."""
    from bcgen.warpsim import split_warps
    for seed in range(9100, 9160):
        recs, tb = random_trace(seed)
        r2, g2, _ = split_warps(recs, tb.geom.as_dict(), ws)
        assert_parity(r2, g2)


@pytest.mark.parametrize("ws", [16, 8, 4, 32])
def test_split_warps_in_libbc(ws):
    """bc_split_warps (the re-split inside libbc) produces the same records and origins
    as the input transform of bcgen.warpsim (the fixture the oracle tests use), and the GPU check of the
    GPU-split trace equals the oracle on it."""
    from bcgen.warpsim import split_warps
    for seed in list(range(9300, 9330)) + [None]:
        if seed is None:
            plan = ConfigPlan(3, n_blocks=6, iters=2, tpb=64)
            recs, geom = plan.records(), plan.geometry
        else:
            recs, tb = random_trace(seed)
            geom = tb.geom.as_dict()
        r2, g2, org = split_warps(recs, geom, ws)
        d, gg, dorg = bc.split_warps(recs, geom, ws)
        got = d.cpu().numpy().view(bcgen.RECORD_DTYPE)
        assert len(got) == len(r2), (seed, len(got), len(r2))
        assert np.array_equal(got.view(np.uint8), r2.view(np.uint8)), seed
        o = dorg.cpu().numpy()
        assert np.array_equal(o >> 5, org[:, 0]) and np.array_equal(o & 31, org[:, 1])
        st_o, want, _ = oracle.detect_geom(r2, g2)
        res = bc.detect(d, gg, device="cuda:0")
        assert res.status == st_o
        if st_o == 0:
            assert np.array_equal(res.races.view(np.uint8), want.view(np.uint8))


@pytest.mark.parametrize("cfg,kw", [(2, dict(n_blocks=4, iters=3)), (3, dict(n_blocks=6, iters=2, tpb=64)),
                                    (4, dict(n_blocks=8, log2_nodes=13, nodes_per_thread=2, inj_scale=4))])
def test_warpsim_configs(cfg, kw):
    """C2-C4 shapes with 16- and 8-lane virtual warps (block sizes up to 256 threads = 32 virtual
    warps of 8)."""
    from bcgen.warpsim import split_warps
    plan = ConfigPlan(cfg, **kw)
    recs = plan.records()
    for ws in (16, 8):
        r2, g2, _ = split_warps(recs, plan.geometry, ws)
        assert_parity(r2, g2)


# ------------------------------------------------ full-size configs (bench launch configuration)
def _golden(name):
    from test_oracle_pins import _golden as g
    return g(name)


def _device_trace(plan, chunk=1 << 20):
    """The plan's records generated straight into one device buffer, chunk by chunk through a pinned
    host buffer (C5's 52 GB trace never exists in host memory)."""
    import torch
    n = plan.n_records
    dev = torch.empty(n * 272, dtype=torch.uint8, device="cuda")
    host = torch.empty(min(n, chunk) * 272, dtype=torch.uint8).pin_memory()
    for b in range(0, n, chunk):
        e = min(n, b + chunk)
        plan.fill(host, b, e)
        dev[b * 272:e * 272].copy_(host[:(e - b) * 272], non_blocking=False)
    return dev


def _assert_same(got, want):
    assert len(got) == len(want), (len(got), len(want))
    assert np.array_equal(got.view(np.uint8), want.view(np.uint8)), _first_diff(got, want)


@pytest.mark.slow
def test_c2_full_size_injected():
    """C2 at the bench size with its injected variant (8 blocks with an unsynchronised exchange): the
    GPU list equals the stored oracle list byte for byte (tools/make_golden.py) and the generator's
    closed form (32 INTRA_BLOCK races per injected block)."""
    plan = ConfigPlan(2, inject=1)
    head, want = _golden("c2_inj")
    assert plan.n_records == int(head["records"])
    res = _gpu(plan.records(), plan.geometry)
    assert res.status == 0
    _assert_same(res.races, want)
    assert np.array_equal(np.sort(want.view("V32")), np.sort(plan.truth().view("V32")))


@pytest.mark.slow
def test_c3_full_size():
    """C3 at the bench size (4096 x 256 threads, ~50 M events, 4096 AR_GLB tickets): race-free by
    construction (every shared access is ordered by a barrier, the partial sums by fence + ticket,
    P:L314-336; the oracle confirms it up to 256 blocks), and its injected variant (block 0's ticket
    without the fence) reports exactly the generator's two races; at 256 blocks the injected list
    equals the stored oracle list."""
    plan = ConfigPlan(3)
    res = _gpu(plan.records(), plan.geometry)
    assert res.status == 0
    assert len(res.races) == 0 and res.stats["lane_events"] > 40_000_000
    plan = ConfigPlan(3, inject=1)
    res = _gpu(plan.records(), plan.geometry)
    truth = plan.truth()
    assert res.status == 0 and len(truth) == 2
    assert np.array_equal(np.sort(res.races.view("V32")), np.sort(truth.view("V32")))
    head, want = _golden("c3_inj")
    plan = ConfigPlan(3, inject=1, n_blocks=256)  # tools/make_golden.py GOLDEN["c3_inj"]
    assert plan.n_records == int(head["records"])
    res = _gpu(plan.records(), plan.geometry)
    _assert_same(res.races, want)


@pytest.mark.slow
@pytest.mark.parametrize("we", [0, 1 << 27])
def test_c4_full_size_golden(we):
    """C4 at the bench size (1 M threads, 218 M lane events, 38 M records), one window and ~4 windows:
    the race list equals the oracle's full-size list byte for byte (tests/golden/c4_oracle_races.txt,
    800 s of oracle time, written by tools/make_golden.py)."""
    plan = ConfigPlan(4)
    head, want = _golden("c4")
    assert plan.n_records == int(head["records"])
    res = bc.detect(_device_trace(plan), plan.geometry, device="cuda:0", window_events=we)
    assert res.status == 0
    assert res.stats["windows"] == (1 if we == 0 else 4)
    _assert_same(res.races, want)


@pytest.mark.slow
def test_c5_full_size_truth():
    """C5 at full size (16384 x 256 = 4 M threads, 193 M records, 1.09 G lane events, a 52 GB trace) on
    one B200: more than 2^27 records, so the check runs in windows with the shadow state carried
    between them; the race set equals the generator's injected set (4x C4's counts).  (The oracle
    cannot run this size: SURVEY §8(d.4).)"""
    import torch
    plan = ConfigPlan(5)
    assert plan.n_records > (1 << 27)
    truth = plan.truth()
    res = bc.detect(_device_trace(plan), plan.geometry, device="cuda:0")
    assert res.status == 0
    assert res.stats["windows"] > 1 and res.stats["lane_events"] > 1_000_000_000
    assert len(truth) > 0
    assert np.array_equal(np.sort(res.races.view("V32")), np.sort(truth.view("V32")))
    torch.cuda.empty_cache()


# ------------------------------------------------------------------ sampled page set (k_header)
def test_sampled_page_set_miss_reruns_exactly():
    """k_header marks written pages from each write record's first and last active lanes only; a page
    written solely by middle lanes is missing from the sample.  K4 sees the write, flags it and the
    detect re-runs with every write address marked: the races on that page (a write by block 0's middle
    lanes, read and rewritten by block 1) must all be found, bit-identical to the oracle."""
    MB = 1 << 20
    tb = TraceBuilder(grid=(2, 1, 1), block=(32, 1, 1))
    w0, w1 = tb.warp(0), tb.warp(1)
    # lanes 0 and 31 write page 0, lanes 1..30 write page 5 (never sampled)
    tb.st(w0, lambda l: GLOBAL_BASE + (0 if l in (0, 31) else 5 * MB) + 4 * l)
    tb.ld(w1, lambda l: GLOBAL_BASE + 5 * MB + 4 * l)
    tb.st(w1, lambda l: GLOBAL_BASE + 5 * MB + 4 * l)
    recs = tb.records()
    want, res = assert_parity(recs, tb.geom.as_dict())
    assert len(want) == 2 * 30  # WR then WW on each of the 30 middle granules
    # the same with several windows (the miss is found in the first one)
    assert_parity(recs, tb.geom.as_dict(), window_events=40)
