"""Pins of the CPU oracle against things other than itself (CPU only).

* Fig. 4 message-passing verdicts and Fig. 1's worked trace (tests/golden/).
* The C1 litmus config: its race set follows from the rules by hand.
* The §3.2 definition: a brute-force transitive closure (oracle/bf.py).
  Theorem 1 + Lemmas 1-2 give: every reported pair is unordered
  (soundness, always), and on granules where the printed atomic rules agree
  with §3.2 (SURVEY §8(c.4) amb. 3) the first racy access per granule — and
  so the per-granule verdict — is the same.  Checked on an exhaustive family
  of tiny traces and on random feasible traces.
* The FastTrack invariant of §3.4, asserted after every record.
* 66 re-authored litmus traces (§6.1 categories), expected multisets by hand.
* Closed forms: race-free-by-construction configs (C2, C3 at reduced size)
  report nothing; C4 reports exactly its injected races.
* Infeasible traces are rejected.
"""
import itertools
import json
import os

import numpy as np
import pytest

import bcgen
import oracle
from bcgen import TraceBuilder, GLOBAL_BASE
from bcgen.configs import ConfigPlan
from bcgen.fuzz import random_trace
from bcgen.format import KIND_NAMES
from oracle.bf import brute_force, valid_granules

import litmus

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
KIND = {n: i for i, n in enumerate(bcgen.KIND_NAMES)}
CLS = {n: i for i, n in enumerate(bcgen.CLS_NAMES)}


def run(recs, geom, flags=0):
    st, races, stats = oracle.detect_geom(recs, geom, flags)
    assert st == 0, st
    return races


def loc_of(r, G=2):
    sp = int(r["space"])
    return (sp, int(r["block"]) if sp == 1 else 0, int(r["addr"]) >> G)


def check_against_bf(recs, geom, races, strict=True, values=None):
    """Soundness always; first racy event + verdict per valid granule."""
    G = geom["granule_log2"]
    bf = brute_force(recs, geom["grid"], geom["block"], G, values=values, warp_size=geom.get("warp_size", 32))
    bfset = bf.race_set()
    orset = {(loc_of(r, G), int(r["prior_event"]), int(r["cur_event"])) for r in races if r["cls"] != 4}
    assert orset <= bfset, sorted(orset - bfset)[:5]
    if not strict:
        return bf
    valid = valid_granules(bf)
    first_bf, first_or = {}, {}
    for (l, p, c) in bfset:
        first_bf[l] = min(c, first_bf.get(l, c))
    for (l, p, c) in orset:
        first_or[l] = min(c, first_or.get(l, c))
    for l in valid:
        assert first_bf.get(l) == first_or.get(l), (l, first_bf.get(l), first_or.get(l))
    return bf


# --------------------------------------------------------------- golden pins
def test_fig4_message_passing():
    cases = json.load(open(os.path.join(GOLDEN, "fig4_mp.json")))["cases"]
    x, y = GLOBAL_BASE, GLOBAL_BASE + 0x100000
    for c in cases:
        tb = TraceBuilder(grid=(2,), block=(1,))
        st_rec = tb.st(0, x)
        tb.rel(0, y, scope=c["rel"])
        tb.acq(1, y, scope=c["acq"])
        ld_rec = tb.ld(1, x)
        races = run(tb.records(), tb.geom.as_dict())
        assert len(races) == len(c["races"]), c
        for r, e in zip(races, c["races"]):
            assert r["kind"] == KIND[e["kind"]] and r["cls"] == CLS[e["cls"]] and r["space"] == 0
            assert r["addr"] == x and r["prior_event"] == st_rec << 5 and r["cur_event"] == ld_rec << 5
        check_against_bf(tb.records(), tb.geom.as_dict(), races)


def test_fig1_translation():
    g = json.load(open(os.path.join(GOLDEN, "fig1.json")))
    a, b, d = GLOBAL_BASE, GLOBAL_BASE + 0x100, GLOBAL_BASE + 0x200
    tb = TraceBuilder(block=(2,))
    tb.ld(0, a); tb.if_(0, [0]); tb.st(0, b); tb.else_(0); tb.fi(0); tb.rel(0, d, scope="blk")
    recs = tb.records()
    assert [bcgen.OP_NAMES[o] for o in recs["op"]] == [r["op"] for r in g["records"]]
    assert list(recs["mask"]) == [3, 3, 1, 1, 2, 3]
    st, races, stats = oracle.detect_geom(recs, tb.geom.as_dict())
    assert st == 0 and len(races) == len(g["races"]) == 0
    # thread ops in Fig. 1(b): 2 rd + 1 wr + 2 relBlk lane events; if/else/fi control
    assert stats["lane_events"] == 5 and stats["control_events"] == 3
    check_against_bf(recs, tb.geom.as_dict(), races)


def test_c1_litmus():
    recs, tb = bcgen.configs.make_c1()
    races = run(recs, tb.geom.as_dict())
    assert len(races) == 1
    r = races[0]
    assert (r["kind"], r["cls"], r["space"]) == (KIND["WW"], CLS["INTER_BLOCK"], 0)
    assert r["addr"] == GLOBAL_BASE + 0x200000
    # prior = block 0 lane 5's store, cur = block 1 lane 5's store
    assert recs[int(r["prior_event"]) >> 5]["warp"] == 0 and int(r["prior_event"]) & 31 == 5
    assert recs[int(r["cur_event"]) >> 5]["warp"] == 1 and int(r["cur_event"]) & 31 == 5
    check_against_bf(recs, tb.geom.as_dict(), races)
    recs2, tb2 = bcgen.configs.make_c1(with_sync=False)
    races2 = run(recs2, tb2.geom.as_dict())
    kinds = sorted(int(x["kind"]) for x in races2)
    assert kinds == [KIND["WW"]] + [KIND["WR"]] * 32
    check_against_bf(recs2, tb2.geom.as_dict(), races2)


# ------------------------------------------------------------- litmus suite
@pytest.mark.parametrize("entry", litmus.SUITE, ids=[e[0] for e in litmus.SUITE])
def test_litmus(entry):
    name, fn, expected, opts = entry
    tb = fn()
    recs, geom = tb.records(), tb.geom.as_dict()
    races = run(recs, geom, oracle.F_CHECK_INVARIANT)
    got = sorted((int(r["kind"]), int(r["cls"]), int(r["space"])) for r in races)
    assert got == expected, (name, got, expected)
    bf = check_against_bf(recs, geom, races, strict=not opts.get("atomic_gap"))
    if opts.get("atomic_gap"):
        assert len(bf.race_set()) == 1  # §3.2 has the race the printed rules miss
    if "overwrite_expected" in opts:
        races_o = run(recs, geom, oracle.F_RELEASE_OVERWRITE)
        got_o = sorted((int(r["kind"]), int(r["cls"]), int(r["space"])) for r in races_o)
        assert got_o == sorted(opts["overwrite_expected"])


def test_same_value_filter_flag():
    tb = TraceBuilder(block=(32,))
    tb.st(0, lambda l: GLOBAL_BASE if l < 3 else GLOBAL_BASE + 4 * l, same_value=True)
    assert len(run(tb.records(), tb.geom.as_dict())) == 0
    races = run(tb.records(), tb.geom.as_dict(), oracle.F_NO_SAME_VALUE_FILTER)
    assert len(races) == 2 and all(r["cls"] == CLS["SAME_INSN"] for r in races)


# ----------------------------------------------------- brute-force property
@pytest.mark.parametrize("chunk", range(8))
def test_random_traces_vs_bruteforce(chunk):
    for seed in range(chunk * 60, chunk * 60 + 60):
        recs, tb = random_trace(seed)
        geom = tb.geom.as_dict()
        st, races, _ = oracle.detect_geom(recs, geom, oracle.F_CHECK_INVARIANT)
        assert st == 0, (seed, st)
        check_against_bf(recs, geom, races)


def test_random_traces_vector_and_granule():
    for seed in range(1000, 1060):
        for G in (0, 3):
            recs, tb = random_trace(seed, granule_log2=G)
            geom = tb.geom.as_dict()
            st, races, _ = oracle.detect_geom(recs, geom, oracle.F_CHECK_INVARIANT)
            assert st == 0
            check_against_bf(recs, geom, races)


def _alphabet():
    g0, g1, s = GLOBAL_BASE, GLOBAL_BASE + 4, GLOBAL_BASE + 0x1000

    def addr(pat):
        return {0: lambda l: g0 if l == 0 else g1, 1: lambda l: g1 if l == 0 else g0,
                2: lambda l: g0}[pat]
    ops = [("ld", 0), ("st", 0), ("st", 2), ("atom", 2), ("ld", 1), ("rel", None), ("acq", None),
           ("br", None)]
    return ops, addr, s


def test_exhaustive_two_warps_two_lanes():
    """Every program of 2 ops per warp over an 8-op alphabet, for two 2-lane
    warps in different blocks, under every interleaving of the 4 ops."""
    ops, addr, s = _alphabet()
    orders = [o for o in itertools.product([0, 1], repeat=4) if sum(o) == 2]
    n = 0
    for p0 in itertools.product(range(len(ops)), repeat=2):
        for p1 in itertools.product(range(len(ops)), repeat=2):
            for order in orders:
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
                recs, geom = tb.records(), tb.geom.as_dict()
                races = run(recs, geom)
                check_against_bf(recs, geom, races)
                n += 1
    assert n == 8 ** 4 * 6


# ------------------------------------------------------------ closed forms
def test_c2_reduced_race_free():
    plan = ConfigPlan(2, n_blocks=3, iters=3)
    races = run(plan.records(), plan.geometry)
    assert len(races) == 0


def test_c3_reduced_race_free():
    plan = ConfigPlan(3, n_blocks=8, iters=2, tpb=64)
    races = run(plan.records(), plan.geometry)
    assert len(races) == 0


def test_c3_small_vs_bruteforce():
    plan = ConfigPlan(3, n_blocks=3, iters=1, tpb=32)
    recs = plan.records()
    races = run(recs, plan.geometry)
    assert len(races) == 0
    bf = brute_force(recs, plan.geometry["grid"], plan.geometry["block"], 2)
    assert len(bf.race_set()) == 0


def test_c4_reduced_exactly_injected():
    plan = ConfigPlan(4, n_blocks=12, log2_nodes=14, nodes_per_thread=2, inj_scale=4)
    recs = plan.records()
    races = run(recs, plan.geometry)
    truth = plan.truth()
    assert len(truth) > 0
    assert np.array_equal(np.sort(races.view("V32")), np.sort(truth.view("V32")))


@pytest.mark.parametrize("kw", [dict(n_blocks=8, iters=6, inj_scale=3), dict(n_blocks=5, iters=4, tpb=96, inj_scale=2)])
def test_c2_injected_exactly_truth(kw):
    """C2's injected variant (a missing barrier): warp 0 stores scratch[lane] and warp 1
    loads it in one barrier interval of a seeded iteration -> exactly one WR / RW INTRA_BLOCK race per
    lane in each injected block, and nothing else races; brute force (§3.2) confirms the smallest."""
    plan = ConfigPlan(2, inject=1, **kw)
    recs = plan.records()
    races = run(recs, plan.geometry)
    truth = plan.truth()
    assert len(truth) == 32 * kw["inj_scale"]
    assert set(truth["cls"]) == {2} and set(truth["space"]) == {1}
    assert np.array_equal(np.sort(races.view("V32")), np.sort(truth.view("V32")))


def test_c2_injected_vs_bruteforce():
    plan = ConfigPlan(2, inject=1, n_blocks=2, iters=2, tpb=64, inj_scale=1)
    recs = plan.records()
    races = run(recs, plan.geometry)
    assert len(races) == 32
    check_against_bf(recs, plan.geometry, races)


@pytest.mark.parametrize("kw", [dict(n_blocks=16, iters=2, tpb=64), dict(n_blocks=24, iters=1, tpb=128)])
def test_c3_injected_exactly_truth(kw):
    """C3's injected variant: block 0 takes its ticket with a plain atomicInc (no fence, so no release,
    P:L314-336): the last block's read of part[0] races with block 0's store (WR INTER_BLOCK) and its
    final count = 0 with block 0's atomic (AW INTER_BLOCK) -- exactly these two."""
    plan = ConfigPlan(3, inject=1, **kw)
    recs = plan.records()
    races = run(recs, plan.geometry)
    truth = plan.truth()
    assert sorted(truth["kind"].tolist()) == [1, 4] and set(truth["cls"]) == {3}
    assert np.array_equal(np.sort(races.view("V32")), np.sort(truth.view("V32")))


def test_c3_injected_vs_bruteforce():
    plan = ConfigPlan(3, inject=1, n_blocks=3, iters=1, tpb=32)
    recs = plan.records()
    races = run(recs, plan.geometry)
    assert len(races) == 2
    check_against_bf(recs, plan.geometry, races)


def _golden(name):
    """tests/golden/<name>_oracle_races.txt (tools/make_golden.py: written by the oracle alone)"""
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", f"{name}_oracle_races.txt")
    head, rows = {}, []
    for line in open(path):
        if line.startswith("#"):
            for tok in line[1:].split():
                if "=" in tok:
                    k, v = tok.split("=", 1)
                    head[k] = v
            continue
        a, p, c, kind, cls, space, blk = line.split()
        rows.append((int(a, 16), int(p, 16), int(c, 16), int(kind), int(cls), int(space), 0, int(blk)))
    return head, np.array(rows, dtype=bcgen.RACE_DTYPE)


def test_golden_c4_is_the_injected_set():
    """The stored full-size C4 oracle list (13 min of oracle time) is exactly the generator's
    injected set, and covers the three injected kinds (WW INTER_BLOCK, WR BRANCH, AR INTER_BLOCK)."""
    head, races = _golden("c4")
    assert int(head["races"]) == len(races) == 2304
    kinds = {(int(k), int(c)) for k, c in zip(races["kind"], races["cls"])}
    assert kinds == {(0, 3), (1, 1), (6, 3)}
    plan = ConfigPlan(4)
    assert plan.n_records == int(head["records"])
    truth = plan.truth()
    assert np.array_equal(np.sort(races.view("V32")), np.sort(truth.view("V32")))


# ---------------------------------------------------------------- infeasible
def _infeasible_traces():
    X = GLOBAL_BASE
    out = []
    tb = TraceBuilder(block=(32,)); tb.raw(0, 0xFFFF, bcgen.OP_LD, addrs=lambda l: X)  # mask != top
    out.append(("mask_mismatch", tb))
    tb = TraceBuilder(block=(32,)); tb.raw(0, 0xFFFFFFFF, bcgen.OP_ELSE)
    out.append(("else_without_if", tb))
    tb = TraceBuilder(block=(32,)); tb.if_(0, [0]); tb.raw(0, 1, bcgen.OP_FI)
    out.append(("fi_without_else", tb))
    tb = TraceBuilder(block=(64,)); tb.bar(0); tb.ld(0, X)
    out.append(("record_while_waiting", tb))
    tb = TraceBuilder(block=(64,)); tb.bar(0)
    out.append(("incomplete_barrier", tb))
    tb = TraceBuilder(block=(32,)); tb.ld(0, X + 2)
    out.append(("misaligned", tb))
    tb = TraceBuilder(block=(32,), smem_bytes=64); tb.ld(0, lambda l: 4 * l, space=1)
    out.append(("shared_oob", tb))
    tb = TraceBuilder(block=(32,)); tb.raw(0, 0xFFFFFFFF, bcgen.OP_IF, aux=0x1_0000_0000 - 1)
    tb.if_(0, [0]); tb.raw(0, 1, bcgen.OP_IF, aux=2)
    out.append(("if_aux_outside_mask", tb))
    tb = TraceBuilder(block=(32,)); tb.if_(0, 0); tb.raw(0, 0, bcgen.OP_LD)
    out.append(("empty_mask_memory", tb))
    tb = TraceBuilder(block=(32,))
    for _ in range(33):
        tb.if_(0, 0xFFFFFFFF)
    out.append(("depth_33", tb))
    tb = TraceBuilder(block=(40,)); tb.raw(1, 0x1FF, bcgen.OP_LD, addrs=lambda l: X)
    out.append(("lane_beyond_partial_warp", tb))
    tb = TraceBuilder(block=(32,)); tb.raw(1, 0xFFFFFFFF, bcgen.OP_LD, addrs=lambda l: X)
    out.append(("warp_out_of_range", tb))
    return out


@pytest.mark.parametrize("case", _infeasible_traces(), ids=lambda c: c[0])
def test_infeasible_rejected(case):
    name, tb = case
    st, races, _ = oracle.detect_geom(tb.records(), tb.geom.as_dict())
    assert st == oracle.INFEASIBLE, name


def test_depth_32_accepted():
    tb = TraceBuilder(block=(32,))
    for _ in range(32):
        tb.if_(0, 0xFFFFFFFF)
    tb.st(0, lambda l: GLOBAL_BASE + 4 * l)
    for _ in range(32):
        tb.else_(0); tb.fi(0)
    st, races, _ = oracle.detect_geom(tb.records(), tb.geom.as_dict())
    assert st == 0 and len(races) == 0


# ------------------------------------------------- lock-heavy hashtable
def _c6(bug, **kw):
    kw.setdefault("n_blocks", 2)
    kw.setdefault("tpb", 32)
    kw.setdefault("iters", 1)
    kw.setdefault("log2_buckets", 3)
    plan = ConfigPlan(6, bug=bug, **kw)
    return plan.records(), plan.geometry


def _c6_buckets(recs):
    """head address -> set of threads that insert into it (from the trace itself)"""
    from bcgen.format import OP_ST
    heads = {}
    region = 1 << 34
    for r in recs:
        if int(r["op"]) != OP_ST:
            continue
        for l in range(32):
            if (int(r["mask"]) >> l) & 1:
                a = int(r["addr"][l])
                if GLOBAL_BASE + 2 * region <= a < GLOBAL_BASE + 3 * region:
                    heads.setdefault(a, set()).add((int(r["warp"]), l))
    return heads


@pytest.mark.parametrize("bug", [0, 1, 2, 3])
def test_c6_hashtable_vs_bruteforce(bug):
    """the fixed hashtable (CAS + fence acquire, fence + exch release) is race-free
    under §3.2; each bug (CAS without fence, unlock by plain store) makes the bucket heads of
    contended buckets race.  The oracle's pairs are §3.2 races and its first race per granule is
    §3.2's on the valid class."""
    recs, geom = _c6(bug)
    races = run(recs, geom)
    bf = check_against_bf(recs, geom, races)
    if bug == 0:
        assert len(races) == 0 and len(bf.race_set()) == 0
    else:
        assert len(races) > 0


@pytest.mark.parametrize("bug", [0, 1, 2, 3])
def test_c6_hashtable_race_structure(bug):
    """Closed form of where the races are: none without a bug; with either bug exactly the
    bucket heads written by two or more threads race (a bucket with one inserter has nothing to
    race with); the lock word races only when the unlock is a plain store (bug bit 1): WW
    against the next plain unlock, or WA against the next lock attempt when the CAS is a plain
    atomic too (both bugs)."""
    recs, geom = _c6(bug, n_blocks=6, tpb=64, iters=2, log2_buckets=5)
    races = run(recs, geom)
    region = 1 << 34
    heads = _c6_buckets(recs)
    head_races = {int(r["addr"]) for r in races if GLOBAL_BASE + 2 * region <= int(r["addr"]) < GLOBAL_BASE + 3 * region}
    lock_races = [r for r in races if GLOBAL_BASE + region <= int(r["addr"]) < GLOBAL_BASE + 2 * region]
    other = [r for r in races if not (GLOBAL_BASE + region <= int(r["addr"]) < GLOBAL_BASE + 3 * region)]
    assert not other
    if bug == 0:
        assert len(races) == 0
        return
    assert head_races == {a for a, th in heads.items() if len(th) >= 2}
    kinds = {int(r["kind"]) for r in lock_races}
    if bug == 1:
        assert not lock_races
    elif bug == 2:
        assert lock_races and kinds == {KIND_NAMES.index("WW")}
    else:
        assert lock_races and kinds == {KIND_NAMES.index("WA")}


# ------------------------------------------- per-lane store values (reading R6b)
def test_values_worked_example():
    """P:L577-581 with values: four lanes of ONE store record write one granule with values
    (a, a, b, a).  Lanes run in ascending order (R5): lane 1 stores lane 0's value (filtered),
    lane 2 differs from lane 1 (race), lane 3 differs from lane 2 (race): exactly two WW
    SAME_INSN races, (l1, l2) and (l2, l3).  The SAME_VALUE flag alone would filter all three."""
    tb = TraceBuilder(block=(32,))
    r = tb.st(0, lambda l: GLOBAL_BASE if l < 4 else GLOBAL_BASE + 64 + 4 * l)
    recs = tb.records()
    vals = np.zeros((len(recs), 32), dtype=np.uint64)
    vals[0, :4] = [7, 7, 9, 7]
    st, races, _ = oracle.detect_geom(recs, tb.geom.as_dict(), values=vals)
    assert st == 0
    got = sorted((int(x["prior_event"]) & 31, int(x["cur_event"]) & 31, int(x["kind"]), int(x["cls"])) for x in races)
    assert got == [(1, 2, KIND_NAMES.index("WW"), 0), (2, 3, KIND_NAMES.index("WW"), 0)]
    # all equal -> no race; the flag gives the same answer as uniform values
    vals[0, :4] = 5
    assert len(oracle.detect_geom(recs, tb.geom.as_dict(), values=vals)[1]) == 0


@pytest.mark.parametrize("chunk", range(3))
def test_values_uniform_equals_flag(chunk):
    """Special case that reduces to the flag: values that are uniform inside every SAME_VALUE
    record and pairwise distinct elsewhere give exactly the flag's race set."""
    from bcgen.format import OP_ST, FLAG_SAME_VALUE
    for seed in range(6000 + 40 * chunk, 6040 + 40 * chunk):
        recs, tb = random_trace(seed, same_value=True)
        geom = tb.geom.as_dict()
        vals = np.zeros((len(recs), 32), dtype=np.uint64)
        for i, r in enumerate(recs):
            if int(r["op"]) == OP_ST:
                vals[i, :] = 1 if int(r["flags"]) & FLAG_SAME_VALUE else np.arange(32) + 100
        st1, want, _ = oracle.detect_geom(recs, geom)
        st2, got, _ = oracle.detect_geom(recs, geom, values=vals)
        assert st1 == st2
        assert np.array_equal(got.view(np.uint8), want.view(np.uint8))


@pytest.mark.parametrize("chunk", range(3))
def test_values_vs_bruteforce(chunk):
    """With per-lane values the oracle's pairs are §3.2 pairs under the value filter, and its
    first race per granule is brute force's on the valid class."""
    from bcgen.fuzz import random_values
    for seed in range(7000 + 40 * chunk, 7040 + 40 * chunk):
        recs, tb = random_trace(seed, same_value=True, n_glob=2)
        geom = tb.geom.as_dict()
        vals = random_values(recs, seed)
        st, races, _ = oracle.detect_geom(recs, geom, values=vals)
        if st != 0:
            continue
        check_against_bf(recs, geom, races, values=vals)


# ------------------------------------------------ warp-size simulation
def _exchange_trace():
    """one 32-thread block: st.shared s[lane]; ld.shared s[lane ^ 16] (warp-synchronous exchange,
    correct only because the 32 lanes execute in lock step)"""
    tb = TraceBuilder(block=(32,), smem_bytes=256)
    from bcgen import SPACE_SHARED
    tb.st(0, lambda l: 4 * l, space=SPACE_SHARED)
    tb.ld(0, lambda l: 4 * (l ^ 16), space=SPACE_SHARED)
    return tb.records(), tb.geom.as_dict()


def test_warpsim_identity_at_32():
    from bcgen.warpsim import split_warps
    recs, tb = random_trace(11)
    r2, g2, org = split_warps(recs, tb.geom.as_dict(), 32)
    assert np.array_equal(r2.view(np.uint8), recs.view(np.uint8))
    assert np.array_equal(run(r2, g2).view(np.uint8), run(recs, tb.geom.as_dict()).view(np.uint8))


@pytest.mark.parametrize("ws", [16, 8, 4])
def test_warpsim_exchange_worked_example(ws):
    """The exchange is race-free with 32-wide warps (the endi of the store orders every lane's
    store before every lane's load) and has exactly 32 WR INTRA_BLOCK races with
    virtual warps of 16, 8 or 4 lanes: every load reads a granule stored by a lane 16 away, which
    is in another virtual warp, and nothing orders two warps of a block but a barrier."""
    from bcgen.warpsim import split_warps
    recs, geom = _exchange_trace()
    assert len(run(recs, geom)) == 0
    r2, g2, org = split_warps(recs, geom, ws)
    races = run(r2, g2)
    assert len(races) == 32
    assert {(int(r["kind"]), int(r["cls"])) for r in races} == {(KIND_NAMES.index("WR"), 2)}
    # reported against the recorded trace: prior = the store of lane l ^ 16, current = the load of lane l
    for r in races:
        pr, pl = org[int(r["prior_event"]) >> 5][0], org[int(r["prior_event"]) >> 5][1] + (int(r["prior_event"]) & 31)
        cr, cl = org[int(r["cur_event"]) >> 5][0], org[int(r["cur_event"]) >> 5][1] + (int(r["cur_event"]) & 31)
        assert (pr, cr) == (0, 1) and pl == cl ^ 16
    check_against_bf(r2, g2, races)


@pytest.mark.parametrize("ws", [16, 8])
def test_warpsim_random_vs_bruteforce(ws):
    from bcgen.warpsim import split_warps
    for seed in range(9000, 9040):
        recs, tb = random_trace(seed, p_bar=0.0, max_bars=0)
        r2, g2, _ = split_warps(recs, tb.geom.as_dict(), ws)
        st, races, _ = oracle.detect_geom(r2, g2)
        if st != 0:
            continue
        check_against_bf(r2, g2, races)


@pytest.mark.parametrize("entry", litmus.OVERWRITE_SUITE, ids=[e[0] for e in litmus.OVERWRITE_SUITE])
def test_release_readings(entry):
    """Hand-derived races under both readings of the release rule (litmus.OVERWRITE_SUITE); the join
    results also match the brute-force §3.2 definition."""
    name, fn, want_join, want_ow = entry
    tb = fn()
    recs, geom = tb.records(), tb.geom.as_dict()
    races = run(recs, geom, oracle.F_CHECK_INVARIANT)
    assert sorted((int(r["kind"]), int(r["cls"]), int(r["space"])) for r in races) == want_join
    check_against_bf(recs, geom, races, strict=True)
    races_o = run(recs, geom, oracle.F_RELEASE_OVERWRITE)
    assert sorted((int(r["kind"]), int(r["cls"]), int(r["space"])) for r in races_o) == want_ow
