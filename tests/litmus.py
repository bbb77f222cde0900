"""66 re-authored concurrency litmus traces (§6.1).

The paper's 66 CUDA programs are not listed, only their categories: "data
races or race-free behavior via global memory, shared memory, within and
across warps and blocks, and using a variety of atomic and memory fence
instructions to implement locks, whole-grid barriers and flag
synchronization" (L1400-1406).  These traces follow SURVEY.md §8(c.5)'s
matrix over those categories (parity unpinned for the exact programs).  The
expected race multiset of each trace is derived by hand from the rules of
§3.3 and cross-checked against the brute-force §3.2 definition in
tests/test_oracle_pins.py; the two traces that rely on a reading (release
join vs overwrite, the atomic-chain gap) say so.

Each entry: (name, build() -> (records, geom dict), expected, options)
expected = sorted list of (kind, cls, space) per reported race.
"""
from __future__ import annotations

from bcgen import GLOBAL_BASE, SPACE_GLOBAL, SPACE_SHARED, TraceBuilder

WW, WR, RW, WA, AW, RA, AR = range(7)
SAME, BRANCH, INTRA, INTER, BDIV = range(5)
G, S = SPACE_GLOBAL, SPACE_SHARED

X = GLOBAL_BASE            # a data location
Y = GLOBAL_BASE + 0x1000   # a second data location
F = GLOBAL_BASE + 0x200000 # a flag / lock
H = GLOBAL_BASE + 0x300000 # another flag


def _addr(space, base_g, off):
    return (base_g if space == G else 0) + off


SUITE = []


def lit(name, expected, **opts):
    def deco(fn):
        SUITE.append((name, fn, sorted(expected), opts))
        return fn
    return deco


def own(space, k=0):
    """lane l -> a distinct granule per lane (never colliding)."""
    base = _addr(space, X + 0x10000 * k, 0x400 + 0x200 * k)
    return lambda l: base + 4 * l


# ---------------------------------------------------------------------------
# 1. intra-warp, same instruction (footnote 2)  — 10 traces
for sp in (G, S):
    sn = "g" if sp == G else "s"
    x = _addr(sp, X, 0)

    @lit(f"intra_warp_ww_distinct_{sn}", [(WW, SAME, sp)])
    def _b(sp=sp, x=x):
        tb = TraceBuilder(block=(32,))
        tb.st(0, lambda l: x if l < 2 else x + 4 * l, space=sp)
        return tb

    @lit(f"intra_warp_ww_same_value_{sn}", [])
    def _b(sp=sp, x=x):
        tb = TraceBuilder(block=(32,))
        tb.st(0, lambda l: x if l < 2 else x + 4 * l, space=sp, same_value=True)
        return tb

    @lit(f"intra_warp_rr_{sn}", [])
    def _b(sp=sp, x=x):
        tb = TraceBuilder(block=(32,))
        tb.ld(0, x, space=sp)
        return tb

    @lit(f"intra_warp_wr_lockstep_{sn}", [])
    def _b(sp=sp, x=x):
        tb = TraceBuilder(block=(32,))
        tb.st(0, lambda l: x + 4 * l, space=sp)
        tb.ld(0, lambda l: x + 4 * ((l + 1) % 32), space=sp)
        return tb

    @lit(f"intra_warp_aa_{sn}", [])
    def _b(sp=sp, x=x):
        tb = TraceBuilder(block=(32,))
        tb.atom(0, x, space=sp)
        return tb

# ---------------------------------------------------------------------------
# 2. branch ordering races  — 12 traces
for sp in (G, S):
    sn = "g" if sp == G else "s"
    x = _addr(sp, X, 0)
    o = own(sp, 1)

    @lit(f"branch_then_w_else_r_{sn}", [(WR, BRANCH, sp)])
    def _b(sp=sp, x=x, o=o):
        tb = TraceBuilder(block=(32,))
        tb.if_(0, [0]); tb.st(0, x, space=sp)
        tb.else_(0); tb.ld(0, lambda l: x if l == 1 else o(l), space=sp)
        tb.fi(0)
        return tb

    @lit(f"branch_then_w_else_w_{sn}", [(WW, BRANCH, sp)])
    def _b(sp=sp, x=x, o=o):
        tb = TraceBuilder(block=(32,))
        tb.if_(0, [0]); tb.st(0, x, space=sp)
        tb.else_(0); tb.st(0, lambda l: x if l == 1 else o(l), space=sp)
        tb.fi(0)
        return tb

    @lit(f"branch_then_r_else_r_{sn}", [])
    def _b(sp=sp, x=x, o=o):
        tb = TraceBuilder(block=(32,))
        tb.if_(0, [0]); tb.ld(0, x, space=sp)
        tb.else_(0); tb.ld(0, lambda l: x if l == 1 else o(l), space=sp)
        tb.fi(0)
        return tb

    @lit(f"branch_then_w_post_fi_r_{sn}", [])
    def _b(sp=sp, x=x):
        tb = TraceBuilder(block=(32,))
        tb.if_(0, [0]); tb.st(0, x, space=sp)
        tb.else_(0); tb.fi(0)
        tb.ld(0, x, space=sp)
        return tb

    @lit(f"branch_nested_inner_then_w_outer_else_r_{sn}", [(WR, BRANCH, sp)])
    def _b(sp=sp, x=x, o=o):
        tb = TraceBuilder(block=(32,))
        tb.if_(0, [0, 1])
        tb.if_(0, [0]); tb.st(0, x, space=sp); tb.else_(0); tb.fi(0)
        tb.else_(0)
        tb.ld(0, lambda l: x if l == 2 else o(l), space=sp)
        tb.fi(0)
        return tb

    @lit(f"branch_empty_else_{sn}", [])
    def _b(sp=sp, x=x):
        tb = TraceBuilder(block=(32,))
        tb.if_(0, range(32)); tb.st(0, lambda l: x + 4 * l, space=sp)
        tb.else_(0); tb.fi(0)
        tb.ld(0, lambda l: x + 4 * ((l + 7) % 32), space=sp)
        return tb

# ---------------------------------------------------------------------------
# 3. intra-block, across warps (2 warps in one block)  — 18 traces
for sp in (G, S):
    sn = "g" if sp == G else "s"
    x = _addr(sp, X, 0)
    f = _addr(sp, F, 0x80)
    o0, o1 = own(sp, 2), own(sp, 3)

    def lane0(addr, other):
        return lambda l: addr if l == 0 else other(l)

    @lit(f"xwarp_no_bar_{sn}", [(WR, INTRA, sp)])
    def _b(sp=sp, x=x, o0=o0, o1=o1):
        tb = TraceBuilder(block=(64,))
        tb.st(0, lane0(x, o0), space=sp)
        tb.ld(1, lane0(x, o1), space=sp)
        return tb

    @lit(f"xwarp_bar_{sn}", [])
    def _b(sp=sp, x=x, o0=o0, o1=o1):
        tb = TraceBuilder(block=(64,))
        tb.st(0, lane0(x, o0), space=sp)
        tb.bar(0); tb.bar(1)
        tb.ld(1, lane0(x, o1), space=sp)
        return tb

    @lit(f"xwarp_read_before_bar_write_after_{sn}", [])
    def _b(sp=sp, x=x, o0=o0, o1=o1):
        tb = TraceBuilder(block=(64,))
        tb.ld(1, lane0(x, o1), space=sp)
        tb.bar(1); tb.bar(0)
        tb.st(0, lane0(x, o0), space=sp)
        return tb

    @lit(f"xwarp_barrier_divergence_{sn}", [(0xFF, BDIV, 2)])
    def _b(sp=sp, x=x, o0=o0, o1=o1):
        tb = TraceBuilder(block=(64,))
        tb.st(0, lane0(x, o0), space=sp)
        tb.if_(0, [0]); tb.bar(0)
        tb.bar(1)
        tb.else_(0); tb.fi(0)
        tb.ld(1, lane0(x, o1), space=sp)
        return tb

    @lit(f"xwarp_relblk_acqblk_flag_{sn}", [])
    def _b(sp=sp, x=x, f=f, o0=o0, o1=o1):
        tb = TraceBuilder(block=(64,))
        tb.st(0, lane0(x, o0), space=sp)
        tb.if_(0, [0]); tb.rel(0, f, scope="blk", space=sp); tb.else_(0); tb.fi(0)
        tb.if_(1, [0]); tb.acq(1, f, scope="blk", space=sp); tb.else_(1); tb.fi(1)
        tb.ld(1, lane0(x, o1), space=sp)
        return tb

    @lit(f"xwarp_acquire_before_release_{sn}", [(WR, INTRA, sp)])
    def _b(sp=sp, x=x, f=f, o0=o0, o1=o1):
        tb = TraceBuilder(block=(64,))
        tb.if_(1, [0]); tb.acq(1, f, scope="blk", space=sp); tb.else_(1); tb.fi(1)
        tb.st(0, lane0(x, o0), space=sp)
        tb.if_(0, [0]); tb.rel(0, f, scope="blk", space=sp); tb.else_(0); tb.fi(0)
        tb.ld(1, lane0(x, o1), space=sp)
        return tb

    @lit(f"xwarp_atm_vs_wr_{sn}", [(AW, INTRA, sp)])
    def _b(sp=sp, x=x, o0=o0, o1=o1):
        tb = TraceBuilder(block=(64,))
        tb.atom(0, lane0(x, o0), space=sp)
        tb.st(1, lane0(x, o1), space=sp)
        return tb

    @lit(f"xwarp_atm_vs_rd_{sn}", [(AR, INTRA, sp)])
    def _b(sp=sp, x=x, o0=o0, o1=o1):
        tb = TraceBuilder(block=(64,))
        tb.atom(0, lane0(x, o0), space=sp)
        tb.ld(1, lane0(x, o1), space=sp)
        return tb

    @lit(f"xwarp_atm_only_{sn}", [])
    def _b(sp=sp, x=x):
        tb = TraceBuilder(block=(64,))
        tb.atom(0, x, space=sp)
        tb.atom(1, x, space=sp)
        return tb

# ---------------------------------------------------------------------------
# 4. inter-block, global memory  — 15 traces (1 thread/warp/block unless noted)


def one(nb, tpb=1):
    return TraceBuilder(grid=(nb,), block=(tpb,))


@lit("xblock_plain_ww", [(WW, INTER, G)])
def _b():
    tb = one(2); tb.st(0, X); tb.st(1, X); return tb


def _mp(rel_scope, acq_scope):
    # Fig. 4 message passing: T1: st x; fence; st y.  T2: ld y; fence; ld x.
    tb = one(2)
    tb.st(0, X)
    tb.rel(0, F, scope=rel_scope)
    tb.acq(1, F, scope=acq_scope)
    tb.ld(1, X)
    return tb


@lit("mp_cta_cta", [(WR, INTER, G)])
def _b(): return _mp("blk", "blk")


@lit("mp_cta_gl", [])
def _b(): return _mp("blk", "glb")


@lit("mp_gl_cta", [])
def _b(): return _mp("glb", "blk")


@lit("mp_gl_gl", [])
def _b(): return _mp("glb", "glb")


@lit("lock_cas_fence", [])
def _b():
    # atom.cas + fence -> acquire; fence + atom.exch -> release
    tb = one(2)
    for b in (0, 1):
        tb.acq(b, F); tb.st(b, X); tb.ld(b, X); tb.rel(b, F)
    return tb


@lit("lock_cas_no_fence_hashtable_bug1", [(WW, INTER, G), (RW, INTER, G)])
def _b():
    # §6.3: atomicCAS without a fence is a plain atomic, so no acquire
    tb = one(2)
    for b in (0, 1):
        tb.atom(b, F); tb.st(b, X); tb.ld(b, Y); tb.rel(b, F)
    tb.st(1, Y)
    return tb


@lit("lock_plain_unlock_hashtable_bug2", [(WW, INTER, G), (WW, INTER, G)])
def _b():
    # §6.3: releasing the lock with a non-atomic write without a fence
    tb = one(2)
    for b in (0, 1):
        tb.acq(b, F); tb.st(b, X); tb.st(b, F)
    return tb


@lit("grid_barrier_arglb_chain", [])
def _b():
    tb = one(3)
    for b in range(3):
        tb.st(b, X + 4 * b); tb.ar(b, F)
    for b in range(3):
        tb.acq(b, F)
        for o in range(3):
            if o != b:
                tb.ld(b, X + 4 * o)
    return tb


@lit("thread_fence_reduction_small", [])
def _b():
    tb = TraceBuilder(grid=(2,), block=(32,), smem_bytes=256)
    for b in (0, 1):
        tb.st(b, lambda l: 4 * l, space=S)
        tb.bar(b)
        tb.if_(b, [0]); tb.st(b, X + 4 * b); tb.ar(b, F); tb.else_(b); tb.fi(b)
        tb.bar(b)
    tb.if_(1, [0, 1]); tb.ld(1, lambda l: X + 4 * l); tb.else_(1); tb.fi(1)
    return tb


@lit("shoc_bfs_flag", [(WW, INTER, G), (WW, INTER, G)])
def _b():
    # §6.3 SHOC bfs: cross-block distance updates and a flag set without atomics/fences
    tb = one(2)
    for b in (0, 1):
        tb.st(b, X); tb.st(b, F)
    return tb


@lit("two_releasers_join", [], overwrite_expected=[(WR, INTER, G)])
def _b():
    # reading R1: S_x[b] := S_x[b] ⊔ C_t.  Under the printed overwrite the
    # second release erases the first and the load of X races.
    tb = one(3)
    tb.st(0, X); tb.rel(0, F)
    tb.st(1, Y); tb.rel(1, F)
    tb.acq(2, F); tb.ld(2, X); tb.ld(2, Y)
    return tb


@lit("arblk_chain_across_blocks", [(WR, INTER, G)])
def _b():
    tb = one(2)
    tb.st(0, X); tb.ar(0, F, scope="blk")
    tb.ar(1, F, scope="blk"); tb.ld(1, X)
    return tb


@lit("acqglb_of_relblk", [])
def _b():
    tb = one(2)
    tb.st(0, X); tb.rel(0, F, scope="blk")
    tb.acq(1, F, scope="glb"); tb.ld(1, X)
    return tb


@lit("relglb_acqblk_then_relblk_acqblk_transitive", [])
def _b():
    tb = TraceBuilder(grid=(2,), block=(64,))
    w10, w11 = tb.warp(1, 0), tb.warp(1, 1)
    tb.st(0, lambda l: X if l == 0 else Y + 4 * l)
    tb.if_(0, [0]); tb.rel(0, F); tb.else_(0); tb.fi(0)
    tb.if_(w10, [0]); tb.acq(w10, F, scope="blk"); tb.rel(w10, H, scope="blk"); tb.else_(w10); tb.fi(w10)
    tb.if_(w11, [0]); tb.acq(w11, H, scope="blk"); tb.ld(w11, X); tb.else_(w11); tb.fi(w11)
    return tb

# ---------------------------------------------------------------------------
# 5. geometry / format  — 11 traces


@lit("partial_last_warp", [(WR, INTRA, G)] * 8)
def _b():
    tb = TraceBuilder(block=(40,))
    tb.st(1, lambda l: X + 4 * l)                       # warp 1 has 8 lanes
    tb.ld(0, lambda l: X + 4 * l if l < 8 else Y + 4 * l)
    return tb


@lit("block_2d_no_bar_and_bar", [(WR, INTRA, G)])
def _b():
    tb = TraceBuilder(block=(8, 8))
    tb.st(0, lambda l: X + 4 * l)
    tb.ld(1, lambda l: X if l == 0 else Y + 4 * l)       # races with lane 0's store
    tb.bar(0); tb.bar(1)
    tb.ld(1, lambda l: X + 4 * l)                        # ordered by the barrier
    return tb


@lit("vector16_overlap", [(WR, INTRA, G)])
def _b():
    tb = TraceBuilder(block=(64,))
    tb.st(0, lambda l: X + 16 * l, size=16)             # lane 0 covers X..X+15
    tb.ld(1, lambda l: X + 8 if l == 0 else Y + 4 * l)
    return tb


@lit("nesting_3_levels", [(WR, BRANCH, G)] * 3)
def _b():
    tb = TraceBuilder(block=(32,))
    o = own(G, 4)
    tb.if_(0, range(16))
    tb.if_(0, range(8))
    tb.if_(0, range(4)); tb.st(0, lambda l: X if l == 0 else o(l))
    tb.else_(0); tb.ld(0, lambda l: X if l == 4 else o(l)); tb.fi(0)
    tb.else_(0); tb.ld(0, lambda l: X if l == 8 else o(l)); tb.fi(0)
    tb.else_(0); tb.ld(0, lambda l: X if l == 16 else o(l)); tb.fi(0)
    return tb


@lit("sparse_acquire_inside_branch", [(WR, INTER, G)])
def _b():
    tb = TraceBuilder(grid=(2,), block=(32,))
    o = own(G, 5)
    tb.st(0, lambda l: X if l == 0 else o(l))
    tb.if_(0, [0]); tb.rel(0, F); tb.else_(0); tb.fi(0)
    w = tb.warp(1)
    tb.if_(w, [3]); tb.acq(w, F); tb.ld(w, X)
    tb.else_(w); tb.ld(w, lambda l: X if l == 4 else o(l) + 0x1000)
    tb.fi(w)
    tb.ld(w, X)
    return tb


@lit("fig1_64_threads_2_warps", [])
def _b():
    tb = TraceBuilder(block=(64,), smem_bytes=64)
    for w in (0, 1):
        a, bb, d = X + 0x100 * w, Y + 0x100 * w, F + 0x100 * w
        tb.ld(w, a)
        tb.if_(w, [0]); tb.st(w, bb); tb.else_(w); tb.fi(w)
        tb.rel(w, d, scope="blk")
    return tb


@lit("lockstep_through_reconvergence", [])
def _b():
    tb = TraceBuilder(block=(32,))
    tb.if_(0, [0]); tb.st(0, X); tb.else_(0); tb.fi(0)
    tb.ld(0, lambda l: X if l == 1 else Y + 4 * l)
    return tb


@lit("reads_inflate_then_write", [(RW, INTRA, G)])
def _b():
    tb = TraceBuilder(block=(64,))
    tb.ld(0, lambda l: X if l == 0 else Y + 4 * l)
    tb.ld(1, lambda l: X if l == 0 else Y + 0x100 + 4 * l)
    tb.st(0, lambda l: X if l == 0 else Y + 0x200 + 4 * l)
    return tb


@lit("rr_then_w_three_blocks", [(RW, INTER, G), (RW, INTER, G)])
def _b():
    tb = one(3)
    tb.ld(0, X); tb.ld(1, X); tb.ld(2, X); tb.st(2, X)
    return tb


@lit("atm_after_plain_write_ordered", [])
def _b():
    tb = TraceBuilder(block=(64,))
    tb.st(0, lambda l: X if l == 0 else Y + 4 * l)
    tb.bar(0); tb.bar(1)
    tb.atom(1, lambda l: X if l == 0 else Y + 0x100 + 4 * l)
    return tb


@lit("atomic_chain_gap_3i", [], atomic_gap=True)
def _b():
    # SURVEY §8(c.4) amb. 3(i): atm(t1), atm(t2), wr(t3) with t2 -> t3 and
    # t1 || t3.  The printed ATOM rule never re-checks the earlier atomic, so
    # the rules report nothing; the §3.2 definition has a race.
    tb = one(3)
    tb.atom(0, X); tb.atom(1, X); tb.rel(1, F)
    tb.acq(2, F); tb.st(2, X)
    return tb


assert len(SUITE) == 66, len(SUITE)


def build(entry):
    name, fn, expected, opts = entry
    tb = fn()
    return tb.records(), tb.geom.as_dict()


# ---------------------------------------------------------------------------
# Release join (reading R1) vs the printed overwrite S_x := C_t (Fig. 3 RELBLOCK / RELGLOBAL,
# P:L754-758; ACQREL joins the slot before writing it).  Not part of the
# 66: these separate the two readings.  Each entry: (name, build, expected_join, expected_overwrite);
# each warp uses 32 lanes on distinct granules, so a racing warp pair is 32 races.
OVERWRITE_SUITE = []


def lit_ow(name, join, overwrite):
    def deco(fn):
        OVERWRITE_SUITE.append((name, fn, sorted(join), sorted(overwrite)))
        return fn
    return deco


@lit_ow("ow_second_release_erases", [], [(WR, INTRA, G)] * 32)
def _b():
    # one block, warps 0-2: w1's release replaces w0's in S_F[0]; w2 acquires only C_w1
    tb = TraceBuilder(block=(96,))
    tb.st(0, own(G)); tb.rel(0, F, scope="blk")
    tb.rel(1, F, scope="blk")
    tb.acq(2, F, scope="blk"); tb.ld(2, own(G))
    return tb


@lit_ow("ow_acqrel_keeps_slot", [], [])
def _b():
    # w1's ACQREL writes C_w1 ⊔ S_F[0] (which holds C_w0): w2 still learns w0's stores
    tb = TraceBuilder(block=(96,))
    tb.st(0, own(G)); tb.rel(0, F, scope="blk")
    tb.ar(1, F, scope="blk")
    tb.acq(2, F, scope="blk"); tb.ld(2, own(G))
    return tb


@lit_ow("ow_block_release_after_global", [], [(WR, INTER, G)] * 32)
def _b():
    # blocks 0 (warps 0, 1) and 1 (warps 2, 3): w0's global release fills every slot, w2's block
    # release then replaces slot 1 only -- w3 (block 1) misses w0's stores, w1 (block 0) does not
    tb = TraceBuilder(grid=(2,), block=(64,))
    tb.st(0, own(G)); tb.rel(0, F, scope="glb")
    tb.rel(2, F, scope="blk")
    tb.acq(3, F, scope="blk"); tb.ld(3, own(G))
    tb.acq(1, F, scope="blk"); tb.ld(1, own(G))
    return tb


@lit_ow("ow_global_release_overrides_block", [], [(WR, INTRA, G)] * 32)
def _b():
    # w0's block release fills slot 0; w2's (block 1) global release overwrites every slot
    tb = TraceBuilder(grid=(2,), block=(64,))
    tb.st(0, own(G)); tb.rel(0, F, scope="blk")
    tb.rel(2, F, scope="glb")
    tb.acq(1, F, scope="blk"); tb.ld(1, own(G))
    return tb


@lit_ow("ow_global_acquire_joins_slots", [], [])
def _b():
    # ⊔_b S_F[b]: slot 0 and 2 hold w0's global release, slot 1 w1's block release
    tb = TraceBuilder(grid=(3,), block=(32,))
    tb.st(0, own(G)); tb.rel(0, F, scope="glb")
    tb.rel(1, F, scope="blk")
    tb.acq(2, F, scope="glb"); tb.ld(2, own(G))
    return tb


@lit_ow("ow_global_acquire_after_global_release", [], [(WR, INTER, G)] * 32)
def _b():
    # w1's global release overwrites slot 0 (w0's block release): no slot holds C_w0 any more
    tb = TraceBuilder(grid=(3,), block=(32,))
    tb.st(0, own(G)); tb.rel(0, F, scope="blk")
    tb.rel(1, F, scope="glb")
    tb.acq(2, F, scope="glb"); tb.ld(2, own(G))
    return tb


@lit_ow("ow_global_acqrel_chain", [], [])
def _b():
    # w1's global ACQREL joins every slot (slot 0 = C_w0) and writes the join everywhere
    tb = TraceBuilder(grid=(3,), block=(32,))
    tb.st(0, own(G)); tb.rel(0, F, scope="blk")
    tb.ar(1, F, scope="glb")
    tb.acq(2, F, scope="blk"); tb.ld(2, own(G))
    return tb
