"""Seeded random *feasible* traces for property / parity tests.

A small interleaving scheduler runs per-warp random programs: memory ops on
a tiny pool of granules (so lanes, warps and blocks collide), nested
if/else/fi with arbitrary masks (including empty paths), barriers (possibly
inside branches, i.e. barrier divergence), and acquire/release/acq-rel ops at
block and global scope on a few synchronisation locations.  Feasibility
 is maintained: each record carries exactly the warp's
active mask, branches are properly nested, every warp of a block arrives at
each barrier once and issues nothing until the barrier completes.

No race-detection arithmetic lives here.
"""
from __future__ import annotations

import random

import numpy as np

from .builder import TraceBuilder
from .format import GLOBAL_BASE, SPACE_GLOBAL, SPACE_SHARED

_FULL = 0xFFFFFFFF


def _random_submask(rng, mask):
    out = 0
    lanes = [l for l in range(32) if (mask >> l) & 1]
    mode = rng.random()
    if mode < 0.15:
        return 0
    if mode < 0.3:
        return mask
    if mode < 0.5 and lanes:
        return 1 << rng.choice(lanes)
    for l in lanes:
        if rng.random() < 0.5:
            out |= 1 << l
    return out


def random_trace(seed: int, *, max_blocks=3, max_tpb=72, ops_per_warp=(3, 14), n_glob=4,
                 n_shared=3, n_sync=2, p_sync=0.12, p_if=0.18, max_depth=4, p_bar=0.12,
                 max_bars=3, same_value=False, vector=True, sync=True, atomics=True,
                 granule_log2=2, tpb=None, n_blocks=None):
    """Return (records, TraceBuilder) for a random feasible trace."""
    rng = random.Random(seed)
    nb = n_blocks if n_blocks is not None else rng.randint(1, max_blocks)
    t = tpb if tpb is not None else rng.choice([rng.randint(1, max_tpb), 32, 64, rng.randint(1, 40)])
    G = 1 << granule_log2
    sbase = ((n_shared * G + 15) // 16) * 16 + 16
    smem = sbase + 16 * max(1, n_sync // 2) + 64
    tb = TraceBuilder(grid=(nb, 1, 1), block=(t, 1, 1), smem_bytes=smem, granule_log2=granule_log2)
    geom = tb.geom
    nw = geom.n_warps
    bars_planned = {b: rng.randint(0, max_bars) for b in range(nb)}
    budget = {w: rng.randint(*ops_per_warp) for w in range(nw)}
    phase = {w: [] for w in range(nw)}          # per open if: 'then' | 'else'
    bars_done = {w: 0 for w in range(nw)}
    waiting = {w: False for w in range(nw)}
    arrived = {b: 0 for b in range(nb)}
    finished = {w: False for w in range(nw)}

    def gaddr_for(lane, size):
        # granule pool of n_glob granules in one global page; aligned to size
        if size >= G:
            per = size // G
            k = rng.randrange(max(1, n_glob // per)) * per
            return GLOBAL_BASE + k * G
        k = rng.randrange(n_glob)
        return GLOBAL_BASE + k * G + rng.randrange(G // size) * size

    def saddr_for(lane, size):
        if size >= G:
            per = size // G
            k = rng.randrange(max(1, n_shared // per)) * per
            return k * G
        k = rng.randrange(n_shared)
        return k * G + rng.randrange(G // size) * size

    sync_g = [GLOBAL_BASE + 0x100000 + i * 64 for i in range(n_sync)]
    sync_s = [sbase + 16 * i for i in range(max(1, n_sync // 2))]

    def step(w):
        b = geom.block_of_warp(w)
        top = tb.top(w)
        ph = phase[w]
        # empty active set: only the branch-closing ops are executable
        if top == 0:
            if ph[-1] == "then":
                tb.else_(w); ph[-1] = "else"
            else:
                tb.fi(w); ph.pop()
            return
        if ph and rng.random() < 0.25:
            if ph[-1] == "then":
                tb.else_(w); ph[-1] = "else"
            else:
                tb.fi(w); ph.pop()
            return
        need_bar = bars_done[w] < bars_planned[b]
        if need_bar and (budget[w] <= 0 or rng.random() < p_bar):
            tb.bar(w)
            bars_done[w] += 1
            waiting[w] = True
            arrived[b] += 1
            if arrived[b] == geom.wpb:
                arrived[b] = 0
                for ww in range(b * geom.wpb, (b + 1) * geom.wpb):
                    waiting[ww] = False
            return
        if budget[w] <= 0:
            if ph:
                if ph[-1] == "then":
                    tb.else_(w); ph[-1] = "else"
                else:
                    tb.fi(w); ph.pop()
                return
            finished[w] = True
            return
        budget[w] -= 1
        r = rng.random()
        if r < p_if and len(ph) < max_depth:
            tb.if_(w, _random_submask(rng, top))
            ph.append("then")
            return
        r = rng.random()
        if sync and r < p_sync:
            kind = rng.choice(["acq", "rel", "ar"])
            scope = rng.choice(["glb", "blk"])
            if rng.random() < 0.7:
                space = SPACE_GLOBAL
                same = rng.random() < 0.7
                x0 = rng.choice(sync_g)
                addrs = (lambda l: x0) if same else (lambda l: rng.choice(sync_g))
            else:
                space = SPACE_SHARED
                x0 = rng.choice(sync_s)
                addrs = lambda l: x0
            getattr(tb, kind)(w, addrs, scope=scope, space=space)
            return
        if rng.random() < 0.04:
            tb.fence(w)
            return
        size = 4
        if vector and rng.random() < 0.15:
            size = rng.choice([1, 2, 8, 16])
        space = SPACE_GLOBAL if rng.random() < 0.55 else SPACE_SHARED
        af = gaddr_for if space == SPACE_GLOBAL else saddr_for
        # lanes often share one address (broadcast / intra-warp collisions)
        if rng.random() < 0.3:
            a0 = af(0, size)
            addrs = lambda l: a0
        else:
            cache = {}
            addrs = lambda l: cache.setdefault(l, af(l, size))
        kinds = ["ld", "st", "atom"] if atomics else ["ld", "st"]
        op = rng.choice(kinds)
        if op == "st":
            tb.st(w, addrs, space=space, size=size,
                  same_value=(same_value and rng.random() < 0.4))
        else:
            getattr(tb, op)(w, addrs, space=space, size=size)

    while True:
        runnable = [w for w in range(nw) if not finished[w] and not waiting[w]]
        if not runnable:
            break
        step(rng.choice(runnable))
    assert all(not waiting[w] for w in range(nw))
    return tb.records(), tb


def random_values(records, seed: int, p_uniform: float = 0.4, n_distinct: int = 3):
    """Per-lane store values [n_records, 32] (uint64) for SURVEY row f3: for each store record,
    with probability p_uniform every lane stores one value, otherwise each lane draws from
    n_distinct values (so some lane pairs agree and some do not).  Input fixture only."""
    import numpy as np
    from .format import OP_ST
    rng = random.Random(seed * 7919 + 17)
    vals = np.zeros((len(records), 32), dtype=np.uint64)
    for i, r in enumerate(records):
        if int(r["op"]) != OP_ST:
            continue
        if rng.random() < p_uniform:
            vals[i, :] = rng.randrange(1 << 62)
        else:
            vals[i, :] = [rng.randrange(n_distinct) for _ in range(32)]
    return vals
