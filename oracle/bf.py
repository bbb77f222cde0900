"""Brute-force checker of the §3.2 definition — TEST INFRASTRUCTURE ONLY.

Builds the synchronization order <σ of PAPER.md §3.2 (L368-399) explicitly as
the transitive closure of its generating edges and enumerates every pair of
conflicting, unordered accesses.  This is independent of the vector-clock
rules of §3.3 and is used to pin the oracle (Theorem 1: the rules
accept a trace iff it has no race).

Generating edges (a occurs before b in the trace):
  * intra-thread program order: a and b performed by the same thread;
  * endi(w), if(w), else(w), fi(w), bar(b) are "barrier"-style operations
    performed by every thread in their set tids(·) (L858-864): endi over the
    active lanes, if over the then-lanes, else over the else-lanes, fi over
    the reconverged lanes (reading R13, SURVEY §8(c.4) amb. 13), bar over all
    threads of the block.  Being "performed by" t, they are ordered with t's
    other operations by program order;
  * release a / acquire b on the same location x, both block-scope in the
    same block, or at least one global-scope (L388-392).  AR ops are both.
A data race: same location, at least one write (wr or atm), not both atm,
unordered (L394-399).  Same-value intra-warp stores are filtered when the
record carries SAME_VALUE (L577-581).

Bitsets are Python ints; sized for traces of up to a few thousand ops.
"""
from __future__ import annotations

from collections import defaultdict

import numpy as np

LD, ST, ATOM = 0, 1, 2
ACQ_BLK, ACQ_GLB, REL_BLK, REL_GLB, AR_BLK, AR_GLB = 3, 4, 5, 6, 7, 8
FENCE, BAR, IF, ELSE, FI = 9, 10, 11, 12, 13
ACQUIRES = (ACQ_BLK, ACQ_GLB, AR_BLK, AR_GLB)
RELEASES = (REL_BLK, REL_GLB, AR_BLK, AR_GLB)
GLOBAL_SCOPE = (ACQ_GLB, REL_GLB, AR_GLB)

# kind of a race from (prior access type, current access type)
_KIND = {(ST, ST): 0, (ST, LD): 1, (LD, ST): 2, (ST, ATOM): 3, (ATOM, ST): 4, (LD, ATOM): 5,
         (ATOM, LD): 6}


class BFResult:
    def __init__(self):
        self.pairs = {}          # (space, block_or_0, granule) -> list of (prior_ev, cur_ev, kind)
        self.accesses = defaultdict(list)  # loc -> [(node, ev, type, rec)]
        self.anc = []            # node -> bitset of ancestors
        self.node_of_ev = {}

    def race_set(self):
        out = set()
        for loc, lst in self.pairs.items():
            for (p, c, k) in lst:
                out.add((loc, p, c))
        return out

    def ordered(self, ev_a, ev_b):
        na, nb = self.node_of_ev[ev_a], self.node_of_ev[ev_b]
        return bool((self.anc[nb] >> na) & 1) or bool((self.anc[na] >> nb) & 1)


def brute_force(records: np.ndarray, grid=(1, 1, 1), block=(32, 1, 1), granule_log2=2,
                same_value_filter=True, values=None, warp_size=32):
    """values: optional per-lane store values [n_records, 32] (reading R6b): two stores of one
    record race only if they store different values (instead of the SAME_VALUE flag)."""
    vals = None if values is None else np.asarray(values, dtype=np.uint64).reshape(-1)
    grid = tuple(grid) + (1,) * (3 - len(grid))
    block = tuple(block) + (1,) * (3 - len(block))
    nb = grid[0] * grid[1] * grid[2]
    tpb = block[0] * block[1] * block[2]
    ws = warp_size
    wpb = (tpb + ws - 1) // ws
    G = granule_log2

    def init_mask(w):
        lanes = min(ws, tpb - (w % wpb) * ws)
        return (1 << lanes) - 1

    def tid(w, l):
        return (w // wpb) * tpb + (w % wpb) * ws + l

    res = BFResult()
    anc = res.anc
    last = {}                         # thread -> last node performed by it
    stacks = defaultdict(list)
    arrived = defaultdict(int)
    releases = defaultdict(list)      # x -> [(node, op, block)]

    def new_node(threads, extra_preds=()):
        n = len(anc)
        a = 0
        for t in threads:
            p = last.get(t)
            if p is not None:
                a |= anc[p] | (1 << p)
        for p in extra_preds:
            a |= anc[p] | (1 << p)
        anc.append(a)
        for t in threads:
            last[t] = n
        return n

    for r, rec in enumerate(records):
        w, mask, op = int(rec["warp"]), int(rec["mask"]), int(rec["op"])
        b = w // wpb
        st = stacks[w]
        if not st:
            st.append(init_mask(w))
        lanes = [l for l in range(32) if (mask >> l) & 1]
        if op <= AR_GLB:
            size = 1 << int(rec["size_log2"])
            space = int(rec["space"])
            for l in lanes:
                t = tid(w, l)
                ev = (r << 5) | l
                a = int(rec["addr"][l])
                if op <= ATOM:
                    n = new_node([t])
                    res.node_of_ev[ev] = n
                    for gr in range(a >> G, ((a + size - 1) >> G) + 1):
                        loc = (space, b if space == 1 else 0, gr)
                        res.accesses[loc].append((n, ev, op, r, int(rec["flags"]) & 1))
                else:
                    x = (space, b if space == 1 else 0, a >> G)
                    preds = []
                    if op in ACQUIRES:
                        for (pn, pop, pb) in releases[x]:
                            if (op in GLOBAL_SCOPE or pop in GLOBAL_SCOPE) or pb == b:
                                preds.append(pn)
                    n = new_node([t], preds)
                    res.node_of_ev[ev] = n
                    if op in RELEASES:
                        releases[x].append((n, op, b))
            new_node([tid(w, l) for l in range(32) if (st[-1] >> l) & 1])  # endi(w)
        elif op == IF:
            top = st[-1]
            then, els = top & int(rec["aux"]), top & ~int(rec["aux"])
            st.append(els)
            st.append(then)
            new_node([tid(w, l) for l in range(32) if (then >> l) & 1])
        elif op in (ELSE, FI):
            st.pop()
            top = st[-1]
            new_node([tid(w, l) for l in range(32) if (top >> l) & 1])
        elif op == BAR:
            arrived[b] += 1
            if arrived[b] == wpb:
                arrived[b] = 0
                new_node([b * tpb + i for i in range(tpb)])
        # FENCE: no trace operation

    for loc, lst in res.accesses.items():
        out = []
        for j in range(len(lst)):
            nj, evj, tj, rj, svj = lst[j]
            for i in range(j):
                ni, evi, ti, ri, svi = lst[i]
                if ti == LD and tj == LD:
                    continue
                if ti == ATOM and tj == ATOM:
                    continue
                if ni == nj:
                    continue
                if (anc[nj] >> ni) & 1:
                    continue
                sv = (vals[evi] == vals[evj]) if vals is not None else svj
                if same_value_filter and ti == ST and tj == ST and ri == rj and sv:
                    continue
                out.append((evi, evj, _KIND[(ti, tj)]))
        if out:
            res.pairs[loc] = out
    return res


def valid_granules(res: BFResult):
    """Granules on which the printed atomic rules coincide with §3.2 (SURVEY
    §8(c.4) amb. 3): either no plain access, or all atomics pairwise ordered."""
    ok = set()
    for loc, lst in res.accesses.items():
        atoms = [n for (n, ev, t, r, sv) in lst if t == ATOM]
        plain = any(t != ATOM for (n, ev, t, r, sv) in lst)
        good = True
        if plain and len(atoms) > 1:
            for j in range(len(atoms)):
                for i in range(j):
                    if not ((res.anc[atoms[j]] >> atoms[i]) & 1):
                        good = False
                        break
                if not good:
                    break
        if good:
            ok.add(loc)
    return ok
