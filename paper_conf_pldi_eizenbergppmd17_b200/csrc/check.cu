// check.cu — K6+K7 per-address shadow check, the hot kernel.
//
// Input: items sorted by shadow granule, each granule's accesses in trace order (stable sort).
// The rules of Fig. 2 / Fig. 3 for one granule x (readings R2-R8):
//   rd  : W_x ⪯ C_t, then READEXCL (R_x ⪯ C_t -> R_x := E(t)) | READINFLATE (-> VC) | READSHARED
//   wr  : W_x ⪯ C_t, R_x ⪯/⊑ C_t; R_x := ⊥, W_x := (E(t), plain)
//   atm : W_x ⪯ C_t only if W_x is plain; R_x ⪯/⊑ C_t; R_x := ⊥, W_x := (E(t), atomic)
// depend on the state only through (a) the last writer before each access, and (b) for each
// writer, the reads since the previous writer: R_x is the epoch of the last read unless some read
// in that run found its predecessor unordered (READINFLATE), in which case R_x is the vector of the
// latest read per thread from the read before the first inflation on ("K7 exactly as
// the oracle").  So the whole automaton is two segmented scans over the sorted items —
//   LW(i) = last writer before i in its granule          (segmented max)
//   FI(i) = first inflating read in the run ending at i  (segmented min, reset at writers)
// plus independent happens-before queries per item, evaluated with warp ballots over rounds of 32
// sorted items (below).  Arbitrarily long (hot) granule segments cost the same per item as short
// ones, and the shadow state never has to be materialised in memory.
#include <cstdlib>
#include <cstring>

#include "common.cuh"
#include "kernels.cuh"

namespace bc {

namespace {

struct Sum {
  u32 fk, lk, lw, fi, bits;  // bits: 1 = one key throughout, 2 = tail key run holds a writer
};

__device__ __forceinline__ Sum sum_ident() { return Sum{NONE, NONE, 0u, NONE, 0u}; }

__device__ __forceinline__ Sum combine(const Sum& L, const Sum& R) {
  if (L.fk == NONE) return R;
  if (R.fk == NONE) return L;
  Sum o;
  o.fk = L.fk;
  o.lk = R.lk;
  if ((R.bits & 1u) && R.fk == L.lk) {
    bool rw = R.bits & 2u;
    o.lw = rw ? R.lw : L.lw;
    o.fi = rw ? R.fi : min(L.fi, R.fi);
    o.bits = (L.bits & 1u) | ((L.bits | R.bits) & 2u);
  } else {
    o.lw = R.lw;
    o.fi = R.fi;
    o.bits = R.bits & 2u;
  }
  return o;
}

struct CheckArgs {
  HbCtx c;
  const u32* keys;  // (granule key << 2) | op
  const u32* evs;   // (record << 5) | lane
  const u64* n_dev;
  uint4* races;  // (key, cur_ev, prior_ev, kind)
  u32* race_cnt;
  u32 race_cap;
  u64* seg_cnt;  // [0] segments, [1] clock snapshot gathers
  const u64* values;  // per-lane store values (row f3), nullable
};

// intra-warp same-value filter: two stores of one record; with per-lane values
// (reading R6b) they must store the same value, else the record's SAME_VALUE flag decides
// (the item op is IOP_ST_SV)
__device__ __forceinline__ bool same_value(const CheckArgs& a, u32 ev_prior, u32 ev_cur) {
  return (ev_prior >> 5) == (ev_cur >> 5) && (!a.values || a.values[ev_prior] == a.values[ev_cur]);
}

__device__ __forceinline__ void emit(const CheckArgs& a, u32 key, u32 cur, u32 prior, u32 kind) {
  u32 at = atomicAdd(a.race_cnt, 1u);
  if (at < a.race_cap) a.races[at] = make_uint4(key, cur, prior, kind);
}

// the analysis context of the running K7 launch (set by launch_check; one K7 at a time)
__constant__ HbCtx cHC;

// slow path of the happens-before query: divergent intra-warp walk and foreign knowledge
static __device__ __noinline__ bool hb_slow(u32 ev1, u32 w1, u32 ev2, u32 s2w, u32 s2ps, u32 s2node, u32 s2blab) {
  const Snap s2{s2w, s2ps, s2node, s2blab};
  return hb(cHC, ev1 >> 5, ev1 & 31u, w1, ev2 >> 5, ev2 & 31u, s2);
}

// happens-before of event ev1 (by warp w1) before event ev2 whose record snapshot is s2.
// Inline fast path: same record / same thread / barrier label / converged warp.
__device__ __forceinline__ bool hb_ev(const HbCtx& c, u32 ev1, u32 w1, u32 ev2, const Snap& s2) {
  const u32 r1 = ev1 >> 5, r2 = ev2 >> 5, l1 = ev1 & 31u, l2 = ev2 & 31u;
  if (r1 == r2) return l1 == l2;                 // lanes of one instruction are concurrent
  if (w1 == s2.warp) {
    if (l1 == l2) return true;                   // program order
    if (s2.node == s2.warp && s2.ps >= r1 + 1u) return true;  // converged warp, endi join
  }
  const bool sameb = blk_of(c.g, w1) == blk_of(c.g, s2.warp);
  if (sameb && r1 + 1u <= s2.blab) return true;  // completed barrier (Fig. 3 BAR)
  if (c.n_acq == 0 && !(w1 == s2.warp && s2.node != s2.warp)) return false;
  return hb_slow(ev1, w1, ev2, s2.warp, s2.ps, s2.node, s2.blab);
}

// Same query, evaluated branch-free up to the rare slow case (divergent intra-warp walk or foreign
// knowledge): lane-sequential K7 lanes sit at different items, so every branch of the query would
// be executed by the whole warp.
__device__ __forceinline__ bool hbq(const HbCtx& c, u32 ev1, u32 w1, u32 ev2, const Snap& s2) {
  const u32 r1 = ev1 >> 5, r2 = ev2 >> 5;
  const bool samel = ((ev1 ^ ev2) & 31u) == 0u;
  const bool samew = w1 == s2.warp;
  const bool conv = s2.node == s2.warp;
  const bool ord = (samew && (samel || (conv && s2.ps > r1))) ||
                   (blk_of(c.g, w1) == blk_of(c.g, s2.warp) && s2.blab > r1);  // program order / endi / barrier
  if (r1 == r2) return samel;  // lanes of one instruction are concurrent
  if (ord) return true;
  if (c.n_acq == 0 && !(samew && !conv)) return false;
  return hb_slow(ev1, w1, ev2, s2.warp, s2.ps, s2.node, s2.blab);
}

// R_x is a vector clock at writer (ev2, s2): its entries are the latest read per thread among
// items [lo, hi] (all reads of this granule).  Check each (Fig. 2 WRITESHARED, Fig. 3 *ATOMSHARED).
static __device__ __noinline__ void vc_check(const u32* __restrict__ evs, uint4* races, u32* race_cnt, u32 race_cap,
                                             u64 lo, u64 hi, u32 ev2, u32 s2w, u32 s2ps, u32 s2node, u32 s2blab,
                                             u32 key, u32 kind) {
  const Snap s2{s2w, s2ps, s2node, s2blab};
  const HbCtx& c = cHC;
  u32 seen[32];
  int ns = 0;
  for (u64 j = hi + 1; j-- > lo;) {
    u32 ev = evs[j];
    u32 w1 = __ldg(&c.snap[ev >> 5].x);
    u32 tid = (w1 << 5) | (ev & 31u);
    bool dup = false;
    for (int q = 0; q < ns; ++q)
      if (seen[q] == tid) { dup = true; break; }
    if (!dup && ns == 32) {
      // overflow of the small set: look for a later read of the same thread directly
      for (u64 q = j + 1; q <= hi; ++q) {
        u32 e2 = evs[q];
        if (((__ldg(&c.snap[e2 >> 5].x) << 5) | (e2 & 31u)) == tid) { dup = true; break; }
      }
    }
    if (dup) continue;
    if (ns < 32) seen[ns++] = tid;
    if (!hb(c, ev >> 5, ev & 31u, w1, ev2 >> 5, ev2 & 31u, s2)) {
      u32 at = atomicAdd(race_cnt, 1u);
      if (at < race_cap) races[at] = make_uint4(key, ev2, ev, kind);
    }
  }
}

// ---------------------------------------------------------------------------------------
// Persistent warp-range formulation.  The grid is sized to be fully co-resident; warp w owns
// the contiguous item range [beg_w, end_w) and walks it in rounds of 32 (lane i = item r*32+i),
// carrying the automaton state (LW, FI of the current granule) from round to round; per lane,
// LW / FI inside a round come from ballots.  The state entering the range depends only on the
// items of the same granule before beg_w, so the warp recomputes it by walking backwards from
// beg_w (usually a few items: a writer or the start of the granule ends the walk); only if that
// walk exceeds K7_WALK_CAP items does the warp wait for warp w-1 to publish its final state.
// Items are read exactly once (plus the short walk), with a K7_PF-round register prefetch.
constexpr int K7_WARPS = 8;
constexpr int K7_PF = 4;
constexpr u32 K7_WALK_CAP = 1u << 14;

__device__ __forceinline__ u32 hibit(u32 m) { return 31u - __clz(m); }  // m != 0

// summary of one round (standalone), uniform across the warp
__device__ __forceinline__ Sum round_sum(u32 V, u32 Kin, u32 W, u32 I, u32 key, u64 base_r) {
  Sum r = sum_ident();
  if (!V) return r;
  const u32 last = hibit(V);
  r.fk = __shfl_sync(0xFFFFFFFFu, key, 0);
  r.lk = __shfl_sync(0xFFFFFFFFu, key, last);
  const u32 kc = Kin & ~1u & V;                 // key changes inside the round
  const u32 ts = kc ? hibit(kc) : 0u;           // start lane of the tail key run
  const u32 Wt = W & V & (~0u << ts);
  const bool hasW = Wt != 0;
  const u32 rs = hasW ? hibit(Wt) + 1u : ts;    // start of the trailing read run
  const u32 It = rs < 32 ? (I & V & (~0u << rs)) : 0u;
  r.lw = hasW ? (u32)(base_r + hibit(Wt)) + 1u : 0u;
  r.fi = It ? (u32)(base_r + __ffs(It) - 1) : NONE;
  r.bits = (kc ? 0u : 1u) | (hasW ? 2u : 0u);
  return r;
}

struct WarpEnd {  // final state of a warp's range (for the fallback of warp w+1)
  u32 flag, lk, lw, fi;
};

// READINFLATE flag of item i (a read): its predecessor i-1 is a read of the same granule that
// does not happen before it (Fig. 2, READINFLATE).
__device__ __forceinline__ bool infl_flag(const HbCtx& c, u32 qev, u32 ev) {
  const Snap s2 = load_snap(c.snap, ev >> 5);
  const u32 qw = __ldg(&c.snap[qev >> 5].x);
  return !hb_ev(c, qev, qw, ev, s2);
}

// State (lk, lw, fi) after item s-1 restricted to the granule of item s-1, computed from the
// items before s.  Returns false if the walk exceeded the cap.
__device__ bool walk_back(const CheckArgs& a, u64 s, Sum& out) {
  const HbCtx& c = a.c;
  const int lane = threadIdx.x & 31;
  const u32 k0 = a.keys[s - 1] >> 2;
  out = sum_ident();
  out.fk = k0;
  out.lk = k0;
  out.bits = 1u;
  u32 fi = NONE;
  u64 hi = s - 1;  // highest item of the current window
  for (u32 walked = 0;; walked += 32) {
    if (walked >= K7_WALK_CAP) return false;
    const u64 lo = hi >= 31 ? hi - 31 : 0;
    const u64 i = lo + lane;
    const bool in = i <= hi;
    const u32 kx = in ? a.keys[i] : NONE, ev = in ? a.evs[i] : 0u;
    const bool inkey = in && (kx >> 2) == k0;
    const u32 W = __ballot_sync(0xFFFFFFFFu, inkey && (kx & 3u) != IOP_LD);
    const u32 B = __ballot_sync(0xFFFFFFFFu, in && !inkey);  // other granules (below, keys sorted)
    const int hw = W ? (int)hibit(W) : -1, hb_ = B ? (int)hibit(B) : -1;
    const int bnd = hw > hb_ ? hw : hb_;  // the read run is (bnd, top]
    // inflation flags of the run's reads (predecessor inside the run)
    u32 qkx = __shfl_up_sync(0xFFFFFFFFu, kx, 1), qev = __shfl_up_sync(0xFFFFFFFFu, ev, 1);
    if (lane == 0 && lo > 0) {
      qkx = a.keys[lo - 1];
      qev = a.evs[lo - 1];
    }
    const bool inrun = in && lane > bnd;
    const bool e = inrun && (lane > 0 || lo > 0) && qkx != NONE && (qkx >> 2) == k0 && (qkx & 3u) == IOP_LD &&
                   infl_flag(c, qev, ev);
    const u32 I = __ballot_sync(0xFFFFFFFFu, e);
    if (I) fi = (u32)(lo + __ffs(I) - 1);  // earlier windows hold earlier items
    if (bnd >= 0 || lo == 0) {
      if (hw >= 0 && hw > hb_) {
        out.lw = (u32)(lo + hw) + 1u;
        out.bits |= 2u;
      }
      out.fi = fi;
      return true;
    }
    hi = lo - 1;
  }
}

// Software pipeline per warp: items (key, ev) are loaded K7_PF rounds ahead, the 16-B clock
// snapshot of each item's record K7_PS rounds ahead (its address is the item's ev, which arrived
// K7_PF - K7_PS rounds earlier), so the happens-before queries of a round touch registers only.
// The predecessor item's warp (for READINFLATE and the epoch R check) comes from the lane below by
// a shuffle; the last writer's (key, ev, warp) is carried in registers across rounds.
// An item's snapshot is gathered only if some query of the round can read it: an item alone in its
// granule never needs one, nor does an atomic whose same-granule neighbours are atomics (its W check
// is elided against the atomic before it, it is not a read, and the next item, if atomic, does not
// check against it).  Every other consumer -- READINFLATE (both reads), the W check
// (the current item and the last writer, which is followed by a read or by the checking item), the
// R check at a writer (the writer and the read before it) -- lies inside this set.  On atomic-heavy
// traces (C4/C5 cost/mask) this removes almost all random 16-B gathers.
constexpr int K7_PS = 2;

__device__ __forceinline__ uint4 snap_if_needed(const HbCtx& c, u32 k, u32 e, u32 kprev0, u32 knext31) {
  const int lane = threadIdx.x & 31;
  u32 kp = __shfl_up_sync(0xFFFFFFFFu, k, 1), kn = __shfl_down_sync(0xFFFFFFFFu, k, 1);
  if (lane == 0) kp = kprev0;
  if (lane == 31) kn = knext31;
  if (k == NONE) return make_uint4(0, 0, 0, 0);
  const u32 key = k >> 2;
  const bool sp = kp != NONE && (kp >> 2) == key, sn = kn != NONE && (kn >> 2) == key;
  const bool atm_only = (k & 3u) == IOP_ATOM && (!sp || (kp & 3u) == IOP_ATOM) && (!sn || (kn & 3u) == IOP_ATOM);
  if ((!sp && !sn) || atm_only) return make_uint4(0, 0, 0, 0);
  return __ldg(c.snap + (e >> 5));
}

__global__ void __launch_bounds__(K7_WARPS * 32, 2) k_check(CheckArgs a, WarpEnd* wend, u32 nw) {
  const u64 n = *a.n_dev;
  const u32 w = blockIdx.x * K7_WARPS + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  const HbCtx& c = a.c;
  const u32 lt = lanemask_lt();
  const u64 nr = (n + 31) / 32;  // rounds in total
  const u64 beg = (nr * w / nw) * 32, end = min(n, (nr * (w + 1) / nw) * 32);

  // ---- incoming state
  Sum carry = sum_ident();
  u32 pkx = NONE, pev = 0, pw = 0;      // item beg-1 (the predecessor of lane 0 in the first round)
  u32 cwk = 0, cwe = 0, cww = 0;        // carried last writer: key word, event, warp
  if (beg > 0 && beg < end) {
    pkx = a.keys[beg - 1];
    pev = a.evs[beg - 1];
    pw = __ldg(&c.snap[pev >> 5].x);
    if ((pkx >> 2) == (a.keys[beg] >> 2)) {  // the first granule straddles the boundary
      if (!walk_back(a, beg, carry)) {
        // very long read run: take warp w-1's final state (all warps are co-resident)
        volatile WarpEnd* pe = &wend[w - 1];
        while (pe->flag == 0) {
        }
        __threadfence();
        carry.fk = carry.lk = pe->lk;
        carry.lw = pe->lw;
        carry.fi = pe->fi;
        carry.bits = 1u | (carry.lw ? 2u : 0u);
      }
      if (carry.lw) {
        cwk = a.keys[carry.lw - 1];
        cwe = a.evs[carry.lw - 1];
        cww = __ldg(&c.snap[cwe >> 5].x);
      }
    }
  }

  // ---- the range, round by round
  const u32 no_sv = c.g.flags & BC_F_NO_SAME_VALUE_FILTER;
  u32 segs = 0;
  u32 pf_k[K7_PF], pf_e[K7_PF];
  uint4 pf_s[K7_PS];
#pragma unroll
  for (int q = 0; q < K7_PF; ++q) {
    const u64 i = beg + (u64)q * 32 + lane;
    pf_k[q] = i < end ? a.keys[i] : NONE;
    pf_e[q] = i < end ? a.evs[i] : 0u;
  }
#pragma unroll
  for (int q = 0; q < K7_PS; ++q) {
    const u32 kp0 = q == 0 ? pkx : __shfl_sync(0xFFFFFFFFu, pf_k[q > 0 ? q - 1 : 0], 31);
    const u32 kn31 = __shfl_sync(0xFFFFFFFFu, pf_k[q + 1], 0);
    pf_s[q] = snap_if_needed(c, pf_k[q], pf_e[q], kp0, kn31);
  }
  for (u64 base_r = beg; base_r < end; base_r += 32) {
    const u64 i = base_r + lane;
    const bool valid = i < end;
    const u32 kx = pf_k[0], ev = pf_e[0];
    const Snap s2 = to_snap(pf_s[0]);
#pragma unroll
    for (int q = 0; q + 1 < K7_PF; ++q) {
      pf_k[q] = pf_k[q + 1];
      pf_e[q] = pf_e[q + 1];
    }
#pragma unroll
    for (int q = 0; q + 1 < K7_PS; ++q) pf_s[q] = pf_s[q + 1];
    {
      const u64 ip = base_r + (u64)K7_PF * 32 + lane;
      pf_k[K7_PF - 1] = ip < end ? a.keys[ip] : NONE;
      pf_e[K7_PF - 1] = ip < end ? a.evs[ip] : 0u;
      const u32 kp0 = __shfl_sync(0xFFFFFFFFu, K7_PS >= 2 ? pf_k[K7_PS >= 2 ? K7_PS - 2 : 0] : kx, 31);
      const u32 kn31 = __shfl_sync(0xFFFFFFFFu, pf_k[K7_PS], 0);
      pf_s[K7_PS - 1] = snap_if_needed(c, pf_k[K7_PS - 1], pf_e[K7_PS - 1], kp0, kn31);
    }
    u32 qkx = __shfl_up_sync(0xFFFFFFFFu, kx, 1);
    u32 qev = __shfl_up_sync(0xFFFFFFFFu, ev, 1);
    u32 qw = __shfl_up_sync(0xFFFFFFFFu, s2.warp, 1);
    if (lane == 0) {
      qkx = pkx;
      qev = pev;
      qw = pw;
    }
    const u32 key = kx >> 2, op = kx & 3u;
    const bool same = qkx != NONE && (qkx >> 2) == key;
    const bool e = valid && op == IOP_LD && same && (qkx & 3u) == IOP_LD && !hb_ev(c, qev, qw, ev, s2);
    const u32 V = __ballot_sync(0xFFFFFFFFu, valid);
    const u32 I = __ballot_sync(0xFFFFFFFFu, e);
    const u32 W = __ballot_sync(0xFFFFFFFFu, valid && op != IOP_LD);
    const u32 K = __ballot_sync(0xFFFFFFFFu, valid && !same);
    segs += __popc(K);
    const bool cont_key = carry.fk != NONE && carry.lk == key;
    // segment start of this lane inside the round (-1: the key run continues from before)
    const u32 Kle = K & (lt | (1u << lane));
    const int sstart = Kle ? (int)hibit(Kle) : -1;
    const u32 segm = sstart >= 0 ? (~0u << sstart) : ~0u;
    const u32 cand = W & lt & segm;
    const int lwl = cand ? (int)hibit(cand) : -1;
    const u32 src = lwl >= 0 ? (u32)lwl : (u32)lane;
    const u32 wkx = __shfl_sync(0xFFFFFFFFu, kx, src);
    const u32 wev = __shfl_sync(0xFFFFFFFFu, ev, src);
    const u32 wwp = __shfl_sync(0xFFFFFFFFu, s2.warp, src);
    if (valid) {
      u32 pkx2 = 0, pev2 = 0, pw2 = 0;
      bool haveW = false;
      if (lwl >= 0) {
        pkx2 = wkx; pev2 = wev; pw2 = wwp; haveW = true;
      } else if (sstart < 0 && cont_key && carry.lw) {
        pkx2 = cwk; pev2 = cwe; pw2 = cww; haveW = true;
      }
      const bool patm = (pkx2 & 3u) == IOP_ATOM;
      const bool needW = valid && haveW && !(op == IOP_ATOM && patm);
      const bool needR = valid && op != IOP_LD && same && (qkx & 3u) == IOP_LD;
      // W_x check (every rule of Fig. 2; atomics only against a plain last write)
      if (needW && !hb_ev(c, pev2, pw2, ev, s2)) {
        if (op == IOP_LD) {
          emit(a, key, ev, pev2, patm ? BC_KIND_AR : BC_KIND_WR);
        } else if (op == IOP_ATOM) {
          emit(a, key, ev, pev2, BC_KIND_WA);
        } else {
          const bool filtered = !patm && op == IOP_ST_SV && !no_sv && same_value(a, pev2, ev);
          if (!filtered) emit(a, key, ev, pev2, patm ? BC_KIND_AW : BC_KIND_WW);
        }
      }
      // R_x check at writers (WRITE* / *ATOM*: R_x ⪯ C_t as an epoch, R_x ⊑ C_t as a vector)
      if (needR) {
        const u32 kind = op == IOP_ATOM ? BC_KIND_RA : BC_KIND_RW;
        // first READINFLATE in the read run ending at this writer
        const int rs = lwl >= 0 ? lwl + 1 : sstart;  // -1: the run started before this round
        const u32 Ir = I & lt & (rs >= 0 ? (~0u << rs) : ~0u);
        u32 fi = NONE;
        if (rs < 0 && cont_key && carry.fi != NONE) fi = carry.fi;  // the run's first inflation came earlier
        else if (Ir) fi = (u32)(base_r + __ffs(Ir) - 1);
        if (fi == NONE) {
          if (!hb_ev(c, qev, qw, ev, s2)) emit(a, key, ev, qev, kind);
        } else {
          vc_check(a.evs, a.races, a.race_cnt, a.race_cap, (u64)fi - 1, i - 1, ev, s2.warp, s2.ps, s2.node,
                   s2.blab, key, kind);
        }
      }
    }
    const Sum rsum = round_sum(V, K, W, I, key, base_r);
    if (rsum.bits & 2u) {  // the round's tail key run holds a writer: it is the new carried writer
      const u32 lwln = (u32)(rsum.lw - 1u - (u32)base_r);
      cwk = __shfl_sync(0xFFFFFFFFu, kx, lwln);
      cwe = __shfl_sync(0xFFFFFFFFu, ev, lwln);
      cww = __shfl_sync(0xFFFFFFFFu, s2.warp, lwln);
    }
    carry = combine(carry, rsum);
    const u32 last = hibit(V);
    pkx = __shfl_sync(0xFFFFFFFFu, kx, last);
    pev = __shfl_sync(0xFFFFFFFFu, ev, last);
    pw = __shfl_sync(0xFFFFFFFFu, s2.warp, last);
  }
  if (lane == 0) {
    if (segs) atomicAdd((unsigned long long*)a.seg_cnt, (unsigned long long)segs);
    volatile WarpEnd* me = &wend[w];
    me->lk = carry.lk;
    me->lw = carry.lw;
    me->fi = carry.fi;
    __threadfence();
    me->flag = 1u;
  }
}

// ---------------------------------------------------------------------------------------
// Lane-sequential formulation with shared-memory staged clocks and a query buffer (default;
// BC_K7=ballot selects k_check above).  Same persistent warp ranges and incoming state
// (walk_back / WarpEnd) as k_check; each range is processed in blocks of 32 * KT_IPL items:
//   load    : the block's (key, ev) words land in shared memory by cp.async, one block ahead
//             (row pitch KT_IPL+1 words: lane l reading item l*KT_IPL+j is bank-conflict free)
//   gather  : lane l walks ITS KT_IPL consecutive items; for each item some query can read (the
//             snap_if_needed rule) it issues a 16-B cp.async of the record snapshot into shared
//             memory (up to 32*KT_IPL gathers in flight per warp, no registers held), and for
//             each read preceded by a read of the same granule it queues a READINFLATE query
//   eval    : the queued happens-before queries are evaluated in uniform rounds (lane l, round i:
//             its own i-th query), so the warp runs ONE copy of the query code instead of the
//             union of every branch its lanes are in
//   summary : lane l walks its items again: chunk summary Sum (last key, last writer, first
//             inflation after it) from the READINFLATE flags (Fig. 2)
//   scan    : a 5-step warp scan of the summaries (the associative combine of k_check) gives every
//             lane the automaton state (LW, FI) entering its chunk, and the block carry
//   rules   : lane l replays the rules of Fig. 2 / Fig. 3 over its chunk from that state and queues
//             the checks they make (W check, R check against the epoch or the read vector, with
//             the same-value filter applied at queueing), then the queries are evaluated as above.
// A query is one u32: item index (current event), source index (prior event; two codes name
// per-lane registers holding an event from before the block), kind.  Every query reads shared
// memory only; values carried across blocks are loaded from global memory once per lane.
#ifndef KT_IPL_
#define KT_IPL_ 16
#endif
constexpr int KT_IPL = KT_IPL_;              // items per lane per block
constexpr int KT_BLK = 32 * KT_IPL;          // items per warp block
constexpr int KT_PITCH = 32 * (KT_IPL + 1);  // padded entries per array
#ifndef KT_DB
#define KT_DB 0  // 1: keys / events of the next block staged during this one (double buffer)
#endif
#ifndef KT_NWARPS
#define KT_NWARPS 16  // 16 x 128 registers fill the register file; the single-buffered stage fits 16
#endif
constexpr int KT_WARPS = KT_NWARPS;
// per warp: snapshots [KT_PITCH] uint4, keys / evs double-buffered [2][2][KT_PITCH] u32
constexpr size_t KT_WARP_BYTES = (size_t)KT_PITCH * (sizeof(uint4) + (KT_DB ? 4 : 2) * sizeof(u32));

__device__ __forceinline__ u32 tpad(u32 i) { return i + i / KT_IPL; }

__device__ __forceinline__ void cp_async4(void* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// stage the (key, ev) words of items [bb, bb + nb) of the range into sK / sE (lane l copies items
// r*32 + l); tail entries up to KT_BLK are NONE / 0
__device__ __forceinline__ void kt_stage(const CheckArgs& a, u64 bb, u32 nb, u32* sK, u32* sE, u32 lane) {
#pragma unroll 4
  for (u32 r = 0; r < (u32)KT_IPL; ++r) {
    const u32 li = r * 32u + lane;
    if (li < nb) {
      cp_async4(sK + tpad(li), a.keys + bb + li);
      cp_async4(sE + tpad(li), a.evs + bb + li);
    } else {
      sK[tpad(li)] = NONE;
      sE[tpad(li)] = 0u;
    }
  }
  cp_async_commit();
}

__device__ __forceinline__ Sum shfl_up_sum(const Sum& s, int o) {
  Sum r;
  r.fk = __shfl_up_sync(0xFFFFFFFFu, s.fk, o);
  r.lk = __shfl_up_sync(0xFFFFFFFFu, s.lk, o);
  r.lw = __shfl_up_sync(0xFFFFFFFFu, s.lw, o);
  r.fi = __shfl_up_sync(0xFFFFFFFFu, s.fi, o);
  r.bits = __shfl_up_sync(0xFFFFFFFFu, s.bits, o);
  return r;
}
__device__ __forceinline__ Sum shfl_sum(const Sum& s, int src) {
  Sum r;
  r.fk = __shfl_sync(0xFFFFFFFFu, s.fk, src);
  r.lk = __shfl_sync(0xFFFFFFFFu, s.lk, src);
  r.lw = __shfl_sync(0xFFFFFFFFu, s.lw, src);
  r.fi = __shfl_sync(0xFFFFFFFFu, s.fi, src);
  r.bits = __shfl_sync(0xFFFFFFFFu, s.bits, src);
  return r;
}

__global__ void __launch_bounds__(KT_WARPS * 32, 1) k_check_tile(CheckArgs a, WarpEnd* wend, u32 nw) {
  extern __shared__ __align__(16) unsigned char kt_smem[];
  const int wi = threadIdx.x >> 5;
  uint4* sS = reinterpret_cast<uint4*>(kt_smem + (size_t)wi * KT_WARP_BYTES);
  u32* const sKE = reinterpret_cast<u32*>(sS + KT_PITCH);  // [buf][key|ev][KT_PITCH]
  const u64 n = *a.n_dev;
  const u32 w = blockIdx.x * KT_WARPS + wi;
  const u32 lane = threadIdx.x & 31;
  const HbCtx& c = a.c;
  const u64 nr = (n + 31) / 32;
  const u64 beg = (nr * w / nw) * 32, end = min(n, (nr * (w + 1) / nw) * 32);
  const u32 no_sv = c.g.flags & BC_F_NO_SAME_VALUE_FILTER;

  // ---- incoming state of the range (as k_check)
  Sum carry = sum_ident();
  u32 pkx = NONE, pev = 0;  // the item before the block
  u32 cwk = 0, cwe = 0;     // key word / event of carry.lw
  if (beg > 0 && beg < end) {
    pkx = a.keys[beg - 1];
    pev = a.evs[beg - 1];
    if ((pkx >> 2) == (a.keys[beg] >> 2)) {
      if (!walk_back(a, beg, carry)) {
        volatile WarpEnd* pe = &wend[w - 1];
        while (pe->flag == 0) {
        }
        __threadfence();
        carry.fk = carry.lk = pe->lk;
        carry.lw = pe->lw;
        carry.fi = pe->fi;
        carry.bits = 1u | (carry.lw ? 2u : 0u);
      }
      if (carry.lw) {
        cwk = a.keys[carry.lw - 1];
        cwe = a.evs[carry.lw - 1];
      }
    }
  }

  u32 segs = 0;
  const u32 l0 = lane * KT_IPL;
  if (beg < end) kt_stage(a, beg, (u32)(end - beg < (u64)KT_BLK ? end - beg : (u64)KT_BLK), sKE, sKE + KT_PITCH, lane);
  for (u64 bb = beg; bb < end; bb += KT_BLK) {
    const u32 nb = (u32)(end - bb < (u64)KT_BLK ? end - bb : (u64)KT_BLK);
    // ---- this block's (key, ev) words were staged one iteration ago (or by the prologue)
    const u32 buf = KT_DB ? (u32)(((bb - beg) / KT_BLK) & 1u) : 0u;
    u32* const sK = sKE + buf * 2 * KT_PITCH;
    u32* const sE = sK + KT_PITCH;
    const u32 knext = bb + nb < end ? a.keys[bb + nb] : NONE;  // first item after the block
    cp_async_wait<0>();
    __syncwarp();

    const u32 cnt = l0 < nb ? min((u32)KT_IPL, nb - l0) : 0u;
    const u32 ppk = lane == 0 ? pkx : sK[tpad(l0 - 1)];
    const u32 ppe = lane == 0 ? pev : sE[tpad(l0 - 1)];
    // warp of the item before the lane's chunk (read only if that item is a same-granule read,
    // which has a successor, so it was gathered; lane 0: the item before the block)
    const u32 gbb = (u32)bb;

    // ---- gather the snapshots some query can read
    {
      u32 kp = ppk, k = cnt ? sK[tpad(l0)] : NONE;
      for (u32 j = 0; j < cnt; ++j) {
        const u32 li = l0 + j;
        const u32 kn = li + 1 < nb ? sK[tpad(li + 1)] : knext;
        const u32 key = k >> 2;
        const bool sp = kp != NONE && (kp >> 2) == key, sn = kn != NONE && (kn >> 2) == key;
        const bool atm_only =
            (k & 3u) == IOP_ATOM && (!sp || (kp & 3u) == IOP_ATOM) && (!sn || (kn & 3u) == IOP_ATOM);
        if ((sp || sn) && !atm_only) cp_async16(sS + tpad(li), c.snap + (sE[tpad(li)] >> 5));
        kp = k;
        k = kn;
      }
    }
    cp_async_commit();
    if (KT_DB && bb + nb < end) {  // stage the next block now: its loads overlap this block's work
      const u64 b2 = bb + nb;
      kt_stage(a, b2, (u32)(end - b2 < (u64)KT_BLK ? end - b2 : (u64)KT_BLK), sKE + (buf ^ 1u) * 2 * KT_PITCH,
               sKE + (buf ^ 1u) * 2 * KT_PITCH + KT_PITCH, lane);
    }
    const u32 pw0 = (lane == 0 && ppk != NONE) ? __ldg(&c.snap[pev >> 5].x) : 0u;
    if (KT_DB && bb + nb < end) cp_async_wait<1>(); else cp_async_wait<0>();
    __syncwarp();

    // ---- READINFLATE flags (Fig. 2: a read whose predecessor is an unordered read of the same
    // granule) and the chunk summary
    Sum sm = sum_ident();
    u32 imask = 0;
    if (cnt) {
      u32 pk = ppk, pe = ppe, pw = lane ? sS[tpad(l0 - 1)].x : pw0, tlw = 0, tfi = NONE;
      bool kc = false;
      sm.fk = sK[tpad(l0)] >> 2;
      for (u32 j = 0; j < cnt; ++j) {
        const u32 li = l0 + j;
        const u32 k = sK[tpad(li)], e = sE[tpad(li)];
        const uint4 sv = sS[tpad(li)];
        const u32 gi = gbb + li;
        const bool same = pk != NONE && (pk >> 2) == (k >> 2);
        if (!same) {
          ++segs;
          kc |= j > 0;
          tlw = 0;
          tfi = NONE;
        }
        if ((k & 3u) != IOP_LD) {
          tlw = gi + 1u;
          tfi = NONE;
        } else if (same && (pk & 3u) == IOP_LD && !hbq(c, pe, pw, e, to_snap(sv))) {
          imask |= 1u << j;
          if (tfi == NONE) tfi = gi;
        }
        pk = k;
        pe = e;
        pw = sv.x;
      }
      sm.lk = pk >> 2;
      sm.lw = tlw;
      sm.fi = tfi;
      sm.bits = (kc ? 0u : 1u) | (tlw ? 2u : 0u);
    }

    // ---- scan of the chunk summaries -> state entering each chunk; block carry
    Sum incl = sm;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const Sum up = shfl_up_sum(incl, o);
      if ((int)lane >= o) incl = combine(up, incl);
    }
    Sum ex = shfl_up_sum(incl, 1);
    if (lane == 0) ex = sum_ident();
    const Sum in = combine(carry, ex);
    const Sum blk = shfl_sum(incl, 31);

    // ---- the rules of Fig. 2 / Fig. 3, lane-sequentially
    if (cnt) {
      u32 lw = (in.fk != NONE) ? in.lw : 0u, fi = (in.fk != NONE) ? in.fi : NONE;
      u32 wk = 0, we = 0, ww = 0;
      if (lw) {
        if ((u64)(lw - 1) >= bb) {
          const u32 wl = (u32)(lw - 1 - bb);
          wk = sK[tpad(wl)];
          we = sE[tpad(wl)];
          ww = sS[tpad(wl)].x;  // gathered: the writer has a same-granule successor in the block
        } else {
          wk = cwk;
          we = cwe;
          ww = __ldg(&c.snap[cwe >> 5].x);
        }
      }
      u32 pk = ppk, pe = ppe, pw = lane ? sS[tpad(l0 - 1)].x : pw0;
      for (u32 j = 0; j < cnt; ++j) {
        const u32 li = l0 + j;
        const u32 k = sK[tpad(li)], e = sE[tpad(li)];
        const uint4 sv = sS[tpad(li)];
        const Snap s2 = to_snap(sv);
        const u32 op = k & 3u;
        const u32 gi = gbb + li;
        const bool same = pk != NONE && (pk >> 2) == (k >> 2);
        if (!same) {
          lw = 0;
          fi = NONE;
        }
        if (op == IOP_LD && ((imask >> j) & 1u) && fi == NONE) fi = gi;
        const bool patm = (wk & 3u) == IOP_ATOM;
        // W_x check (every rule of Fig. 2; atomics only against a plain last write)
        if (lw && !(op == IOP_ATOM && patm) && !hbq(c, we, ww, e, s2)) {
          const u32 kind = op == IOP_LD ? (patm ? BC_KIND_AR : BC_KIND_WR)
                                        : op == IOP_ATOM ? BC_KIND_WA : (patm ? BC_KIND_AW : BC_KIND_WW);
          const bool filtered = !patm && op == IOP_ST_SV && !no_sv && same_value(a, we, e);
          if (!filtered) emit(a, k >> 2, e, we, kind);
        }
        if (op != IOP_LD) {
          if (same && (pk & 3u) == IOP_LD) {  // R_x check at a writer: epoch, or vector after READINFLATE
            const u32 kind = op == IOP_ATOM ? BC_KIND_RA : BC_KIND_RW;
            if (fi == NONE) {
              if (!hbq(c, pe, pw, e, s2)) emit(a, k >> 2, e, pe, kind);
            } else {
              const u64 lo = (u64)fi - 1;
              if (lo >= bb && gi - (u32)lo <= 64u) {
                // the read run is staged in this block: the latest read of each thread in it
                const u32 jl = (u32)(lo - bb);
                for (u32 jj = li; jj-- > jl;) {
                  const u32 ev1 = sE[tpad(jj)], w1 = sS[tpad(jj)].x;
                  bool dup = false;
                  for (u32 q = jj + 1; q < li && !dup; ++q)
                    dup = sS[tpad(q)].x == w1 && ((sE[tpad(q)] ^ ev1) & 31u) == 0u;
                  if (!dup && !hbq(c, ev1, w1, e, s2)) emit(a, k >> 2, e, ev1, kind);
                }
              } else {
                vc_check(a.evs, a.races, a.race_cnt, a.race_cap, lo, (u64)gi - 1, e, s2.warp, s2.ps, s2.node,
                         s2.blab, k >> 2, kind);
              }
            }
          }
          lw = gi + 1u;
          wk = k;
          we = e;
          ww = sv.x;
          fi = NONE;
        }
        pk = k;
        pe = e;
        pw = sv.x;
      }
    }

    // ---- block carry
    carry = combine(carry, blk);
    if (carry.lw && (u64)(carry.lw - 1) >= bb) {
      cwk = sK[tpad((u32)(carry.lw - 1 - bb))];
      cwe = sE[tpad((u32)(carry.lw - 1 - bb))];
    }
    pkx = sK[tpad(nb - 1)];
    pev = sE[tpad(nb - 1)];
    __syncwarp();
    if (!KT_DB && bb + nb < end) {  // single buffer: stage the next block once this one is done
      const u64 b2 = bb + nb;
      kt_stage(a, b2, (u32)(end - b2 < (u64)KT_BLK ? end - b2 : (u64)KT_BLK), sKE, sKE + KT_PITCH, lane);
    }
  }
  segs = __reduce_add_sync(0xFFFFFFFFu, segs);
  if (lane == 0) {
    if (segs) atomicAdd((unsigned long long*)a.seg_cnt, (unsigned long long)segs);
    volatile WarpEnd* me = &wend[w];
    me->lk = carry.lk;
    me->lw = carry.lw;
    me->fi = carry.fi;
    __threadfence();
    me->flag = 1u;
  }
}

// Statistics only (bc_config.flags & BC_F_COUNT_GATHERS): the number of items whose record clock
// snapshot K7 reads -- the snap_if_needed rule over the sorted items -- for the roofline's
// algorithmic bytes.  A separate pass so that the hot kernels carry no counter.
__global__ void k_count_gathers(const u32* __restrict__ keys, const u64* __restrict__ n_dev, u64* __restrict__ out) {
  const u64 n = *n_dev;
  u32 cnt = 0;
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x) {
    const u32 k = keys[i], kp = i ? keys[i - 1] : NONE, kn = i + 1 < n ? keys[i + 1] : NONE;
    const u32 key = k >> 2;
    const bool sp = kp != NONE && (kp >> 2) == key, sn = kn != NONE && (kn >> 2) == key;
    const bool atm_only = (k & 3u) == IOP_ATOM && (!sp || (kp & 3u) == IOP_ATOM) && (!sn || (kn & 3u) == IOP_ATOM);
    cnt += (sp || sn) && !atm_only;
  }
  cnt = __reduce_add_sync(0xFFFFFFFFu, cnt);
  if ((threadIdx.x & 31) == 0 && cnt) atomicAdd((unsigned long long*)out, (unsigned long long)cnt);
}

}  // namespace

void launch_count_gathers(const u32* keys, const u64* n_dev, u64* out, cudaStream_t st) {
  k_count_gathers<<<148 * 8, 256, 0, st>>>(keys, n_dev, out);
  ++g_launches;
}

size_t check_status_bytes(u64 n) { return (size_t)148 * 64 * sizeof(WarpEnd) + 256; }

void launch_check(const HbCtx& c, const u32* keys, const u32* evs, const u64* n_dev, u64 n_max, void* status,
                  uint4* races, u32* race_cnt, u32 race_cap, u64* seg_cnt, const u64* values, cudaStream_t st) {
  if (n_max == 0) return;
  // K7 variant: lane-sequential with shared-memory staged clocks (default) or ballot rounds
  // (BC_K7=ballot); read at every launch so that tests can switch it
  const char* v = getenv("BC_K7");
  const int use_tile = (v && !strcmp(v, "ballot")) ? 0 : 1;
  static int grid_tile = 0, grid_ballot = 0;
  const size_t smem_tile = (size_t)KT_WARPS * KT_WARP_BYTES;
  int& grid = use_tile ? grid_tile : grid_ballot;
  if (grid == 0) {
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (use_tile) {
      cudaFuncSetAttribute(k_check_tile, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_tile);
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_check_tile, KT_WARPS * 32, smem_tile);
    } else {
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_check, K7_WARPS * 32, 0);
    }
    if (per < 1) per = 1;
    const int wpc = use_tile ? KT_WARPS : K7_WARPS;
    grid = sms * per;
    if (grid * wpc > 148 * 64) grid = 148 * 64 / wpc;
  }
  const u32 nw = (u32)grid * (use_tile ? KT_WARPS : K7_WARPS);
  cudaMemsetAsync(status, 0, (size_t)nw * sizeof(WarpEnd), st);
  cudaMemcpyToSymbolAsync(cHC, &c, sizeof(HbCtx), 0, cudaMemcpyHostToDevice, st);
  CheckArgs a;
  a.c = c;
  a.keys = keys;
  a.evs = evs;
  a.n_dev = n_dev;
  a.races = races;
  a.race_cnt = race_cnt;
  a.race_cap = race_cap;
  a.seg_cnt = seg_cnt;
  a.values = values;
  if (use_tile) {
    k_check_tile<<<grid, KT_WARPS * 32, smem_tile, st>>>(a, (WarpEnd*)status, nw);
  } else {
    k_check<<<grid, K7_WARPS * 32, 0, st>>>(a, (WarpEnd*)status, nw);
  }
  ++g_launches;
}

}  // namespace bc
