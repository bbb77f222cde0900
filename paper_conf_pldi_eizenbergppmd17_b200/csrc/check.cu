// check.cu — K6+K7 per-address shadow check, the hot kernel.
//
// Input: the items of one trace WINDOW (a contiguous record range [R0, R1)) sorted
// by shadow granule, each granule's accesses in trace order (stable sort); an item is
// (granule key << 2 | op, (record - R0) << 5 | lane).
// The rules of Fig. 2 / Fig. 3 for one granule x (readings R2-R8):
//   rd  : W_x ⪯ C_t, then READEXCL (R_x ⪯ C_t -> R_x := E(t)) | READINFLATE (-> VC) | READSHARED
//   wr  : W_x ⪯ C_t, R_x ⪯/⊑ C_t; R_x := ⊥, W_x := (E(t), plain)
//   atm : W_x ⪯ C_t only if W_x is plain; R_x ⪯/⊑ C_t; R_x := ⊥, W_x := (E(t), atomic)
// depend on the state only through (a) the last writer before each access, and (b) for each
// writer, the reads since the previous writer: R_x is the epoch of the last read unless some read
// in that run found its predecessor unordered (READINFLATE), in which case R_x is the vector of the
// latest read per thread from the read before the first inflation on ("K7 exactly as
// the oracle").  Inside a window the automaton is two segmented scans over the sorted items —
//   LW(i) = last writer before i in its granule          (segmented max)
//   FI(i) = first inflating read in the run ending at i  (segmented min, reset at writers)
// plus independent happens-before queries per item.
//
// Across windows the granule's state is carried in the paper's per-location shadow entry
// (Fig. 8; shadow memory §4.3.3), 32 B per granule:
//   e0 = {W rec, W lane, W flags (valid | atomic), R mode (none | epoch | vector)}
//   e1 = {R rec | vector offset, R lane | vector length, key, 0}
// (a thread is (record, lane): its warp is snap[record].warp, looked up only when a check against the
// carried access is made, so writing an entry never needs the record's clock snapshot)
// The entry of granule k acts as virtual items in front of k's first item of the window: its W is
// the last writer until the first writer of the window, its R the read state the first reads of the
// window extend (a carried read vector counts as already inflated).  Read
// vectors live in an append-only pool of (record, warp << 5 | lane) entries.  The entries are read
// from one table and written to another (double buffer), so no lane ever sees a half-updated state.
#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "common.cuh"
#include "kernels.cuh"

namespace bc {

namespace {

// ----------------------------------------------------------------- scan summary of an item span
// bits: SB_ONE = one key throughout; SB_W = the tail key run holds a writer (lw = its index + 1);
//       SB_CI = the tail run (no writer) starts at its granule's first item of the window and the
//       carried read state makes it a read vector ("carried inflation")
constexpr u32 SB_ONE = 1u, SB_W = 2u, SB_CI = 4u;

struct Sum {
  u32 fk, lk, lw, fi, bits;  // first / last granule, last writer (+1) and first inflation of the tail run
};

__device__ __forceinline__ Sum sum_ident() { return Sum{NONE, NONE, 0u, NONE, 0u}; }

__device__ __forceinline__ Sum combine(const Sum& L, const Sum& R) {
  if (L.fk == NONE) return R;
  if (R.fk == NONE) return L;
  Sum o;
  o.fk = L.fk;
  o.lk = R.lk;
  if ((R.bits & SB_ONE) && R.fk == L.lk) {  // R continues L's tail granule throughout
    const bool rw = R.bits & SB_W;
    o.lw = rw ? R.lw : L.lw;
    o.fi = rw ? R.fi : min(L.fi, R.fi);
    o.bits = (L.bits & SB_ONE) | ((L.bits | R.bits) & SB_W) | (rw ? 0u : (L.bits & SB_CI));
  } else {
    o.lw = R.lw;
    o.fi = R.fi;
    o.bits = R.bits & (SB_W | SB_CI);
  }
  return o;
}

// ----------------------------------------------------------------- shadow entry (carried state)
constexpr u32 SH_W_VALID = 1u, SH_W_ATOM = 2u;
constexpr u32 SH_R_NONE = 0u, SH_R_EPOCH = 1u, SH_R_VC = 2u;

struct Carry {
  u32 wr, wwl, wf;   // carried writer: record, lane, flags
  u32 rm, rr, rwl;   // carried read state: mode; epoch (record, lane) or vector (offset, length)
};
__device__ __forceinline__ Carry no_carry() { return Carry{0u, 0u, 0u, SH_R_NONE, 0u, 0u}; }

// Everything the out-of-line slow paths need (device copy per launch, per context: no __constant__
// state shared between contexts or devices)
struct K7Ctx {
  HbCtx c;
  const u32* keys;
  const u32* evs;
  u32 R0;               // global record index of the window's first record
  const uint4* sh_in;   // [n_keys][2] carried entries, or null (first window: nothing carried)
  uint4* sh_out;        // [n_keys][2] entries after this window, or null (last window)
  uint2* pool;          // read-vector pool: entries [0, *pool_cnt) carried, appended by this launch
  u32* pool_cnt;
  u32 pool_cap;
  uint4* races;         // (key, cur rec, prior rec, cur lane | prior lane << 5 | kind << 10)
  u32* race_cnt;
  u32 race_cap;
  u64* seg_cnt;         // [0] segments
  const u64* values;    // per-lane store values (row f3), nullable
  const u64* n_dev;
};

struct CheckArgs {
  const K7Ctx* k;       // device copy
  HbCtx c;              // by value: the inline fast path reads kernel parameters
  const u32* keys;
  const u32* evs;
  const u64* n_dev;
  u32 R0;
  const uint4* sh_in;
  uint4* sh_out;
  u32 no_sv;
  const u64* values;
};

__device__ __forceinline__ Carry load_carry(const uint4* sh, u32 key) {
  Carry k = no_carry();
  if (sh) {
    const uint4 e0 = __ldg(sh + 2 * (u64)key), e1 = __ldg(sh + 2 * (u64)key + 1);
    k.wr = e0.x;
    k.wwl = e0.y;
    k.wf = e0.z;
    k.rm = e0.w;
    k.rr = e1.x;
    k.rwl = e1.y;
  }
  return k;
}

__device__ __forceinline__ void emit(const K7Ctx* k, u32 key, u32 rc, u32 lc, u32 rp, u32 lp, u32 kind) {
  const u32 at = atomicAdd(k->race_cnt, 1u);
  if (at < k->race_cap) k->races[at] = make_uint4(key, rc, rp, lc | (lp << 5) | (kind << 10));
}

// slow path of the happens-before query: divergent intra-warp walk and foreign knowledge
static __device__ __noinline__ bool hb_slow(const K7Ctx* k, u32 r1, u32 l1, u32 w1, u32 r2, u32 l2, u32 s2w,
                                           u32 s2ps, u32 s2node, u32 s2blab) {
  const Snap s2{s2w, s2ps, s2node, s2blab};
  return hb(k->c, r1, l1, w1, r2, l2, s2);
}

// Does the access of (record r1, lane l1, warp w1) happen before (record r2, lane l2) whose record
// snapshot is s2?  Global record indices, r1 <= r2.  Branch-free up to the rare slow case (divergent
// intra-warp walk or foreign knowledge): lane-sequential K7 lanes sit at different items, so every
// branch of the query would be executed by the whole warp.
__device__ __forceinline__ bool hbq(const K7Ctx* k, const HbCtx& c, u32 r1, u32 l1, u32 w1, u32 r2, u32 l2,
                                    const Snap& s2) {
  const bool samel = l1 == l2;
  const bool samew = w1 == s2.warp;
  const bool conv = s2.node == s2.warp;
  const bool ord = (samew && (samel || (conv && s2.ps > r1))) ||
                   (blk_of(c.g, w1) == blk_of(c.g, s2.warp) && s2.blab > r1);  // program order / endi / barrier
  if (r1 == r2) return samel;  // lanes of one instruction are concurrent
  if (ord) return true;
  if (c.n_acq == 0 && !(samew && !conv)) return false;
  return hb_slow(k, r1, l1, w1, r2, l2, s2.warp, s2.ps, s2.node, s2.blab);
}

__device__ __forceinline__ u32 item_warp(const K7Ctx* k, u32 ev) { return __ldg(&k->c.snap[k->R0 + (ev >> 5)].x); }
// warp of a carried access (global record index)
__device__ __forceinline__ u32 rec_warp(const HbCtx& c, u32 rec) { return __ldg(&c.snap[rec].x); }

// first item of item i's granule in the window (keys sorted): lower bound of its key
static __device__ __noinline__ u64 seg_start(const K7Ctx* k, u64 i) {
  const u32 key = __ldg(k->keys + i) >> 2;
  u64 lo = 0, hi = i;
  while (lo < hi) {
    const u64 m = (lo + hi) >> 1;
    if ((__ldg(k->keys + m) >> 2) < key) lo = m + 1; else hi = m;
  }
  return lo;
}

// R_x is a read vector at the writer (r2, l2, s2): its entries are the latest read per thread among the
// in-window items [lo, hi] (all reads of this granule; lo > hi: none) and, when cm != SH_R_NONE, the
// carried read state (epoch (crr, crwl) or vector pool[crr, crr + crwl)), which lies before them.
// Check each (Fig. 2 WRITESHARED, Fig. 3 *ATOMSHARED); one race per unordered entry.
static __device__ __noinline__ void vc_check(const K7Ctx* k, u64 lo, u64 hi, u32 r2, u32 l2, u32 s2w, u32 s2ps,
                                             u32 s2node, u32 s2blab, u32 key, u32 kind, u32 cm, u32 crr,
                                             u32 crwl) {
  const Snap s2{s2w, s2ps, s2node, s2blab};
  const HbCtx& c = k->c;
  u32 seen[32];
  int ns = 0;
  auto dup_of = [&](u32 tid, u64 j_in, u32 q_car) -> bool {
    for (int q = 0; q < ns; ++q)
      if (seen[q] == tid) return true;
    if (ns < 32) return false;
    // overflow of the small set: look for a later read of the same thread directly
    for (u64 q = j_in; q <= hi && q >= lo && lo <= hi; ++q) {
      const u32 e2 = __ldg(k->evs + q);
      if (((item_warp(k, e2) << 5) | (e2 & 31u)) == tid) return true;
    }
    if (cm == SH_R_VC)
      for (u32 q = q_car; q < crwl; ++q)
        if (k->pool[crr + q].y == tid) return true;
    return false;
  };
  if (lo <= hi) {
    for (u64 j = hi + 1; j-- > lo;) {
      const u32 ev = __ldg(k->evs + j);
      const u32 r1 = k->R0 + (ev >> 5), l1 = ev & 31u, w1 = item_warp(k, ev);
      const u32 tid = (w1 << 5) | l1;
      if (dup_of(tid, j + 1, crwl)) continue;
      if (ns < 32) seen[ns++] = tid;
      if (!hb(c, r1, l1, w1, r2, l2, s2)) emit(k, key, r2, l2, r1, l1, kind);
    }
  }
  const u32 nc = cm == SH_R_VC ? crwl : (cm == SH_R_EPOCH ? 1u : 0u);
  for (u32 q = nc; q-- > 0;) {
    const uint2 e = cm == SH_R_VC ? k->pool[crr + q] : make_uint2(crr, (rec_warp(c, crr) << 5) | crwl);
    const u32 tid = e.y;
    if (dup_of(tid, lo, q + 1)) continue;
    if (ns < 32) seen[ns++] = tid;
    if (!hb(c, e.x, tid & 31u, tid >> 5, r2, l2, s2)) emit(k, key, r2, l2, e.x, tid & 31u, kind);
  }
}

// Shadow entry of a granule after the window: writer (wr, wwl, wf); read state: none, the epoch of
// in-window item `hi`, or a read vector = the carried read state (when cm != SH_R_NONE) followed by the
// in-window reads [lo, hi], in trace order (appended to the pool; readers keep the latest per thread).
static __device__ __noinline__ void put_state(const K7Ctx* k, u32 key, u32 wr, u32 wwl, u32 wf, u32 mode, u64 lo,
                                              u64 hi, u32 cm, u32 crr, u32 crwl) {
  uint4 e0 = make_uint4(wr, wwl, wf, mode), e1 = make_uint4(0, 0, key, 0);
  if (mode == SH_R_EPOCH) {
    const u32 ev = __ldg(k->evs + hi);
    e1.x = k->R0 + (ev >> 5);
    e1.y = ev & 31u;
  } else if (mode == SH_R_VC) {
    const u32 nc = cm == SH_R_VC ? crwl : (cm == SH_R_EPOCH ? 1u : 0u);
    const u32 m = nc + (u32)(hi + 1 - lo);
    const u32 off = atomicAdd(k->pool_cnt, m);
    if ((u64)off + m > k->pool_cap) {
      set_err(k->c.err, ERR_OVERFLOW);  // cannot happen: the host sizes the pool for the worst case
      return;
    }
    for (u32 q = 0; q < nc; ++q)
      k->pool[off + q] = cm == SH_R_VC ? k->pool[crr + q] : make_uint2(crr, (rec_warp(k->c, crr) << 5) | crwl);
    for (u64 j = lo; j <= hi; ++j) {
      const u32 ev = __ldg(k->evs + j);
      k->pool[off + nc + (u32)(j - lo)] = make_uint2(k->R0 + (ev >> 5), (item_warp(k, ev) << 5) | (ev & 31u));
    }
    e1.x = off;
    e1.y = m;
  }
  k->sh_out[2 * (u64)key] = e0;
  k->sh_out[2 * (u64)key + 1] = e1;
}

// intra-warp same-value filter: two stores of one record; with per-lane values
// (reading R6b) they must store the same value, else the record's SAME_VALUE flag decides
// (the item op is IOP_ST_SV).  ev: window-local events.
__device__ __forceinline__ bool same_value(const CheckArgs& a, u32 ev_prior, u32 ev_cur) {
  return (ev_prior >> 5) == (ev_cur >> 5) &&
         (!a.values || a.values[((u64)a.R0 << 5) + ev_prior] == a.values[((u64)a.R0 << 5) + ev_cur]);
}

__device__ __forceinline__ u32 hibit(u32 m) { return 31u - __clz(m); }  // m != 0

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

// warp range of the persistent K7 grid (K7a and K7b use the same partition)
__device__ __forceinline__ void warp_range(u64 n, u32 w, u32 nw, u64& beg, u64& end) {
  const u64 nr = (n + 31) / 32;
  beg = (nr * w / nw) * 32;
  end = min(n, (nr * (w + 1) / nw) * 32);
  if (beg > end) beg = end;
}

// Carried inflation of a read run that starts at the granule's first item s of the window (a read):
// the carried read state is a vector, or an epoch the read at s does not know (READINFLATE).
__device__ __forceinline__ bool carried_infl(const K7Ctx* k, const Carry& C, u32 ev_s, const Snap& s_s) {
  if (C.rm == SH_R_VC) return true;
  if (C.rm != SH_R_EPOCH) return false;
  return !hbq(k, k->c, C.rr, C.rwl, rec_warp(k->c, C.rr), k->R0 + (ev_s >> 5), ev_s & 31u, s_s);
}

// ---------------------------------------------------------------------- tail summary of an item range
// Summary (Sum) of the items [beg, end): the tail granule run's last writer and first inflation after
// it, found by walking back from the end (usually a few items: a writer or the granule's start ends
// the walk; never past beg).  Warp-cooperative; uniform result.
__device__ Sum tail_sum(const K7Ctx* kc, u64 beg, u64 end) {
  const int lane = threadIdx.x & 31;
  const HbCtx& c = kc->c;
  const u32* const keys = kc->keys;
  const u32* const evs = kc->evs;
  const u32 R0 = kc->R0;
  Sum s = sum_ident();
  if (beg >= end) return s;
  const u32 k0 = __ldg(keys + end - 1) >> 2;
  s.fk = __ldg(keys + beg) >> 2;
  s.lk = k0;
  u32 bits = s.fk == k0 ? SB_ONE : 0u, lw = 0, fi = NONE;
  u64 hi = end - 1;
  for (;;) {
    const u64 lo = hi >= beg + 31 ? hi - 31 : beg;
    const u64 i = lo + lane;
    const bool in = i <= hi;
    const u32 kx = in ? __ldg(keys + i) : NONE, ev = in ? __ldg(evs + i) : 0u;
    const bool inkey = in && (kx >> 2) == k0;
    const u32 W = __ballot_sync(0xFFFFFFFFu, inkey && (kx & 3u) != IOP_LD);
    const u32 B = __ballot_sync(0xFFFFFFFFu, in && !inkey);  // other granules (below: keys sorted)
    const int hw = W ? (int)hibit(W) : -1, hbk = B ? (int)hibit(B) : -1;
    const int bnd = hw > hbk ? hw : hbk;  // the read run is (bnd, top]
    u32 qkx = __shfl_up_sync(0xFFFFFFFFu, kx, 1), qev = __shfl_up_sync(0xFFFFFFFFu, ev, 1);
    if (lane == 0) {
      qkx = lo > 0 ? __ldg(keys + lo - 1) : NONE;
      qev = lo > 0 ? __ldg(evs + lo - 1) : 0u;
    }
    const bool inrun = in && lane > bnd;
    bool e = false;
    if (inrun && qkx != NONE && (qkx >> 2) == k0 && (qkx & 3u) == IOP_LD) {
      const Snap s2 = load_snap(c.snap, R0 + (ev >> 5));
      const u32 qw = __ldg(&c.snap[R0 + (qev >> 5)].x);
      e = !hbq(kc, c, R0 + (qev >> 5), qev & 31u, qw, R0 + (ev >> 5), ev & 31u, s2);
    }
    const u32 I = __ballot_sync(0xFFFFFFFFu, e);
    if (I) fi = (u32)(lo + __ffs(I) - 1);  // earlier rounds hold later items
    bool seg_at = false;                   // the run starts at its granule's first item s
    u64 sidx = 0;
    bool done = false;
    if (bnd >= 0) {
      if (hw >= 0 && hw > hbk) {
        lw = (u32)(lo + hw) + 1u;
        bits |= SB_W;
      } else {
        seg_at = true;
        sidx = lo + hbk + 1;
      }
      done = true;
    } else if (lo == beg) {
      seg_at = beg == 0 || (__ldg(keys + beg - 1) >> 2) != k0;
      sidx = beg;
      done = true;
    }
    if (done) {
      if (seg_at && kc->sh_in) {
        const Carry C = load_carry(kc->sh_in, k0);
        const u32 evs_ = __ldg(evs + sidx);
        if (carried_infl(kc, C, evs_, load_snap(c.snap, R0 + (evs_ >> 5)))) bits |= SB_CI;
      }
      break;
    }
    hi = lo - 1;
  }
  s.lw = lw;
  s.fi = fi;
  s.bits = bits;
  return s;
}

#ifndef KT_IPL_
#define KT_IPL_ 8  // A/B (K7b on C2 / C3 / C4): 16 -> 8 took 699 / 375 / 53 us to 369 / 223 / 25 us
#endif
constexpr int KT_IPL = KT_IPL_;              // items per lane per block
constexpr int KT_BLK = 32 * KT_IPL;          // items per warp block
constexpr int KT_PITCH = 32 * (KT_IPL + 1);  // padded entries per array
#ifndef KT_NWARPS
#define KT_NWARPS 12  // A/B (K7b, C2 / C3 / C4): 16 -> 12 took 376 / 231 / 25.6 us to 332 / 219 / 24.2 us
#endif
constexpr int KT_WARPS = KT_NWARPS;
constexpr size_t KT_WARP_BYTES = (size_t)KT_PITCH * (sizeof(uint4) + 2 * sizeof(u32));

// Partition of a window's items among K7a's persistent CTAs, from the device-side item count (the host
// knows only the window's upper bound, which can be far larger: C4's never-written pages drop 38 % of
// the slots): CTA c owns the blocks [c * G, (c + 1) * G), G a multiple of 64 (whole K7a chunks, and
// whole 8-block chunks), nct <= K7A_CTAS CTAs with blocks.
#ifndef KA_MINB
#define KA_MINB 4  // K7a CTAs per SM
#endif
constexpr u32 K7A_CTAS = 148 * KA_MINB;
struct K7Part {
  u32 nblk, G, nct;
};
__device__ __forceinline__ K7Part k7_part(u64 n) {
  K7Part p;
  p.nblk = (u32)((n + KT_BLK - 1) / KT_BLK);
  u32 G = (p.nblk + K7A_CTAS - 1) / K7A_CTAS;
  p.G = G < 64u ? 64u : (G + 63u) & ~63u;
  p.nct = (p.nblk + p.G - 1) / p.G;
  return p;
}

// ---------------------------------------------------------------------- state entering a block
// The automaton state entering block b = the exclusive prefix of the block summaries, of which only
// the tail matters (the last granule's last writer, first inflation, carried inflation).  A summary
// whose tail granule starts inside its block, or that holds a writer, fixes that tail whatever lies
// before it (see combine), so the walk back over the summaries stops there: usually at block b - 1,
// a run of one read-only granule over many blocks takes one step per 32 blocks.  Warp-cooperative.
__device__ Sum enter_state(const Sum* __restrict__ sums, u32 b) {
  const u32 lane = threadIdx.x & 31;
  Sum acc = sum_ident();
  u32 j = b;
  while (j > 0) {
    const u32 lo = j >= 32 ? j - 32 : 0;
    const u32 i = lo + lane;
    Sum incl = i < j ? sums[i] : sum_ident();  // identities after the range keep the order
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const Sum up = shfl_up_sum(incl, o);
      if ((int)lane >= o) incl = combine(up, incl);
    }
    acc = combine(shfl_sum(incl, 31), acc);
    j = lo;
    if (acc.fk != NONE && (!(acc.bits & SB_ONE) || (acc.bits & SB_W))) break;
  }
  return acc;
}

// ---------------------------------------------------------------------------------------
// K7b: lane-sequential check with shared-memory staged clocks.  Persistent warp ranges (state
// entering each from enter_state); each listed block of 32 * KT_IPL items is processed as:
//   load    : the block's (key, ev) words land in shared memory by cp.async
//             (row pitch KT_IPL+1 words: lane l reading item l*KT_IPL+j is bank-conflict free)
//   gather  : lane l walks ITS KT_IPL consecutive items; for each item some query can read it issues
//             a 16-B cp.async of the record snapshot into shared memory
//   summary : lane l walks its items: READINFLATE flags (Fig. 2) and the chunk summary Sum; at a
//             granule's first item the carried shadow entry decides the carried inflation
//   scan    : a 5-step warp scan of the summaries gives every lane the automaton state (LW, FI)
//             entering its chunk, and the block carry
//   rules   : lane l replays the rules of Fig. 2 / Fig. 3 over its chunk from that state (W check, R
//             check against the epoch or the read vector, same-value filter), with the carried
//             entry as the state before a granule's first item; at a granule's last item it writes
//             the granule's entry for the next window

__device__ __forceinline__ u32 tpad(u32 i) { return i + i / KT_IPL; }

__device__ __forceinline__ void cp_async4(void* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait0() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

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

// ---------------------------------------------------------------------- K7a: block summaries
// Persistent CTAs, CTA c owning the contiguous blocks [c * G, (c + 1) * G) of KT_BLK sorted items.
// Phase 1, one warp per block (the next block's key words prefetched while this one is summarised):
// from the key words alone (vector loads) it counts the granules starting in the block and decides
// whether any item makes a check -- with one window and nothing carried, an item alone in its granule
// or an atomic between atomics (its W check is elided, and no read follows it) checks
// nothing.  Such a block only advances the automaton state: its summary comes from the keys.  Any other
// block is summarised by a bounded tail walk (never past the block start) and listed for K7b, which
// finds the state entering it by walking back over the summaries (enter_state).
constexpr int KT_SWARPS = 8;
__device__ __forceinline__ void load_keys16(const u32* __restrict__ keys, u64 bb, u32 nb, u32 l0, u32 (&kr)[KT_IPL]) {
  const u32 cntf = l0 < nb ? min((u32)KT_IPL, nb - l0) : 0u;
  if (cntf == (u32)KT_IPL) {
    const uint4* kv = reinterpret_cast<const uint4*>(keys + bb + l0);  // 64-B aligned: bb, l0 are x16
#pragma unroll
    for (int q = 0; q < KT_IPL / 4; ++q) {
      const uint4 v = __ldg(kv + q);
      kr[4 * q] = v.x;
      kr[4 * q + 1] = v.y;
      kr[4 * q + 2] = v.z;
      kr[4 * q + 3] = v.w;
    }
  } else {
#pragma unroll
    for (int j = 0; j < KT_IPL; ++j) kr[j] = (u32)j < cntf ? __ldg(keys + bb + l0 + j) : NONE;
  }
}

static __device__ __noinline__ Sum tail_sum_nl(const K7Ctx* k, u64 beg, u64 end) { return tail_sum(k, beg, end); }

// A block with no bad pair (see k_blk_sum) in a run of several windows.  Its granule-first items are
// checked against the carried entries: the block stays trivial iff no entry holds a read state and no
// entry holds a writer the item's W check would see (only an atomic after an atomic is elided,
// P:L661-670) -- then no item makes a check at all.  A trivial block then writes the entry of each of
// its granule-last items for the next window: a writer (ST / ATOM) is the new W with no read state; a
// read is alone in its granule in the window (no bad pair), found no carried writer or read state, so
// its entry is no writer and the read's epoch (Fig. 8).  sk: the block's key words in
// shared memory (sk[-1]: the item before, sk[nb]: the item after).  Warp-uniform result.
static __device__ __forceinline__ bool sh_block(const CheckArgs& a, const u32* sk, u64 bb, u32 nb, u64 n, u32 lane) {
  const u32 kb = bb > 0 ? sk[-1] : NONE, ka = bb + nb < n ? sk[nb] : NONE;
  if (a.sh_in) {
    bool need = false;
#pragma unroll
    for (int q = 0; q < KT_BLK / 128; ++q) {
#pragma unroll
      for (int t = 0; t < 4; ++t) {
        const u32 i = (u32)q * 128u + lane * 4u + (u32)t;
        if (i < nb) {
          const u32 k = sk[i], kp = i ? sk[i - 1] : kb;
          if (kp == NONE || (kp >> 2) != (k >> 2)) {
            const uint4 e0 = __ldg(a.sh_in + 2 * (u64)(k >> 2));
            need |= e0.w != SH_R_NONE || ((e0.z & SH_W_VALID) && !((k & 3u) == IOP_ATOM && (e0.z & SH_W_ATOM)));
          }
        }
      }
    }
    if (__any_sync(0xFFFFFFFFu, need)) return false;
  }
  if (a.sh_out) {
#pragma unroll
    for (int q = 0; q < KT_BLK / 128; ++q) {
      const u32 i0 = (u32)q * 128u + lane * 4u;
      u32 ev[4];
      if (i0 + 4 <= nb) {
        const uint4 v = __ldg(reinterpret_cast<const uint4*>(a.evs + bb + i0));
        ev[0] = v.x; ev[1] = v.y; ev[2] = v.z; ev[3] = v.w;
      } else {
#pragma unroll
        for (int t = 0; t < 4; ++t) ev[t] = i0 + t < nb ? __ldg(a.evs + bb + i0 + t) : 0u;
      }
#pragma unroll
      for (int t = 0; t < 4; ++t) {
        const u32 i = i0 + (u32)t;
        if (i < nb) {
          const u32 k = sk[i], kn = i + 1 < nb ? sk[i + 1] : ka;
          if (kn == NONE || (kn >> 2) != (k >> 2)) {
            const u32 op = k & 3u, rec = a.R0 + (ev[t] >> 5), ln = ev[t] & 31u;
            uint4* const o = a.sh_out + 2 * (u64)(k >> 2);
            if (op != IOP_LD) {
              o[0] = make_uint4(rec, ln, SH_W_VALID | (op == IOP_ATOM ? SH_W_ATOM : 0u), SH_R_NONE);
              o[1] = make_uint4(0u, 0u, k >> 2, 0u);
            } else {
              o[0] = make_uint4(0u, 0u, 0u, SH_R_EPOCH);
              o[1] = make_uint4(rec, ln, k >> 2, 0u);
            }
          }
        }
      }
    }
  }
  return true;
}

// key words stream through shared memory: one chunk = KT_SWARPS warp tiles of KA_TILE items, each
// KA_BPT blocks (+ 4 words on each side for
// the neighbours of the first / last item), KB_STAGES chunks in flight per CTA (1-D TMA bulk copies)
#ifndef KB_STAGES_
#define KB_STAGES_ 2
#endif
constexpr int KB_STAGES = KB_STAGES_;
#ifndef KA_UNROLL
#define KA_UNROLL 2  // the tile's blocks interleaved (A/B on C4: 159 -> 150 us)
#endif
constexpr int KA_UNR = KA_UNROLL;
constexpr int KA_TILE = 512;
constexpr u32 KA_MAXG = 8192;  // blocks per K7a CTA: a window holds < 2^30 items, so G <= 7104                     // items per K7a warp per chunk (independent of the block size:
constexpr int KA_BPT = KA_TILE / KT_BLK;         //  K7b's blocks are shorter, K7a's tiles stay long)
static_assert(KA_TILE % KT_BLK == 0 && KT_BLK % 128 == 0, "K7a tiles hold whole blocks of whole 128-item rounds");
constexpr int KB_CHUNK = KT_SWARPS * KA_TILE;    // items per chunk
constexpr int KB_ROW = KB_CHUNK + 8;             // words per stage
constexpr size_t KB_SMEM = (size_t)KB_STAGES * KB_ROW * sizeof(u32);
__global__ void __launch_bounds__(KT_SWARPS * 32, KA_MINB) k_blk_sum(CheckArgs a, Sum* __restrict__ sums,
                                                            u32* __restrict__ wl, u32* __restrict__ wl_cnt) {
  extern __shared__ __align__(128) u32 kb_smem[];  // [KB_STAGES][KB_ROW] key words
  u32 (*const s_keys)[KB_ROW] = reinterpret_cast<u32 (*)[KB_ROW]>(kb_smem);
  __shared__ u64 s_bar[KB_STAGES];
  __shared__ u32 s_nt[KA_MAXG / 32];  // the CTA's blocks with a check (bitmap)
  const u32 wi = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const u64 n = *a.n_dev;
  const K7Part P = k7_part(n);
  const u32 nblk = P.nblk, G = P.G;
  if (blockIdx.x >= P.nct) return;  // CTA-uniform
  const bool fast_ok = a.sh_in == nullptr && a.sh_out == nullptr;
  const u32 b0 = blockIdx.x * G, b1 = min(nblk, b0 + G);
  const u32 l0 = lane * KT_IPL;
  const u64 i0 = (u64)b0 * KT_BLK, i1 = min(n, (u64)b1 * KT_BLK);  // the CTA's items
  const u32 n_chunks = i1 > i0 ? (u32)((i1 - i0 + KB_CHUNK - 1) / KB_CHUNK) : 0u;
  // chunk c covers items [i0 + c * KB_CHUNK, ...); the stage holds words from item (c0 - 4) at index 0
  auto issue = [&](u32 c, int st) {
    const u64 c0 = i0 + (u64)c * KB_CHUNK;
    const u64 lo = c0 >= 4 ? c0 - 4 : 0;                  // 16-B aligned: c0 is a multiple of 512
    const u64 hi = min(n, c0 + KB_CHUNK + 4);
    const u32 bytes = (u32)(((hi - lo) + 3) & ~3ull) * 4u;  // whole 16-B units (buffers are padded)
    mbar_expect_tx(&s_bar[st], bytes);
    bulk_g2s(&s_keys[st][c0 >= 4 ? 0 : 4], a.keys + lo, bytes, &s_bar[st]);
  };
  if (threadIdx.x == 0) {
    for (int q = 0; q < KB_STAGES; ++q) mbar_init(&s_bar[q], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  for (u32 q = threadIdx.x; q < KA_MAXG / 32; q += KT_SWARPS * 32) s_nt[q] = 0;
  __syncthreads();
  if (threadIdx.x == 0)
    for (int q = 0; q < KB_STAGES; ++q)
      if ((u32)q < n_chunks) issue(q, q);
  for (u32 c = 0; c < n_chunks; ++c) {
    const int st = (int)(c % KB_STAGES);
    mbar_wait(&s_bar[st], (c / KB_STAGES) & 1u);
    const u64 c0 = i0 + (u64)c * KB_CHUNK;
    const u32* sk = &s_keys[st][4];  // sk[j] = key word of item c0 + j (sk[-1]: the item before)
#pragma unroll (KA_UNR)
    for (int sb = 0; sb < KA_BPT; ++sb) {  // the warp's tile: KA_BPT consecutive blocks
    const u32 blk = b0 + (c * KT_SWARPS + wi) * KA_BPT + sb;
    const u64 bb = (u64)blk * KT_BLK;
    const u32 nb = (blk < b1 && bb < n) ? (u32)(n - bb < (u64)KT_BLK ? n - bb : (u64)KT_BLK) : 0u;
    Sum bs = sum_ident();
    if (nb) {
      const u32 off = (wi * KA_BPT + sb) * KT_BLK;  // the block's first item in the chunk
      // KT_BLK / 128 rounds of 128 items; in round q lane l holds items 128 q + 4 l .. + 3 (one conflict-free
      // 16-B shared-memory read); neighbours across lanes / rounds by shuffles and broadcast reads
      const u32 lkw = sk[off + nb - 1];                           // the block's last item
      const u32 fkw = sk[off];
      u32 pk_round = bb > 0 ? sk[(int)off - 1] : NONE;            // item before the round
      // A block makes no check iff no two neighbouring items (including the items just before and
      // after it) share a granule unless both are atomics.  Absent items are NONE: granule 0x3FFFFFFF
      // (never a real key, keys < 2^30 - 1) with the atomic op bits, so they never form a bad pair.
      u32 bad = 0;
      const bool full = nb == (u32)KT_BLK;
#pragma unroll
      for (int q = 0; q < KT_BLK / 128; ++q) {
        const u32 base = (u32)q * 128u + lane * 4u;  // item index within the block
        const uint4 v = *reinterpret_cast<const uint4*>(sk + off + base);
        u32 kk[4] = {v.x, v.y, v.z, v.w};
        if (!full) {
#pragma unroll
          for (int t = 0; t < 4; ++t) kk[t] = base + (u32)t < nb ? kk[t] : NONE;
        }
        u32 kprev = __shfl_up_sync(0xFFFFFFFFu, kk[3], 1);
        kprev = lane == 0 ? pk_round : kprev;
        u32 knext = __shfl_down_sync(0xFFFFFFFFu, kk[0], 1);
        {  // lane 31: the next round's first item, or the item after the block (a broadcast read)
          const u32 nx = (u32)q * 128u + 128u;
          const u32 k31 = sk[off + (nx < nb ? nx : nb)];
          const u32 kn31 = (nx < nb || bb + nb < n) ? k31 : NONE;
          knext = lane == 31 ? kn31 : knext;
        }
        pk_round = __shfl_sync(0xFFFFFFFFu, kk[3], 31);
        u32 kpv = kprev;
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          const u32 k = kk[t];
          bad |= ((k ^ kpv) < 4u) & ((k & kpv & 3u) != 3u);
          kpv = k;
        }
        bad |= ((kk[3] ^ knext) < 4u) & ((kk[3] & knext & 3u) != 3u);
      }
      bool triv = __all_sync(0xFFFFFFFFu, bad == 0u);
      // several windows: the carried entries decide too, and a trivial block writes its granules'
      // entries for the next window here instead of in K7b
      if (!fast_ok && triv) triv = sh_block(a, sk + off, bb, nb, n, lane);
      if (triv) {
        // no read has a same-granule read before it (no READINFLATE flags), so the summary is closed-form:
        // first and last granule, and the last writer of the last granule.  Keys are sorted, so the last
        // granule's items are the block's tail run, and in a block without bad pairs that run is a single
        // item or a run of atomics: its last writer is the block's last item unless that is a read (then
        // the run is that read alone and holds no writer).
        const u32 mlw = (lkw & 3u) != IOP_LD ? (u32)bb + nb : 0u;
        bs.fk = fkw >> 2;
        bs.lk = lkw >> 2;
        bs.lw = mlw;
        bs.fi = NONE;
        bs.bits = (bs.fk == bs.lk ? SB_ONE : 0u) | (mlw ? SB_W : 0u);
        if (lane == 0) sums[blk] = bs;
      } else if (lane == 0) {  // tail-walked after the stream (no call in the hot loop), listed for K7b
        atomicOr(&s_nt[(blk - b0) >> 5], 1u << ((blk - b0) & 31));
      }
    }
    }
    (void)c0;
    __syncthreads();  // every warp is done with stage st: refill it
    if (threadIdx.x == 0 && c + KB_STAGES < n_chunks) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      issue(c + KB_STAGES, st);
    }
  }
  // the blocks with a check: a bounded tail walk each (their words are L2-hot), then listed for K7b
  for (u32 wd = wi; wd < (b1 - b0 + 31) / 32; wd += KT_SWARPS) {
    u32 m = s_nt[wd];
    while (m) {
      const u32 blk = b0 + wd * 32 + (u32)(__ffs(m) - 1);
      m &= m - 1;
      const u64 bb = (u64)blk * KT_BLK;
      const u32 nb = (u32)(n - bb < (u64)KT_BLK ? n - bb : (u64)KT_BLK);
      const Sum bs = tail_sum_nl(a.k, bb, bb + nb);
      if (lane == 0) {
        sums[blk] = bs;
        wl[atomicAdd(wl_cnt, 1u)] = blk;
      }
    }
  }
}

// ---------------------------------------------------------------------- K7b: the listed blocks
// SH (several windows: carried entries in and / or entries out): 8 warps per CTA, and per warp
// the carried entries of the block's granule-first items staged in shared memory with the snapshots
// (cp.async, all of a lane's loads in flight together), so the lane-sequential rules never wait on a
// dependent global load per granule.
template <bool SH>
struct KtCfg {
  static constexpr int WARPS = SH ? 8 : KT_WARPS;
  static constexpr size_t WARP_BYTES =
      KT_WARP_BYTES + (SH ? (size_t)KT_PITCH * (sizeof(uint4) + sizeof(uint2)) : 0);
};

__device__ __forceinline__ void cp_async8(void* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}

__device__ __forceinline__ Carry carry_of(const uint4& e0, const uint2& e1) {
  return Carry{e0.x, e0.y, e0.z, e0.w, e1.x, e1.y};
}

template <bool SH>
__global__ void __launch_bounds__(KtCfg<SH>::WARPS * 32, 1) k_check_tile(CheckArgs a, const u32* __restrict__ wl,
                                                                         const u32* __restrict__ wl_cnt,
                                                                         const Sum* __restrict__ sums, u32 nblk) {
  constexpr int NWARP = KtCfg<SH>::WARPS;
  extern __shared__ __align__(16) unsigned char kt_smem[];
  const int wi = threadIdx.x >> 5;
  uint4* sS = reinterpret_cast<uint4*>(kt_smem + (size_t)wi * KtCfg<SH>::WARP_BYTES);
  u32* const sK = reinterpret_cast<u32*>(sS + KT_PITCH);
  u32* const sE = sK + KT_PITCH;
  uint4* const sC0 = reinterpret_cast<uint4*>(sE + KT_PITCH);  // SH: carried e0 of granule-first items
  uint2* const sC1 = reinterpret_cast<uint2*>(sC0 + KT_PITCH);  // SH: carried (e1.x, e1.y)
  const u64 n = *a.n_dev;
  const u32 w = blockIdx.x * NWARP + wi, nw = gridDim.x * NWARP;
  const u32 lane = threadIdx.x & 31;
  const HbCtx& c = a.c;
  const K7Ctx* const kx = a.k;
  const u32 R0 = a.R0;
  const bool shadow = a.sh_in != nullptr;
  const u32 n_tasks = *wl_cnt;
  u32 segs = 0;
  const u32 l0 = lane * KT_IPL;
  for (u32 task = w; task < n_tasks; task += nw) {
    // a listed block (the loop below also serves runs of blocks carrying the state through)
    const u32 blk0 = wl[task], blk1 = min(nblk, blk0 + 1);
    Sum carry = enter_state(sums, blk0);
    u32 pkx = blk0 > 0 ? __ldg(a.keys + (u64)blk0 * KT_BLK - 1) : NONE;  // the item before the block
    for (u32 bi = blk0; bi < blk1; ++bi) {
    const u64 bb = (u64)bi * KT_BLK;
    if (bb >= n) break;
    const u32 nb = (u32)(n - bb < (u64)KT_BLK ? n - bb : (u64)KT_BLK);
    const u32 knext = bb + nb < n ? __ldg(a.keys + bb + nb) : NONE;  // first item after the block
    kt_stage(a, bb, nb, sK, sE, lane);
    cp_async_wait0();
    __syncwarp();

    const u32 cnt = l0 < nb ? min((u32)KT_IPL, nb - l0) : 0u;
    const u32 ppk = lane == 0 ? pkx : sK[tpad(l0 - 1)];
    const u32 ppe = lane == 0 ? (bb > 0 ? __ldg(a.evs + bb - 1) : 0u) : sE[tpad(l0 - 1)];
    const u32 gbb = (u32)bb;

    // ---- gather the snapshots some query can read: an item with a same-granule neighbour (unless an
    // atomic among atomics: its W check is elided and no read follows it), and with carried
    // state every granule's first item (it checks against the carried entry)
    if (SH && shadow) {  // first the carried entries of the granule-first items (they decide which
                         // of those items make a check at all)
      u32 kp = ppk;
      for (u32 j = 0; j < cnt; ++j) {
        const u32 li = l0 + j;
        const u32 k = sK[tpad(li)];
        if (kp == NONE || (kp >> 2) != (k >> 2)) {
          cp_async16(sC0 + tpad(li), a.sh_in + 2 * (u64)(k >> 2));
          cp_async8(sC1 + tpad(li), a.sh_in + 2 * (u64)(k >> 2) + 1);
        }
        kp = k;
      }
      cp_async_commit();
      cp_async_wait0();
      __syncwarp();
    }
    {
      u32 kp = ppk, k = cnt ? sK[tpad(l0)] : NONE;
      for (u32 j = 0; j < cnt; ++j) {
        const u32 li = l0 + j;
        const u32 kn = li + 1 < nb ? sK[tpad(li + 1)] : knext;
        const u32 key = k >> 2;
        const bool sp = kp != NONE && (kp >> 2) == key, sn = kn != NONE && (kn >> 2) == key;
        const bool atm_only =
            (k & 3u) == IOP_ATOM && (!sp || (kp & 3u) == IOP_ATOM) && (!sn || (kn & 3u) == IOP_ATOM);
        // a granule-first item checks against the carried entry iff it holds a read state, or a writer
        // the item's W check is not elided for (an atomic after an atomic)
        bool need = (sp || sn) && !atm_only;
        if (SH && shadow && !sp) {
          const uint4 e0 = sC0[tpad(li)];
          need |= e0.w != SH_R_NONE ||
                  ((e0.z & SH_W_VALID) && !((k & 3u) == IOP_ATOM && (e0.z & SH_W_ATOM)));
        }
        if (need) cp_async16(sS + tpad(li), c.snap + R0 + (sE[tpad(li)] >> 5));
        kp = k;
        k = kn;
      }
    }
    cp_async_commit();
    const u32 pw0 = (lane == 0 && ppk != NONE) ? __ldg(&c.snap[R0 + (ppe >> 5)].x) : 0u;
    cp_async_wait0();
    __syncwarp();

    // ---- READINFLATE flags and the chunk summary
    Sum sm = sum_ident();
    u32 imask = 0, cmask = 0;
    if (cnt) {
      u32 pk = ppk, pe = ppe, pw = lane ? sS[tpad(l0 - 1)].x : pw0, tlw = 0, tfi = NONE;
      bool kc = false, tci = false;
      sm.fk = sK[tpad(l0)] >> 2;
      for (u32 j = 0; j < cnt; ++j) {
        const u32 li = l0 + j;
        const u32 k = sK[tpad(li)], e = sE[tpad(li)];
        const uint4 sv = sS[tpad(li)];
        const u32 gi = gbb + li;
        const bool same = pk != NONE && (pk >> 2) == (k >> 2);
        if (!same) {
          kc |= j > 0;
          tlw = 0;
          tfi = NONE;
          tci = false;
          if (shadow && (k & 3u) == IOP_LD &&
              carried_infl(kx, SH ? carry_of(sC0[tpad(li)], sC1[tpad(li)]) : load_carry(a.sh_in, k >> 2), e,
                           to_snap(sv))) {
            tci = true;
            cmask |= 1u << j;
          }
        }
        if ((k & 3u) != IOP_LD) {
          tlw = gi + 1u;
          tfi = NONE;
          tci = false;
        } else if (same && (pk & 3u) == IOP_LD &&
                   !hbq(kx, c, R0 + (pe >> 5), pe & 31u, pw, R0 + (e >> 5), e & 31u, to_snap(sv))) {
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
      sm.bits = (kc ? 0u : SB_ONE) | (tlw ? SB_W : 0u) | (tci ? SB_CI : 0u);
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
      u32 lw = 0, fi = NONE;
      bool ci = false;
      if (in.fk != NONE) {
        lw = in.lw;
        fi = in.fi;
        ci = (in.bits & SB_CI) != 0;
      }
      u32 wk = 0, we = 0, ww = 0;  // in-window last writer: key word, event, warp
      if (lw) {
        if ((u64)(lw - 1) >= bb) {
          const u32 wl = (u32)(lw - 1 - bb);
          wk = sK[tpad(wl)];
          we = sE[tpad(wl)];
          ww = sS[tpad(wl)].x;  // gathered: the writer has a same-granule successor in the block
        } else {  // the last writer lies before the block
          wk = __ldg(a.keys + lw - 1);
          we = __ldg(a.evs + lw - 1);
          ww = __ldg(&c.snap[R0 + (we >> 5)].x);
        }
      }
      u32 pk = ppk, pe = ppe, pw = lane ? sS[tpad(l0 - 1)].x : pw0;
      Carry C = no_carry();
      if (shadow && pk != NONE && (pk >> 2) == (sK[tpad(l0)] >> 2) && lw == 0) C = load_carry(a.sh_in, pk >> 2);
      for (u32 j = 0; j < cnt; ++j) {
        const u32 li = l0 + j;
        const u32 k = sK[tpad(li)], e = sE[tpad(li)];
        const uint4 sv = sS[tpad(li)];
        const Snap s2 = to_snap(sv);
        const u32 op = k & 3u;
        const u32 gi = gbb + li;
        const u32 r2 = R0 + (e >> 5), l2 = e & 31u;
        const bool same = pk != NONE && (pk >> 2) == (k >> 2);
        if (!same) {
          lw = 0;
          fi = NONE;
          ci = (cmask >> j) & 1u;
          C = shadow ? (SH ? carry_of(sC0[tpad(li)], sC1[tpad(li)]) : load_carry(a.sh_in, k >> 2)) : no_carry();
        }
        if (op == IOP_LD && ((imask >> j) & 1u) && fi == NONE) fi = gi;
        // W_x check (every rule of Fig. 2; atomics only against a plain last write)
        if (lw) {
          const bool patm = (wk & 3u) == IOP_ATOM;
          if (!(op == IOP_ATOM && patm) && !hbq(kx, c, R0 + (we >> 5), we & 31u, ww, r2, l2, s2)) {
            const u32 kind = op == IOP_LD ? (patm ? BC_KIND_AR : BC_KIND_WR)
                                          : op == IOP_ATOM ? BC_KIND_WA : (patm ? BC_KIND_AW : BC_KIND_WW);
            const bool filtered = !patm && op == IOP_ST_SV && !a.no_sv && same_value(a, we, e);
            if (!filtered) emit(kx, k >> 2, r2, l2, R0 + (we >> 5), we & 31u, kind);
          }
        } else if (C.wf & SH_W_VALID) {  // the carried writer (an earlier window: never the same record)
          const bool patm = (C.wf & SH_W_ATOM) != 0;
          if (!(op == IOP_ATOM && patm) && !hbq(kx, c, C.wr, C.wwl, rec_warp(c, C.wr), r2, l2, s2)) {
            const u32 kind = op == IOP_LD ? (patm ? BC_KIND_AR : BC_KIND_WR)
                                          : op == IOP_ATOM ? BC_KIND_WA : (patm ? BC_KIND_AW : BC_KIND_WW);
            emit(kx, k >> 2, r2, l2, C.wr, C.wwl, kind);
          }
        }
        if (op != IOP_LD) {
          const u32 kind = op == IOP_ATOM ? BC_KIND_RA : BC_KIND_RW;
          if (same && (pk & 3u) == IOP_LD) {  // R_x check at a writer after in-window reads
            if (lw == 0 && ci) {
              // the carried read state and every in-window read of the granule so far
              vc_check(kx, seg_start(kx, gi), (u64)gi - 1, r2, l2, s2.warp, s2.ps, s2.node, s2.blab, k >> 2, kind,
                       C.rm, C.rr, C.rwl);
            } else if (fi == NONE) {
              if (!hbq(kx, c, R0 + (pe >> 5), pe & 31u, pw, r2, l2, s2)) emit(kx, k >> 2, r2, l2, R0 + (pe >> 5), pe & 31u, kind);
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
                  if (!dup && !hbq(kx, c, R0 + (ev1 >> 5), ev1 & 31u, w1, r2, l2, s2))
                    emit(kx, k >> 2, r2, l2, R0 + (ev1 >> 5), ev1 & 31u, kind);
                }
              } else {
                vc_check(kx, lo, (u64)gi - 1, r2, l2, s2.warp, s2.ps, s2.node, s2.blab, k >> 2, kind, SH_R_NONE,
                         0u, 0u);
              }
            }
          } else if (!same && C.rm != SH_R_NONE) {  // the granule's first item: the carried read state
            if (C.rm == SH_R_EPOCH) {
              if (!hbq(kx, c, C.rr, C.rwl, rec_warp(c, C.rr), r2, l2, s2)) emit(kx, k >> 2, r2, l2, C.rr, C.rwl, kind);
            } else {
              vc_check(kx, 1, 0, r2, l2, s2.warp, s2.ps, s2.node, s2.blab, k >> 2, kind, C.rm, C.rr, C.rwl);
            }
          }
          lw = gi + 1u;
          wk = k;
          we = e;
          ww = sv.x;
          fi = NONE;
          ci = false;
        }
        // ---- the granule's last item of the window: its shadow entry for the next window
        if (SH && a.sh_out) {
          const u32 kn = li + 1 < nb ? sK[tpad(li + 1)] : knext;
          if (kn == NONE || (kn >> 2) != (k >> 2)) {
            u32 wr = C.wr, wwl = C.wwl, wf = C.wf;
            if (lw) {
              wr = R0 + (we >> 5);
              wwl = we & 31u;
              wf = SH_W_VALID | ((wk & 3u) == IOP_ATOM ? SH_W_ATOM : 0u);
            }
            // no read state (a writer ends the window's run) or an epoch (the last read, gathered): two
            // stores inline; a read vector (pool append) out of line
            if (op != IOP_LD || (!(lw == 0 && ci) && fi == NONE)) {
              uint4* const o = a.sh_out + 2 * (u64)(k >> 2);
              const bool ep = op == IOP_LD;
              o[0] = make_uint4(wr, wwl, wf, ep ? SH_R_EPOCH : SH_R_NONE);
              o[1] = make_uint4(ep ? R0 + (e >> 5) : 0u, ep ? e & 31u : 0u, k >> 2, 0u);
            } else if (lw == 0 && ci) {
              put_state(kx, k >> 2, wr, wwl, wf, SH_R_VC, seg_start(kx, gi), gi, C.rm, C.rr, C.rwl);
            } else {
              put_state(kx, k >> 2, wr, wwl, wf, SH_R_VC, (u64)fi - 1, gi, SH_R_NONE, 0, 0);
            }
          }
        }
        pk = k;
        pe = e;
        pw = sv.x;
      }
    }

    carry = combine(carry, blk);
    pkx = sK[tpad(nb - 1)];
    __syncwarp();
    }
  }
  (void)segs;
}

// Statistics only (bc_config.flags & BC_F_COUNT_GATHERS): the number of items whose record clock
// snapshot K7 reads -- the gather rule over the sorted items -- for the roofline's algorithmic
// bytes.  A separate pass so that the hot kernel carries no counter.
__global__ void k_count_gathers(const u32* __restrict__ keys, const u64* __restrict__ n_dev, u64* __restrict__ out,
                                u64* __restrict__ segs) {
  const u64 n = *n_dev;
  u32 cnt = 0, sg = 0;
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x) {
    const u32 k = keys[i], kp = i ? keys[i - 1] : NONE, kn = i + 1 < n ? keys[i + 1] : NONE;
    const u32 key = k >> 2;
    const bool sp = kp != NONE && (kp >> 2) == key, sn = kn != NONE && (kn >> 2) == key;
    const bool atm_only = (k & 3u) == IOP_ATOM && (!sp || (kp & 3u) == IOP_ATOM) && (!sn || (kn & 3u) == IOP_ATOM);
    cnt += (sp || sn) && !atm_only;
    sg += !sp;  // the granule's first item of the window
  }
  cnt = __reduce_add_sync(0xFFFFFFFFu, cnt);
  sg = __reduce_add_sync(0xFFFFFFFFu, sg);
  if ((threadIdx.x & 31) == 0 && cnt) atomicAdd((unsigned long long*)out, (unsigned long long)cnt);
  if ((threadIdx.x & 31) == 0 && sg) atomicAdd((unsigned long long*)segs, (unsigned long long)sg);
}

// Shadow commit after a window: K7 read the carried entries from `tab` and wrote the entry of every
// granule the window touched into `out` (at the granule's last item), so `tab` could not be updated in
// place while K7 ran.  Now copy exactly the touched entries back: one per granule segment of the sorted
// items (its last item).  Untouched entries are already current in `tab`, so a window costs 4 B per item
// + 64 B per touched granule instead of a copy of the whole table (32 B x every granule key).
__global__ void k_shadow_commit(const u32* __restrict__ keys, const u64* __restrict__ n_dev,
                                const uint4* __restrict__ out, uint4* __restrict__ tab) {
  const u64 n = *n_dev;
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x) {
    const u32 k = __ldg(keys + i) >> 2;
    if (i + 1 < n && (__ldg(keys + i + 1) >> 2) == k) continue;
    const uint4 e0 = __ldg(out + 2 * (u64)k), e1 = __ldg(out + 2 * (u64)k + 1);
    tab[2 * (u64)k] = e0;
    tab[2 * (u64)k + 1] = e1;
  }
}

}  // namespace

void launch_shadow_commit(const u32* keys, const u64* n_dev, u64 n_max, const uint4* out, uint4* tab,
                          cudaStream_t st) {
  if (n_max == 0) return;
  const u64 want = (n_max + 255) / 256;
  k_shadow_commit<<<(unsigned)std::min<u64>(want, 148 * 16), 256, 0, st>>>(keys, n_dev, out, tab);
  ++g_launches;
}

void launch_count_gathers(const u32* keys, const u64* n_dev, u64* out, u64* segs, cudaStream_t st) {
  k_count_gathers<<<148 * 8, 256, 0, st>>>(keys, n_dev, out, segs);
  ++g_launches;
}

// per device: K7b grid (fully co-resident persistent CTAs) and its shared-memory opt-in
template <bool SH>
static int k7_grid(int dev) {
  static int grid[64] = {};
  if (dev < 0 || dev >= 64) dev = 0;
  if (!grid[dev]) {
    constexpr int NW = KtCfg<SH>::WARPS;
    const size_t smem_tile = (size_t)NW * KtCfg<SH>::WARP_BYTES;
    int sms = 0, per = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaFuncSetAttribute(k_check_tile<SH>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_tile);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_check_tile<SH>, NW * 32, smem_tile);
    if (per < 1) per = 1;
    int g = sms * per;
    if (g * NW > 148 * 64) g = 148 * 64 / NW;
    grid[dev] = g;
  }
  return grid[dev];
}

// status scratch: [K7Ctx][Sum sums[nblk]][u32 wl[nblk]][u32 wl_cnt]
size_t check_status_bytes(u64 n) {
  const u64 nblk = (n + KT_BLK - 1) / KT_BLK + 1;
  return 256 + ((sizeof(K7Ctx) + 255) & ~(size_t)255) + (nblk + 4) * sizeof(Sum) + (nblk + 64) * sizeof(u32) +
         1024;
}

void launch_check(const CheckLaunch& L, cudaStream_t st) {
  if (L.n_max == 0) return;
  int dev = 0;
  cudaGetDevice(&dev);
  const bool SH = L.sh_in || L.sh_out;
  const int grid = SH ? k7_grid<true>(dev) : k7_grid<false>(dev);
  const u64 nblk = (L.n_max + KT_BLK - 1) / KT_BLK;  // upper bound (array sizes); the kernels partition the
                                                      // device-side item count (k7_part)
  char* base = (char*)L.status;
  K7Ctx* kdev = reinterpret_cast<K7Ctx*>(base);
  Sum* sums = reinterpret_cast<Sum*>(base + ((sizeof(K7Ctx) + 255) & ~(size_t)255));
  u32* wl = reinterpret_cast<u32*>(sums + nblk + 1);
  u32* wl_cnt = wl + nblk + 1;
  K7Ctx k{};
  k.c = L.c;
  k.keys = L.keys;
  k.evs = L.evs;
  k.R0 = L.R0;
  k.sh_in = L.sh_in;
  k.sh_out = L.sh_out;
  k.pool = L.pool;
  k.pool_cnt = L.pool_cnt;
  k.pool_cap = L.pool_cap;
  k.races = L.races;
  k.race_cnt = L.race_cnt;
  k.race_cap = L.race_cap;
  k.seg_cnt = L.seg_cnt;
  k.values = L.values;
  k.n_dev = L.n_dev;
  cudaMemcpyAsync(kdev, &k, sizeof(K7Ctx), cudaMemcpyHostToDevice, st);
  cudaMemsetAsync(wl_cnt, 0, sizeof(u32), st);
  CheckArgs a;
  a.k = kdev;
  a.c = L.c;
  a.keys = L.keys;
  a.evs = L.evs;
  a.n_dev = L.n_dev;
  a.R0 = L.R0;
  a.sh_in = L.sh_in;
  a.sh_out = L.sh_out;
  a.no_sv = L.c.g.flags & BC_F_NO_SAME_VALUE_FILTER;
  a.values = L.values;
  static bool kb_attr[64] = {};
  if (dev >= 0 && dev < 64 && !kb_attr[dev]) {
    cudaFuncSetAttribute(k_blk_sum, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)KB_SMEM);
    kb_attr[dev] = true;
  }
  k_blk_sum<<<K7A_CTAS, KT_SWARPS * 32, KB_SMEM, st>>>(a, sums, wl, wl_cnt);
  if (SH)
    k_check_tile<true><<<grid, KtCfg<true>::WARPS * 32, (size_t)KtCfg<true>::WARPS * KtCfg<true>::WARP_BYTES, st>>>(
        a, wl, wl_cnt, sums, (u32)nblk);
  else
    k_check_tile<false><<<grid, KtCfg<false>::WARPS * 32, (size_t)KtCfg<false>::WARPS * KtCfg<false>::WARP_BYTES,
                          st>>>(a, wl, wl_cnt, sums, (u32)nblk);
  g_launches += 2;
}

void preload_check() {
  preload(k_blk_sum, k_check_tile<false>, k_check_tile<true>, k_count_gathers,
          k_shadow_commit);
}

}  // namespace bc
