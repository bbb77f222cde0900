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
// plus independent happens-before queries per item.  One tile = 2048 items; the scan state crosses
// tiles by decoupled look-back, so arbitrarily long (hot) granule segments cost the same per item
// as short ones, and the shadow state never has to be materialised in memory within a window.
#include "common.cuh"
#include "kernels.cuh"

namespace bc {

namespace {

constexpr int CK_THREADS = 256;
constexpr int CK_IPT = 8;
constexpr int CK_TILE = CK_THREADS * CK_IPT;

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

__device__ __forceinline__ Sum shfl_up_sum(const Sum& s, int o) {
  Sum r;
  r.fk = __shfl_up_sync(0xFFFFFFFFu, s.fk, o);
  r.lk = __shfl_up_sync(0xFFFFFFFFu, s.lk, o);
  r.lw = __shfl_up_sync(0xFFFFFFFFu, s.lw, o);
  r.fi = __shfl_up_sync(0xFFFFFFFFu, s.fi, o);
  r.bits = __shfl_up_sync(0xFFFFFFFFu, s.bits, o);
  return r;
}

struct TileStatus {  // 32 B
  u32 flag, fk, lk, lw, fi, bits, pad0, pad1;
};

__device__ __forceinline__ void publish(TileStatus* ts, const Sum& s, u32 flag) {
  volatile TileStatus* v = ts;
  v->fk = s.fk;
  v->lk = s.lk;
  v->lw = s.lw;
  v->fi = s.fi;
  v->bits = s.bits;
  __threadfence();
  v->flag = flag;
}

struct CheckArgs {
  HbCtx c;
  const u32* keys;  // (granule key << 2) | op
  const u32* evs;   // (record << 5) | lane
  u64 n;
  TileStatus* status;
  u32* tile_counter;
  uint4* races;  // (key, cur_ev, prior_ev, kind)
  u32* race_cnt;
  u32 race_cap;
  u64* seg_cnt;
};

__device__ __forceinline__ void emit(const CheckArgs& a, u32 key, u32 cur, u32 prior, u32 kind) {
  u32 at = atomicAdd(a.race_cnt, 1u);
  if (at < a.race_cap) a.races[at] = make_uint4(key, cur, prior, kind);
}

// lazily loaded snapshot of the current item's record
struct Cur {
  u32 ev, rec, lane;
  bool have;
  Snap s;
};
__device__ __forceinline__ const Snap& cur_snap(const CheckArgs& a, Cur& cu) {
  if (!cu.have) {
    cu.s = load_snap(a.c.snap, cu.rec);
    cu.have = true;
  }
  return cu.s;
}
__device__ __forceinline__ bool hb_ev(const CheckArgs& a, u32 ev1, Cur& cu) {
  u32 r1 = ev1 >> 5, l1 = ev1 & 31u;
  if (r1 == cu.rec) return l1 == cu.lane;
  const Snap& s2 = cur_snap(a, cu);
  u32 w1 = __ldg(&a.c.snap[r1].x);
  return hb(a.c, r1, l1, w1, cu.rec, cu.lane, s2);
}

// thread identity of an event (warp << 5 | lane)
__device__ __forceinline__ u32 ev_tid(const CheckArgs& a, u32 ev) { return (__ldg(&a.c.snap[ev >> 5].x) << 5) | (ev & 31u); }

// R_x is a vector clock at writer `cu` (index i): entries = latest read per thread among items
// [lo, hi] (all reads of this granule).  Check each entry (Fig. 2 WRITESHARED, Fig. 3 *ATOMSHARED).
__device__ __noinline__ void vc_check(const CheckArgs& a, u64 lo, u64 hi, Cur& cu, u32 key, u32 kind) {
  u32 seen[32];
  int ns = 0;
  for (u64 j = hi + 1; j-- > lo;) {
    u32 ev = a.evs[j];
    u32 tid = ev_tid(a, ev);
    bool dup = false;
    for (int q = 0; q < ns; ++q)
      if (seen[q] == tid) { dup = true; break; }
    if (!dup && ns == 32) {
      // overflow of the small set: look for a later read of the same thread directly
      for (u64 q = j + 1; q <= hi; ++q)
        if (ev_tid(a, a.evs[q]) == tid) { dup = true; break; }
    }
    if (dup) continue;
    if (ns < 32) seen[ns++] = tid;
    if (!hb_ev(a, ev, cu)) emit(a, key, cu.ev, ev, kind);
  }
}

__global__ void __launch_bounds__(CK_THREADS) k_check(CheckArgs a) {
  __shared__ u32 s_tile;
  __shared__ Sum s_wt[CK_THREADS / 32];
  __shared__ Sum s_prefix;
  __shared__ u32 s_segs;
  const int t = threadIdx.x, w = t >> 5, lane = t & 31;
  if (t == 0) {
    s_tile = atomicAdd(a.tile_counter, 1u);
    s_segs = 0;
  }
  __syncthreads();
  const u32 tile = s_tile;
  const u64 base = (u64)tile * CK_TILE + (u64)t * CK_IPT;

  u32 kx[CK_IPT], ev[CK_IPT];
  u32 infl = 0;  // bit j: item j is a read that found its predecessor read unordered (READINFLATE)
  u32 segs = 0;
  u32 pk = NONE, pop = 0, pev = 0;  // previous item
  if (base > 0 && base - 1 < a.n) {
    pk = a.keys[base - 1];
    pev = a.evs[base - 1];
    pop = pk & 3u;
    pk >>= 2;
  }
#pragma unroll
  for (int j = 0; j < CK_IPT; ++j) {
    u64 i = base + j;
    if (i < a.n) {
      kx[j] = a.keys[i];
      ev[j] = a.evs[i];
    } else {
      kx[j] = NONE;
      ev[j] = 0;
    }
  }
  Sum mine = sum_ident();
#pragma unroll
  for (int j = 0; j < CK_IPT; ++j) {
    u64 i = base + j;
    if (i >= a.n) break;
    u32 key = kx[j] >> 2, op = kx[j] & 3u;
    if (key != pk) ++segs;
    if (op == IOP_LD && key == pk && pop == IOP_LD) {
      Cur cu{ev[j], ev[j] >> 5, ev[j] & 31u, false, Snap{}};
      if (!hb_ev(a, pev, cu)) infl |= 1u << j;
    }
    Sum it;
    it.fk = key;
    it.lk = key;
    it.lw = op != IOP_LD ? (u32)i + 1u : 0u;
    it.fi = ((infl >> j) & 1u) ? (u32)i : NONE;
    it.bits = 1u | (op != IOP_LD ? 2u : 0u);
    mine = combine(mine, it);
    pk = key;
    pop = op;
    pev = ev[j];
  }
  // block scan of thread summaries
  Sum incl = mine;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    Sum left = shfl_up_sum(incl, o);
    if (lane >= o) incl = combine(left, incl);
  }
  Sum excl = shfl_up_sum(incl, 1);
  if (lane == 0) excl = sum_ident();
  if (lane == 31) s_wt[w] = incl;
  if (segs) atomicAdd(&s_segs, segs);
  __syncthreads();
  Sum wp = sum_ident();
  for (int ww = 0; ww < w; ++ww) wp = combine(wp, s_wt[ww]);
  if (t == 0) {
    Sum agg = sum_ident();
    for (int ww = 0; ww < CK_THREADS / 32; ++ww) agg = combine(agg, s_wt[ww]);
    Sum P = sum_ident();
    if (tile == 0) {
      publish(&a.status[0], agg, 2u);
    } else {
      publish(&a.status[tile], agg, 1u);
      int pt = (int)tile - 1;
      while (true) {
        volatile TileStatus* v = &a.status[pt];
        u32 f = v->flag;
        if (f == 0) continue;
        __threadfence();
        Sum s{v->fk, v->lk, v->lw, v->fi, v->bits};
        P = combine(s, P);
        if (f == 2u) break;
        --pt;
      }
      publish(&a.status[tile], combine(P, agg), 2u);
    }
    s_prefix = P;
    if (s_segs) atomicAdd((unsigned long long*)a.seg_cnt, (unsigned long long)s_segs);
  }
  __syncthreads();
  Sum st = combine(s_prefix, combine(wp, excl));

  // per-item checks with the exact incoming state
  const u32 no_sv = a.c.g.flags & BC_F_NO_SAME_VALUE_FILTER;
  u32 lk = st.lk, lw = st.lw, fi = st.fi;
  if (base > 0 && base - 1 < a.n) {
    pk = a.keys[base - 1];
    pev = a.evs[base - 1];
    pop = pk & 3u;
    pk >>= 2;
  } else {
    pk = NONE;
  }
#pragma unroll 1
  for (int j = 0; j < CK_IPT; ++j) {
    u64 i = base + j;
    if (i >= a.n) break;
    u32 key = kx[j] >> 2, op = kx[j] & 3u;
    if (key != lk) {
      lk = key;
      lw = 0;
      fi = NONE;
    }
    Cur cu{ev[j], ev[j] >> 5, ev[j] & 31u, false, Snap{}};
    // W_x check (every rule of Fig. 2; atomics only against a plain last write)
    if (lw) {
      u32 pk2 = a.keys[lw - 1], pev2 = a.evs[lw - 1];
      bool patm = (pk2 & 3u) == IOP_ATOM;
      if (op == IOP_LD) {
        if (!hb_ev(a, pev2, cu)) emit(a, key, cu.ev, pev2, patm ? BC_KIND_AR : BC_KIND_WR);
      } else if (op == IOP_ATOM) {
        if (!patm && !hb_ev(a, pev2, cu)) emit(a, key, cu.ev, pev2, BC_KIND_WA);
      } else {
        if (!hb_ev(a, pev2, cu)) {
          bool filtered = !patm && op == IOP_ST_SV && !no_sv && (pev2 >> 5) == cu.rec;
          if (!filtered) emit(a, key, cu.ev, pev2, patm ? BC_KIND_AW : BC_KIND_WW);
        }
      }
    }
    // R_x check at writers (WRITE*/ATOM*: R_x ⪯ C_t or R_x ⊑ C_t)
    if (op != IOP_LD && key == pk && pop == IOP_LD) {
      u32 kind = op == IOP_ATOM ? BC_KIND_RA : BC_KIND_RW;
      if (fi == NONE) {
        if (!hb_ev(a, pev, cu)) emit(a, key, cu.ev, pev, kind);
      } else {
        vc_check(a, (u64)fi - 1, i - 1, cu, key, kind);
      }
    }
    // state update
    if (op != IOP_LD) {
      lw = (u32)i + 1u;
      fi = NONE;
    } else if (((infl >> j) & 1u) && fi == NONE) {
      fi = (u32)i;
    }
    pk = key;
    pop = op;
    pev = ev[j];
  }
}

}  // namespace

size_t check_status_bytes(u64 n) { return ((n + CK_TILE - 1) / CK_TILE + 1) * sizeof(TileStatus); }

void launch_check(const HbCtx& c, const u32* keys, const u32* evs, u64 n, void* status, u32* tile_counter,
                  uint4* races, u32* race_cnt, u32 race_cap, u64* seg_cnt, cudaStream_t st) {
  if (n == 0) return;
  u64 tiles = (n + CK_TILE - 1) / CK_TILE;
  cudaMemsetAsync(status, 0, tiles * sizeof(TileStatus), st);
  cudaMemsetAsync(tile_counter, 0, sizeof(u32), st);
  CheckArgs a;
  a.c = c;
  a.keys = keys;
  a.evs = evs;
  a.n = n;
  a.status = (TileStatus*)status;
  a.tile_counter = tile_counter;
  a.races = races;
  a.race_cnt = race_cnt;
  a.race_cap = race_cap;
  a.seg_cnt = seg_cnt;
  k_check<<<(unsigned)tiles, CK_THREADS, 0, st>>>(a);
}

}  // namespace bc
