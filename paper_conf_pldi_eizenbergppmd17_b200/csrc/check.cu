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
  const bool sameb = (w1 / c.g.wpb) == (s2.warp / c.g.wpb);
  if (sameb && r1 + 1u <= s2.blab) return true;  // completed barrier (Fig. 3 BAR)
  if (c.n_acq == 0 && !(w1 == s2.warp && s2.node != s2.warp)) return false;
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

// warp 0: exclusive prefix of this tile from its predecessors' published summaries,
// 32 predecessors per round (decoupled look-back, non-commutative combine in tile order).
__device__ __forceinline__ Sum warp_lookback(TileStatus* status, u32 tile, const Sum& agg, int lane) {
  if (tile == 0) {
    if (lane == 0) publish(&status[0], agg, 2u);
    return sum_ident();
  }
  if (lane == 0) publish(&status[tile], agg, 1u);
  Sum P = sum_ident();
  int hi = (int)tile - 1;
  while (true) {
    int idx = hi - lane;  // lane 0 = nearest predecessor
    u32 f = 2u;
    Sum s = sum_ident();
    if (idx >= 0) {
      f = ((volatile TileStatus*)&status[idx])->flag;
    }
    // all lanes spin together until every inspected predecessor has published
    while (__any_sync(0xFFFFFFFFu, f == 0u)) {
      if (f == 0u) f = ((volatile TileStatus*)&status[idx])->flag;
    }
    __threadfence();
    if (idx >= 0) {
      volatile TileStatus* v = &status[idx];
      s = Sum{v->fk, v->lk, v->lw, v->fi, v->bits};
    }
    u32 incm = __ballot_sync(0xFFFFFFFFu, idx >= 0 && f == 2u);
    int last = incm ? (__ffs(incm) - 1) : 31;  // nearest inclusive predecessor ends this round
    if (hi - last < 0) last = hi;                // fewer than 32 tiles left (tile 0 is inclusive)
    // P = combine(s[last], ..., s[1], s[0], P)
    Sum acc = sum_ident();
    for (int k = last; k >= 0; --k) {
      Sum sk;
      sk.fk = __shfl_sync(0xFFFFFFFFu, s.fk, k);
      sk.lk = __shfl_sync(0xFFFFFFFFu, s.lk, k);
      sk.lw = __shfl_sync(0xFFFFFFFFu, s.lw, k);
      sk.fi = __shfl_sync(0xFFFFFFFFu, s.fi, k);
      sk.bits = __shfl_sync(0xFFFFFFFFu, s.bits, k);
      acc = combine(acc, sk);
    }
    P = combine(acc, P);
    if (incm) break;
    hi -= 32;
  }
  if (lane == 0) publish(&status[tile], combine(P, agg), 2u);
  return P;
}

__global__ void __launch_bounds__(CK_THREADS) k_check(CheckArgs a) {
  __shared__ u32 s_kx[CK_TILE];
  __shared__ u32 s_ev[CK_TILE];
  __shared__ u32 s_w[CK_TILE];
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
  const u64 tbase = (u64)tile * CK_TILE;
  const u64 base = tbase + (u64)t * CK_IPT;
  const HbCtx& c = a.c;

  // ---- A: items + their records' snapshots (all gathers in flight together)
  u32 kx[CK_IPT], ev[CK_IPT];
  uint4 sn[CK_IPT];
#pragma unroll
  for (int j = 0; j < CK_IPT; ++j) {
    u64 i = base + j;
    kx[j] = i < a.n ? a.keys[i] : NONE;
    ev[j] = i < a.n ? a.evs[i] : 0u;
  }
#pragma unroll
  for (int j = 0; j < CK_IPT; ++j) sn[j] = base + j < a.n ? __ldg(c.snap + (ev[j] >> 5)) : make_uint4(0, 0, 0, 0);
  // previous item (the last item of thread t-1, or the item before the tile)
  u32 pkx = __shfl_up_sync(0xFFFFFFFFu, kx[CK_IPT - 1], 1);
  u32 pev = __shfl_up_sync(0xFFFFFFFFu, ev[CK_IPT - 1], 1);
  u32 pw = __shfl_up_sync(0xFFFFFFFFu, sn[CK_IPT - 1].x, 1);
  if (lane == 0) {
    if (base > 0 && base - 1 < a.n) {
      pkx = a.keys[base - 1];
      pev = a.evs[base - 1];
      pw = __ldg(&c.snap[pev >> 5].x);
    } else {
      pkx = NONE;
    }
  }
#pragma unroll
  for (int j = 0; j < CK_IPT; ++j) {
    s_kx[t * CK_IPT + j] = kx[j];
    s_ev[t * CK_IPT + j] = ev[j];
    s_w[t * CK_IPT + j] = sn[j].x;
  }

  // ---- B: READINFLATE flags (a read whose predecessor read of the granule is unordered)
  u32 infl = 0, segs = 0;
  Sum mine = sum_ident();
#pragma unroll
  for (int j = 0; j < CK_IPT; ++j) {
    const u64 i = base + j;
    const u32 qkx = j ? kx[j - 1] : pkx;
    const u32 qev = j ? ev[j - 1] : pev;
    const u32 qw = j ? sn[j - 1].x : pw;
    if (i < a.n) {
      const u32 key = kx[j] >> 2, op = kx[j] & 3u;
      const bool same = qkx != NONE && (qkx >> 2) == key;
      if (!same) ++segs;
      if (op == IOP_LD && same && (qkx & 3u) == IOP_LD && !hb_ev(c, qev, qw, ev[j], to_snap(sn[j]))) infl |= 1u << j;
      Sum it;
      it.fk = key;
      it.lk = key;
      it.lw = op != IOP_LD ? (u32)i + 1u : 0u;
      it.fi = ((infl >> j) & 1u) ? (u32)i : NONE;
      it.bits = 1u | (op != IOP_LD ? 2u : 0u);
      mine = combine(mine, it);
    }
  }

  // ---- C: block scan of thread summaries + look-back across tiles
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
  if (w == 0) {
    Sum agg = sum_ident();
    for (int ww = 0; ww < CK_THREADS / 32; ++ww) agg = combine(agg, s_wt[ww]);
    Sum P = warp_lookback(a.status, tile, agg, lane);
    if (lane == 0) {
      s_prefix = P;
      if (s_segs) atomicAdd((unsigned long long*)a.seg_cnt, (unsigned long long)s_segs);
    }
  }
  Sum wp = sum_ident();
  for (int ww = 0; ww < w; ++ww) wp = combine(wp, s_wt[ww]);
  __syncthreads();
  const Sum st = combine(s_prefix, combine(wp, excl));

  // ---- D: per-item checks with the exact incoming state
  const u32 no_sv = c.g.flags & BC_F_NO_SAME_VALUE_FILTER;
  u32 lk = st.lk, lw = st.lw, fi = st.fi;
#pragma unroll
  for (int j = 0; j < CK_IPT; ++j) {
    const u64 i = base + j;
    if (i < a.n) {
      const u32 key = kx[j] >> 2, op = kx[j] & 3u;
      const Snap s2 = to_snap(sn[j]);
      const u32 qkx = j ? kx[j - 1] : pkx;
      const u32 qev = j ? ev[j - 1] : pev;
      const u32 qw = j ? sn[j - 1].x : pw;
      if (key != lk) {
        lk = key;
        lw = 0;
        fi = NONE;
      }
      // W_x check (every rule of Fig. 2; atomics only against a plain last write)
      if (lw) {
        const u64 li = (u64)lw - 1;
        u32 pkx2, pev2, pw2;
        if (li >= tbase) {
          pkx2 = s_kx[li - tbase];
          pev2 = s_ev[li - tbase];
          pw2 = s_w[li - tbase];
        } else {
          pkx2 = a.keys[li];
          pev2 = a.evs[li];
          pw2 = __ldg(&c.snap[pev2 >> 5].x);
        }
        const bool patm = (pkx2 & 3u) == IOP_ATOM;
        if (op == IOP_LD) {
          if (!hb_ev(c, pev2, pw2, ev[j], s2)) emit(a, key, ev[j], pev2, patm ? BC_KIND_AR : BC_KIND_WR);
        } else if (op == IOP_ATOM) {
          if (!patm && !hb_ev(c, pev2, pw2, ev[j], s2)) emit(a, key, ev[j], pev2, BC_KIND_WA);
        } else if (!hb_ev(c, pev2, pw2, ev[j], s2)) {
          const bool filtered = !patm && op == IOP_ST_SV && !no_sv && (pev2 >> 5) == (ev[j] >> 5);
          if (!filtered) emit(a, key, ev[j], pev2, patm ? BC_KIND_AW : BC_KIND_WW);
        }
      }
      // R_x check at writers (WRITE* / *ATOM*: R_x ⪯ C_t as an epoch, R_x ⊑ C_t as a vector)
      if (op != IOP_LD && qkx != NONE && (qkx >> 2) == key && (qkx & 3u) == IOP_LD) {
        const u32 kind = op == IOP_ATOM ? BC_KIND_RA : BC_KIND_RW;
        if (fi == NONE) {
          if (!hb_ev(c, qev, qw, ev[j], s2)) emit(a, key, ev[j], qev, kind);
        } else {
          vc_check(a.evs, a.races, a.race_cnt, a.race_cap, (u64)fi - 1, i - 1, ev[j], s2.warp, s2.ps, s2.node,
                   s2.blab, key, kind);
        }
      }
      if (op != IOP_LD) {
        lw = (u32)i + 1u;
        fi = NONE;
      } else if (((infl >> j) & 1u) && fi == NONE) {
        fi = (u32)i;
      }
    }
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
  cudaMemcpyToSymbolAsync(cHC, &c, sizeof(HbCtx), 0, cudaMemcpyHostToDevice, st);
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
  k_check<<<(unsigned)tiles, CK_THREADS, 0, st>>>(a); ++g_launches;
}

}  // namespace bc
