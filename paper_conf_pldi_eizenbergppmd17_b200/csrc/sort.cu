// sort.cu — hand-written stable LSD radix sort (8- to 10-bit digits, reduce-then-scan per pass)
// and a device-wide exclusive scan, for sm_100a.
//
// The radix sort is the paper's per-location serialisation (a spinlock per shadow
// entry orders the host threads' accesses) turned into data parallelism: a STABLE sort of
// (location key, trace position) items groups each location's accesses into one contiguous
// segment that is still in trace order.
// Per pass:
//   k_rs_up    : per 6144-key tile (24 keys / thread), the digit counts (reads 4 B / item)
//   k_rs_rows  : one CTA per digit scans that digit's counts over all tiles (independent rows: no
//                serial chain across tiles, unlike a decoupled look-back whose first wave of ~450
//                co-resident tiles walks back one L2 round trip per step), and its total
//   k_rs_bins  : exclusive scan of the digit totals (digit start offsets); kept-item count
//                (default RS_FUSED_BINS: done by every k_rs_down CTA itself, no launch)
//   k_rs_down  : per tile: stable in-tile rank (MATCH.ANY + per-warp histograms), scatter through
//                shared memory so that each digit's run is written contiguously (8 B in, 8 B out).
#include <algorithm>
#include <cstdlib>

#include "common.cuh"
#include "kernels.cuh"

namespace bc {

namespace {

constexpr int RS_THREADS = 256;
#ifndef RS_ITEMS_
#define RS_ITEMS_ 24
#endif
constexpr int RS_ITEMS = RS_ITEMS_;  // keys per thread per tile
constexpr int RS_TILE = RS_THREADS * RS_ITEMS;  // 6144 (A/B on C2 / C4: 24 keys per thread beat 8-32)
constexpr int RS_WARPS = RS_THREADS / 32;
constexpr int RS_MAXB = 2048;                   // bins of the widest digit (11 bits)
constexpr int RS_MAXP = 4;
#ifndef RS_MATCH_ANY
#define RS_MATCH_ANY 1  // warp peers of a digit by one MATCH.ANY instead of RB+1 ballots
#endif
// temp header: digit totals [RS_MAXP][RS_MAXB], gbase[RS_MAXP][RS_MAXB]; the (digit, tile) table follows
constexpr size_t RS_HDR_BYTES = (2 * RS_MAXP * RS_MAXB + 64) * sizeof(u32);

// Lanes of the warp holding the same (RB+1)-bit label (digit, or 1 << RB = no item): RB+1 ballots,
// a fixed cost independent of how many distinct digits the warp holds.
template <int RB>
__device__ __forceinline__ u32 match_label(u32 d) {
  u32 m = 0xFFFFFFFFu;
#pragma unroll
  for (int b = 0; b <= RB; ++b) {
    const bool bit = (d >> b) & 1u;
    const u32 bal = __ballot_sync(0xFFFFFFFFu, bit);
    m &= bit ? bal : ~bal;
  }
  return m;
}

// add 1 per lane to h[d]; a warp that holds one digit only (the common case for the high digits of
// sorted-ish keys) does a single atomic
__device__ __forceinline__ void warp_hist_add(u32* h, u32 d, bool ok, u32 lt) {
  const u32 vm = __ballot_sync(0xFFFFFFFFu, ok);
  const u32 d0 = __shfl_sync(0xFFFFFFFFu, d, vm ? __ffs(vm) - 1 : 0);
  if (__all_sync(0xFFFFFFFFu, !ok || d == d0)) {
    if (vm && (lt & vm) == 0 && ok) atomicAdd(&h[d], (u32)__popc(vm));
  } else if (ok) {
    atomicAdd(&h[d], 1u);
  }
}

// gbase[d] = exclusive prefix of the digit totals; *n_out = kept items (all digits).  BINS threads.
template <int RB>
__global__ void __launch_bounds__((1 << RB) < 1024 ? (1 << RB) : 1024) k_rs_bins(const u32* __restrict__ ghist,
                                                                               u32* __restrict__ gbase,
                                                                               u64* __restrict__ n_out) {
  constexpr int BINS = 1 << RB;
  constexpr int T = BINS < 1024 ? BINS : 1024, PER = BINS / T;  // thread t: digits [t*PER, t*PER+PER)
  __shared__ u32 wsum[T / 32];
  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  u32 v[PER], sum = 0;
#pragma unroll
  for (int q = 0; q < PER; ++q) {
    v[q] = ghist[t * PER + q];
    sum += v[q];
  }
  const u32 x = warp_incl_sum(sum);
  if (l == 31) wsum[w] = x;
  __syncthreads();
  u32 off = 0, tot = 0;
  for (int ww = 0; ww < T / 32; ++ww) {
    if (ww < w) off += wsum[ww];
    tot += wsum[ww];
  }
  u32 run = off + x - sum;
#pragma unroll
  for (int q = 0; q < PER; ++q) {
    gbase[t * PER + q] = run;
    run += v[q];
  }
  if (t == 0 && n_out) *n_out = tot;
}

// Upsweep of one pass: the digit counts of every tile, digit-major (counts[d * tiles + tile]);
// tiles past the (device-side) item count write zeros.
template <int RB>
__global__ void __launch_bounds__(RS_THREADS) k_rs_up(const u32* __restrict__ kin, u64 n_max,
                                                      const u64* __restrict__ n_dev, int drop, int shift,
                                                      u32* __restrict__ counts, u64 tiles) {
  constexpr int BINS = 1 << RB;
  __shared__ u32 h[BINS];
  const int t = threadIdx.x;
  for (int i = t; i < BINS; i += RS_THREADS) h[i] = 0;
  __syncthreads();
  const u64 n = n_dev ? *n_dev : n_max;
  const u64 base = (u64)blockIdx.x * RS_TILE;
  const u32 lt = lanemask_lt();
  if (base < n) {
    u32 k[RS_ITEMS];
#pragma unroll
    for (int j = 0; j < RS_ITEMS; ++j) {
      const u64 idx = base + (u64)j * RS_THREADS + t;
      k[j] = idx < n ? kin[idx] : KEY_DROP;
    }
#pragma unroll
    for (int j = 0; j < RS_ITEMS; ++j) {
      const u64 idx = base + (u64)j * RS_THREADS + t;
      const bool ok = idx < n && !(drop && k[j] == KEY_DROP);
      warp_hist_add(h, ok ? (k[j] >> shift) & (BINS - 1) : 0u, ok, lt);
    }
  }
  __syncthreads();
  for (int d = t; d < BINS; d += RS_THREADS) counts[(u64)d * tiles + blockIdx.x] = h[d];
}

// One CTA per digit d: offs[d * tiles + tile] = items of digit d in tiles < tile; rowtot[d] = all items
// of digit d (their exclusive scan over the digits, k_rs_bins, is the digit's output base).
// The rows are independent, so there is no serial chain across tiles (unlike a decoupled
// look-back, whose first wave of ~450 co-resident tiles walks back one L2 round trip per step).
__global__ void __launch_bounds__(RS_THREADS) k_rs_rows(u32* __restrict__ counts, u64 tiles,
                                                        u32* __restrict__ rowtot) {
  __shared__ u32 wsum[RS_WARPS];
  __shared__ u32 s_carry;
  const int t = threadIdx.x, w = t >> 5, l = t & 31, d = blockIdx.x;
  u32* row = counts + (u64)d * tiles;
  if (t == 0) s_carry = 0;
  __syncthreads();
  constexpr int PER = 8;
  for (u64 c0 = 0; c0 < tiles; c0 += RS_THREADS * PER) {
    u32 v[PER], sum = 0;
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      const u64 i = c0 + (u64)t * PER + q;
      v[q] = i < tiles ? row[i] : 0u;
      sum += v[q];
    }
    const u32 x = warp_incl_sum(sum);
    if (l == 31) wsum[w] = x;
    __syncthreads();
    u32 off = 0, tot = 0;
    for (int ww = 0; ww < RS_WARPS; ++ww) {
      if (ww < w) off += wsum[ww];
      tot += wsum[ww];
    }
    u32 run = s_carry + off + x - sum;
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      const u64 i = c0 + (u64)t * PER + q;
      if (i < tiles) row[i] = run;
      run += v[q];
    }
    __syncthreads();
    if (t == 0) s_carry += tot;
    __syncthreads();
  }
  if (t == 0) rowtot[d] = s_carry;
}

// Downsweep of one pass: stable in-tile rank (ballot match + per-warp histograms), scatter through
// shared memory so that each digit's run is written contiguously (8 B in, 8 B out per item).
// Persistent CTAs; each tile's keys arrive in shared memory by 1-D TMA bulk copies issued
// RS_DSTAGES tiles ahead (mbarrier ring), so the load latency that dominated a one-tile-per-CTA kernel
// overlaps the ranking of the previous tile; the tile's values are loaded into registers at the start
// of the tile and land while it is ranked.  Once scattered, the stage holds the permuted values.
#ifndef RS_FASTRANK
#define RS_FASTRANK 0  // shuffle + vote fast paths (all-distinct / all-equal digits) before MATCH.ANY:
                       // A/B lost (C2 sort 0.279 -> 0.291 ms, C4 4.38 -> 4.69 ms; profiles/r1_ab_fastrank.txt)
#endif
#ifndef RS_FUSED_BINS
#define RS_FUSED_BINS 1  // digit bases scanned inside k_rs_down (no k_rs_bins launch per pass)
#endif
#ifndef RS_DSTAGES_
#define RS_DSTAGES_ 2
#endif
constexpr int RS_DSTAGES = RS_DSTAGES_;
template <int RB>
constexpr size_t rs_dsmem() {
  return (size_t)RS_DSTAGES * RS_TILE * sizeof(u32) + RS_TILE * sizeof(u32) +
         (size_t)(RS_WARPS + 2) * (1 << RB) * sizeof(u32) + 64 + RS_DSTAGES * 8;
}

template <int RB>
__global__ void __launch_bounds__(RS_THREADS, 2) k_rs_down(const u32* __restrict__ kin, const u32* __restrict__ vin,
                                                           u32* __restrict__ kout, u32* __restrict__ vout, u64 n_max,
                                                           const u64* __restrict__ n_dev, int drop, int shift,
                                                           const u32* __restrict__ offs, u64 tiles,
                                                           const u32* __restrict__ gbase,
                                                           const u32* __restrict__ rowtot, u64* __restrict__ n_out) {
  constexpr int BINS = 1 << RB;
  constexpr int DPT = BINS / RS_THREADS;  // digits per thread (1, 2 or 4)
  extern __shared__ __align__(128) unsigned char rs_smem[];
  u32* stage = reinterpret_cast<u32*>(rs_smem);                 // [RS_DSTAGES][RS_TILE] keys
  u32* skeys = stage + RS_DSTAGES * RS_TILE;                    // [RS_TILE]
  u32* whist = skeys + RS_TILE;                                 // [RS_WARPS][BINS]
  u32* tofs = whist + RS_WARPS * BINS;                          // [BINS]
  u32* gstart = tofs + BINS;                                    // [BINS]
  u32* wsum = gstart + BINS;                                    // [RS_WARPS]
  u32* s_kept = wsum + RS_WARPS;
  u64* bar = reinterpret_cast<u64*>(rs_smem + rs_dsmem<RB>() - RS_DSTAGES * 8);

  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  const u64 n = n_dev ? *n_dev : n_max;
  const u64 n_tiles = (n + RS_TILE - 1) / RS_TILE;
  auto issue = [&](u64 tile, int st) {
    const u64 base = tile * RS_TILE;
    const u64 cnt = n - base < (u64)RS_TILE ? n - base : (u64)RS_TILE;
    const u32 bytes = (u32)(((cnt + 3) & ~3ull) * sizeof(u32));  // whole 16-B units (buffers are padded)
    mbar_expect_tx(&bar[st], bytes);
    bulk_g2s(stage + st * RS_TILE, kin + base, bytes, &bar[st]);
  };
  if (t == 0) {
    for (int q = 0; q < RS_DSTAGES; ++q) mbar_init(&bar[q], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (t == 0)
    for (int q = 0; q < RS_DSTAGES; ++q) {
      const u64 tl = blockIdx.x + (u64)q * gridDim.x;
      if (tl < n_tiles) issue(tl, q);
    }
  const u32 lt = lanemask_lt();
  // digit bases: with rowtot (RS_FUSED_BINS) every CTA scans the digit totals itself, once (thread t
  // owns digits t + q * RS_THREADS, i.e. q-th block of RS_THREADS consecutive digits), instead of a
  // separate one-CTA k_rs_bins launch per pass; CTA 0 publishes the kept-item count
  u32 gb[DPT];
  if (rowtot) {
    u32 carry = 0;
#pragma unroll
    for (int q = 0; q < DPT; ++q) {
      const u32 v0 = __ldg(&rowtot[t + q * RS_THREADS]);
      const u32 x = warp_incl_sum(v0);
      if (l == 31) wsum[w] = x;
      __syncthreads();
      u32 off = 0, tot = 0;
      for (int ww = 0; ww < RS_WARPS; ++ww) {
        if (ww < w) off += wsum[ww];
        tot += wsum[ww];
      }
      gb[q] = carry + off + x - v0;
      carry += tot;
      __syncthreads();
    }
    if (n_out && blockIdx.x == 0 && t == 0) *n_out = carry;
  } else {
#pragma unroll
    for (int q = 0; q < DPT; ++q) gb[q] = __ldg(&gbase[t + q * RS_THREADS]);
  }
  u32 it = 0;
  for (u64 tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
    const int st = (int)(it % RS_DSTAGES);
    const u32 phase = (it / RS_DSTAGES) & 1u;
    u32* sk = stage + st * RS_TILE;
    const u64 base = tile * RS_TILE;
    u32 v[RS_ITEMS];
    if (vin) {
#pragma unroll
      for (int j = 0; j < RS_ITEMS; ++j) {
        const u64 idx = base + (u64)w * (RS_ITEMS * 32) + j * 32 + l;
        v[j] = idx < n ? vin[idx] : 0u;
      }
    }
    for (int i = t; i < RS_WARPS * BINS; i += RS_THREADS) whist[i] = 0;
    // this tile's digit offsets: loaded now, stored to shared memory after the ranking (their
    // latency overlaps it instead of stalling the tile start)
    u32 go[DPT];
#pragma unroll
    for (int q = 0; q < DPT; ++q)
      go[q] = gb[q] + __ldg(&offs[(u64)(t + q * RS_THREADS) * tiles + tile]);
    __syncthreads();
    mbar_wait(&bar[st], phase);
    u32 rank[RS_ITEMS];  // (digit << 16) | rank in the warp's digit run, NONE = no item
#pragma unroll
    // digits and warp peers of all items first (independent MATCH.ANYs in flight together), then the
    // per-warp running counts in item order
    u32 dg[RS_ITEMS], pr[RS_ITEMS];
#pragma unroll
    for (int j = 0; j < RS_ITEMS; ++j) {
      const u32 li = w * (RS_ITEMS * 32) + j * 32 + l;
      const u64 idx = base + li;
      const u32 k = idx < n ? sk[li] : KEY_DROP;
      dg[j] = (idx < n && !(drop && k == KEY_DROP)) ? ((k >> shift) & (BINS - 1)) : (u32)BINS;
#if RS_FASTRANK
      // warp-uniform fast paths before the (MIO-bound) MATCH.ANY: 32 strictly increasing digits are
      // all distinct (low digits of consecutive granules), 32 equal digits are one run (high digits)
      const u32 dprev = __shfl_up_sync(0xFFFFFFFFu, dg[j], 1);
      if (__all_sync(0xFFFFFFFFu, l == 0 || dg[j] > dprev))
        pr[j] = 1u << l;
      else if (__all_sync(0xFFFFFFFFu, dg[j] == __shfl_sync(0xFFFFFFFFu, dg[j], 0)))
        pr[j] = 0xFFFFFFFFu;
      else
#endif
      pr[j] = RS_MATCH_ANY ? __match_any_sync(0xFFFFFFFFu, dg[j]) : match_label<RB>(dg[j]);
    }
#pragma unroll
    for (int j = 0; j < RS_ITEMS; ++j) {
      const u32 d = dg[j], peers = pr[j];
      u32* hw = whist + w * BINS;
      const u32 old = d < (u32)BINS ? hw[d] : 0u;
      __syncwarp();
      if (d < (u32)BINS && (peers & lt) == 0) hw[d] = old + __popc(peers);
      __syncwarp();
      rank[j] = d < (u32)BINS ? ((d << 16) | (old + __popc(peers & lt))) : NONE;
    }
#pragma unroll
    for (int q = 0; q < DPT; ++q) gstart[t + q * RS_THREADS] = go[q];
    __syncthreads();
    // per digit: prefix over warps, tile total; thread t owns digits [t*DPT, t*DPT + DPT)
    u32 tsum = 0, dtot[DPT];
#pragma unroll
    for (int q = 0; q < DPT; ++q) {
      const int d = t * DPT + q;
      u32 total = 0;
#pragma unroll
      for (int ww = 0; ww < RS_WARPS; ++ww) {
        const u32 c = whist[ww * BINS + d];
        whist[ww * BINS + d] = total;
        total += c;
      }
      dtot[q] = total;
      tsum += total;
    }
    {
      const u32 x = warp_incl_sum(tsum);
      if (l == 31) wsum[w] = x;
      __syncthreads();
      u32 off = 0;
      for (int ww = 0; ww < w; ++ww) off += wsum[ww];
      u32 run = off + x - tsum;
#pragma unroll
      for (int q = 0; q < DPT; ++q) {
        tofs[t * DPT + q] = run;
        run += dtot[q];
      }
      if (t == RS_THREADS - 1) *s_kept = run;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < RS_ITEMS; ++j) {
      if (rank[j] != NONE) {
        const u32 d = rank[j] >> 16;
        skeys[tofs[d] + whist[w * BINS + d] + (rank[j] & 0xFFFFu)] = sk[w * (RS_ITEMS * 32) + j * 32 + l];
      }
    }
    __syncthreads();
    const u32 tile_n = *s_kept;
    if (vout) {
      // values: the same permutation, staged in the (consumed) key stage; keys and values then leave
      // in one pass over the tile
#pragma unroll
      for (int j = 0; j < RS_ITEMS; ++j) {
        if (rank[j] != NONE) {
          const u32 d = rank[j] >> 16;
          sk[tofs[d] + whist[w * BINS + d] + (rank[j] & 0xFFFFu)] = v[j];
        }
      }
      __syncthreads();
      for (u32 q = t; q < tile_n; q += RS_THREADS) {
        const u32 kk = skeys[q];
        const u32 d = (kk >> shift) & (BINS - 1);
        const u64 o = (u64)gstart[d] + (q - tofs[d]);
        kout[o] = kk;
        vout[o] = sk[q];
      }
    } else {
      for (u32 q = t; q < tile_n; q += RS_THREADS) {
        const u32 kk = skeys[q];
        const u32 d = (kk >> shift) & (BINS - 1);
        kout[(u64)gstart[d] + (q - tofs[d])] = kk;
      }
    }
    __syncthreads();  // stage st and the per-tile tables are free: refill the stage
    if (t == 0) {
      const u64 tn = tile + (u64)RS_DSTAGES * gridDim.x;
      if (tn < n_tiles) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        issue(tn, st);
      }
    }
  }
}

// ---------------------------------------------------------------------- scan
constexpr int SC_THREADS = 256, SC_ITEMS = 8, SC_TILE = SC_THREADS * SC_ITEMS;

// reduce-then-scan: per-tile sums, one CTA scans the tile sums, then every tile scans itself
__global__ void __launch_bounds__(SC_THREADS) k_scan_tsum(const u32* __restrict__ in, u64 n, u64* __restrict__ tsum) {
  __shared__ u64 wsum[SC_THREADS / 32];
  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  const u64 base = (u64)blockIdx.x * SC_TILE;
  u64 sum = 0;
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    const u64 i = base + (u64)j * SC_THREADS + t;
    sum += i < n ? in[i] : 0u;
  }
  const u64 x = warp_incl_sum(sum);
  if (l == 31) wsum[w] = x;
  __syncthreads();
  if (t == 0) {
    u64 tot = 0;
    for (int ww = 0; ww < SC_THREADS / 32; ++ww) tot += wsum[ww];
    tsum[blockIdx.x] = tot;
  }
}

__global__ void __launch_bounds__(1024) k_scan_tiles(u64* __restrict__ tsum, u64 tiles, u64* __restrict__ total_out) {
  __shared__ u64 wsum[32];
  __shared__ u64 s_carry;
  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  if (t == 0) s_carry = 0;
  __syncthreads();
  for (u64 c0 = 0; c0 < tiles; c0 += 1024) {
    const u64 i = c0 + t;
    const u64 v = i < tiles ? tsum[i] : 0ull;
    const u64 x = warp_incl_sum(v);
    if (l == 31) wsum[w] = x;
    __syncthreads();
    u64 off = 0, tot = 0;
    for (int ww = 0; ww < 32; ++ww) {
      if (ww < w) off += wsum[ww];
      tot += wsum[ww];
    }
    const u64 carry = s_carry;
    if (i < tiles) tsum[i] = carry + off + x - v;
    __syncthreads();
    if (t == 0) s_carry = carry + tot;
    __syncthreads();
  }
  if (t == 0 && total_out) *total_out = s_carry;
}

// small inputs: one CTA scans the whole array in chunks of 1024 with a running carry (one launch)
constexpr u64 SC_SMALL = 8192;
template <typename TO>
__global__ void __launch_bounds__(1024) k_scan_small(const u32* __restrict__ in, TO* __restrict__ out, u64 n,
                                                     u64* __restrict__ total_out) {
  __shared__ u64 wsum[32];
  __shared__ u64 s_carry;
  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  if (t == 0) s_carry = 0;
  // every chunk's input is loaded before the first scan step: one memory round trip, not one per chunk
  constexpr int CH = (int)(SC_SMALL / 1024);
  u32 pre[CH];
#pragma unroll
  for (int j = 0; j < CH; ++j) pre[j] = (u64)j * 1024 + t < n ? in[(u64)j * 1024 + t] : 0u;
  __syncthreads();
#pragma unroll
  for (int j = 0; j < CH; ++j) {
    const u64 c0 = (u64)j * 1024;
    if (c0 >= n) break;
    const u64 i = c0 + t;
    const u64 v = pre[j];
    const u64 x = warp_incl_sum(v);
    if (l == 31) wsum[w] = x;
    __syncthreads();
    u64 off = 0, tot = 0;
    for (int ww = 0; ww < 32; ++ww) {
      if (ww < w) off += wsum[ww];
      tot += wsum[ww];
    }
    const u64 carry = s_carry;
    if (i < n) out[i] = (TO)(carry + off + x - v);
    __syncthreads();
    if (t == 0) s_carry = carry + tot;
    __syncthreads();
  }
  if (t == 0 && total_out) *total_out = s_carry;
}

template <typename TO>
__global__ void __launch_bounds__(SC_THREADS) k_scan_u32(const u32* __restrict__ in, TO* __restrict__ out, u64 n,
                                                         const u64* __restrict__ texcl) {
  __shared__ u64 wsum[SC_THREADS / 32];
  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  const u64 base = (u64)blockIdx.x * SC_TILE + (u64)t * SC_ITEMS;
  static_assert(SC_ITEMS == 8, "two 16-B loads per thread");
  u32 v[SC_ITEMS];
  u64 sum = 0;
  // vector path: a whole 8-word group and 16-B aligned arrays (base is a multiple of 8 words; callers may
  // pass arrays that start inside a buffer, e.g. the barrier counts after the IF counts)
  const bool full = base + SC_ITEMS <= n && (((uintptr_t)in | (uintptr_t)out) & 15u) == 0;
  if (full) {
    const uint4 a = __ldg(reinterpret_cast<const uint4*>(in + base));
    const uint4 b = __ldg(reinterpret_cast<const uint4*>(in + base) + 1);
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
  } else {
#pragma unroll
    for (int j = 0; j < SC_ITEMS; ++j) v[j] = base + j < n ? in[base + j] : 0u;
  }
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) sum += v[j];
  const u64 x = warp_incl_sum(sum);
  if (l == 31) wsum[w] = x;
  __syncthreads();
  u64 off = 0;
  for (int ww = 0; ww < w; ++ww) off += wsum[ww];
  u64 run = texcl[blockIdx.x] + off + x - sum;
  TO o[SC_ITEMS];
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    o[j] = (TO)run;
    run += v[j];
  }
  if (full) {  // 16-B stores (out + base is 32-B / 64-B aligned)
    constexpr int PER16 = 16 / (int)sizeof(TO);
#pragma unroll
    for (int j = 0; j < SC_ITEMS; j += PER16) {
      if constexpr (sizeof(TO) == 8) {
        *reinterpret_cast<ulonglong2*>(out + base + j) = make_ulonglong2(o[j], o[j + 1]);
      } else {
        *reinterpret_cast<uint4*>(out + base + j) = make_uint4(o[j], o[j + 1], o[j + 2], o[j + 3]);
      }
    }
  } else {
#pragma unroll
    for (int j = 0; j < SC_ITEMS; ++j)
      if (base + j < n) out[base + j] = o[j];
  }
}

}  // namespace

// ------------------------------------------------------------------ host side
size_t scan_temp_bytes(u64 n);
size_t rs_temp_bytes(u64 n) {
  const u64 tiles = (n + RS_TILE - 1) / RS_TILE;
  // histograms + bases, then the (digit, tile) count / offset table of one pass
  return RS_HDR_BYTES + (size_t)(tiles ? tiles : 1) * RS_MAXB * sizeof(u32) + 256;
}

// Small sorts (n <= RS_SMALL, e.g. the K3 sync-skeleton tables, K1 of small traces): one CTA sorts in
// shared memory and gathers keys / values into the alternate buffers: one launch instead of four
// kernels per digit pass.
constexpr u32 RS_SMALL = 8192;
// One CTA, 1024 threads, up to RS_SMALL keys resident in shared memory: LSD radix passes of 8 bits
// over (digit, input index) pairs.  Per pass every warp ranks its 256 keys (32 consecutive keys per
// step, MATCH.ANY peers + per-warp running digit counts, so equal digits keep their order), the CTA
// turns the 32 x 256 warp counts into scatter bases (digit-major, warp-minor), and the pairs move to
// the other buffer -- 8 barriers per pass instead of a bitonic network's ~90.  The input index
// travels along, so the last step gathers keys / values from global memory in sorted order.
constexpr int SS_THREADS = 1024, SS_WARPS = SS_THREADS / 32, SS_PER = RS_SMALL / SS_THREADS;  // 8
constexpr size_t SS_SMEM = (size_t)RS_SMALL * 4 * sizeof(u32) + (size_t)SS_WARPS * 256 * sizeof(u32) + 64;
__global__ void __launch_bounds__(SS_THREADS) k_sort_small(const u32* __restrict__ kin, const u32* __restrict__ vin,
                                                           u32* __restrict__ kout, u32* __restrict__ vout, u64 n_max,
                                                           const u64* __restrict__ n_dev, int drop, int bit_lo,
                                                           int bits, u64* __restrict__ n_out) {
  extern __shared__ __align__(16) u32 ss[];
  u32* dA = ss;                      // digits-source keys (already shifted / masked), buffer A
  u32* iA = dA + RS_SMALL;           // input indices, buffer A
  u32* dB = iA + RS_SMALL;           // buffer B
  u32* iB = dB + RS_SMALL;
  u32* wh = iB + RS_SMALL;           // [SS_WARPS][256] warp digit counts -> scatter bases
  __shared__ u32 s_kept;
  const u32 t = threadIdx.x, w = t >> 5, l = t & 31;
  const u32 n = (u32)(n_dev ? *n_dev : n_max);
  const u32 dmask = bits >= 32 ? 0xFFFFFFFFu : ((1u << bits) - 1u);
  // compact the kept keys (drop: KEY_DROP removed) in input order: one warp-aggregated pass
  if (t == 0) s_kept = 0;
  __syncthreads();
  for (u32 c0 = 0; c0 < n; c0 += SS_THREADS) {
    const u32 i = c0 + t;
    const u32 k = i < n ? kin[i] : KEY_DROP;
    const bool keep = i < n && !(drop && k == KEY_DROP);
    const u32 bal = __ballot_sync(0xFFFFFFFFu, keep);
    __shared__ u32 s_wbase[SS_WARPS];
    if (l == 0) s_wbase[w] = __popc(bal);
    __syncthreads();
    if (t == 0) {  // 32 warp counts -> bases (tiny serial scan)
      u32 run = s_kept;
      for (u32 q = 0; q < SS_WARPS; ++q) {
        const u32 c = s_wbase[q];
        s_wbase[q] = run;
        run += c;
      }
      s_kept = run;
    }
    __syncthreads();
    if (keep) {
      const u32 at = s_wbase[w] + __popc(bal & lanemask_lt());
      dA[at] = (k >> bit_lo) & dmask;
      iA[at] = i;
    }
    __syncthreads();
  }
  const u32 nk = s_kept;
  const int passes = (bits + 7) / 8;
  for (int p = 0; p < passes; ++p) {
    const u32 sh = 8u * (u32)p;
    for (u32 q = t; q < SS_WARPS * 256; q += SS_THREADS) wh[q] = 0;
    __syncthreads();
    u32 rk[SS_PER], dg[SS_PER];
#pragma unroll
    for (int j = 0; j < SS_PER; ++j) {  // warp w owns keys [w*256, w*256+256), 32 per step in order
      const u32 i = (u32)w * 256u + (u32)j * 32u + l;
      const u32 d = i < nk ? (dA[i] >> sh) & 255u : 256u;
      const u32 peers = __match_any_sync(0xFFFFFFFFu, d);
      u32 old = 0;
      if (d < 256u) old = wh[w * 256 + d];
      __syncwarp();
      if (d < 256u && (peers & lanemask_lt()) == 0) wh[w * 256 + d] = old + __popc(peers);
      __syncwarp();
      dg[j] = d;
      rk[j] = old + __popc(peers & lanemask_lt());
    }
    __syncthreads();
    // scatter bases: digit-major, warp-minor exclusive prefix over the 32 x 256 counts
    if (t < 256) {
      u32 tot = 0;
      for (u32 q = 0; q < SS_WARPS; ++q) {
        const u32 c = wh[q * 256 + t];
        wh[q * 256 + t] = tot;
        tot += c;
      }
      // exclusive scan of the 256 digit totals (8 warps x 32)
      const u32 x = warp_incl_sum(tot);
      __shared__ u32 s_dsum[8];
      if (l == 31) s_dsum[w] = x;
      __syncwarp();
      asm volatile("bar.sync 1, 256;" ::: "memory");
      u32 off = 0;
      for (u32 q = 0; q < w; ++q) off += s_dsum[q];
      const u32 base = off + x - tot;
      for (u32 q = 0; q < SS_WARPS; ++q) wh[q * 256 + t] += base;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < SS_PER; ++j) {
      const u32 i = (u32)w * 256u + (u32)j * 32u + l;
      if (dg[j] < 256u) {
        const u32 at = wh[w * 256 + dg[j]] + rk[j];
        dB[at] = dA[i];
        iB[at] = iA[i];
      }
    }
    __syncthreads();
    u32* tmp = dA; dA = dB; dB = tmp;
    tmp = iA; iA = iB; iB = tmp;
  }
  for (u32 i = t; i < nk; i += SS_THREADS) {
    const u32 src = iA[i];
    kout[i] = kin[src];
    if (vout) vout[i] = vin[src];
  }
  if (t == 0 && n_out) *n_out = nk;
}

// One pass of RB-bit digits at `shift` (pass index p: its row of the digit-total tables).
template <int RB>
static void rs_pass(u32*& ki, u32*& vi, u32*& ko, u32*& vo, u64 n, const u64*& nd, int shift, int p, bool dr,
                    void* temp, cudaStream_t st, u64* n_out_dev) {
  constexpr int BINS = 1 << RB;
  const u64 tiles = (n + RS_TILE - 1) / RS_TILE;
  u32* ghist = (u32*)temp;                           // [RS_MAXP][RS_MAXB]
  u32* gbase = ghist + RS_MAXP * RS_MAXB;            // [RS_MAXP][RS_MAXB]
  u32* counts = (u32*)((char*)temp + RS_HDR_BYTES);  // [BINS][tiles]
  static int grid_of[64] = {};  // per device: shared-memory opt-in + occupancy-derived persistent grid
  constexpr size_t dsmem = rs_dsmem<RB>();
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) dev = 0;
  if (!grid_of[dev]) {
    int sms = 148, per = 1;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaFuncSetAttribute(k_rs_down<RB>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsmem);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_rs_down<RB>, RS_THREADS, dsmem);
    grid_of[dev] = sms * (per > 0 ? per : 1);
  }
  const int down_grid = grid_of[dev];
  k_rs_up<RB><<<(unsigned)tiles, RS_THREADS, 0, st>>>(ki, n, nd, dr ? 1 : 0, shift, counts, tiles); ++g_launches;
  k_rs_rows<<<BINS, RS_THREADS, 0, st>>>(counts, tiles, ghist + p * RS_MAXB); ++g_launches;
  // the digit bases come from the downsweep's own scan of the row totals, unless the kept count it
  // publishes would overwrite the item count the same launch reads (n_dev == n_out_dev)
  const bool fused = RS_FUSED_BINS && !(dr && nd == n_out_dev);
  if (!fused) {
    k_rs_bins<RB><<<1, BINS < 1024 ? BINS : 1024, 0, st>>>(ghist + p * RS_MAXB, gbase + p * RS_MAXB,
                                                          dr ? n_out_dev : nullptr);
    ++g_launches;
  }
  k_rs_down<RB><<<(unsigned)std::min<u64>(tiles, (u64)down_grid), RS_THREADS, dsmem, st>>>(
      ki, vi, ko, vo, n, nd, dr ? 1 : 0, shift, counts, tiles, gbase + p * RS_MAXB,
      fused ? ghist + p * RS_MAXB : nullptr, fused && dr ? n_out_dev : nullptr);
  ++g_launches;
  if (dr) nd = n_out_dev;
  u32* tk = ki; ki = ko; ko = tk;
  u32* tv = vi; vi = vo; vo = tv;
}

static void rs_pass_any(int rb, u32*& ki, u32*& vi, u32*& ko, u32*& vo, u64 n, const u64*& nd, int shift, int p,
                        bool dr, void* temp, cudaStream_t st, u64* n_out_dev) {
  if (rb == 8) rs_pass<8>(ki, vi, ko, vo, n, nd, shift, p, dr, temp, st, n_out_dev);
  else if (rb == 9) rs_pass<9>(ki, vi, ko, vo, n, nd, shift, p, dr, temp, st, n_out_dev);
  else if (rb == 10) rs_pass<10>(ki, vi, ko, vo, n, nd, shift, p, dr, temp, st, n_out_dev);
  else rs_pass<11>(ki, vi, ko, vo, n, nd, shift, p, dr, temp, st, n_out_dev);
}

// Stable sort of (keys, vals) by key bits [bit_lo, bit_hi) (vals may be null: keys only).  Result is
// in (keys, vals) when the function returns false, else in (keys_alt, vals_alt).  n is the (upper
// bound of the) item count; with n_dev the exact count is read on the device.  drop: the first pass
// removes items whose key is KEY_DROP and writes the number kept to *n_out_dev (at least one pass
// is run).  Digit width: the fewest passes of at most 10 bits, each pass 8, 9 or 10 bits wide.  Per
// pass: k_rs_up (digit counts per tile) -> k_rs_rows (independent per-digit row scans + totals) ->
// k_rs_bins (digit bases from the totals) -> k_rs_down (rank + scatter).
bool radix_sort_pairs(u32* keys, u32* vals, u32* keys_alt, u32* vals_alt, u64 n, int bit_lo, int bit_hi, void* temp,
                      cudaStream_t st, const u64* n_dev, u64* n_out_dev, bool drop) {
  if (!drop && (n <= 1 || bit_hi <= bit_lo)) return false;
  if (n == 0) {
    if (n_out_dev) cudaMemsetAsync(n_out_dev, 0, 8, st);
    return false;
  }
  const int bits = std::max(bit_hi - bit_lo, 1);
  if (n <= RS_SMALL) {
    static bool attr[64] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if (!attr[dev]) {
      cudaFuncSetAttribute(k_sort_small, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SS_SMEM);
      attr[dev] = true;
    }
    k_sort_small<<<1, SS_THREADS, SS_SMEM, st>>>(keys, vals, keys_alt, vals_alt, n, n_dev, drop ? 1 : 0, bit_lo,
                                                 bits, drop ? n_out_dev : nullptr);
    ++g_launches;
    return true;
  }
  static int maxb = 0;
  if (!maxb) {
    const char* e = getenv("BC_RS_MAXBITS");  // widest digit of a multi-pass sort (8..10); experiments only
    maxb = e ? std::max(8, std::min(10, atoi(e))) : 10;
  }
  // an 11-bit digit only when it makes the sort single-pass (K1 of 2048-warp traces): the 2048-bin
  // downsweep runs one CTA per SM, which loses to one more 8-10-bit pass when both need passes
  const int mb = bits == 11 ? 11 : maxb;
  const int passes = std::min((bits + mb - 1) / mb, RS_MAXP);
  // digit widths: the fewest passes; the extra bits of a uniform split go to the first passes only
  // (bits - 8 * passes of them): the other passes run 8-bit digits (256 bins: longer digit runs per
  // tile, better-coalesced scatter) -- e.g. 25 bits as 9 + 8 + 8 rather than 9 + 9 + 9
  u32 *ki = keys, *vi = vals, *ko = keys_alt, *vo = vals_alt;
  const u64* nd = n_dev;
  int shift = bit_lo, left = bits;
  for (int p = 0; p < passes; ++p) {
    const int rem = passes - p;
    const int rb = std::max(8, std::min(mb, (left + rem - 1) / rem));
    rs_pass_any(rb, ki, vi, ko, vo, n, nd, shift, p, drop && p == 0, temp, st, n_out_dev);
    shift += rb;
    left -= rb;
  }
  return (passes & 1) != 0;
}

size_t scan_temp_bytes(u64 n) { return ((n + SC_TILE - 1) / SC_TILE + 1) * sizeof(u64) + 64; }

// exclusive scan in -> out (out may alias in); total written to *total_dev if non-null
template <typename TO>
static void exclusive_scan_t(const u32* in, TO* out, u64 n, void* temp, u64* total_dev, cudaStream_t st) {
  const u64 tiles = (n + SC_TILE - 1) / SC_TILE;
  u64* tsum = (u64*)temp;
  if (tiles == 0) {
    if (total_dev) cudaMemsetAsync(total_dev, 0, 8, st);
    return;
  }
  if (n <= SC_SMALL) {
    k_scan_small<TO><<<1, 1024, 0, st>>>(in, out, n, total_dev); ++g_launches;
    return;
  }
  k_scan_tsum<<<(unsigned)tiles, SC_THREADS, 0, st>>>(in, n, tsum); ++g_launches;
  k_scan_tiles<<<1, 1024, 0, st>>>(tsum, tiles, total_dev); ++g_launches;
  k_scan_u32<TO><<<(unsigned)tiles, SC_THREADS, 0, st>>>(in, out, n, tsum); ++g_launches;
}
void exclusive_scan_u32(const u32* in, u32* out, u64 n, void* temp, u64* total_dev, cudaStream_t st) {
  exclusive_scan_t<u32>(in, out, n, temp, total_dev, st);
}
// u64 prefix of u32 values (record window weights: totals beyond 2^32)
void exclusive_scan_u32_u64(const u32* in, u64* out, u64 n, void* temp, u64* total_dev, cudaStream_t st) {
  exclusive_scan_t<u64>(in, out, n, temp, total_dev, st);
}

void preload_sort() {
  preload(k_rs_bins<8>, k_rs_bins<9>, k_rs_bins<10>, k_rs_bins<11>, k_rs_up<8>, k_rs_up<9>, k_rs_up<10>, k_rs_up<11>,
          k_rs_down<8>, k_rs_down<9>, k_rs_down<10>, k_rs_down<11>, k_rs_rows, k_sort_small, k_scan_small<u32>,
          k_scan_small<u64>, k_scan_u32<u32>, k_scan_u32<u64>, k_scan_tiles, k_scan_tsum);
}

}  // namespace bc
