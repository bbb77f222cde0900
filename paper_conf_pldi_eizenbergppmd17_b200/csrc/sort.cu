// sort.cu — hand-written stable LSD radix sort (8-bit digits, reduce-then-scan per pass) and a
// device-wide exclusive scan, for sm_100a.
//
// The radix sort is the paper's per-location serialisation (a spinlock per shadow
// entry orders the host threads' accesses) turned into data parallelism: a STABLE sort of
// (location key, trace position) items groups each location's accesses into one contiguous
// segment that is still in trace order.
//   k_rs_hist  : one read of the keys -> the global 256-bin histogram of every digit pass
//   k_rs_bins  : exclusive scan of each pass's histogram (digit start offsets); kept-item count
//   k_rs_up    : per 4096-key tile, the digit counts (reads 4 B / item)
//   k_rs_rows  : one CTA per digit scans that digit's counts over all tiles (256 independent rows:
//                no serial chain across tiles, unlike a decoupled look-back whose first wave of
//                ~450 co-resident tiles walks back one L2 round trip per step)
//   k_rs_down  : per tile: stable in-tile rank (ballot match + per-warp histograms), scatter through
//                shared memory so that each digit's run is written contiguously (8 B in, 8 B out).
#include <algorithm>

#include "common.cuh"
#include "kernels.cuh"

namespace bc {

namespace {

constexpr int RS_THREADS = 256;
constexpr int RS_ITEMS = 16;
constexpr int RS_TILE = RS_THREADS * RS_ITEMS;  // 4096
constexpr int RS_WARPS = RS_THREADS / 32;
constexpr int RS_BINS = 256;
constexpr int RS_MAXP = 4;
// temp header: ghist[RS_MAXP][256], gbase[RS_MAXP][256]; the (digit, tile) table follows
constexpr size_t RS_HDR_BYTES = (2 * RS_MAXP * 256 + 64) * sizeof(u32);

// Lanes of the warp holding the same 9-bit label (digit, or 256 = no item): 9 ballots, a fixed
// cost independent of how many distinct digits the warp holds.
__device__ __forceinline__ u32 match9(u32 d) {
  u32 m = 0xFFFFFFFFu;
#pragma unroll
  for (int b = 0; b < 9; ++b) {
    const bool bit = (d >> b) & 1u;
    const u32 bal = __ballot_sync(0xFFFFFFFFu, bit);
    m &= bit ? bal : ~bal;
  }
  return m;
}

constexpr int RS_HIST_ITEMS = 8;

// Global digit histograms of all passes in one read.  Same-digit keys of a warp are combined
// (match9) before the shared-memory atomic (sorted-ish inputs hit one bin hard).  Each thread keeps
// RS_HIST_ITEMS loads in flight.
__global__ void __launch_bounds__(RS_THREADS) k_rs_hist(const u32* __restrict__ kin, u64 n_max,
                                                        const u64* __restrict__ n_dev, int drop, int bit_lo,
                                                        int passes, u32* __restrict__ ghist) {
  __shared__ u32 h[RS_MAXP][RS_BINS];
  const int t = threadIdx.x;
  for (int i = t; i < RS_MAXP * RS_BINS; i += RS_THREADS) (&h[0][0])[i] = 0;
  __syncthreads();
  const u64 n = n_dev ? *n_dev : n_max;
  const u32 lt = lanemask_lt();
  constexpr int CH = RS_THREADS * RS_HIST_ITEMS;
  const u64 stride = (u64)gridDim.x * CH;
  for (u64 base = (u64)blockIdx.x * CH; base < n; base += stride) {
    u32 k[RS_HIST_ITEMS];
#pragma unroll
    for (int j = 0; j < RS_HIST_ITEMS; ++j) {
      const u64 idx = base + (u64)j * RS_THREADS + t;
      k[j] = idx < n ? kin[idx] : KEY_DROP;
    }
#pragma unroll
    for (int j = 0; j < RS_HIST_ITEMS; ++j) {
      const u64 idx = base + (u64)j * RS_THREADS + t;
      const bool ok = idx < n && !(drop && k[j] == KEY_DROP);
      const u32 vm = __ballot_sync(0xFFFFFFFFu, ok);
      for (int p = 0; p < passes; ++p) {
        const u32 d = ok ? (k[j] >> (bit_lo + 8 * p)) & 0xFFu : 0x100u;
        // one digit across the warp (the common case for the high digits): one atomic
        const u32 d0 = __shfl_sync(0xFFFFFFFFu, d, vm ? __ffs(vm) - 1 : 0);
        if (__all_sync(0xFFFFFFFFu, !ok || d == d0)) {
          if (vm && (lt & vm) == 0 && ok) atomicAdd(&h[p][d], (u32)__popc(vm));
        } else if (ok) {
          atomicAdd(&h[p][d], 1u);
        }
      }
    }
  }
  __syncthreads();
  for (int i = t; i < passes * RS_BINS; i += RS_THREADS) {
    const u32 v = (&h[0][0])[i];
    if (v) atomicAdd(&ghist[i], v);
  }
}

// gbase[p][d] = exclusive prefix of ghist[p][*]; *n_out = kept items (pass 0 total)
__global__ void __launch_bounds__(RS_BINS) k_rs_bins(const u32* __restrict__ ghist, u32* __restrict__ gbase,
                                                     u64* __restrict__ n_out) {
  __shared__ u32 wsum[RS_BINS / 32];
  const int t = threadIdx.x, w = t >> 5, l = t & 31, p = blockIdx.x;
  const u32 v = ghist[p * RS_BINS + t];
  const u32 x = warp_incl_sum(v);
  if (l == 31) wsum[w] = x;
  __syncthreads();
  u32 off = 0, tot = 0;
  for (int ww = 0; ww < RS_BINS / 32; ++ww) {
    if (ww < w) off += wsum[ww];
    tot += wsum[ww];
  }
  gbase[p * RS_BINS + t] = off + x - v;
  if (p == 0 && t == 0 && n_out) *n_out = tot;
}

// Upsweep of one pass: the digit counts of every tile, digit-major (counts[d * tiles + tile]);
// tiles past the (device-side) item count write zeros.
__global__ void __launch_bounds__(RS_THREADS) k_rs_up(const u32* __restrict__ kin, u64 n_max,
                                                      const u64* __restrict__ n_dev, int drop, int shift,
                                                      u32* __restrict__ counts, u64 tiles) {
  __shared__ u32 h[RS_BINS];
  const int t = threadIdx.x;
  h[t] = 0;
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
      const u32 d = ok ? (k[j] >> shift) & 0xFFu : 0x100u;
      const u32 vm = __ballot_sync(0xFFFFFFFFu, ok);
      const u32 d0 = __shfl_sync(0xFFFFFFFFu, d, vm ? __ffs(vm) - 1 : 0);
      if (__all_sync(0xFFFFFFFFu, !ok || d == d0)) {
        if (vm && (lt & vm) == 0 && ok) atomicAdd(&h[d], (u32)__popc(vm));
      } else if (ok) {
        atomicAdd(&h[d], 1u);
      }
    }
  }
  __syncthreads();
  counts[(u64)t * tiles + blockIdx.x] = h[t];
}

// One CTA per digit d: offs[d * tiles + tile] = gbase[d] + (items of digit d in tiles < tile).
// The 256 rows are independent, so there is no serial chain across tiles.
__global__ void __launch_bounds__(RS_THREADS) k_rs_rows(u32* __restrict__ counts, u64 tiles,
                                                        const u32* __restrict__ gbase) {
  __shared__ u32 wsum[RS_WARPS];
  __shared__ u32 s_carry;
  const int t = threadIdx.x, w = t >> 5, l = t & 31, d = blockIdx.x;
  u32* row = counts + (u64)d * tiles;
  if (t == 0) s_carry = gbase[d];
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
}

// Downsweep of one pass: stable in-tile rank (ballot match + per-warp histograms), scatter through
// shared memory so that each digit's run is written contiguously (8 B in, 8 B out per item).
// Persistent CTAs; each tile's keys and values arrive in shared memory by 1-D TMA bulk copies issued
// RS_DSTAGES tiles ahead (mbarrier ring), so the global-load latency that dominated a one-tile-per-CTA
// kernel overlaps the ranking and scattering of the previous tile.  The staged keys are read in input
// order for ranking; once scattered, the stage's key half holds the permuted values.
constexpr int RS_DSTAGES = 2;
constexpr size_t RS_DSMEM = (size_t)RS_DSTAGES * 2 * RS_TILE * sizeof(u32) + RS_TILE * sizeof(u32) +
                            RS_WARPS * RS_BINS * sizeof(u32) + 3 * RS_BINS * sizeof(u32) + 64 + RS_DSTAGES * 8;

__global__ void __launch_bounds__(RS_THREADS, 2) k_rs_down(const u32* __restrict__ kin, const u32* __restrict__ vin,
                                                           u32* __restrict__ kout, u32* __restrict__ vout, u64 n_max,
                                                           const u64* __restrict__ n_dev, int drop, int shift,
                                                           const u32* __restrict__ offs, u64 tiles) {
  extern __shared__ __align__(128) unsigned char rs_smem[];
  u32* stage = reinterpret_cast<u32*>(rs_smem);                 // [RS_DSTAGES][2][RS_TILE] (keys, vals)
  u32* skeys = stage + RS_DSTAGES * 2 * RS_TILE;                // [RS_TILE]
  u32(*whist)[RS_BINS] = reinterpret_cast<u32(*)[RS_BINS]>(skeys + RS_TILE);
  u32* tofs = &whist[RS_WARPS][0];
  u32* gstart = tofs + RS_BINS;
  u32* wsum = gstart + RS_BINS;                                 // [RS_WARPS]
  u32* s_kept = wsum + RS_WARPS;
  u64* bar = reinterpret_cast<u64*>(rs_smem + RS_DSMEM - RS_DSTAGES * 8);

  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  const u64 n = n_dev ? *n_dev : n_max;
  const u64 n_tiles = (n + RS_TILE - 1) / RS_TILE;
  auto issue = [&](u64 tile, int st) {
    const u64 base = tile * RS_TILE;
    const u64 cnt = n - base < (u64)RS_TILE ? n - base : (u64)RS_TILE;
    const u32 bytes = (u32)(((cnt + 3) & ~3ull) * sizeof(u32));  // whole 16-B units (buffers are padded)
    mbar_expect_tx(&bar[st], vin ? 2 * bytes : bytes);
    bulk_g2s(stage + st * 2 * RS_TILE, kin + base, bytes, &bar[st]);
    if (vin) bulk_g2s(stage + st * 2 * RS_TILE + RS_TILE, vin + base, bytes, &bar[st]);
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
  u32 it = 0;
  for (u64 tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
    const int st = (int)(it % RS_DSTAGES);
    const u32 phase = (it / RS_DSTAGES) & 1u;
    u32* sk = stage + st * 2 * RS_TILE;
    u32* sv = sk + RS_TILE;
    const u64 base = tile * RS_TILE;
    for (int i = t; i < RS_WARPS * RS_BINS; i += RS_THREADS) (&whist[0][0])[i] = 0;
    gstart[t] = offs[(u64)t * tiles + tile];
    __syncthreads();
    mbar_wait(&bar[st], phase);
    u32 rank[RS_ITEMS];  // (digit << 16) | rank in the warp's digit run, NONE = no item
#pragma unroll
    for (int j = 0; j < RS_ITEMS; ++j) {
      const u32 li = w * (RS_ITEMS * 32) + j * 32 + l;
      const u64 idx = base + li;
      const u32 k = idx < n ? sk[li] : KEY_DROP;
      const u32 d = (idx < n && !(drop && k == KEY_DROP)) ? ((k >> shift) & 0xFFu) : 256u;
      const u32 peers = match9(d);
      const u32 old = d < 256u ? whist[w][d] : 0u;
      __syncwarp();
      if (d < 256u && (peers & lt) == 0) whist[w][d] = old + __popc(peers);
      __syncwarp();
      rank[j] = d < 256u ? ((d << 16) | (old + __popc(peers & lt))) : NONE;
    }
    __syncthreads();
    // per digit (thread t): prefix over warps, tile total; tile-local exclusive scan of the totals
    u32 total = 0;
#pragma unroll
    for (int ww = 0; ww < RS_WARPS; ++ww) {
      const u32 c = whist[ww][t];
      whist[ww][t] = total;
      total += c;
    }
    {
      const u32 x = warp_incl_sum(total);
      if (l == 31) wsum[w] = x;
      __syncthreads();
      u32 off = 0;
      for (int ww = 0; ww < w; ++ww) off += wsum[ww];
      tofs[t] = off + x - total;
      if (t == RS_BINS - 1) *s_kept = off + x;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < RS_ITEMS; ++j) {
      if (rank[j] != NONE) {
        const u32 d = rank[j] >> 16;
        skeys[tofs[d] + whist[w][d] + (rank[j] & 0xFFFFu)] = sk[w * (RS_ITEMS * 32) + j * 32 + l];
      }
    }
    __syncthreads();
    const u32 tile_n = *s_kept;
    for (u32 q = t; q < tile_n; q += RS_THREADS) {
      const u32 kk = skeys[q];
      const u32 d = (kk >> shift) & 0xFFu;
      kout[(u64)gstart[d] + (q - tofs[d])] = kk;
    }
    if (vout) {
      // values: the same permutation, staged in the stage's (now consumed) key half
#pragma unroll
      for (int j = 0; j < RS_ITEMS; ++j) {
        if (rank[j] != NONE) {
          const u32 d = rank[j] >> 16;
          sk[tofs[d] + whist[w][d] + (rank[j] & 0xFFFFu)] = sv[w * (RS_ITEMS * 32) + j * 32 + l];
        }
      }
      __syncthreads();
      for (u32 q = t; q < tile_n; q += RS_THREADS) {
        const u32 d = (skeys[q] >> shift) & 0xFFu;
        vout[(u64)gstart[d] + (q - tofs[d])] = sk[q];
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

__global__ void __launch_bounds__(SC_THREADS) k_scan_u32(const u32* __restrict__ in, u32* __restrict__ out, u64 n,
                                                         const u64* __restrict__ texcl) {
  __shared__ u64 wsum[SC_THREADS / 32];
  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  const u64 base = (u64)blockIdx.x * SC_TILE + (u64)t * SC_ITEMS;
  u32 v[SC_ITEMS];
  u64 sum = 0;
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    v[j] = base + j < n ? in[base + j] : 0u;
    sum += v[j];
  }
  const u64 x = warp_incl_sum(sum);
  if (l == 31) wsum[w] = x;
  __syncthreads();
  u64 off = 0;
  for (int ww = 0; ww < w; ++ww) off += wsum[ww];
  u64 run = texcl[blockIdx.x] + off + x - sum;
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    if (base + j < n) out[base + j] = (u32)run;
    run += v[j];
  }
}

}  // namespace

// ------------------------------------------------------------------ host side
size_t scan_temp_bytes(u64 n);
size_t rs_temp_bytes(u64 n) {
  const u64 tiles = (n + RS_TILE - 1) / RS_TILE;
  // histograms + bases, then the (digit, tile) count / offset table of one pass
  return RS_HDR_BYTES + (size_t)(tiles ? tiles : 1) * RS_BINS * sizeof(u32) + 256;
}

// Stable sort of (keys, vals) by key bits [bit_lo, bit_hi) (vals may be null: keys only).  Result is
// in (keys, vals) when the function returns false, else in (keys_alt, vals_alt).  n is the (upper
// bound of the) item count; with n_dev the exact count is read on the device.  drop: the first pass
// removes items whose key is KEY_DROP and writes the number kept to *n_out_dev (at least one pass
// is run).  Per pass: k_rs_up (digit counts per tile) -> k_rs_rows (256 independent row scans) ->
// k_rs_down (rank + scatter); one k_rs_hist read up front gives every pass's digit bases.
bool radix_sort_pairs(u32* keys, u32* vals, u32* keys_alt, u32* vals_alt, u64 n, int bit_lo, int bit_hi, void* temp,
                      cudaStream_t st, const u64* n_dev, u64* n_out_dev, bool drop) {
  if (!drop && (n <= 1 || bit_hi <= bit_lo)) return false;
  if (n == 0) {
    if (n_out_dev) cudaMemsetAsync(n_out_dev, 0, 8, st);
    return false;
  }
  int passes = (bit_hi - bit_lo + 7) / 8;
  if (passes > RS_MAXP) passes = RS_MAXP;
  if (passes < 1) passes = 1;
  const u64 tiles = (n + RS_TILE - 1) / RS_TILE;
  u32* ghist = (u32*)temp;                           // [RS_MAXP][256]
  u32* gbase = ghist + RS_MAXP * RS_BINS;            // [RS_MAXP][256]
  u32* counts = (u32*)((char*)temp + RS_HDR_BYTES);  // [256][tiles]
  cudaMemsetAsync(ghist, 0, RS_MAXP * RS_BINS * sizeof(u32), st);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  static int down_grid = 0;
  if (!down_grid) {
    int per = 1;
    cudaFuncSetAttribute(k_rs_down, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)RS_DSMEM);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_rs_down, RS_THREADS, RS_DSMEM);
    down_grid = sms * (per > 0 ? per : 1);
  }
  const unsigned hgrid =
      (unsigned)std::min<u64>((n + RS_THREADS * RS_HIST_ITEMS - 1) / (RS_THREADS * RS_HIST_ITEMS), (u64)sms * 8);
  k_rs_hist<<<hgrid, RS_THREADS, 0, st>>>(keys, n, n_dev, drop ? 1 : 0, bit_lo, passes, ghist); ++g_launches;
  k_rs_bins<<<passes, RS_BINS, 0, st>>>(ghist, gbase, drop ? n_out_dev : nullptr); ++g_launches;
  u32 *ki = keys, *vi = vals, *ko = keys_alt, *vo = vals_alt;
  const u64* nd = n_dev;
  for (int p = 0; p < passes; ++p) {
    const int shift = bit_lo + 8 * p;
    const int dr = (drop && p == 0) ? 1 : 0;
    k_rs_up<<<(unsigned)tiles, RS_THREADS, 0, st>>>(ki, n, nd, dr, shift, counts, tiles); ++g_launches;
    k_rs_rows<<<RS_BINS, RS_THREADS, 0, st>>>(counts, tiles, gbase + p * RS_BINS); ++g_launches;
    k_rs_down<<<(unsigned)std::min<u64>(tiles, (u64)down_grid), RS_THREADS, RS_DSMEM, st>>>(ki, vi, ko, vo, n, nd, dr,
                                                                                           shift, counts, tiles);
    ++g_launches;
    if (dr) nd = n_out_dev;
    u32* tk = ki; ki = ko; ko = tk;
    u32* tv = vi; vi = vo; vo = tv;
  }
  return (passes & 1) != 0;
}

size_t scan_temp_bytes(u64 n) { return ((n + SC_TILE - 1) / SC_TILE + 1) * sizeof(u64) + 64; }

// exclusive scan in -> out (out may alias in); total written to *total_dev if non-null
void exclusive_scan_u32(const u32* in, u32* out, u64 n, void* temp, u64* total_dev, cudaStream_t st) {
  const u64 tiles = (n + SC_TILE - 1) / SC_TILE;
  u64* tsum = (u64*)temp;
  if (tiles == 0) {
    if (total_dev) cudaMemsetAsync(total_dev, 0, 8, st);
    return;
  }
  k_scan_tsum<<<(unsigned)tiles, SC_THREADS, 0, st>>>(in, n, tsum); ++g_launches;
  k_scan_tiles<<<1, 1024, 0, st>>>(tsum, tiles, total_dev); ++g_launches;
  k_scan_u32<<<(unsigned)tiles, SC_THREADS, 0, st>>>(in, out, n, tsum); ++g_launches;
}

}  // namespace bc
