// sort.cu — hand-written stable LSD radix sort (onesweep-style, decoupled look-back) and
// device-wide exclusive scan for sm_100a.
//
// The radix sort is the paper's per-location serialisation (a spinlock per shadow
// entry orders the host threads' accesses) turned into data parallelism: a STABLE sort of
// (location key, trace position) items groups each location's accesses into one contiguous
// segment that is still in trace order.  8-bit digits, 4096 keys per tile, one global
// per pass: upsweep (per-tile digit counts), one exclusive scan over (digit, tile), downsweep
// (stable in-tile rank, scatter through shared memory).
#include "common.cuh"
#include "kernels.cuh"

namespace bc {

namespace {

constexpr int RS_THREADS = 256;
constexpr int RS_ITEMS = 16;
constexpr int RS_TILE = RS_THREADS * RS_ITEMS;  // 4096
constexpr int RS_WARPS = RS_THREADS / 32;
constexpr int RS_BINS = 256;

// upsweep: per-tile digit counts, digit-major (counts[d * tiles + tile]) so that one exclusive
// scan gives every (digit, tile) its global output offset
// n = *n_dev when n_dev is set (item count known only on the device), else n_max.
// drop: keys equal to KEY_DROP are not counted (first pass of a compacting sort).
__global__ void __launch_bounds__(RS_THREADS) k_rs_upsweep(const u32* __restrict__ kin, u64 n_max,
                                                           const u64* __restrict__ n_dev, int drop, int shift,
                                                           u64 tiles, u32* __restrict__ counts) {
  __shared__ u32 h[RS_BINS];
  const int t = threadIdx.x;
  const u64 n = n_dev ? *n_dev : n_max;
  h[t] = 0;
  __syncthreads();
  const u64 base = (u64)blockIdx.x * RS_TILE;
#pragma unroll 4
  for (int j = 0; j < RS_ITEMS; ++j) {
    u64 idx = base + (u64)j * RS_THREADS + t;
    if (idx < n) {
      const u32 k = kin[idx];
      if (!(drop && k == KEY_DROP)) atomicAdd(&h[(k >> shift) & 0xFFu], 1u);
    }
  }
  __syncthreads();
  counts[(u64)t * tiles + blockIdx.x] = h[t];
}

// downsweep: stable rank inside the tile, then scatter through shared memory
__global__ void __launch_bounds__(RS_THREADS, 2) k_rs_downsweep(const u32* __restrict__ kin, const u32* __restrict__ vin,
                                                               u32* __restrict__ kout, u32* __restrict__ vout, u64 n_max,
                                                               const u64* __restrict__ n_dev, int drop, int shift,
                                                               const u32* __restrict__ offs, u64 tiles) {
  __shared__ u32 skeys[RS_TILE];
  __shared__ u32 svals[RS_TILE];
  __shared__ u32 whist[RS_WARPS][RS_BINS];
  __shared__ u32 tofs[RS_BINS];
  __shared__ u32 gstart[RS_BINS];
  __shared__ u32 s_kept;

  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  const u64 n = n_dev ? *n_dev : n_max;
  const u32 tile = blockIdx.x;
  const u64 base = (u64)tile * RS_TILE;
  if (base >= n) return;
  for (int i = t; i < RS_WARPS * RS_BINS; i += RS_THREADS) (&whist[0][0])[i] = 0;
  __syncthreads();

  u32 k[RS_ITEMS], rank[RS_ITEMS];
#pragma unroll
  for (int j = 0; j < RS_ITEMS; ++j) {
    u64 idx = base + (u64)w * (RS_ITEMS * 32) + j * 32 + l;
    k[j] = idx < n ? kin[idx] : 0u;
  }
  const u32 lt = lanemask_lt();
#pragma unroll
  for (int j = 0; j < RS_ITEMS; ++j) {
    u64 idx = base + (u64)w * (RS_ITEMS * 32) + j * 32 + l;
    u32 d = (idx < n && !(drop && k[j] == KEY_DROP)) ? ((k[j] >> shift) & 0xFFu) : 256u;
    u32 peers = __match_any_sync(0xFFFFFFFFu, d);
    u32 old = d < 256u ? whist[w][d] : 0u;
    __syncwarp();
    if (d < 256u && (peers & lt) == 0) whist[w][d] = old + __popc(peers);
    __syncwarp();
    rank[j] = old + __popc(peers & lt);
  }
  __syncthreads();
  // per digit: exclusive prefix over warps, tile total
  u32 total = 0;
#pragma unroll
  for (int ww = 0; ww < RS_WARPS; ++ww) {
    u32 c = whist[ww][t];
    whist[ww][t] = total;
    total += c;
  }
  gstart[t] = offs[(u64)t * tiles + tile];
  // tile-local exclusive scan of totals over digits
  {
    u32 x = warp_incl_sum(total);
    __shared__ u32 wsum[RS_WARPS];
    if (l == 31) wsum[w] = x;
    __syncthreads();
    u32 off = 0;
    for (int ww = 0; ww < w; ++ww) off += wsum[ww];
    tofs[t] = off + x - total;
    if (t == RS_BINS - 1) s_kept = off + x;  // kept items of the tile
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < RS_ITEMS; ++j) {
    u64 idx = base + (u64)w * (RS_ITEMS * 32) + j * 32 + l;
    if (idx < n && !(drop && k[j] == KEY_DROP)) {
      u32 d = (k[j] >> shift) & 0xFFu;
      u32 pos = tofs[d] + whist[w][d] + rank[j];
      skeys[pos] = k[j];
      svals[pos] = vin[idx];
    }
  }
  __syncthreads();
  const u32 tile_n = s_kept;
  for (u32 q = t; q < tile_n; q += RS_THREADS) {
    u32 kk = skeys[q];
    u32 d = (kk >> shift) & 0xFFu;
    u64 op = (u64)gstart[d] + (q - tofs[d]);
    kout[op] = kk;
    vout[op] = svals[q];
  }
}

// ---------------------------------------------------------------------- scan
constexpr int SC_THREADS = 256, SC_ITEMS = 8, SC_TILE = SC_THREADS * SC_ITEMS;

__global__ void __launch_bounds__(SC_THREADS) k_scan_u32(const u32* __restrict__ in, u32* __restrict__ out, u64 n,
                                                         u64* status, u32* tile_counter, u64* total_out) {
  __shared__ u32 s_tile;
  __shared__ u64 wsum[SC_THREADS / 32];
  __shared__ u64 s_excl;
  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  if (t == 0) s_tile = atomicAdd(tile_counter, 1u);
  __syncthreads();
  const u32 tile = s_tile;
  const u64 base = (u64)tile * SC_TILE + (u64)t * SC_ITEMS;
  u32 v[SC_ITEMS];
  u64 sum = 0;
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    v[j] = base + j < n ? in[base + j] : 0u;
    sum += v[j];
  }
  u64 x = warp_incl_sum(sum);
  if (l == 31) wsum[w] = x;
  __syncthreads();
  u64 off = 0, agg = 0;
  for (int ww = 0; ww < SC_THREADS / 32; ++ww) {
    if (ww < w) off += wsum[ww];
    agg += wsum[ww];
  }
  if (w == 0) {
    u64 e = lookback_u64_warp(status, tile, agg, l);
    if (l == 0) s_excl = e;
  }
  __syncthreads();
  u64 run = s_excl + off + x - sum;
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    if (base + j < n) out[base + j] = (u32)run;
    run += v[j];
  }
  if (total_out && base < n && base + SC_ITEMS >= n) *total_out = run;
  if (total_out && n == 0 && tile == 0 && t == 0) *total_out = 0;
}

}  // namespace

// ------------------------------------------------------------------ host side
size_t scan_temp_bytes(u64 n);
size_t rs_temp_bytes(u64 n) {
  u64 tiles = (n + RS_TILE - 1) / RS_TILE;
  return ((tiles * RS_BINS * sizeof(u32) + 255) & ~(u64)255) + scan_temp_bytes(tiles * RS_BINS) + 256;
}

// Stable sort of (keys, vals) by key bits [bit_lo, bit_hi).  Result is in (keys, vals) when
// the function returns false, else in (keys_alt, vals_alt).  n is the (upper bound of the) item
// count; with n_dev the exact count is read on the device.  drop: the first pass removes items
// whose key is KEY_DROP and writes the number kept to *n_out_dev (at least one pass is run).
bool radix_sort_pairs(u32* keys, u32* vals, u32* keys_alt, u32* vals_alt, u64 n, int bit_lo, int bit_hi, void* temp,
                      cudaStream_t st, const u64* n_dev, u64* n_out_dev, bool drop) {
  if (!drop && (n <= 1 || bit_hi <= bit_lo)) return false;
  if (n == 0) {
    if (n_out_dev) cudaMemsetAsync(n_out_dev, 0, 8, st);
    return false;
  }
  int passes = (bit_hi - bit_lo + 7) / 8;
  if (passes > 4) passes = 4;
  if (passes < 1) passes = 1;
  const u64 tiles = (n + RS_TILE - 1) / RS_TILE;
  u32* counts = (u32*)temp;
  void* stemp = (char*)temp + ((tiles * RS_BINS * sizeof(u32) + 255) & ~(u64)255);
  u32 *ki = keys, *vi = vals, *ko = keys_alt, *vo = vals_alt;
  const u64* nd = n_dev;
  for (int p = 0; p < passes; ++p) {
    const int shift = bit_lo + 8 * p;
    const int dr = (drop && p == 0) ? 1 : 0;
    k_rs_upsweep<<<(unsigned)tiles, RS_THREADS, 0, st>>>(ki, n, nd, dr, shift, tiles, counts); ++g_launches;
    exclusive_scan_u32(counts, counts, tiles * RS_BINS, stemp, dr ? n_out_dev : nullptr, st);
    k_rs_downsweep<<<(unsigned)tiles, RS_THREADS, 0, st>>>(ki, vi, ko, vo, n, nd, dr, shift, counts, tiles);
    ++g_launches;
    if (dr) nd = n_out_dev;
    u32* tk = ki; ki = ko; ko = tk;
    u32* tv = vi; vi = vo; vo = tv;
  }
  return (passes & 1) != 0;
}

size_t scan_temp_bytes(u64 n) { return 64 + ((n + SC_TILE - 1) / SC_TILE + 1) * sizeof(u64) + 64; }

// exclusive scan in -> out (out may alias in); total written to *total_dev if non-null
void exclusive_scan_u32(const u32* in, u32* out, u64 n, void* temp, u64* total_dev, cudaStream_t st) {
  u64 tiles = (n + SC_TILE - 1) / SC_TILE;
  if (tiles == 0) tiles = 1;
  u32* counter = (u32*)temp;
  u64* status = (u64*)((char*)temp + 64);
  cudaMemsetAsync(temp, 0, 64 + tiles * sizeof(u64), st);
  k_scan_u32<<<(unsigned)tiles, SC_THREADS, 0, st>>>(in, out, n, status, counter, total_dev); ++g_launches;
}

}  // namespace bc
