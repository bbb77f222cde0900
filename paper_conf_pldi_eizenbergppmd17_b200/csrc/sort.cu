// sort.cu — hand-written stable LSD radix sort (onesweep-style, decoupled look-back) and
// device-wide exclusive scan for sm_100a.
//
// The radix sort is the paper's per-location serialisation (a spinlock per shadow
// entry orders the host threads' accesses) turned into data parallelism: a STABLE sort of
// (location key, trace position) items groups each location's accesses into one contiguous
// segment that is still in trace order.  8-bit digits, 4096 keys per tile, one global
// histogram pass for all digits, then one scatter pass per digit with decoupled look-back.
#include "common.cuh"
#include "kernels.cuh"

namespace bc {

namespace {

constexpr int RS_THREADS = 256;
constexpr int RS_ITEMS = 16;
constexpr int RS_TILE = RS_THREADS * RS_ITEMS;  // 4096
constexpr int RS_WARPS = RS_THREADS / 32;
constexpr int RS_BINS = 256;

__global__ void __launch_bounds__(256) k_rs_hist(const u32* __restrict__ keys, u64 n, int bit_lo, int passes,
                                                 u32* __restrict__ hist) {
  __shared__ u32 sh[4][RS_BINS];
  for (int i = threadIdx.x; i < 4 * RS_BINS; i += blockDim.x) (&sh[0][0])[i] = 0;
  __syncthreads();
  u64 stride = (u64)gridDim.x * blockDim.x;
  for (u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    u32 k = keys[i];
    for (int p = 0; p < passes; ++p) atomicAdd(&sh[p][(k >> (bit_lo + 8 * p)) & 0xFFu], 1u);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < passes * RS_BINS; i += blockDim.x) {
    u32 v = (&sh[0][0])[i];
    if (v) atomicAdd(&hist[i], v);
  }
}

// exclusive scan of each pass's 256-bin histogram (one block of 256 threads)
__global__ void k_rs_hist_scan(u32* hist, int passes) {
  __shared__ u32 s[RS_BINS];
  for (int p = 0; p < passes; ++p) {
    u32 v = hist[p * RS_BINS + threadIdx.x];
    s[threadIdx.x] = v;
    __syncthreads();
    for (int o = 1; o < RS_BINS; o <<= 1) {
      u32 t = threadIdx.x >= (u32)o ? s[threadIdx.x - o] : 0;
      __syncthreads();
      s[threadIdx.x] += t;
      __syncthreads();
    }
    hist[p * RS_BINS + threadIdx.x] = s[threadIdx.x] - v;
    __syncthreads();
  }
}

__global__ void __launch_bounds__(RS_THREADS) k_rs_onesweep(const u32* __restrict__ kin, const u32* __restrict__ vin,
                                                            u32* __restrict__ kout, u32* __restrict__ vout, u64 n,
                                                            int shift, const u32* __restrict__ digit_base,
                                                            u64* status, u32* tile_counter) {
  __shared__ u32 skeys[RS_TILE];
  __shared__ u32 svals[RS_TILE];
  __shared__ u32 whist[RS_WARPS][RS_BINS];
  __shared__ u32 tofs[RS_BINS];
  __shared__ u32 gstart[RS_BINS];
  __shared__ u32 s_tile;

  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  if (t == 0) s_tile = atomicAdd(tile_counter, 1u);
  for (int i = t; i < RS_WARPS * RS_BINS; i += RS_THREADS) (&whist[0][0])[i] = 0;
  __syncthreads();
  const u32 tile = s_tile;
  const u64 base = (u64)tile * RS_TILE;

  u32 k[RS_ITEMS], v[RS_ITEMS], rank[RS_ITEMS];
#pragma unroll
  for (int j = 0; j < RS_ITEMS; ++j) {
    u64 idx = base + (u64)w * (RS_ITEMS * 32) + j * 32 + l;
    if (idx < n) {
      k[j] = kin[idx];
      v[j] = vin[idx];
    } else {
      k[j] = 0;
      v[j] = 0;
    }
  }
  const u32 lt = lanemask_lt();
#pragma unroll
  for (int j = 0; j < RS_ITEMS; ++j) {
    u64 idx = base + (u64)w * (RS_ITEMS * 32) + j * 32 + l;
    u32 d = idx < n ? ((k[j] >> shift) & 0xFFu) : 256u;
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
  // decoupled look-back per digit
  {
    volatile u64* st = status;
    u64 excl = 0;
    if (tile == 0) {
      st[t] = LB_INC | total;
    } else {
      st[(u64)tile * RS_BINS + t] = LB_AGG | total;
      int pt = (int)tile - 1;
      while (true) {
        u64 s = st[(u64)pt * RS_BINS + t];
        u64 f = s & ~LB_MASK;
        if (f == 0) continue;
        excl += s & LB_MASK;
        if (f == LB_INC) break;
        --pt;
      }
      __threadfence();
      st[(u64)tile * RS_BINS + t] = LB_INC | (excl + total);
    }
    gstart[t] = digit_base[t] + (u32)excl;
  }
  // tile-local exclusive scan of totals over digits
  {
    u32 x = warp_incl_sum(total);
    __shared__ u32 wsum[RS_WARPS];
    if (l == 31) wsum[w] = x;
    __syncthreads();
    u32 off = 0;
    for (int ww = 0; ww < w; ++ww) off += wsum[ww];
    tofs[t] = off + x - total;
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < RS_ITEMS; ++j) {
    u64 idx = base + (u64)w * (RS_ITEMS * 32) + j * 32 + l;
    if (idx < n) {
      u32 d = (k[j] >> shift) & 0xFFu;
      u32 pos = tofs[d] + whist[w][d] + rank[j];
      skeys[pos] = k[j];
      svals[pos] = v[j];
    }
  }
  __syncthreads();
  u32 tile_n = (u32)((n - base) < (u64)RS_TILE ? (n - base) : (u64)RS_TILE);
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
  if (t == 0) s_excl = lookback_u64(status, tile, agg);
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
size_t rs_temp_bytes(u64 n) {
  u64 tiles = (n + RS_TILE - 1) / RS_TILE;
  return 4 * RS_BINS * sizeof(u32) + 64 + tiles * RS_BINS * sizeof(u64) + 256;
}

// Stable sort of (keys, vals) by key bits [bit_lo, bit_hi).  Result is in (keys, vals) when
// the function returns false, else in (keys_alt, vals_alt).
bool radix_sort_pairs(u32* keys, u32* vals, u32* keys_alt, u32* vals_alt, u64 n, int bit_lo, int bit_hi,
                      void* temp, cudaStream_t st) {
  if (n <= 1 || bit_hi <= bit_lo) return false;
  int passes = (bit_hi - bit_lo + 7) / 8;
  if (passes > 4) passes = 4;
  char* tp = (char*)temp;
  u32* hist = (u32*)tp;
  u32* counter = (u32*)(tp + 4 * RS_BINS * sizeof(u32));
  u64* status = (u64*)(tp + 4 * RS_BINS * sizeof(u32) + 64);
  u64 tiles = (n + RS_TILE - 1) / RS_TILE;
  cudaMemsetAsync(hist, 0, 4 * RS_BINS * sizeof(u32), st);
  int blocks = (int)((n + 255) / 256);
  if (blocks > 148 * 8) blocks = 148 * 8;
  k_rs_hist<<<blocks, 256, 0, st>>>(keys, n, bit_lo, passes, hist); ++g_launches;
  k_rs_hist_scan<<<1, RS_BINS, 0, st>>>(hist, passes); ++g_launches;
  u32 *ki = keys, *vi = vals, *ko = keys_alt, *vo = vals_alt;
  for (int p = 0; p < passes; ++p) {
    cudaMemsetAsync(counter, 0, sizeof(u32), st);
    cudaMemsetAsync(status, 0, tiles * RS_BINS * sizeof(u64), st);
    k_rs_onesweep<<<(unsigned)tiles, RS_THREADS, 0, st>>>(ki, vi, ko, vo, n, bit_lo + 8 * p, hist + p * RS_BINS,
                                                           status, counter); ++g_launches;
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
