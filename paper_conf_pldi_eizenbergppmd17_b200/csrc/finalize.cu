// finalize.cu — K8 race finalize: canonical order and classification.
//
// Races leave K7 as (granule key, current record, prior record, current lane | prior lane << 5 |
// kind << 10) in arbitrary order (global record indices: any trace length).  The dense key order is
// the canonical location order (global granules by address, then shared granules by (block,
// offset)), so a stable LSD sort by prior (lane, record), then current (lane, record), then key gives
// the canonical (location, current event, prior event) order, event = record << 5 | lane (up to
// FR_SMALL races: one CTA bitonic-sorts by that composite key directly; the records are distinct).  Classification from the two events
// (reading R9): same record -> SAME_INSN; same warp -> BRANCH (branch ordering,
// P:L591-630); same block -> INTRA_BLOCK; else INTER_BLOCK.  Barrier-divergence findings
// come first, ordered by (block, record).
#include "common.cuh"
#include "kernels.cuh"

namespace bc {

namespace {

inline unsigned nb(u64 n) { return (unsigned)((n + 255) / 256); }

__global__ void k_field(const uint4* __restrict__ r, u32 n, int f, u32* __restrict__ out) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint4 v = r[i];
  out[i] = f == 0 ? v.x : f == 1 ? v.y : f == 2 ? v.z : f == 3 ? (v.w & 31u) : ((v.w >> 5) & 31u);
}

// rank -> page number, from the sorted list of non-zero bitmap words (k_page_rank)
__global__ void k_page_list(const u32* __restrict__ words, const u32* __restrict__ wl_prefix,
                            const u32* __restrict__ bits, u64 n_words, u32* __restrict__ page_num) {
  u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n_words) return;
  const u32 wd = words[i];
  u32 b = bits[wd];
  u32 k = wl_prefix[i];
  while (b) {
    int j = __ffs(b) - 1;
    b &= b - 1;
    page_num[k++] = wd * 32u + (u32)j;
  }
}

__global__ void k_emit_races(const uint4* __restrict__ r, const u32* __restrict__ perm, u32 n, Geo g,
                             const uint4* __restrict__ snap, const u32* __restrict__ page_num, u32 shared_base,
                             bc_race* __restrict__ out) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint4 v = r[perm[i]];
  const u32 key = v.x, cr = v.y, pr = v.z, cl = v.w & 31u, pl = (v.w >> 5) & 31u, kind = (v.w >> 10) & 0xFFu;
  bc_race o;
  u32 cw = snap[cr].x, pw = snap[pr].x;
  if (key < shared_base) {
    u32 sh = 20 - g.G;
    u64 page = page_num[key >> sh];
    o.addr = (page << 20) | ((u64)(key & ((1u << sh) - 1u)) << g.G);
    o.space = BC_SPACE_GLOBAL;
    o.block = cw / g.wpb;
  } else {
    u32 k = key - shared_base;
    o.addr = (u64)(k % g.smem_gran) << g.G;
    o.space = BC_SPACE_SHARED;
    o.block = k / g.smem_gran;
  }
  o.prior_event = ((u64)pr << 5) | pl;
  o.cur_event = ((u64)cr << 5) | cl;
  o.kind = (uint8_t)kind;
  if (cr == pr) o.cls = BC_CLS_SAME_INSN;
  else if (cw == pw) o.cls = BC_CLS_BRANCH;
  else if (cw / g.wpb == pw / g.wpb) o.cls = BC_CLS_INTRA_BLOCK;
  else o.cls = BC_CLS_INTER_BLOCK;
  o.pad = 0;
  out[i] = o;
}

__global__ void k_emit_findings(const u32* __restrict__ fblk, const u32* __restrict__ frec,
                                const u32* __restrict__ perm, u32 n, bc_race* __restrict__ out) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  u32 p = perm[i];
  bc_race o;
  o.addr = 0;
  o.prior_event = ~0ull;
  o.cur_event = (u64)frec[p] << 5;
  o.kind = BC_KIND_NONE;
  o.cls = BC_CLS_BARRIER_DIVERGENCE;
  o.space = BC_SPACE_NONE;
  o.pad = 0;
  o.block = fblk[p];
  out[i] = o;
}

// Few races (n <= FR_SMALL): one CTA sorts the permutation in shared memory by the canonical key
// (granule key, current record, current lane, prior record, prior lane) -- a bitonic sort over the race
// records themselves (they are distinct: one per failed check) -- instead of five LSD passes of
// (field extraction + radix sort + gather) launches.
constexpr u32 FR_SMALL = 4096;
__device__ __forceinline__ bool race_less(const uint4& a, const uint4& b) {
  if (a.x != b.x) return a.x < b.x;
  if (a.y != b.y) return a.y < b.y;
  if ((a.w & 31u) != (b.w & 31u)) return (a.w & 31u) < (b.w & 31u);
  if (a.z != b.z) return a.z < b.z;
  return ((a.w >> 5) & 31u) < ((b.w >> 5) & 31u);
}
__global__ void __launch_bounds__(1024) k_sort_races_small(const uint4* __restrict__ r, u32 n,
                                                           u32* __restrict__ perm) {
  extern __shared__ __align__(16) unsigned char fr_smem[];
  uint4* const sr = reinterpret_cast<uint4*>(fr_smem);                        // [FR_SMALL]
  unsigned short* const si = reinterpret_cast<unsigned short*>(sr + FR_SMALL);  // [FR_SMALL]
  u32 m = 1;
  while (m < n) m <<= 1;
  for (u32 i = threadIdx.x; i < m; i += blockDim.x) {
    sr[i] = i < n ? r[i] : make_uint4(0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu);
    si[i] = (unsigned short)i;
  }
  __syncthreads();
  for (u32 k = 2; k <= m; k <<= 1) {
    for (u32 j = k >> 1; j > 0; j >>= 1) {
      for (u32 i = threadIdx.x; i < m; i += blockDim.x) {
        const u32 l = i ^ j;
        if (l > i) {
          const bool up = (i & k) == 0;
          const uint4 a = sr[i], b = sr[l];
          if (race_less(b, a) == up) {  // out of order for this half: swap
            sr[i] = b;
            sr[l] = a;
            const unsigned short t = si[i];
            si[i] = si[l];
            si[l] = t;
          }
        }
      }
      __syncthreads();
    }
  }
  for (u32 i = threadIdx.x; i < n; i += blockDim.x) perm[i] = si[i];
}

int bits_for(u64 maxval) {
  int b = 0;
  while (b < 32 && (maxval >> b)) ++b;
  return b;
}

}  // namespace

void launch_page_list(const u32* words, const u32* wl_prefix, const u32* page_bits, u64 n_words, u32* page_num,
                      cudaStream_t st) {
  if (!n_words) return;
  k_page_list<<<nb(n_words), 256, 0, st>>>(words, wl_prefix, page_bits, n_words, page_num); ++g_launches;
}

// races[n_r] (key, cur, prior, kind) + findings -> out[n_f + n_r] in canonical order
void finalize_races(const uint4* races, u32 n_r, const u32* fblk, const u32* frec, u32 n_f, const Geo& g,
                    const uint4* snap, const u32* page_num, u32 shared_base, u32 n_keys, bc_race* out, Scratch& S,
                    cudaStream_t st) {
  if (n_f) {
    u32* p = S.alloc<u32>(n_f);
    launch_iota(p, n_f, st);
    sort_perm_by(p, frec, n_f, 32, S, st);
    sort_perm_by(p, fblk, n_f, bits_for(g.n_blocks), S, st);
    k_emit_findings<<<nb(n_f), 256, 0, st>>>(fblk, frec, p, n_f, out); ++g_launches;
  }
  if (n_r && n_r <= FR_SMALL) {
    u32* p = S.alloc<u32>(n_r);
    constexpr size_t smem = FR_SMALL * (sizeof(uint4) + sizeof(unsigned short));
    static bool attr[64] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 0 && dev < 64 && !attr[dev]) {
      cudaFuncSetAttribute(k_sort_races_small, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      attr[dev] = true;
    }
    k_sort_races_small<<<1, 1024, smem, st>>>(races, n_r, p); ++g_launches;
    k_emit_races<<<nb(n_r), 256, 0, st>>>(races, p, n_r, g, snap, page_num, shared_base, out + n_f); ++g_launches;
  } else if (n_r) {
    u32* p = S.alloc<u32>(n_r);
    u32* f = S.alloc<u32>(n_r);
    launch_iota(p, n_r, st);
    const int fields[4] = {4, 2, 3, 1};  // prior lane, prior record, current lane, current record
    for (int q = 0; q < 4; ++q) {
      k_field<<<nb(n_r), 256, 0, st>>>(races, n_r, fields[q], f); ++g_launches;
      sort_perm_by(p, f, n_r, (fields[q] == 3 || fields[q] == 4) ? 5 : bits_for(g.n_recs), S, st);
    }
    k_field<<<nb(n_r), 256, 0, st>>>(races, n_r, 0, f); ++g_launches;
    sort_perm_by(p, f, n_r, bits_for(n_keys), S, st);
    k_emit_races<<<nb(n_r), 256, 0, st>>>(races, p, n_r, g, snap, page_num, shared_base, out + n_f); ++g_launches;
  }
}

void preload_finalize() {
  preload(k_emit_findings, k_emit_races, k_field, k_page_list, k_sort_races_small);
}

}  // namespace bc
