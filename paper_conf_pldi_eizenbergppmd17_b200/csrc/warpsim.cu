// warpsim.cu — warp-size simulation ("in future we could
// simulate the behavior of smaller/larger warps to find additional latent bugs"), reading R17:
// a trace recorded with 32-lane warps is re-split into virtual warps of ws lanes (4, 8, 16).  Record
// (warp w, mask m) becomes, in trace order, one record per virtual warp j of w that executes it --
// warp (block, (w_in_block * 32 + j * ws) / ws), mask (m >> j*ws) & (2^ws - 1), addresses
// addr[j*ws ...].  Control flow per virtual warp follows its own SIMT stack: an IF whose mask has
// none of its lanes is not executed by it, nor the matching ELSE / FI or anything nested.
//
//   1. records grouped by physical warp (stable radix sort, the K1 partition);
//   2. one thread per (physical warp, virtual warp) walks that warp's records in trace order with a
//      bit stack of "this virtual warp executes the construct" flags and marks the records it emits;
//   3. an exclusive scan of the marks in trace order (record-major, virtual-warp-minor) gives every
//      emitted record its position; one warp per output record writes it (272 B) and its origin.
#include <algorithm>

#include "ctx.cuh"

namespace bc {

namespace {

inline unsigned nb(u64 n) { return (unsigned)((n + 255) / 256); }

__global__ void k_ws_keys(const bc_record* __restrict__ recs, u64 n, u32* __restrict__ wk, u32* __restrict__ wv) {
  const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  wk[i] = recs[i].warp;
  wv[i] = (u32)i;
}

// warp_start[w] = lower bound of w in the warp-sorted keys
__global__ void k_ws_start(const u32* __restrict__ sk, u64 n, u32 n_warps, u32* __restrict__ start) {
  const u32 w = blockIdx.x * blockDim.x + threadIdx.x;
  if (w > n_warps) return;
  u64 lo = 0, hi = n;
  while (lo < hi) {
    const u64 m = (lo + hi) >> 1;
    if (sk[m] < w) lo = m + 1; else hi = m;
  }
  start[w] = (u32)lo;
}

// thread (w, j): marks[i * k + j] = 1 iff virtual warp j of physical warp w executes record i
__global__ void k_ws_mark(const bc_record* __restrict__ recs, const u32* __restrict__ wrec,
                          const u32* __restrict__ start, u32 n_warps, u32 k, u32 ws, u32 wpb32, u32 tpb,
                          u32* __restrict__ marks, u32* __restrict__ err) {
  const u64 t = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= (u64)n_warps * k) return;
  const u32 w = (u32)(t / k), j = (u32)(t % k);
  const u32 wib = w % wpb32;
  if (wib * 32 + j * ws >= tpb) return;  // this virtual warp has no threads
  const u32 lm = (1u << ws) - 1u;
  u64 stack = 1;  // bit d = run flag at depth d (depth 0: always executing)
  int depth = 0;
  for (u32 q = start[w]; q < start[w + 1]; ++q) {
    const u32 i = wrec[q];
    const bc_record& r = recs[i];
    const u32 op = r.op, sm = (r.mask >> (j * ws)) & lm;
    bool run;
    if (op == BC_OP_IF) {
      run = ((stack >> depth) & 1ull) && sm != 0;
      if (depth >= 62) {
        atomicOr(err, 1u);
        return;
      }
      ++depth;
      stack = (stack & ~(1ull << depth)) | ((u64)run << depth);
    } else if (op == BC_OP_ELSE) {
      run = depth > 0 && ((stack >> depth) & 1ull);
    } else if (op == BC_OP_FI) {
      run = depth > 0 && ((stack >> depth) & 1ull);
      if (depth > 0) --depth;
    } else {
      run = sm != 0;
    }
    if (run) marks[(u64)i * k + j] = 1u;
  }
}

// one warp per input (record, virtual warp) slot with a mark: write the virtual record
__global__ void k_ws_emit(const bc_record* __restrict__ recs, const u32* __restrict__ marks,
                          const u64* __restrict__ pos, u64 n_slots, u32 k, u32 ws, u32 wpb32, u32 wpb,
                          bc_record* __restrict__ out, u64* __restrict__ origin, u64 cap) {
  const u64 s = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const u32 lane = threadIdx.x & 31;
  if (s >= n_slots || !marks[s]) return;
  const u64 o = pos[s];
  if (o >= cap) return;
  const u64 i = s / k;
  const u32 j = (u32)(s % k);
  const bc_record& r = recs[i];
  const u32 lm = (1u << ws) - 1u;
  const u32 b = r.warp / wpb32, wib = r.warp % wpb32;
  bc_record& d = out[o];
  if (lane == 0) {
    d.warp = b * wpb + (wib * 32 + j * ws) / ws;
    d.mask = (r.mask >> (j * ws)) & lm;
    d.op = r.op;
    d.space = r.space;
    d.size_log2 = r.size_log2;
    d.flags = r.flags;
    d.aux = r.op == BC_OP_IF ? ((r.aux >> (j * ws)) & lm) : 0u;
    origin[o] = (i << 5) | (j * ws);
  }
  d.addr[lane] = lane < ws ? r.addr[j * ws + lane] : 0ull;
}

}  // namespace
}  // namespace bc

using namespace bc;

// C ABI: see include/bc.h
extern "C" bc_status bc_split_warps(bc_ctx* c, const bc_record* recs, uint64_t n, uint32_t ws, bc_record* out,
                                    uint64_t* origin, uint64_t cap, uint64_t* n_out) {
  if (!c || !n_out || (n && !recs)) return BC_ERR_INVALID_ARG;
  if (ws != 4 && ws != 8 && ws != 16 && ws != 32) return fail(c, BC_ERR_INVALID_ARG, "warp size 4, 8, 16 or 32");
  if (c->g.ws != 32) return fail(c, BC_ERR_INVALID_ARG, "the context must describe the recorded 32-lane warps");
  if (n >= (1ull << 32) / 8) return fail(c, BC_ERR_OVERFLOW, "too many records to split");
  cudaSetDevice(c->cfg.device);
  cudaStream_t st = c->stream;
  const u32 k = 32 / ws, wpb32 = c->g.wpb, tpb = c->g.tpb, wpb = (tpb + ws - 1) / ws;
  const u32 n_warps = c->g.n_warps;
  const u64 n_slots = n * k;
  bc_status s = BC_OK;
  {
    Scratch S(st, &c->arena);
    try {
      u32* wk = S.alloc<u32>(n + 1);
      u32* wv = S.alloc<u32>(n + 1);
      u32* wk2 = S.alloc<u32>(n + 1);
      u32* wv2 = S.alloc<u32>(n + 1);
      u32* start = S.alloc<u32>(n_warps + 2);
      u32* marks = S.alloc<u32>(n_slots + 1);
      u64* pos = S.alloc<u64>(n_slots + 1);
      u32* err = S.alloc<u32>(1);
      cudaMemsetAsync(err, 0, 4, st);
      cudaMemsetAsync(marks, 0, (n_slots + 1) * 4, st);
      if (n) {
        k_ws_keys<<<nb(n), 256, 0, st>>>(recs, n, wk, wv);
        ++g_launches;
      }
      const bool alt = radix_sort_pairs(wk, wv, wk2, wv2, n, 0, bits_for(n_warps ? n_warps - 1 : 0),
                                        S.alloc<char>(rs_temp_bytes(n)), st);
      const u32* sk = alt ? wk2 : wk;
      const u32* wrec = alt ? wv2 : wv;
      k_ws_start<<<nb(n_warps + 1), 256, 0, st>>>(sk, n, n_warps, start);
      k_ws_mark<<<nb((u64)n_warps * k), 256, 0, st>>>(recs, wrec, start, n_warps, k, ws, wpb32, tpb, marks, err);
      g_launches += 2;
      exclusive_scan_u32_u64(marks, pos, n_slots, S.alloc<char>(scan_temp_bytes(n_slots)), pos + n_slots, st);
      u64 tot = 0;
      u32 herr = 0;
      cudaMemcpyAsync(&tot, pos + n_slots, 8, cudaMemcpyDeviceToHost, st);
      cudaMemcpyAsync(&herr, err, 4, cudaMemcpyDeviceToHost, st);
      if (cudaStreamSynchronize(st) != cudaSuccess) {
        s = cuda_check(c, "split");
      } else if (herr) {
        s = fail(c, BC_ERR_INFEASIBLE_TRACE, "branch nesting deeper than 62");
      } else {
        *n_out = tot;
        if (out && n_slots) {
          k_ws_emit<<<(unsigned)((n_slots * 32 + 255) / 256), 256, 0, st>>>(recs, marks, pos, n_slots, k, ws, wpb32,
                                                                          wpb, out, origin, cap);
          ++g_launches;
          if (cudaStreamSynchronize(st) != cudaSuccess) s = cuda_check(c, "split");
          else if (tot > cap) s = fail(c, BC_ERR_TRUNCATED, "output capacity below the split record count");
        }
      }
    } catch (const std::bad_alloc&) {
      s = fail(c, BC_ERR_OOM, "split scratch");
    }
  }
  return s;
}
