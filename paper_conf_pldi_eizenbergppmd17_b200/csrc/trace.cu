// trace.cu — the record-level passes of the hot path:
//   k_header   (a1/a2) header validation, event counts, K1 partition keys, write-page marking
//   k_replay   (a3)    K2 compressed clock replay: one analysis warp per traced warp walks its records
//   k_barriers (a3)    block barrier completion labels (§4.3.2 block max)
//   k_expand   (a5)    K4 lane expansion into (granule key | op, event) items in trace order
#include <algorithm>

#include "common.cuh"
#include "kernels.cuh"

namespace bc {

// counters in `cnt` (u64)

// ---------------------------------------------------------------------------- k_header
#ifndef HDR_ROWS
#define HDR_ROWS 8  // write records whose address rows one warp loads at once (page marking)
#endif
// One warp per 32 consecutive records.  Lane l validates record base+l's header (the checks of
// P:L360-366 that need no state; stack / barrier checks are in k_replay / k_barriers), then the
// warp marks the 1-MB pages written by the ST / ATOM global records among the 32 (the paper's
// on-demand global shadow page table, used here to skip never-written memory).
__global__ void __launch_bounds__(256) k_header(const bc_record* __restrict__ recs, Geo g, u32* __restrict__ wkey,
                                                u32* __restrict__ wval, u32* __restrict__ if_cnt,
                                                u32* __restrict__ bar_cnt, u32* __restrict__ sync_list,
                                                u32* __restrict__ page_bits, u32* __restrict__ word_list,
                                                u64* __restrict__ cnt, u32* __restrict__ rec_w,
                                                uint4* __restrict__ hdr16, u32* __restrict__ rec_cnt,
                                                u32* __restrict__ err, int mark_pages) {
  const u32 lane = threadIdx.x & 31;
  const u64 gw = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const u64 r = gw * 32 + lane;
  bool valid = r < g.n_recs;
  Hdr h{};
  u32 bad = 0;
  u32 lane_ev = 0, ctl_ev = 0, is_sync = 0, is_acq = 0, is_mem = 0, is_if = 0, is_bar = 0, ibound = 0;
  if (valid) {
    const uint4 hv = __ldg(reinterpret_cast<const uint4*>(recs + r));
    hdr16[r] = hv;  // compact copy of the 16-B header for K2 (gathered per warp there)
    h.warp = hv.x;
    h.mask = hv.y;
    h.op = hv.z & 0xFFu;
    h.space = (hv.z >> 8) & 0xFFu;
    h.size_log2 = (hv.z >> 16) & 0xFFu;
    h.flags = (hv.z >> 24) & 0xFFu;
    h.aux = hv.w;
    if (h.op > BC_OP_FI || h.warp >= g.n_warps) {
      bad = 1;
    } else {
      if (h.mask & ~init_mask(g, h.warp)) bad = 1;
      if (h.op <= BC_OP_AR_GLB) {
        if (h.mask == 0 || h.size_log2 > 4 || h.space > BC_SPACE_SHARED) bad = 1;
        lane_ev = __popc(h.mask);
        if (h.op <= BC_OP_ATOM) {
          is_mem = 1;
          u32 ng = (1u << (h.size_log2 & 7)) >> g.G;
          ibound = lane_ev * (ng ? ng : 1u);
        } else {
          is_sync = 1;
        }
        if (h.op == BC_OP_ACQ_BLK || h.op == BC_OP_ACQ_GLB || h.op == BC_OP_AR_BLK || h.op == BC_OP_AR_GLB)
          is_acq = 1;
      } else {
        ctl_ev = 1;
        if ((h.op == BC_OP_FENCE || h.op == BC_OP_BAR) && h.mask == 0) bad = 1;
        if (h.op == BC_OP_IF) {
          if (h.mask == 0 || (h.aux & ~h.mask)) bad = 1;
          is_if = 1;
        }
        if (h.op == BC_OP_BAR) is_bar = 1;
      }
    }
    wkey[r] = bad ? 0u : h.warp;
    wval[r] = (u32)r;
    if (!bad) {
      if (is_if) atomicAdd(&if_cnt[h.warp], 1u);
      if (is_bar) atomicAdd(&bar_cnt[h.warp], 1u);
      if (is_sync) {
        u64 at = atomicAdd((unsigned long long*)&cnt[C_SYNC_RECS], 1ull);
        sync_list[at] = (u32)r;
      }
    }
  }
  if (__any_sync(0xFFFFFFFFu, bad) && lane == 0) set_err(err, ERR_INFEASIBLE);
  if (rec_cnt) {  // records per traced warp (K1 CSR offsets by a scan, small grids): one atomic per warp id
    const bool cnt_me = valid && !bad;
    const u32 peers = __match_any_sync(0xFFFFFFFFu, cnt_me ? h.warp : 0xFFFFFFFFu);
    if (cnt_me && (peers & lanemask_lt()) == 0) atomicAdd(&rec_cnt[h.warp], (u32)__popc(peers));
  }
  // warp-reduced counters
  if (bad) ibound = 0;
  if (valid) rec_w[r] = ibound + REC_W;  // window weight: item upper bound (K4 writes at static slots) + REC_W
  u32 v[8] = {lane_ev, ctl_ev, is_acq, is_mem, is_if, is_bar, is_sync ? lane_ev : 0u, ibound};
#pragma unroll
  for (int i = 0; i < 8; ++i) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v[i] += __shfl_down_sync(0xFFFFFFFFu, v[i], o);
  }
  {
    __shared__ unsigned long long s_cnt[8];
    if (threadIdx.x < 8) s_cnt[threadIdx.x] = 0;
    __syncthreads();
    if (lane == 0) {
#pragma unroll
      for (int i = 0; i < 8; ++i)
        if (v[i]) atomicAdd(&s_cnt[i], (unsigned long long)v[i]);
    }
    __syncthreads();
    if (threadIdx.x < 8) {
      const int slot[8] = {C_LANE_EVENTS, C_CONTROL_EVENTS, C_ACQ_RECS, C_MEM_RECS, C_IFS, C_BARS, C_SYNC_LANEOPS,
                           C_ITEM_BOUND};
      if (s_cnt[threadIdx.x]) atomicAdd((unsigned long long*)&cnt[slot[threadIdx.x]], s_cnt[threadIdx.x]);
    }
  }
  // page marking: ST / ATOM on global memory.  mark_pages == 2 (sampled): only the first and last active
  // lanes' addresses of each write record -- one or two 8-B loads instead of its 256-B row; K4 checks every
  // write address against the set and flags a missing page (ERR_PAGES), and the host then re-runs the
  // detect with every address marked (mark_pages == 1), so the page set K4-K7 use is always complete.
  const bool wrec = valid && !bad && (h.op == BC_OP_ST || h.op == BC_OP_ATOM) && h.space == BC_SPACE_GLOBAL;
  if (mark_pages == 2 && wrec) {
    const int la = __ffs(h.mask) - 1, lb = 31 - __clz(h.mask);
    const u64 a0 = __ldg(&recs[r].addr[la]), a1 = __ldg(&recs[r].addr[lb]);
#pragma unroll
    for (int k = 0; k < 2; ++k) {
      const u64 p = (k ? a1 : a0) >> 20;
      if (p >= (1ull << 28)) {
        set_err(err, ERR_OVERFLOW);
      } else {
        const u32 bit = 1u << (p & 31);
        u32* wp = &page_bits[p >> 5];
        if (!(*(volatile u32*)wp & bit) && atomicOr(wp, bit) == 0u) {
          const u64 at = atomicAdd((unsigned long long*)&cnt[C_PAGE_WORDS], 1ull);
          word_list[at] = (u32)(p >> 5);
        }
      }
    }
  }
  u32 wr = __ballot_sync(0xFFFFFFFFu, mark_pages == 1 && wrec);
  while (wr) {  // HDR_ROWS records' address rows in flight at a time
    int js[HDR_ROWS];
    u64 a[HDR_ROWS];
#pragma unroll
    for (int k = 0; k < HDR_ROWS; ++k) {
      js[k] = -1;
      if (wr) {
        js[k] = __ffs(wr) - 1;
        wr &= wr - 1;
      }
    }
#pragma unroll
    for (int k = 0; k < HDR_ROWS; ++k) {
      a[k] = ~0ull;
      if (js[k] >= 0) {
        u32 m = __shfl_sync(0xFFFFFFFFu, h.mask, js[k]);
        if ((m >> lane) & 1u) a[k] = __ldg(&recs[gw * 32 + js[k]].addr[lane]);
      } else {
        __shfl_sync(0xFFFFFFFFu, h.mask, 0);
      }
    }
#pragma unroll
    for (int k = 0; k < HDR_ROWS; ++k) {
      if (a[k] == ~0ull) continue;
      u64 p = a[k] >> 20;
      if (p >= (1ull << 28)) {
        set_err(err, ERR_OVERFLOW);
      } else {
        u32 bit = 1u << (p & 31);
        u32* wp = &page_bits[p >> 5];
        if (!(*(volatile u32*)wp & bit)) {
          // the thread that turns a bitmap word non-zero lists it (ranked by k_page_rank)
          if (atomicOr(wp, bit) == 0u) {
            const u64 at = atomicAdd((unsigned long long*)&cnt[C_PAGE_WORDS], 1ull);
            word_list[at] = (u32)(p >> 5);
          }
        }
      }
    }
  }
}

// Streaming (declared allocations, bc_config.global_ranges): mark every 1-MB page of the ranges; a
// word that turns non-zero is listed for k_page_rank
__global__ void k_mark_ranges(const u64* __restrict__ ranges, u32 n_ranges, u32* __restrict__ page_bits,
                              u32* __restrict__ word_list, u64* __restrict__ cnt, u32* __restrict__ err) {
  for (u32 q = 0; q < n_ranges; ++q) {
    const u64 base = ranges[2 * q], size = ranges[2 * q + 1];
    if (!size) continue;
    const u64 p0 = base >> 20, p1 = (base + size - 1) >> 20;
    if (p1 >= (1ull << 28)) {
      if (threadIdx.x == 0 && blockIdx.x == 0) set_err(err, ERR_OVERFLOW);
      continue;
    }
    for (u64 p = p0 + (u64)blockIdx.x * blockDim.x + threadIdx.x; p <= p1; p += (u64)gridDim.x * blockDim.x) {
      const u32 bit = 1u << (p & 31);
      if (atomicOr(&page_bits[p >> 5], bit) == 0u) {
        const u64 at = atomicAdd((unsigned long long*)&cnt[C_PAGE_WORDS], 1ull);
        word_list[at] = (u32)(p >> 5);
      }
    }
  }
}
void launch_mark_ranges(const u64* ranges, u32 n_ranges, u32* page_bits, u32* word_list, u64* cnt, u32* err,
                        cudaStream_t st) {
  if (!n_ranges) return;
  k_mark_ranges<<<64, 256, 0, st>>>(ranges, n_ranges, page_bits, word_list, cnt, err);
  ++g_launches;
}

// warp_start[w] = first index of warp w in the warp-sorted record list (lower bound)
__global__ void k_warp_start(const u32* __restrict__ skeys, u64 n, u32 n_warps, u32* __restrict__ warp_start) {
  u32 w = blockIdx.x * blockDim.x + threadIdx.x;
  if (w > n_warps) return;
  u64 lo = 0, hi = n;
  while (lo < hi) {
    u64 mid = (lo + hi) >> 1;
    if (skeys[mid] < w) lo = mid + 1; else hi = mid;
  }
  warp_start[w] = (u32)lo;
}

// ---------------------------------------------------------------------------- k_replay
// K2: compressed clock replay (Fig. 7, §4.3.1-4.3.2).  One analysis warp per traced
// warp walks the traced warp's records in trace order with the SIMT stack of Fig. 2 (K_w,
// P:L430-432).  Stack levels are branch-tree nodes: IF pushes the then-node (else-node
// is its sibling, id+1, entered at ELSE); FI pops.  Every join-fork step (endi, if, else, fi, bar)
// is labelled rec+1.  The 32 lanes load 32 consecutive records (index + compact 16-B header) at
// once, one chunk ahead.  Runs of endi records (LD / ST / ATOM / ACQ / REL / AR: only ps changes)
// are resolved in parallel (lane j: ps = rec[j-1] + 1); the control records between them (IF, ELSE,
// FI, BAR, FENCE) are stepped one at a time, uniformly across the lanes (header = broadcast
// shared-memory read, top of the SIMT stack in registers).  Lane j keeps the state record j saw,
// so the per-record snapshot {warp, ps, node, phase} is written by 32 lanes in parallel.  Per IF it writes the two
// nodes {mask, parent, popen}; per BAR its record and the warp's next record (barrier feasibility)
// and a BARRIER_DIVERGENCE finding when the mask is not the warp's initial mask.
__global__ void __launch_bounds__(256, 4) k_replay(const uint4* __restrict__ hdr16, const u32* __restrict__ wrec,
                                                const u32* __restrict__ gidx, const u32* __restrict__ warp_start, Geo g,
                                                const u32* __restrict__ node_base, const u32* __restrict__ bar_base,
                                                uint4* __restrict__ snap, uint4* __restrict__ nodes,
                                                u32* __restrict__ bar_rec, u32* __restrict__ bar_next,
                                                u32* __restrict__ find_blk, u32* __restrict__ find_rec,
                                                u32* __restrict__ find_cnt, u32* __restrict__ err) {
  __shared__ uint4 s_hdr[8][32];  // the chunk's headers / record indices: broadcast reads in the
  __shared__ u32 s_rec[8][32];    // serial steps instead of four shuffles each
  const u32 w = (u32)(((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5);
  const u32 lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  if (w >= g.n_warps) return;  // warp-uniform
  const u32 imask = init_mask(g, w);
  // SIMT stack below the top (the top lives in cur_node / cur_mask): warp-uniform, so one copy per
  // analysis warp in shared memory (a per-lane array would be spilled to local memory 32 times over)
  __shared__ uint2 s_stack[8][33];
  uint2* const stk = s_stack[threadIdx.x >> 5];
  u32 cur_node = w, cur_mask = imask;
  u64 then_bits = 0;  // bit d set: level d is a then-node
  int depth = 0;
  if (lane == 0) nodes[w] = make_uint4(imask, NONE, 0u, 0u);
  u32 ps = 0, phase = 0, nif = 0, nbar = 0;
  bool need_next = false;
  bool bad = false;
  const u32 nb0 = node_base[w], bb0 = bar_base[w];
  const u32 i0 = warp_start[w], i1 = warp_start[w + 1];
  // local record index (hdr16 / snap position) and its global index (the step label is global index + 1;
  // the same unless the context holds a block shard of the trace)
  u32 nr = 0, ng = 0;
  uint4 nh = make_uint4(0, 0, 0, 0);
  if (i0 + lane < i1) {
    nr = wrec[i0 + lane];
    nh = __ldg(hdr16 + nr);
    ng = gidx ? __ldg(gidx + nr) : nr;
  }
  u32 nr2 = i0 + 32 + lane < i1 ? wrec[i0 + 32 + lane] : 0u;
  for (u32 c0 = i0; c0 < i1 && !bad; c0 += 32) {
    const u32 r = nr, rg = ng;
    const uint4 hv = nh;
    const u32 cnt = min(32u, i1 - c0);
    // the next chunk's headers in flight while this one is stepped through (their record indices were
    // loaded one chunk earlier, so the gather does not wait on them), and the indices of the one after
    if (c0 + 32 + lane < i1) {
      nr = nr2;
      nh = __ldg(hdr16 + nr);
      ng = gidx ? __ldg(gidx + nr) : nr;
    }
    if (c0 + 64 + lane < i1) nr2 = wrec[c0 + 64 + lane];
    s_hdr[wib][lane] = hv;
    s_rec[wib][lane] = rg;
    __syncwarp();
    // control records (FENCE, BAR, IF, ELSE, FI) are stepped one by one; the runs of endi records
    // between them (LD / ST / ATOM / ACQ / REL / AR: ps := rec + 1, stack unchanged) in parallel
    const u32 ctl = __ballot_sync(0xFFFFFFFFu, lane < cnt && (hv.z & 0xFFu) >= BC_OP_FENCE);
    const u32 rprev = __shfl_up_sync(0xFFFFFFFFu, rg, 1);
    u32 my_ps = 0, my_node = 0, my_phase = 0;
    bool badl = false;
    u32 sidx = 0;
    while (sidx < cnt) {
      const u32 rest = ctl & (~0u << sidx);
      const u32 f = rest ? (u32)__ffs(rest) - 1u : cnt;
      if (f > sidx) {  // endi run [sidx, f)
        if (lane >= sidx && lane < f) {
          my_ps = lane == sidx ? ps : rprev + 1u;
          my_node = cur_node;
          my_phase = phase;
          badl |= hv.y != cur_mask;  // feasibility: record mask == K_w.peek()
        }
        if (need_next) {
          if (lane == 0) bar_next[bb0 + nbar - 1] = s_rec[wib][sidx];
          need_next = false;
        }
        ps = s_rec[wib][f - 1] + 1u;
      }
      if (f >= cnt) break;
      // control record f
      const uint4 hf = s_hdr[wib][f];
      const u32 rj = s_rec[wib][f], mask = hf.y, op = hf.z & 0xFFu, aux = hf.w;
      if (need_next) {
        if (lane == 0) bar_next[bb0 + nbar - 1] = rj;
        need_next = false;
      }
      if (lane == f) {
        my_ps = ps;
        my_node = cur_node;
        my_phase = phase;
      }
      if (mask != cur_mask) {
        bad = true;
        break;
      }
      switch (op) {
        case BC_OP_FENCE:
          break;  // standalone fence: no trace operation (R14)
        case BC_OP_IF: {
          if (depth >= 32) { bad = true; break; }
          const u32 then = mask & aux;
          const u32 nid = nb0 + 2 * nif;
          ++nif;
          if (lane == 0) {
            nodes[nid] = make_uint4(then, cur_node, ps, 0u);
            nodes[nid + 1] = make_uint4(mask & ~then, cur_node, ps, 0u);
          }
          __syncwarp();  // every lane is done reading the stack (an earlier FI / ELSE at this depth)
          if (lane == 0) stk[depth] = make_uint2(cur_node, cur_mask);
          __syncwarp();
          ++depth;
          cur_node = nid;
          cur_mask = then;
          then_bits |= 1ull << depth;
          ps = rj + 1;
          break;
        }
        case BC_OP_ELSE: {
          if (depth == 0 || !((then_bits >> depth) & 1ull)) { bad = true; break; }
          cur_node += 1;
          cur_mask = stk[depth - 1].y & ~cur_mask;
          then_bits &= ~(1ull << depth);
          ps = rj + 1;
          break;
        }
        case BC_OP_FI: {
          if (depth == 0 || ((then_bits >> depth) & 1ull)) { bad = true; break; }
          --depth;
          const uint2 top = stk[depth];
          cur_node = top.x;
          cur_mask = top.y;
          ps = rj + 1;
          break;
        }
        default: {  // BC_OP_BAR
          if (lane == 0) {
            if (mask != imask) {  // barrier divergence; the barrier still completes (R10)
              const u32 at = atomicAdd(find_cnt, 1u);
              find_blk[at] = blk_of(g, w);
              find_rec[at] = rj;
            }
            bar_rec[bb0 + nbar] = rj;
            bar_next[bb0 + nbar] = NONE;
          }
          ++nbar;
          ++phase;
          need_next = true;
          ps = rj + 1;
          break;
        }
      }
      if (bad) break;
      sidx = f + 1;
    }
    bad |= __any_sync(0xFFFFFFFFu, badl);
    if (lane < cnt) snap[r] = make_uint4(w, my_ps, my_node, my_phase);
    __syncwarp();
  }
  if (bad && lane == 0) set_err(err, ERR_INFEASIBLE);
}

// ---------------------------------------------------------------------------- k_barriers
// Per block: every warp must arrive at every barrier exactly once (R10).  Barrier k completes
// at the last arrival R_k = max over the block's warps of their k-th BAR record; its step is
// labelled R_k + 1 for every thread of the block.  A warp whose next record after its k-th
// BAR precedes R_k issued a record while waiting -> infeasible.  One warp per traced block; lane l
// handles barriers l, l+32, ... and checks the counts of warps l, l+32, ...
__global__ void __launch_bounds__(256) k_barriers(Geo g, const u32* __restrict__ bar_cnt,
                                                  const u32* __restrict__ bar_base, const u32* __restrict__ bar_rec,
                                                  const u32* __restrict__ bar_next, u32* __restrict__ blockR,
                                                  u32* __restrict__ err, int allow_pending) {
  const u32 b = (u32)(((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5);
  const u32 lane = threadIdx.x & 31;
  if (b >= g.n_blocks) return;  // warp-uniform
  const u32 w0 = b * g.wpb;
  // barriers [0, nb) completed (every warp arrived); a prefix of a streamed trace (allow_pending) may end
  // with barrier nb pending: some warps arrived (and may issue nothing more), the others not yet
  u32 mn = NONE, mx = 0;
  for (u32 i = lane; i < g.wpb; i += 32) {  // (wpb > 32: simulated small warps)
    mn = min(mn, bar_cnt[w0 + i]);
    mx = max(mx, bar_cnt[w0 + i]);
  }
  mn = __reduce_min_sync(0xFFFFFFFFu, mn);
  mx = __reduce_max_sync(0xFFFFFFFFu, mx);
  if (mx != mn && !(allow_pending && mx == mn + 1)) {
    if (lane == 0) set_err(err, ERR_INFEASIBLE);
    return;
  }
  const u32 nb = mn;
  for (u32 k = lane; k < nb; k += 32) {
    u32 R = 0, mnx = NONE;
    for (u32 i = 0; i < g.wpb; ++i) {
      u32 bi = bar_base[w0 + i] + k;
      R = max(R, bar_rec[bi]);
      mnx = min(mnx, bar_next[bi]);
    }
    if (mnx != NONE && mnx < R) set_err(err, ERR_INFEASIBLE);
    blockR[bar_base[w0] + k] = R + 1;
  }
  if (mx > nb)  // the pending barrier: a warp that arrived issues nothing until it completes
    for (u32 i = lane; i < g.wpb; i += 32)
      if (bar_cnt[w0 + i] > nb && bar_next[bar_base[w0 + i] + nb] != NONE) set_err(err, ERR_INFEASIBLE);
}

// ---------------------------------------------------------------------------- k_expand
// K4: lowering of each LD / ST / ATOM warp record of one window [R0, R1) into one thread operation
// per active lane and per shadow granule (R7), emitted as 8-byte items
//   key = (dense granule key << 2) | op,   ev = window-local event = ((record - R0) << 5) | lane
// at static slots: record r owns popc(mask) * granules slots (upper bound from k_header) starting
// at its weight prefix within the window (cum[r] - cum[R0] - REC_W * (r - R0)), lane l the
// popc(mask & lanemask_lt) * granules slots of it -- so items land in
// trace order with no synchronisation at all.  Dense keys: global granules of written 1-MB
// pages first (page rank from the write bitmap, so keys follow address order), then shared
// granules (block, offset).  Accesses to never-written global pages cannot take
// part in a race (every race needs a write): their slots get the sentinel key
// KEY_DROP, which the first radix pass removes.  Also validates per-lane alignment / shared
// bounds for every op <= AR_GLB.
//
// Data movement (each address-carrying record is read once, at HBM rate): every warp owns chunks of
// EX_RPW consecutive records (warp-strided over the window) and stages only the 256-B address rows of
// the records that carry addresses (LD / ST / ATOM / ACQ / REL / AR; the headers come from k_header's
// compact copy hdr16), so the rows of control records (IF / ELSE / FI / BAR / FENCE: half of C4's
// records) never leave HBM.  Rows land in the warp's own shared-memory buffer by cp.async (16 B per
// lane: one warp instruction moves two rows), the next chunk in flight while this one is expanded
// (two stages); no CTA-wide barrier, so a warp never waits for another warp's records.  (Round 1-2:
// 64-record chunks by one TMA bulk copy per CTA and stage, 2 stages, whole records: 3.8 ms on C4,
// barrier-stall bound; a bulk copy per run of address-carrying records was slower still: 5.0 ms.)
constexpr int EX_THREADS = 256;
constexpr int EX_WARPS = EX_THREADS / 32;
constexpr int EX_RPW = 8;                          // records per warp chunk
constexpr size_t EX_ROW = 32 * sizeof(u64);        // 256 B: one record's address row
constexpr size_t EX_SMEM = (size_t)EX_WARPS * 2 * EX_RPW * EX_ROW;  // 32 KB per CTA

__global__ void __launch_bounds__(EX_THREADS) k_expand(const bc_record* __restrict__ recs,
                                                       const uint4* __restrict__ hdr16, Geo g,
                                                       const u32* __restrict__ page_bits,
                                                       const u32* __restrict__ page_rank, u32 shared_base,
                                                       const u64* __restrict__ cum, u64 R0, u64 R1,
                                                       const u32* __restrict__ gidx, u64 G0,
                                                       u32* __restrict__ okeys, u32* __restrict__ oevs,
                                                       u32* __restrict__ err) {
  extern __shared__ __align__(128) unsigned char ex_smem[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  u64* const rows = reinterpret_cast<u64*>(ex_smem + (size_t)wid * 2 * EX_RPW * EX_ROW);  // [2][EX_RPW][32]
  const u64 n = R1 - R0;  // records of the window
  const u64 n_chunks = (n + EX_RPW - 1) / EX_RPW;
  const u64 nw = (u64)gridDim.x * EX_WARPS;
  const u64 cum0 = __ldg(cum + R0);
  const u32 lt = lanemask_lt();
  bool bad = false, ovf = false, undecl = false, pmiss = false;
  // per chunk, lane j < EX_RPW holds record j's header, slot offset and event base
  // meta: valid (1) | LD/ST/ATOM (2) | shared (4) | op code << 3 | size_log2 << 5 | (granules - 1) << 8 |
  // writer << 13 -- decoded once per chunk, in parallel over its records
  struct Ch {
    u32 mask, meta, sb, uo, eb, sel;
  };
  // load a chunk's headers / offsets and start copying the address rows of its selected records
  auto issue = [&](u64 chunk, int stg) -> Ch {
    Ch c;
    const u64 r0 = chunk * EX_RPW;
    const u64 rl = r0 + (u64)(lane & (EX_RPW - 1));
    const bool have = lane < EX_RPW && rl < n;
    const uint4 h = have ? __ldg(hdr16 + R0 + rl) : make_uint4(0, 0, 0xFFu, 0);
    c.uo = have ? (u32)(__ldg(cum + R0 + rl) - cum0 - (u64)REC_W * rl) : 0u;
    c.eb = have ? (u32)(((gidx ? (u64)__ldg(gidx + R0 + rl) : R0 + rl) - G0) << 5) : 0u;
    const u32 op = h.z & 0xFFu, space = (h.z >> 8) & 0xFFu, sl = (h.z >> 16) & 0xFFu, fl = (h.z >> 24) & 0xFFu;
    c.sel = __ballot_sync(0xFFFFFFFFu, have && op <= BC_OP_AR_GLB);
    const bool rv = have && op <= BC_OP_AR_GLB && sl <= 4 && space <= 1 && h.x < g.n_warps;
    const u32 nk = rv ? max(1u, (1u << sl) >> g.G) : 1u;
    const u32 opc = op == BC_OP_LD ? IOP_LD : op == BC_OP_ATOM ? IOP_ATOM
                                                             : (((fl & BC_REC_SAME_VALUE) || (g.flags & GEO_F_VALUES))
                                                                    ? IOP_ST_SV : IOP_ST);
    c.mask = h.y;
    c.meta = (u32)rv | ((u32)(op <= BC_OP_ATOM) << 1) | ((u32)(space == BC_SPACE_SHARED) << 2) | (opc << 3) |
             ((sl & 7u) << 5) | ((nk - 1u) << 8) | ((u32)(op != BC_OP_LD) << 13);
    c.sb = (rv && space == BC_SPACE_SHARED) ? shared_base + blk_of(g, h.x) * g.smem_gran : 0u;
    // two rows per instruction: lanes 0-15 the k-th selected record, lanes 16-31 the (k+1)-th
    u32 m = c.sel;
    while (m) {
      const int ja = __ffs(m) - 1;
      m &= m - 1;
      const int jb = m ? __ffs(m) - 1 : -1;
      if (m) m &= m - 1;
      const int j = lane < 16 ? ja : jb;
      if (j >= 0) {
        const int q = lane & 15;  // 16-B piece of the row
        const char* src = reinterpret_cast<const char*>(&recs[R0 + r0 + j].addr[0]) + q * 16;
        char* dst = reinterpret_cast<char*>(rows + ((size_t)stg * EX_RPW + j) * 32) + q * 16;
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
    return c;
  };
  u64 chunk = (u64)blockIdx.x * EX_WARPS + wid;
  int stg = 0;
  Ch cur = chunk < n_chunks ? issue(chunk, 0) : Ch{};
  for (; chunk < n_chunks; chunk += nw, stg ^= 1) {
    Ch nxt{};
    if (chunk + nw < n_chunks) nxt = issue(chunk + nw, stg ^ 1);
    else asm volatile("cp.async.commit_group;" ::: "memory");  // (keeps the group count: wait 1 = current)
    asm volatile("cp.async.wait_group 1;" ::: "memory");
    __syncwarp();
    const u64* const crow = rows + (size_t)stg * EX_RPW * 32;
    u32 mem = cur.sel;
    while (mem) {
      const int j = __ffs(mem) - 1;
      mem &= mem - 1;
      const u32 uoj = __shfl_sync(0xFFFFFFFFu, cur.uo, j);
      const u32 evb = __shfl_sync(0xFFFFFFFFu, cur.eb, j);
      const u32 hmask = __shfl_sync(0xFFFFFFFFu, cur.mask, j), meta = __shfl_sync(0xFFFFFFFFu, cur.meta, j);
      const u32 sb = __shfl_sync(0xFFFFFFFFu, cur.sb, j);
      if (!((meta & 1u) && ((hmask >> lane) & 1u))) continue;
      const u64 a = crow[j * 32 + lane];
      const u32 alo = (u32)a, ahi = (u32)(a >> 32);
      const u32 sl = (meta >> 5) & 7u;
      if (alo & ((1u << sl) - 1u)) bad = true;  // natural alignment
      if ((meta & 4u) && a + (1ull << sl) > g.smem) bad = true;
      if (!(meta & 2u)) continue;  // ACQ / REL / AR: alignment only
      const u32 nk = ((meta >> 8) & 31u) + 1u;
      const u32 opc = (meta >> 3) & 3u;
      u32 key0 = KEY_DROP;
      if (bad) {
      } else if (meta & 4u) {
        key0 = sb + (alo >> g.G);  // shared: a < smem_bytes
      } else if (ahi < (1u << 16)) {  // < 2^48: 2^28 1-MB pages
        const u32 p = (ahi << 12) | (alo >> 20);
        const u32 pw = __ldg(&page_bits[p >> 5]);
        const u32 bit = p & 31u;
        if ((pw >> bit) & 1u)
          key0 = (__ldg(&page_rank[p >> 5]) + __popc(pw & ((1u << bit) - 1u))) << (20 - g.G) | ((alo & 0xFFFFFu) >> g.G);
        else if (g.flags & GEO_F_DECLARED)
          undecl = true;  // streaming: the page set is the declared allocations, nothing may fall outside
        else if (meta & (1u << 13))
          pmiss = true;   // a write outside the (sampled) page set: the set is incomplete
      } else {
        ovf = true;
      }
      const u32 o = uoj + (u32)__popc(hmask & lt) * nk;  // window slots < 2^30
      const u32 ev = evb | (u32)lane;                    // window-local event id
      if (nk == 1 && g.world == 1) {  // one granule, one shard: the common case
        okeys[o] = key0 != KEY_DROP ? ((key0 << 2) | opc) : KEY_DROP;
        oevs[o] = ev;
        continue;
      }
      for (u32 k = 0; k < nk; ++k) {
        const bool mine = key0 != KEY_DROP && (g.world == 1 || shard_of(key0 + k, g.world) == g.rank);
        okeys[o + k] = mine ? (((key0 + k) << 2) | opc) : KEY_DROP;
        oevs[o + k] = ev;
      }
    }
    __syncwarp();  // every lane is done with this stage: the next issue may refill it
    cur = nxt;
  }
  asm volatile("cp.async.wait_group 0;" ::: "memory");
  if (__any_sync(0xFFFFFFFFu, bad) && lane == 0) set_err(err, ERR_INFEASIBLE);
  if (__any_sync(0xFFFFFFFFu, ovf) && lane == 0) set_err(err, ERR_OVERFLOW);
  if (__any_sync(0xFFFFFFFFu, undecl) && lane == 0) set_err(err, ERR_UNDECLARED);
  if (__any_sync(0xFFFFFFFFu, pmiss) && lane == 0) set_err(err, ERR_PAGES);
}

// Window k = the records whose weight prefix cum[r] (exclusive) lies in [k * we, (k + 1) * we):
// starts[k] = lower bound of k * we in cum (n + 1 entries, cum[n] = total), starts[nwin] = n;
// bounds[k] = the window's item upper bound (its weight minus REC_W per record).
__global__ void k_window_starts(const u64* __restrict__ cum, u64 n, u64 we, u32 nwin, u64* __restrict__ starts,
                                u64* __restrict__ bounds) {
  const u32 k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k > nwin) return;
  auto lb = [&](u64 v) {
    u64 lo = 0, hi = n;
    while (lo < hi) {
      const u64 m = (lo + hi) >> 1;
      if (cum[m] < v) lo = m + 1; else hi = m;
    }
    return lo;
  };
  const u64 s0 = k == 0 ? 0 : (k == nwin ? n : lb((u64)k * we));
  starts[k] = s0;
  if (k < nwin) {
    const u64 s1 = k + 1 == nwin ? n : lb((u64)(k + 1) * we);
    bounds[k] = (cum[s1] - cum[s0]) - (u64)REC_W * (s1 - s0);
  }
}
void launch_window_starts(const u64* cum, u64 n, u64 we, u32 nwin, u64* starts, u64* bounds, cudaStream_t st) {
  k_window_starts<<<(nwin + 1 + 255) / 256, 256, 0, st>>>(cum, n, we, nwin, starts, bounds);
  ++g_launches;
}

// Ranks of the written 1-MB pages in address order (the dense global key space):
// `words` = the non-zero bitmap words; unless `presorted`, the CTA first sorts them in shared memory
// (bitonic, up to PR_MAX words; a longer list sets *need_sort and returns, and the host sorts it with
// the radix sort and calls again with presorted = 1).  page_rank[word] = set bits in all lower words;
// wl_prefix[i] = page_rank[words[i]]; *n_pages_dev = written pages.  The CTA walks the list in
// chunks of 1024 with a running carry; only listed words of page_rank are ever read.
constexpr u32 PR_MAX = 8192;
__global__ void __launch_bounds__(1024) k_page_rank(u32* __restrict__ words, const u64* __restrict__ n_words_dev,
                                                    const u32* __restrict__ page_bits, u32* __restrict__ page_rank,
                                                    u32* __restrict__ wl_prefix, u64* __restrict__ n_pages_dev,
                                                    u32* __restrict__ need_sort, int presorted) {
  __shared__ u32 wsum[32];
  __shared__ u32 s_carry;
  __shared__ u32 sw[PR_MAX];
  const u32 t = threadIdx.x, w = t >> 5, l = t & 31;
  const u64 nw = *n_words_dev;
  if (!presorted) {
    if (nw > PR_MAX) {
      if (t == 0) *need_sort = 1u;
      return;
    }
    u32 P = 1;
    while (P < nw) P <<= 1;
    for (u32 i = t; i < P; i += 1024) sw[i] = i < nw ? words[i] : 0xFFFFFFFFu;
    __syncthreads();
    for (u32 k = 2; k <= P; k <<= 1) {
      for (u32 j = k >> 1; j > 0; j >>= 1) {
        for (u32 i = t; i < P; i += 1024) {
          const u32 ij = i ^ j;
          if (ij > i) {
            const u32 a = sw[i], b = sw[ij];
            if (((i & k) == 0) == (a > b)) {
              sw[i] = b;
              sw[ij] = a;
            }
          }
        }
        __syncthreads();
      }
    }
    for (u32 i = t; i < nw; i += 1024) words[i] = sw[i];
  }
  if (t == 0) s_carry = 0;
  __syncthreads();
  for (u64 c0 = 0; c0 < nw; c0 += 1024) {
    const u64 i = c0 + t;
    const u32 wd = i < nw ? words[i] : 0u;
    const u32 v = i < nw ? (u32)__popc(page_bits[wd]) : 0u;
    const u32 x = warp_incl_sum(v);
    if (l == 31) wsum[w] = x;
    __syncthreads();
    u32 off = 0, tot = 0;
    for (u32 ww = 0; ww < 32; ++ww) {
      if (ww < w) off += wsum[ww];
      tot += wsum[ww];
    }
    const u32 carry = s_carry;
    if (i < nw) {
      const u32 r = carry + off + x - v;
      page_rank[wd] = r;
      wl_prefix[i] = r;
    }
    __syncthreads();
    if (t == 0) s_carry = carry + tot;
    __syncthreads();
  }
  if (t == 0) *n_pages_dev = s_carry;
}

// --------------------------------------------------------------------- host launchers
void launch_header(const bc_record* recs, const Geo& g, u32* wkey, u32* wval, u32* if_cnt, u32* bar_cnt,
                   u32* sync_list, u32* page_bits, u32* word_list, u64* cnt, u32* rec_w, uint4* hdr16,
                   u32* rec_cnt, u32* err, cudaStream_t st, int mark_pages) {
  u64 warps = (g.n_recs + 31) / 32;
  if (warps == 0) return;
  u64 blocks = (warps + 7) / 8;
  k_header<<<(unsigned)blocks, 256, 0, st>>>(recs, g, wkey, wval, if_cnt, bar_cnt, sync_list, page_bits, word_list, cnt,
                                             rec_w, hdr16, rec_cnt, err, mark_pages); ++g_launches;
}

void launch_warp_start(const u32* skeys, u64 n, u32 n_warps, u32* warp_start, cudaStream_t st) {
  k_warp_start<<<(n_warps + 1 + 255) / 256, 256, 0, st>>>(skeys, n, n_warps, warp_start); ++g_launches;
}

void launch_replay(const uint4* hdr16, const u32* wrec, const u32* gidx, const u32* warp_start, const Geo& g,
                   const u32* node_base, const u32* bar_base, uint4* snap, uint4* nodes, u32* bar_rec, u32* bar_next,
                   u32* find_blk, u32* find_rec, u32* find_cnt, u32* err, cudaStream_t st) {
  k_replay<<<(unsigned)(((u64)g.n_warps * 32 + 255) / 256), 256, 0, st>>>(hdr16, wrec, gidx, warp_start, g, node_base, bar_base, snap, nodes,
                                                     bar_rec, bar_next, find_blk, find_rec, find_cnt, err); ++g_launches;
}

void launch_barriers(const Geo& g, const u32* bar_cnt, const u32* bar_base, const u32* bar_rec, const u32* bar_next,
                     u32* blockR, u32* err, cudaStream_t st, bool allow_pending) {
  k_barriers<<<(unsigned)(((u64)g.n_blocks * 32 + 255) / 256), 256, 0, st>>>(g, bar_cnt, bar_base, bar_rec, bar_next,
                                                                             blockR, err, allow_pending ? 1 : 0);
  ++g_launches;
}

// snapshot .w: barrier phase -> label of the block's last completed barrier (0 = none)
__global__ void k_snap_blab(uint4* __restrict__ snap, u64 n, u32 wpb, u32 n_warps, u64 n_bars,
                            const u32* __restrict__ bar_base, const u32* __restrict__ blockR) {
  u64 r = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= n) return;
  uint2 v = *reinterpret_cast<const uint2*>(reinterpret_cast<const u32*>(snap + r) + 2);  // (node, phase)
  u32 w = reinterpret_cast<const u32*>(snap + r)[0];
  u32 ph = v.y;
  u32 lab = 0;
  if (ph && w < n_warps) {  // (records after an infeasibility are garbage; results are discarded)
    u64 i = (u64)bar_base[(w / wpb) * wpb] + ph - 1;
    lab = i < n_bars ? blockR[i] : 0u;
  }
  reinterpret_cast<u32*>(snap + r)[3] = lab;
}
void launch_snap_blab(uint4* snap, u64 n, u32 wpb, u32 n_warps, u64 n_bars, const u32* bar_base, const u32* blockR,
                      cudaStream_t st) {
  if (!n || !n_bars) return;  // no barrier: every phase is 0 and k_replay already wrote label 0
  k_snap_blab<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(snap, n, wpb, n_warps, n_bars, bar_base, blockR);
  ++g_launches;
}

void launch_page_rank(u32* words, const u64* n_words_dev, const u32* page_bits, u32* page_rank, u32* wl_prefix,
                      u64* n_pages_dev, u32* need_sort, int presorted, cudaStream_t st) {
  k_page_rank<<<1, 1024, 0, st>>>(words, n_words_dev, page_bits, page_rank, wl_prefix, n_pages_dev, need_sort,
                                  presorted);
  ++g_launches;
}

// Small grids (n_warps <= WS_SMALL): one CTA turns the header's per-warp counters into K1's CSR offsets
// (warp_start = exclusive scan of records per warp, + total), the SIMT-node bases (n_warps + 2 x
// exclusive scan of IFs) and the barrier bases (exclusive scan of BARs) -- one launch instead of a
// binary search per warp and two device-wide scans.
__global__ void __launch_bounds__(1024) k_warp_scans(const u32* __restrict__ rec_cnt, const u32* __restrict__ if_cnt,
                                                     const u32* __restrict__ bar_cnt, u32 n_warps,
                                                     u32* __restrict__ warp_start, u32* __restrict__ node_base,
                                                     u32* __restrict__ bar_base) {
  __shared__ u32 wsum[3][32];
  __shared__ u32 s_carry[3];
  const u32 t = threadIdx.x, wi = t >> 5, l = t & 31;
  if (t < 3) s_carry[t] = 0;
  __syncthreads();
  for (u32 c0 = 0; c0 < n_warps; c0 += 1024) {
    const u32 w = c0 + t;
    u32 v[3], x[3];
    v[0] = w < n_warps ? rec_cnt[w] : 0u;
    v[1] = w < n_warps ? if_cnt[w] : 0u;
    v[2] = w < n_warps ? bar_cnt[w] : 0u;
#pragma unroll
    for (int a = 0; a < 3; ++a) {
      x[a] = warp_incl_sum(v[a]);
      if (l == 31) wsum[a][wi] = x[a];
    }
    __syncthreads();
    u32 off[3] = {0, 0, 0}, tot[3] = {0, 0, 0};
    for (u32 q = 0; q < 32; ++q) {
#pragma unroll
      for (int a = 0; a < 3; ++a) {
        if (q < wi) off[a] += wsum[a][q];
        tot[a] += wsum[a][q];
      }
    }
    u32 ex[3];
#pragma unroll
    for (int a = 0; a < 3; ++a) ex[a] = s_carry[a] + off[a] + x[a] - v[a];
    if (w < n_warps) {
      warp_start[w] = ex[0];
      node_base[w] = n_warps + 2u * ex[1];
      bar_base[w] = ex[2];
    }
    __syncthreads();
    if (t < 3) s_carry[t] += tot[t];
    __syncthreads();
  }
  if (t == 0) warp_start[n_warps] = s_carry[0];
}
void launch_warp_scans(const u32* rec_cnt, const u32* if_cnt, const u32* bar_cnt, u32 n_warps, u32* warp_start,
                       u32* node_base, u32* bar_base, cudaStream_t st) {
  k_warp_scans<<<1, 1024, 0, st>>>(rec_cnt, if_cnt, bar_cnt, n_warps, warp_start, node_base, bar_base);
  ++g_launches;
}

__global__ void k_node_base(const u32* __restrict__ if_excl, u32 n_warps, u32* __restrict__ node_base) {
  u32 w = blockIdx.x * blockDim.x + threadIdx.x;
  if (w < n_warps) node_base[w] = n_warps + 2u * if_excl[w];
}
void launch_node_base(const u32* if_excl, u32 n_warps, u32* node_base, cudaStream_t st) {
  k_node_base<<<(n_warps + 255) / 256, 256, 0, st>>>(if_excl, n_warps, node_base); ++g_launches;
}

void launch_expand(const bc_record* recs, const uint4* hdr16, const Geo& g, const u32* page_bits, const u32* page_rank,
                   u32 shared_base, const u64* cum, u64 R0, u64 R1, const u32* gidx, u64 G0, u32* keys, u32* evs,
                   u32* err, cudaStream_t st) {
  const u64 chunks = (R1 - R0 + EX_RPW - 1) / EX_RPW;
  if (!chunks) return;
  static int grid[64] = {};  // per device: the shared-memory opt-in and the occupancy-derived grid
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) dev = 0;
  if (!grid[dev]) {
    int sms = 148, per = 1;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaFuncSetAttribute(k_expand, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)EX_SMEM);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_expand, EX_THREADS, EX_SMEM);
    grid[dev] = sms * (per > 0 ? per : 1);
  }
  const unsigned gr = (unsigned)std::min<u64>((chunks + EX_WARPS - 1) / EX_WARPS, (u64)grid[dev]);
  k_expand<<<gr, EX_THREADS, EX_SMEM, st>>>(recs, hdr16, g, page_bits, page_rank, shared_base, cum, R0, R1, gidx, G0,
                                            keys, evs, err);
  ++g_launches;
}

void preload_trace() {
  preload(k_barriers, k_expand, k_header, k_mark_ranges, k_node_base, k_page_rank, k_replay, k_snap_blab,
          k_warp_scans, k_warp_start, k_window_starts);
}

}  // namespace bc
