// shard.cu — block-sharded multi-GPU race check (SURVEY.md §8 row e).
//
// Rank r of W holds the records of the traced blocks b with b % W == r (bc_load_trace_shard, with
// their global record indices): the paper's per-block queues as the unit of
// partitioning.  Per bc_detect:
//   1. header, K1 and K2 (clock replay) over the LOCAL records only: every warp, barrier and SIMT
//      stack of a block lives on one rank; step labels are global record indices + 1;
//   2. the clock state every rank needs for the checks it owns is exchanged once: the 16-B record
//      snapshots (all-gather, then scattered to global record positions), the branch nodes (global
//      ids: rank offsets of the IF counts), the written-page set (union), and the sync records
//      (ACQ / REL / AR, 272 B each) on which every rank builds the same K3 sync skeleton ("epoch clock
//      deltas broadcast");
//   3. per trace window (global record ranges): K4 expands the local records; each item goes to the
//      owner of its granule -- shared memory: the block's own rank (no traffic); global memory: a
//      hash of the granule -- by one all-to-all; the owner sorts what it received by (event, then
//      granule), so each granule's accesses are in global trace order, and runs K7 with its own
//      32-B shadow entries carried between windows;
//   4. race records and barrier-divergence findings are gathered to rank 0, whose K8 finalize sorts
//      them into the canonical list.
// Every rank runs the same sequence of collectives; error states are agreed on before any branch.
#include <algorithm>
#include <cstring>
#include <vector>

#include "ctx.cuh"

namespace bc {

namespace {

inline unsigned nb(u64 n) { return (unsigned)((n + 255) / 256); }

// (word index, bits) of the non-zero page-bitmap words this rank listed
__global__ void k_pack_words(const u32* __restrict__ words, const u32* __restrict__ bits, u64 n, uint2* __restrict__ out) {
  const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) out[i] = make_uint2(words[i], bits[words[i]]);
}
// OR every rank's words into the bitmap; a word that turns non-zero is listed (as k_header does)
__global__ void k_merge_words(const uint2* __restrict__ in, u64 n, u32* __restrict__ bits, u32* __restrict__ words,
                              u64* __restrict__ n_words) {
  const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint2 v = in[i];
  if ((bits[v.x] | v.y) == bits[v.x]) return;
  if (atomicOr(&bits[v.x], v.y) == 0u) {
    const u64 at = atomicAdd((unsigned long long*)n_words, 1ull);
    words[at] = v.x;
  }
}
__global__ void k_add_u32(u32* __restrict__ p, u64 n, u32 add) {
  const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] += add;
}
// SIMT root node of every warp (rank-independent: the warp's initial mask)
__global__ void k_roots(uint4* __restrict__ nodes, Geo g) {
  const u32 w = blockIdx.x * blockDim.x + threadIdx.x;
  if (w < g.n_warps) nodes[w] = make_uint4(init_mask(g, w), NONE, 0u, 0u);
}
// dst[idx[i]] = src[i]
__global__ void k_scatter16(const uint4* __restrict__ src, const u32* __restrict__ idx, u64 n, uint4* __restrict__ dst) {
  const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) dst[idx[i]] = src[i];
}
__global__ void k_gather_u32s(const u32* __restrict__ src, const u32* __restrict__ idx, u64 n, u32* __restrict__ dst) {
  const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) dst[i] = src[idx[i]];
}
// compact copy of the local sync records (one warp per record)
__global__ void k_gather_recs(const bc_record* __restrict__ recs, const u32* __restrict__ idx, u64 n,
                              bc_record* __restrict__ dst) {
  const u64 i = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const u32 l = threadIdx.x & 31;
  if (i >= n) return;
  const u32* s = reinterpret_cast<const u32*>(recs + idx[i]);
  u32* d = reinterpret_cast<u32*>(dst + i);
  for (u32 q = l; q < sizeof(bc_record) / 4; q += 32) d[q] = s[q];
}
// window k = global records [k * rw, (k + 1) * rw): first local position and local item bound
__global__ void k_shard_windows(const u32* __restrict__ gidx, u64 nl, const u64* __restrict__ cum, u64 rw, u32 nwin,
                                u64* __restrict__ pstart, u64* __restrict__ pbound) {
  const u32 k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k > nwin) return;
  auto lb = [&](u64 v) {
    u64 lo = 0, hi = nl;
    while (lo < hi) {
      const u64 m = (lo + hi) >> 1;
      if ((u64)gidx[m] < v) lo = m + 1; else hi = m;
    }
    return lo;
  };
  const u64 p0 = lb((u64)k * rw);
  pstart[k] = p0;
  if (k < nwin) {
    const u64 p1 = lb((u64)(k + 1) * rw);
    pbound[k] = (cum[p1] - cum[p0]) - (u64)REC_W * (p1 - p0);
  }
}
// destination rank of an item: its block's rank for shared granules, hash owner for global ones
__global__ void k_dest(const u32* __restrict__ keys, u64 n, u32 shared_base, u32 world, u32 rank,
                       u32* __restrict__ dest, u32* __restrict__ idx) {
  const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const u32 k = keys[i];
  dest[i] = k == KEY_DROP ? KEY_DROP : ((k >> 2) >= shared_base ? rank : shard_of(k >> 2, world));
  idx[i] = (u32)i;
}
// counts per destination of the dest-sorted list (lower bounds)
__global__ void k_dest_counts(const u32* __restrict__ dsorted, const u64* __restrict__ n_dev, u32 world,
                              u64* __restrict__ counts) {
  const u32 r = threadIdx.x;
  if (r > world) return;
  __shared__ u64 lo_r[1025];
  const u64 n = *n_dev;
  u64 lo = 0, hi = n;
  while (lo < hi) {
    const u64 m = (lo + hi) >> 1;
    if (dsorted[m] < r) lo = m + 1; else hi = m;
  }
  lo_r[r] = lo;
  __syncthreads();
  if (r < world) counts[r] = lo_r[r + 1] - lo_r[r];
}
__global__ void k_gather_items(const u32* __restrict__ keys, const u32* __restrict__ evs, const u32* __restrict__ perm,
                               const u64* __restrict__ n_dev, u32* __restrict__ ok, u32* __restrict__ oe) {
  const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= *n_dev) return;
  const u32 p = perm[i];
  ok[i] = keys[p];
  oe[i] = evs[p];
}
__global__ void k_set_u64(u64* p, u64 v) { *p = v; }

}  // namespace
}  // namespace bc

// All ranks agree: the worst (most negative) status any rank reached.
static bc_status agree(bc_ctx* c, bc_status s, u64* dtmp) {
  std::vector<u64> all(c->comm->world);
  const u64 mine = (u64)(int64_t)s;
  if (allgather_u64(c->comm, &mine, 1, all.data(), dtmp, c->stream)) return fail(c, BC_ERR_NCCL, "status exchange");
  bc_status worst = BC_OK;
  for (u64 v : all) worst = std::min(worst, (bc_status)(int64_t)v);
  if (worst != BC_OK && s == BC_OK) c->err = "another rank failed";
  return worst;
}

bc_status detect_sharded(bc_ctx* c, Scratch& S) {
  Comm* cm = c->comm;
  const int W = cm->world, me = cm->rank;
  cudaStream_t st = c->stream;
  Geo g = c->g;
  g.world = 1;  // ownership is decided by the routing below, not by K4's filter
  g.rank = 0;
  g.n_recs = c->n_global;
  const u64 nl = c->n_recs, n = c->n_global;
  const bc_record* recs = c->trace;
  const u32* gidx = c->gidx;
  bc_stats& sx = c->stats;
  memset(&sx, 0, sizeof(sx));
  c->n_races = 0;
  const u64 launches0 = g_launches;
  u64* const hcnt = c->hcnt;
  u64* dtmp = S.alloc<u64>(4 * (size_t)(W + 1) * 8);  // small exchange scratch
  cudaEventRecord(c->ev[0], st);

  // ---- 1. header over the local records
  const u64 nwords = 1ull << 23;
  u64* cnt = S.alloc<u64>(C_N);
  u32* err = reinterpret_cast<u32*>(cnt + C_ERR);
  const u64 nla = std::max<u64>(nl, 1);
  u32* wkey = S.alloc<u32>(nla);
  u32* wval = S.alloc<u32>(nla);
  const bool small_w = g.n_warps <= WS_SMALL;
  u32* wcnt = S.alloc<u32>(3 * (size_t)(g.n_warps + 1));
  u32* if_cnt = wcnt;
  u32* bar_cnt = wcnt + (g.n_warps + 1);
  u32* rec_cnt = small_w ? wcnt + 2 * (size_t)(g.n_warps + 1) : nullptr;
  u32* sync_list = S.alloc<u32>(nla);
  u32* page_bits = S.alloc<u32>(nwords);
  u32* rec_w = S.alloc<u32>(nla);
  uint4* hdr16 = S.alloc<uint4>(nla);
  u32* word_list = S.alloc<u32>(nwords);
  u32* wl2 = S.alloc<u32>(nwords);
  u32* page_rank = S.alloc<u32>(nwords);
  cudaMemsetAsync(cnt, 0, C_N * 8, st);
  cudaMemsetAsync(wcnt, 0, 3 * (size_t)(g.n_warps + 1) * 4, st);
  cudaMemsetAsync(page_bits, 0, nwords * 4, st);
  Geo gl = g;
  gl.n_recs = nl;
  launch_header(recs, gl, wkey, wval, if_cnt, bar_cnt, sync_list, page_bits, word_list, cnt, rec_w, hdr16, rec_cnt, err,
                st);
  cudaMemcpyAsync(hcnt, cnt, C_N * sizeof(u64), cudaMemcpyDeviceToHost, st);
  if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "header");
  std::vector<u64> loc(hcnt, hcnt + C_N);
  bc_status s0 = BC_OK;
  if ((u32)loc[C_ERR] & ERR_INFEASIBLE) s0 = fail(c, BC_ERR_INFEASIBLE_TRACE, "record header violates feasibility");
  else if ((u32)loc[C_ERR] & ERR_OVERFLOW) s0 = fail(c, BC_ERR_OVERFLOW, "global address >= 2^48");
  if (bc_status a = agree(c, s0, dtmp)) return a;
  // global counters (sums over the ranks)
  const int NS = 6;
  const u64 mine[NS] = {loc[C_LANE_EVENTS], loc[C_CONTROL_EVENTS], loc[C_SYNC_LANEOPS], loc[C_SYNC_RECS],
                        loc[C_ACQ_RECS], loc[C_IFS]};
  std::vector<u64> allc((size_t)W * NS);
  if (allgather_u64(cm, mine, NS, allc.data(), dtmp, st)) return fail(c, BC_ERR_NCCL, "counter exchange");
  u64 tot[NS] = {};
  u64 if_off = 0;
  std::vector<u64> nsync(W);
  for (int r = 0; r < W; ++r) {
    for (int q = 0; q < NS; ++q) tot[q] += allc[(size_t)r * NS + q];
    if (r < me) if_off += allc[(size_t)r * NS + 5];
    nsync[r] = allc[(size_t)r * NS + 3];
  }
  sx.records = n;
  sx.lane_events = tot[0];
  sx.control_events = tot[1];
  sx.sync_ops = tot[2];

  // ---- 2a. written pages: union of every rank's bitmap words
  {
    const u64 nw_l = loc[C_PAGE_WORDS];
    std::vector<u64> nw_all(W);
    if (allgather_u64(cm, &nw_l, 1, nw_all.data(), dtmp, st)) return fail(c, BC_ERR_NCCL, "page exchange");
    u64 nw_tot = 0;
    std::vector<u64> bytes(W);
    for (int r = 0; r < W; ++r) {
      bytes[r] = nw_all[r] * sizeof(uint2);
      nw_tot += nw_all[r];
    }
    uint2* mine_w = S.alloc<uint2>(nw_l + 1);
    uint2* all_w = S.alloc<uint2>(nw_tot + 1);
    if (nw_l) { k_pack_words<<<nb(nw_l), 256, 0, st>>>(word_list, page_bits, nw_l, mine_w); ++g_launches; }
    if (cm->allgatherv(mine_w, all_w, bytes.data(), st)) return fail(c, BC_ERR_NCCL, "page exchange");
    if (nw_tot) { k_merge_words<<<nb(nw_tot), 256, 0, st>>>(all_w, nw_tot, page_bits, word_list, cnt + C_PAGE_WORDS); ++g_launches; }
  }
  u32* words = word_list;
  u32* wl_prefix = wl2;
  u32* need_sort = reinterpret_cast<u32*>(cnt + C_NEED_SORT);
  launch_page_rank(words, cnt + C_PAGE_WORDS, page_bits, page_rank, wl_prefix, cnt + C_PAGES, need_sort, 0, st);
  cudaMemcpyAsync(hcnt, cnt, C_N * sizeof(u64), cudaMemcpyDeviceToHost, st);
  if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "pages");
  if ((u32)hcnt[C_NEED_SORT]) {
    const u64 nwl = hcnt[C_PAGE_WORDS];
    if (radix_sort_pairs(word_list, nullptr, wl2, nullptr, nwl, 0, 23, S.alloc<char>(rs_temp_bytes(nwl)), st)) {
      words = wl2;
      wl_prefix = word_list;
    }
    launch_page_rank(words, cnt + C_PAGE_WORDS, page_bits, page_rank, wl_prefix, cnt + C_PAGES, need_sort, 1, st);
    cudaMemcpyAsync(hcnt, cnt, C_N * sizeof(u64), cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "pages");
  }
  const u64 n_pages = hcnt[C_PAGES], n_words = hcnt[C_PAGE_WORDS];
  sx.written_pages = n_pages;
  const u32 shared_base = (u32)std::min<u64>(n_pages << (20 - g.G), 0xFFFFFFFFull);
  const u64 n_keys = (n_pages << (20 - g.G)) + (u64)g.n_blocks * g.smem_gran;
  if (n_keys >= (1ull << 30)) return fail(c, BC_ERR_OVERFLOW, "shadow key space >= 2^30 granules");
  cudaEventRecord(c->ev[1], st);

  // ---- 1b. K1 + K2 over the local records (node ids: this rank's range of the global node table)
  u32* wk2 = S.alloc<u32>(nla);
  u32* wv2 = S.alloc<u32>(nla);
  bool alt = radix_sort_pairs(wkey, wval, wk2, wv2, nl, 0, bits_for(g.n_warps - 1), S.alloc<char>(rs_temp_bytes(nl)), st);
  u32* skeys = alt ? wk2 : wkey;
  u32* wrec = alt ? wv2 : wval;
  u32* warp_start = S.alloc<u32>(g.n_warps + 1);
  u32* node_base = S.alloc<u32>(g.n_warps + 1);
  u32* bar_base = S.alloc<u32>(g.n_warps + 1);
  const u64 n_if_l = loc[C_IFS], n_bar = loc[C_BARS];
  if (small_w) {
    launch_warp_scans(rec_cnt, if_cnt, bar_cnt, g.n_warps, warp_start, node_base, bar_base, st);
  } else {
    launch_warp_start(skeys, nl, g.n_warps, warp_start, st);
    exclusive_scan_u32(if_cnt, node_base, g.n_warps, S.alloc<char>(scan_temp_bytes(g.n_warps)), nullptr, st);
    launch_node_base(node_base, g.n_warps, node_base, st);
    exclusive_scan_u32(bar_cnt, bar_base, g.n_warps, S.alloc<char>(scan_temp_bytes(g.n_warps)), nullptr, st);
  }
  if (if_off) { k_add_u32<<<nb(g.n_warps), 256, 0, st>>>(node_base, g.n_warps, (u32)(2 * if_off)); ++g_launches; }
  const u64 n_if = tot[5];
  const u64 n_nodes = g.n_warps + 2 * n_if;
  uint4* snap_l = S.alloc<uint4>(nla);
  uint4* nodes = S.alloc<uint4>(n_nodes);
  u32* bar_rec = S.alloc<u32>(n_bar + 1);
  u32* bar_next = S.alloc<u32>(n_bar + 1);
  u32* blockR = S.alloc<u32>(n_bar + 1);
  u32* find_blk = S.alloc<u32>(n_bar + 1);
  u32* find_rec = S.alloc<u32>(n_bar + 1);
  u32* find_cnt = reinterpret_cast<u32*>(cnt + C_FINDINGS);
  cudaEventRecord(c->ev[2], st);
  launch_replay(hdr16, wrec, gidx, warp_start, g, node_base, bar_base, snap_l, nodes, bar_rec, bar_next, find_blk,
                find_rec, find_cnt, err, st);
  launch_barriers(g, bar_cnt, bar_base, bar_rec, bar_next, blockR, err, st);
  launch_snap_blab(snap_l, nl, g.wpb, g.n_warps, n_bar, bar_base, blockR, st);
  cudaMemcpyAsync(hcnt, cnt, C_N * sizeof(u64), cudaMemcpyDeviceToHost, st);
  if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "replay");
  const u32 nfind_l = (u32)hcnt[C_FINDINGS];
  s0 = ((u32)hcnt[C_ERR] & ERR_INFEASIBLE) ? fail(c, BC_ERR_INFEASIBLE_TRACE, "SIMT stack / barrier feasibility")
                                           : BC_OK;
  if (bc_status a = agree(c, s0, dtmp)) return a;

  // ---- 2b. global clock tables: record snapshots and branch nodes of every rank
  std::vector<u64> nl_all(W);
  if (allgather_u64(cm, &nl, 1, nl_all.data(), dtmp, st)) return fail(c, BC_ERR_NCCL, "size exchange");
  uint4* snap = S.alloc<uint4>(n + 1);
  {
    std::vector<u64> b16(W), b4(W);
    u64 ntot = 0;
    for (int r = 0; r < W; ++r) {
      b16[r] = nl_all[r] * 16;
      b4[r] = nl_all[r] * 4;
      ntot += nl_all[r];
    }
    if (ntot != n) return fail(c, BC_ERR_INVALID_ARG, "the shards do not add up to the global record count");
    uint4* sall = S.alloc<uint4>(ntot + 1);
    u32* iall = S.alloc<u32>(ntot + 1);
    if (cm->allgatherv(snap_l, sall, b16.data(), st) || cm->allgatherv(gidx, iall, b4.data(), st))
      return fail(c, BC_ERR_NCCL, "snapshot exchange");
    if (ntot) { k_scatter16<<<nb(ntot), 256, 0, st>>>(sall, iall, ntot, snap); ++g_launches; }
    std::vector<u64> bn(W);
    for (int r = 0; r < W; ++r) bn[r] = allc[(size_t)r * NS + 5] * 2 * 16;
    uint4* ifn = nodes + g.n_warps;
    // rank-major IF-node ranges = the node table's order (in place: this rank's range is its send buffer)
    if (cm->allgatherv(ifn + 2 * if_off, ifn, bn.data(), st)) return fail(c, BC_ERR_NCCL, "node exchange");
    k_roots<<<nb(g.n_warps), 256, 0, st>>>(nodes, g);
    ++g_launches;
  }
  cudaEventRecord(c->ev[3], st);

  // ---- 2c. K3: every rank builds the sync skeleton from all sync records
  HbCtx hc{};
  hc.g = g;
  hc.snap = snap;
  hc.nodes = nodes;
  hc.n_nodes = (u32)n_nodes;
  hc.err = err;
  const u64 n_srec = tot[3];
  if (n_srec) {
    const u64 ns_l = loc[C_SYNC_RECS];
    bc_record* srec_l = S.alloc<bc_record>(ns_l + 1);
    u32* sidx_l = S.alloc<u32>(ns_l + 1);
    if (ns_l) {
      // local sync records in local order (= global order) and their global indices
      u32* k2 = S.alloc<u32>(ns_l);
      const bool a2 = radix_sort_pairs(sync_list, nullptr, k2, nullptr, ns_l, 0, bits_for(nl), S.alloc<char>(rs_temp_bytes(ns_l)), st);
      const u32* sl = a2 ? k2 : sync_list;
      k_gather_recs<<<nb(ns_l * 32), 256, 0, st>>>(recs, sl, ns_l, srec_l);
      k_gather_u32s<<<nb(ns_l), 256, 0, st>>>(gidx, sl, ns_l, sidx_l);
      g_launches += 2;
    }
    std::vector<u64> br(W), bi(W);
    for (int r = 0; r < W; ++r) {
      br[r] = nsync[r] * sizeof(bc_record);
      bi[r] = nsync[r] * 4;
    }
    bc_record* srec_a = S.alloc<bc_record>(n_srec);
    u32* sidx_a = S.alloc<u32>(n_srec);
    if (cm->allgatherv(srec_l, srec_a, br.data(), st) || cm->allgatherv(sidx_l, sidx_a, bi.data(), st))
      return fail(c, BC_ERR_NCCL, "sync record exchange");
    // trace order across ranks: sort by global index, gather the records
    u32* perm = S.alloc<u32>(n_srec);
    u32* pk = S.alloc<u32>(n_srec);
    u32* pp = S.alloc<u32>(n_srec);
    launch_iota(perm, (u32)n_srec, st);
    const bool a3 = radix_sort_pairs(sidx_a, perm, pk, pp, n_srec, 0, bits_for(n), S.alloc<char>(rs_temp_bytes(n_srec)), st);
    u32* sidx = a3 ? pk : sidx_a;
    u32* sperm = a3 ? pp : perm;
    bc_record* srecs = S.alloc<bc_record>(n_srec);
    k_gather_recs<<<nb(n_srec * 32), 256, 0, st>>>(srec_a, sperm, n_srec, srecs);
    ++g_launches;
    u64 ne = 0;
    int rs = run_sync_skeleton(srecs, sidx, (u32)n_srec, (u32)tot[2], (u32)tot[4], hc, S, st, &ne);
    if (bc_status a = agree(c, (bc_status)rs, dtmp)) return fail(c, a, "sync skeleton");
  }
  cudaEventRecord(c->ev[4], st);

  // ---- 3. windows: global record ranges of (about) `we` weight
  u64* cum = S.alloc<u64>(nl + 1);
  exclusive_scan_u32_u64(rec_w, cum, nl, S.alloc<char>(scan_temp_bytes(nl)), cum + nl, st);
  u64 wl_tot = 0;
  cudaMemcpyAsync(&wl_tot, cum + nl, 8, cudaMemcpyDeviceToHost, st);
  if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "weights");
  std::vector<u64> wall(W);
  if (allgather_u64(cm, &wl_tot, 1, wall.data(), dtmp, st)) return fail(c, BC_ERR_NCCL, "weight exchange");
  u64 total_w = 0;
  for (u64 v : wall) total_w += v;
  const u64 we = c->cfg.window_events ? std::min<u64>(c->cfg.window_events, WIN_MAX)
                                      : (total_w <= WIN_MAX ? WIN_MAX : (1ull << 28));
  u64 nwin = std::max<u64>(1, (total_w + we - 1) / we);
  u64 rw = (n + nwin - 1) / nwin;
  rw = std::max<u64>(1, std::min<u64>(rw, 1ull << 26));  // < 2^27 records: 32-bit window-local events
  nwin = std::max<u64>(1, (n + rw - 1) / rw);
  if (nwin >= (1ull << 31)) return fail(c, BC_ERR_INVALID_ARG, "window_events too small for this trace");
  std::vector<u64> pst(nwin + 1), pbd(nwin);
  {
    u64* d_ps = S.alloc<u64>(nwin + 1);
    u64* d_pb = S.alloc<u64>(nwin);
    k_shard_windows<<<(unsigned)((nwin + 1 + 255) / 256), 256, 0, st>>>(gidx, nl, cum, rw, (u32)nwin, d_ps, d_pb);
    ++g_launches;
    cudaMemcpyAsync(pst.data(), d_ps, (nwin + 1) * 8, cudaMemcpyDeviceToHost, st);
    cudaMemcpyAsync(pbd.data(), d_pb, nwin * 8, cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "windows");
  }
  u64 maxb = 1;
  for (u64 k = 0; k < nwin; ++k) maxb = std::max(maxb, pbd[k]);
  u32* ikeys = S.alloc<u32>(maxb + 1);
  u32* ievs = S.alloc<u32>(maxb + 1);
  u32* dkeys = S.alloc<u32>(maxb + 1);
  u32* didx = S.alloc<u32>(maxb + 1);
  u32* dk2 = S.alloc<u32>(maxb + 1);
  u32* di2 = S.alloc<u32>(maxb + 1);
  u32* sk = S.alloc<u32>(maxb + 1);
  u32* se = S.alloc<u32>(maxb + 1);
  void* rtmp = S.alloc<char>(rs_temp_bytes(maxb));
  u64* dcnt = S.alloc<u64>(W + 1);
  const bool multi = nwin > 1;
  uint4* sh_cur = multi ? S.alloc<uint4>(2 * n_keys) : nullptr;
  uint4* sh_nxt = multi ? S.alloc<uint4>(2 * n_keys) : nullptr;
  bool have_state = false;
  const int kbits = bits_for(n_keys ? n_keys - 1 : 0);
  u64* n_send_dev = cnt + C_ITEMS;
  u64 n_r = 0, n_items = 0, pool_used = 0;
  float ms_chk = 0;
  for (u64 k = 0; k < nwin; ++k) {
    const u64 R0 = k * rw, R1 = std::min<u64>(n, R0 + rw);
    const u64 p0 = pst[k], p1 = pst[k + 1], b = pbd[k];
    ++sx.windows;
    // ---- K4 over the local records of the window, then route each item to its granule's owner
    launch_expand(recs, hdr16, gl, page_bits, page_rank, shared_base, cum, p0, p1, gidx, R0, ikeys, ievs, err, st);
    if (b) { k_dest<<<nb(b), 256, 0, st>>>(ikeys, b, shared_base, (u32)W, (u32)me, dkeys, didx); ++g_launches; }
    const bool a4 = radix_sort_pairs(dkeys, didx, dk2, di2, b, 0, std::max(1, bits_for((u64)W - 1)), rtmp, st,
                                     nullptr, n_send_dev, true);
    const u32* dsort = a4 ? dk2 : dkeys;
    const u32* dperm = a4 ? di2 : didx;
    k_dest_counts<<<1, 1024, 0, st>>>(dsort, n_send_dev, (u32)W, dcnt);
    k_gather_items<<<nb(b + 1), 256, 0, st>>>(ikeys, ievs, dperm, n_send_dev, sk, se);
    g_launches += 2;
    std::vector<u64> scnt(W);
    cudaMemcpyAsync(scnt.data(), dcnt, W * 8, cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "routing");
    std::vector<u64> all((size_t)W * W);
    if (allgather_u64(cm, scnt.data(), W, all.data(), dtmp, st)) return fail(c, BC_ERR_NCCL, "count exchange");
    std::vector<u64> sb(W), so(W), rb(W), ro(W);
    u64 off = 0, roff = 0;
    for (int r = 0; r < W; ++r) {
      sb[r] = scnt[r] * 4;
      so[r] = off * 4;
      off += scnt[r];
      const u64 rc = all[(size_t)r * W + me];
      rb[r] = rc * 4;
      ro[r] = roff * 4;
      roff += rc;
    }
    const u64 n_recv = roff;
    u32* rk = (u32*)ctx_buffer(c, 0, (n_recv + 1) * 4);
    u32* re = (u32*)ctx_buffer(c, 1, (n_recv + 1) * 4);
    u32* rk2 = (u32*)ctx_buffer(c, 2, (n_recv + 1) * 4);
    u32* re2 = (u32*)ctx_buffer(c, 3, (n_recv + 1) * 4);
    if (!rk || !re || !rk2 || !re2) return fail(c, BC_ERR_OOM, "exchange buffers");
    if (cm->alltoallv(sk, sb.data(), so.data(), rk, rb.data(), ro.data(), st) ||
        cm->alltoallv(se, sb.data(), so.data(), re, rb.data(), ro.data(), st))
      return fail(c, BC_ERR_NCCL, "item exchange");
    // ---- K5 on the received items: by event (trace order), then stably by granule
    void* stmp = ctx_buffer(c, 4, rs_temp_bytes(n_recv + 1));
    if (!stmp) return fail(c, BC_ERR_OOM, "exchange sort scratch");
    u32* fk = rk;
    u32* fe = re;
    if (n_recv > 1) {
      const int ebits = bits_for(((R1 - R0) << 5) - 1);
      bool x = radix_sort_pairs(re, rk, re2, rk2, n_recv, 0, ebits, stmp, st);
      u32* ee = x ? re2 : re;
      u32* kk = x ? rk2 : rk;
      u32* ee2 = x ? re : re2;
      u32* kk2 = x ? rk : rk2;
      const bool y = radix_sort_pairs(kk, ee, kk2, ee2, n_recv, 2, 2 + kbits, stmp, st);
      fk = y ? kk2 : kk;
      fe = y ? ee2 : ee;
    }
    k_set_u64<<<1, 1, 0, st>>>(cnt + C_ITEMS, n_recv);
    ++g_launches;
    // ---- K7 on the owned granules
    uint4* sh_out = (multi && k + 1 < nwin) ? sh_nxt : nullptr;
    if (sh_out && !have_state) cudaMemsetAsync(sh_cur, 0, 2 * n_keys * sizeof(uint4), st);
    CheckLaunch L{};
    L.c = hc;
    L.keys = fk;
    L.evs = fe;
    L.n_dev = cnt + C_ITEMS;
    L.n_max = n_recv;
    L.R0 = (u32)R0;
    L.sh_in = have_state ? sh_cur : nullptr;
    L.sh_out = sh_out;
    L.values = nullptr;
    L.status = ctx_buffer(c, 5, check_status_bytes(n_recv));
    if (!L.status) return fail(c, BC_ERR_OOM, "check scratch");
    WindowOut wo;
    bc_status ws = check_window(c, L, n_recv, cnt, n_r, pool_used, wo);
    if (bc_status a = agree(c, ws, dtmp)) return a;
    n_items += wo.items;
    sx.segments += wo.segments;
    ms_chk += wo.ms_check;
    if (sh_out) {
      launch_shadow_commit(fk, cnt + C_ITEMS, n_recv, sh_nxt, sh_cur, st);
      have_state = true;
    }
  }
  cudaEventRecord(c->ev[7], st);

  // ---- 4. races and findings to rank 0; K8 there
  const u64 mine2[3] = {n_r, nfind_l, n_items};
  std::vector<u64> a2((size_t)W * 3);
  if (allgather_u64(cm, mine2, 3, a2.data(), dtmp, st)) return fail(c, BC_ERR_NCCL, "race count exchange");
  u64 R_tot = 0, F_tot = 0, I_tot = 0;
  for (int r = 0; r < W; ++r) {
    R_tot += a2[(size_t)r * 3];
    F_tot += a2[(size_t)r * 3 + 1];
    I_tot += a2[(size_t)r * 3 + 2];
  }
  sx.items = I_tot;
  sx.vc_pool_entries = pool_used;
  uint4* r_all = S.alloc<uint4>(me == 0 ? R_tot + 1 : 1);
  u32* fb_all = S.alloc<u32>(me == 0 ? F_tot + 1 : 1);
  u32* fr_all = S.alloc<u32>(me == 0 ? F_tot + 1 : 1);
  {
    std::vector<u64> sb(W, 0), so(W, 0), rb(W, 0), ro(W, 0);
    auto to0 = [&](const void* src, void* dst, u64 esz, int col) -> int {
      std::fill(sb.begin(), sb.end(), 0);
      std::fill(rb.begin(), rb.end(), 0);
      sb[0] = a2[(size_t)me * 3 + col] * esz;
      if (me == 0) {
        u64 o = 0;
        for (int r = 0; r < W; ++r) {
          rb[r] = a2[(size_t)r * 3 + col] * esz;
          ro[r] = o;
          o += rb[r];
        }
      }
      return cm->alltoallv(src, sb.data(), so.data(), dst, rb.data(), ro.data(), st);
    };
    if (to0(c->rbuf, r_all, 16, 0) || to0(find_blk, fb_all, 4, 1) || to0(find_rec, fr_all, 4, 1))
      return fail(c, BC_ERR_NCCL, "race gather");
  }
  if (me == 0) {
    const u64 total = R_tot + F_tot;
    if (total > c->races_cap) {
      c->da.free(c->races, c->races_cap * sizeof(bc_race));
      c->races_cap = 0;
      c->races = (bc_race*)c->da.alloc(std::max<u64>(total, 1) * sizeof(bc_race));
      if (!c->races) return fail(c, BC_ERR_OOM, "race list");
      c->races_cap = std::max<u64>(total, 1);
    }
    u32* page_num = S.alloc<u32>(n_pages + 1);
    if (R_tot) launch_page_list(words, wl_prefix, page_bits, n_words, page_num, st);
    finalize_races(r_all, (u32)R_tot, fb_all, fr_all, (u32)F_tot, g, snap, page_num, shared_base, (u32)n_keys, c->races,
                   S, st);
    c->n_races = total;
    sx.races = R_tot;
    sx.findings = F_tot;
  }
  cudaEventRecord(c->ev[PH_N], st);
  if (cudaEventSynchronize(c->ev[PH_N]) != cudaSuccess) return cuda_check(c, "finalize");
  if (bc_status cs = cuda_check(c, "detect")) return cs;
  cudaEventElapsedTime(&sx.ms_total, c->ev[0], c->ev[PH_N]);
  sx.ms_kernel[PH_CHECK] = ms_chk;
  sx.ms_kernel[PH_N] = ms_chk;
  sx.kernel_launches = g_launches - launches0;
  return BC_OK;
}


