// api.cu — the C ABI of include/bc.h: context, trace ownership and the bc_detect pipeline.
//
//   bc_detect = header (a1/a2) -> K1 warp partition (radix sort) -> K2 replay (a3) -> barrier
//               labels -> K3 sync skeleton (a4) -> K4 expansion (a5) -> K5 radix sort (a6)
//               -> K7 shadow check (a7) -> K8 finalize (a8/a9)
// all on cfg.stream; every phase is bracketed by cudaEvents for bc_stats.ms_kernel.
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <string>

#include "common.cuh"
#include "kernels.cuh"

using namespace bc;

namespace bc {
u64 g_launches = 0;
}

struct bc_ctx {
  bc_config cfg;
  Geo g;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  const bc_record* trace = nullptr;  // device
  bc_record* owned = nullptr;
  size_t owned_cap = 0;
  u64 n_recs = 0;
  bool loaded = false;
  bool detected = false;
  const u64* values = nullptr;  // device, per-lane store values (row f3), nullable
  u64* values_owned = nullptr;
  size_t values_cap = 0;
  bc_race* races = nullptr;  // device, findings first
  size_t races_cap = 0;
  u64 n_races = 0;
  bc_stats stats{};
  Arena arena;  // scratch buffers, reused across bc_detect calls
  std::string err;
  cudaEvent_t ev[16] = {};
  u64* hcnt = nullptr;  // pinned host copy of the device counter array (one D2H copy per host sync)
};

static const char* kPhase[] = {"header", "partition", "replay", "sync", "expand", "sort", "check", "finalize",
                               "k_check", "k_sort_items", "k_expand", nullptr};
enum { PH_HEADER = 0, PH_PARTITION, PH_REPLAY, PH_SYNC, PH_EXPAND, PH_SORT, PH_CHECK, PH_FINALIZE, PH_N };

static bc_status fail(bc_ctx* c, bc_status s, const std::string& msg) {
  if (c) c->err = msg;
  return s;
}

static bc_status cuda_check(bc_ctx* c, const char* where) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(c, BC_ERR_CUDA, std::string(where) + ": " + cudaGetErrorString(e));
  return BC_OK;
}

static int bits_for(u64 maxval) {
  int b = 0;
  while (b < 64 && (maxval >> b)) ++b;
  return b;
}

extern "C" {

const char* bc_status_string(bc_status s) {
  switch (s) {
    case BC_OK: return "ok";
    case BC_ERR_INVALID_ARG: return "invalid argument";
    case BC_ERR_INFEASIBLE_TRACE: return "infeasible trace";
    case BC_ERR_OOM: return "out of device memory";
    case BC_ERR_CUDA: return "CUDA error";
    case BC_ERR_NCCL: return "NCCL error";
    case BC_ERR_STATE: return "call out of order";
    case BC_ERR_TRUNCATED: return "output truncated";
    case BC_ERR_OVERFLOW: return "32-bit index overflow";
  }
  return "unknown status";
}

const char* bc_last_error(const bc_ctx* c) { return c ? c->err.c_str() : "null context"; }

const char* bc_phase_name(int i) { return (i >= 0 && i < PH_N + 3) ? kPhase[i] : nullptr; }

bc_status bc_init(const bc_config* cfg, bc_ctx** out) {
  if (!cfg || !out) return BC_ERR_INVALID_ARG;
  *out = nullptr;
  const u32 ws = cfg->warp_size;  // 32, or a simulated smaller warp
  if ((ws != 4 && ws != 8 && ws != 16 && ws != 32) || cfg->granule_log2 > 4) return BC_ERR_INVALID_ARG;
  if (cfg->flags & ~(u32)(BC_F_NO_SAME_VALUE_FILTER | BC_F_COUNT_GATHERS)) return BC_ERR_INVALID_ARG;  // overwrite: not on GPU yet
  if (cfg->world < 0 || cfg->world > 1024) return BC_ERR_INVALID_ARG;
  if (cfg->world > 1 && (cfg->rank < 0 || cfg->rank >= cfg->world)) return BC_ERR_INVALID_ARG;
  u64 nb = (u64)cfg->grid_dim[0] * cfg->grid_dim[1] * cfg->grid_dim[2];
  u64 tpb = (u64)cfg->block_dim[0] * cfg->block_dim[1] * cfg->block_dim[2];
  if (nb == 0 || tpb == 0 || tpb > 1024 || nb * tpb > 0xFFFFFFFFull) return BC_ERR_INVALID_ARG;
  u64 wpb = (tpb + ws - 1) / ws;
  if (nb * wpb >= (1ull << 30) || nb * wpb * wpb >= (1ull << 32)) return BC_ERR_INVALID_ARG;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    return BC_ERR_CUDA;
  }
  if (cfg->device < 0 || cfg->device >= ndev) return BC_ERR_INVALID_ARG;
  if (cudaSetDevice(cfg->device) != cudaSuccess) return BC_ERR_CUDA;
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, cfg->device) != cudaSuccess || prop.major < 10) return BC_ERR_CUDA;
  bc_ctx* c = new bc_ctx();
  c->cfg = *cfg;
  Geo& g = c->g;
  g.n_blocks = (u32)nb;
  g.tpb = (u32)tpb;
  g.wpb = (u32)wpb;
  g.ws = ws;
  g.n_warps = (u32)(nb * wpb);
  g.wpb_m = wpb == 1 ? 0u : (u32)(((1ull << 32) + wpb - 1) / wpb);
  g.world = cfg->world > 1 ? (u32)cfg->world : 1u;
  g.rank = cfg->world > 1 ? (u32)cfg->rank : 0u;
  g.G = cfg->granule_log2;
  g.smem = cfg->smem_bytes_per_block;
  g.smem_gran = (u32)(((u64)g.smem + (1u << g.G) - 1) >> g.G);
  g.flags = cfg->flags;
  g.n_recs = 0;
  if (cfg->stream) {
    c->stream = (cudaStream_t)cfg->stream;
  } else {
    cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking);
    c->own_stream = true;
  }
  // keep pooled scratch memory cached between bc_detect calls
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, cfg->device) == cudaSuccess) {
    uint64_t thr = ~0ull;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  for (int i = 0; i < 16; ++i) cudaEventCreate(&c->ev[i]);
  cudaMallocHost(&c->hcnt, C_N * sizeof(u64));
  if (cudaGetLastError() != cudaSuccess) {
    bc_destroy(c);
    return BC_ERR_CUDA;
  }
  *out = c;
  return BC_OK;
}

void bc_destroy(bc_ctx* c) {
  if (!c) return;
  cudaSetDevice(c->cfg.device);
  if (c->stream) cudaStreamSynchronize(c->stream);
  if (c->owned) cudaFree(c->owned);
  if (c->values_owned) cudaFree(c->values_owned);
  if (c->races) cudaFree(c->races);
  c->arena.free_all();
  if (c->hcnt) cudaFreeHost(c->hcnt);
  for (int i = 0; i < 16; ++i)
    if (c->ev[i]) cudaEventDestroy(c->ev[i]);
  if (c->own_stream) cudaStreamDestroy(c->stream);
  delete c;
}

bc_status bc_load_trace(bc_ctx* c, const bc_record* recs, uint64_t n, int on_device) {
  if (!c) return BC_ERR_INVALID_ARG;
  if (n && !recs) return fail(c, BC_ERR_INVALID_ARG, "null trace");
  if (n >= (1ull << 27)) return fail(c, BC_ERR_OVERFLOW, "more than 2^27 records (event id = rec << 5 | lane)");
  cudaSetDevice(c->cfg.device);
  c->loaded = false;
  c->detected = false;
  c->values = nullptr;
  c->n_recs = n;
  c->g.n_recs = n;
  bool aligned = ((uintptr_t)recs & 15) == 0;
  if (n == 0) {
    c->trace = nullptr;
  } else if (on_device && aligned) {
    c->trace = recs;
  } else {
    size_t bytes = n * sizeof(bc_record);
    if (bytes > c->owned_cap) {
      if (c->owned) cudaFree(c->owned);
      c->owned = nullptr;
      c->owned_cap = 0;
      if (cudaMalloc(&c->owned, bytes) != cudaSuccess) {
        cudaGetLastError();
        return fail(c, BC_ERR_OOM, "trace buffer");
      }
      c->owned_cap = bytes;
    }
    cudaMemcpyAsync(c->owned, recs, bytes, on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice,
                    c->stream);
    if (cudaStreamSynchronize(c->stream) != cudaSuccess) return cuda_check(c, "trace copy");
    c->trace = c->owned;
  }
  c->loaded = true;
  return BC_OK;
}

static bc_status detect_impl(bc_ctx* c, Scratch& S) {
  cudaStream_t st = c->stream;
  Geo g = c->g;
  if (c->values) g.flags |= GEO_F_VALUES;
  const u64 n = g.n_recs;
  const bc_record* recs = c->trace;
  bc_stats& sx = c->stats;
  memset(&sx, 0, sizeof(sx));
  sx.records = n;
  c->n_races = 0;
  const u64 launches0 = g_launches;
  cudaEventRecord(c->ev[0], st);
  if (n == 0) {
    cudaEventRecord(c->ev[PH_N], st);
    cudaEventSynchronize(c->ev[PH_N]);
    cudaEventElapsedTime(&sx.ms_total, c->ev[0], c->ev[PH_N]);
    return BC_OK;
  }
  const u64 nwords = 1ull << 23;  // page bitmap: 2^28 1-MB pages (48-bit addresses)
  u64* cnt = S.alloc<u64>(C_N);
  u32* err = reinterpret_cast<u32*>(cnt + C_ERR);
  u32* wkey = S.alloc<u32>(n);
  u32* wval = S.alloc<u32>(n);
  const bool small_w = g.n_warps <= WS_SMALL;
  u32* wcnt = S.alloc<u32>(3 * (size_t)(g.n_warps + 1));  // IFs, BARs, records per warp
  u32* if_cnt = wcnt;
  u32* bar_cnt = wcnt + (g.n_warps + 1);
  u32* rec_cnt = small_w ? wcnt + 2 * (size_t)(g.n_warps + 1) : nullptr;
  u32* sync_list = S.alloc<u32>(n);
  u32* page_bits = S.alloc<u32>(nwords);
  u32* ub_off = S.alloc<u32>(n + 1);  // per record: upper bound of its items, then its first slot
  uint4* hdr16 = S.alloc<uint4>(n);  // compact record headers (K2 gathers them per warp)
  cudaMemsetAsync(cnt, 0, C_N * 8, st);
  cudaMemsetAsync(wcnt, 0, 3 * (size_t)(g.n_warps + 1) * 4, st);
  cudaMemsetAsync(page_bits, 0, nwords * 4, st);
  // ---- header pass; written pages ranked in address order from the list of non-zero bitmap words
  u32* word_list = S.alloc<u32>(nwords);
  u32* wl2 = S.alloc<u32>(nwords);
  launch_header(recs, g, wkey, wval, if_cnt, bar_cnt, sync_list, page_bits, word_list, cnt, ub_off, hdr16, rec_cnt, err, st);
  u32* words = word_list;
  u32* wl_prefix = wl2;
  u32* page_rank = S.alloc<u32>(nwords);
  u32* need_sort = reinterpret_cast<u32*>(cnt + C_NEED_SORT);
  launch_page_rank(words, cnt + C_PAGE_WORDS, page_bits, page_rank, wl_prefix, cnt + C_PAGES, need_sort, 0, st);
  cudaEventRecord(c->ev[1], st);
  u64 hc_cnt[C_N];
  u64* const hcnt = c->hcnt;
  cudaMemcpyAsync(hcnt, cnt, C_N * sizeof(u64), cudaMemcpyDeviceToHost, st);
  if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "header");
  memcpy(hc_cnt, hcnt, sizeof(hc_cnt));
  u32 herr = (u32)hc_cnt[C_ERR], h_need_sort = (u32)hc_cnt[C_NEED_SORT];
  if (h_need_sort) {  // more non-zero page words than one CTA sorts: radix sort, then rank
    const u64 nwl = hc_cnt[C_PAGE_WORDS];
    if (radix_sort_pairs(word_list, nullptr, wl2, nullptr, nwl, 0, 23, S.alloc<char>(rs_temp_bytes(nwl)), st)) {
      words = wl2;
      wl_prefix = word_list;
    }
    launch_page_rank(words, cnt + C_PAGE_WORDS, page_bits, page_rank, wl_prefix, cnt + C_PAGES, need_sort, 1, st);
    cudaMemcpyAsync(hcnt, cnt, C_N * sizeof(u64), cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "page rank");
    memcpy(hc_cnt, hcnt, sizeof(hc_cnt));
  }
  const u64 n_pages = hc_cnt[C_PAGES], n_words = hc_cnt[C_PAGE_WORDS];
  sx.lane_events = hc_cnt[C_LANE_EVENTS];
  sx.control_events = hc_cnt[C_CONTROL_EVENTS];
  sx.sync_ops = hc_cnt[C_SYNC_LANEOPS];
  sx.written_pages = n_pages;
  if (herr & ERR_INFEASIBLE) return fail(c, BC_ERR_INFEASIBLE_TRACE, "record header violates feasibility");
  if (herr & ERR_OVERFLOW) return fail(c, BC_ERR_OVERFLOW, "global address >= 2^48");
  const u32 shared_base = (u32)std::min<u64>(n_pages << (20 - g.G), 0xFFFFFFFFull);
  const u64 n_keys = (n_pages << (20 - g.G)) + (u64)g.n_blocks * g.smem_gran;
  if (n_keys >= (1ull << 30)) return fail(c, BC_ERR_OVERFLOW, "shadow key space >= 2^30 granules");

  // ---- K1: records grouped by warp (stable -> trace order within a warp)
  u32* wk2 = S.alloc<u32>(n);
  u32* wv2 = S.alloc<u32>(n);
  bool alt = radix_sort_pairs(wkey, wval, wk2, wv2, n, 0, bits_for(g.n_warps - 1), S.alloc<char>(rs_temp_bytes(n)), st);
  u32* skeys = alt ? wk2 : wkey;
  u32* wrec = alt ? wv2 : wval;
  u32* warp_start = S.alloc<u32>(g.n_warps + 1);
  const u64 n_if = hc_cnt[C_IFS], n_bar = hc_cnt[C_BARS];
  u32* node_base = S.alloc<u32>(g.n_warps + 1);
  u32* bar_base = S.alloc<u32>(g.n_warps + 1);
  if (small_w) {
    launch_warp_scans(rec_cnt, if_cnt, bar_cnt, g.n_warps, warp_start, node_base, bar_base, st);
  } else {
    launch_warp_start(skeys, n, g.n_warps, warp_start, st);
    exclusive_scan_u32(if_cnt, node_base, g.n_warps, S.alloc<char>(scan_temp_bytes(g.n_warps)), nullptr, st);
    launch_node_base(node_base, g.n_warps, node_base, st);
    exclusive_scan_u32(bar_cnt, bar_base, g.n_warps, S.alloc<char>(scan_temp_bytes(g.n_warps)), nullptr, st);
  }
  cudaEventRecord(c->ev[2], st);
  // ---- K2: clock replay
  const u64 n_nodes = g.n_warps + 2 * n_if;
  uint4* snap = S.alloc<uint4>(n);
  uint4* nodes = S.alloc<uint4>(n_nodes);
  u32* bar_rec = S.alloc<u32>(n_bar + 1);
  u32* bar_next = S.alloc<u32>(n_bar + 1);
  u32* blockR = S.alloc<u32>(n_bar + 1);
  u32* find_blk = S.alloc<u32>(n_bar + 1);
  u32* find_rec = S.alloc<u32>(n_bar + 1);
  u32* find_cnt = reinterpret_cast<u32*>(cnt + C_FINDINGS);
  launch_replay(hdr16, wrec, warp_start, g, node_base, bar_base, snap, nodes, bar_rec, bar_next, find_blk, find_rec,
                find_cnt, err, st);
  launch_barriers(g, bar_cnt, bar_base, bar_rec, bar_next, blockR, err, st);
  launch_snap_blab(snap, n, g.wpb, g.n_warps, n_bar, bar_base, blockR, st);
  cudaEventRecord(c->ev[3], st);
  bc_status cs = cuda_check(c, "replay");
  if (cs) return cs;
  if (hc_cnt[C_SYNC_RECS]) {  // K3 walks snapshots: make sure the replay accepted the trace
    cudaMemcpyAsync(hcnt, cnt, C_N * sizeof(u64), cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "replay");
    herr = (u32)hcnt[C_ERR];
    if (herr & ERR_INFEASIBLE) return fail(c, BC_ERR_INFEASIBLE_TRACE, "SIMT stack / barrier feasibility");
  }

  HbCtx hc{};
  hc.g = g;
  hc.snap = snap;
  hc.nodes = nodes;
  hc.n_nodes = (u32)n_nodes;
  hc.err = err;
  hc.n_acq = 0;
  hc.n_idx = 0;
  // ---- K3: sync skeleton
  if (hc_cnt[C_SYNC_RECS]) {
    u64 ne = 0;
    int rs = run_sync_skeleton(recs, sync_list, (u32)hc_cnt[C_SYNC_RECS], (u32)hc_cnt[C_SYNC_LANEOPS],
                               (u32)hc_cnt[C_ACQ_RECS], hc, S, st, &ne);
    if (rs) return fail(c, (bc_status)rs, "sync skeleton");
  }
  cudaEventRecord(c->ev[4], st);
  // ---- K4: expansion (static slots from the header's per-record upper bounds)
  const u64 bound = hc_cnt[C_ITEM_BOUND];
  exclusive_scan_u32(ub_off, ub_off, n, S.alloc<char>(scan_temp_bytes(n)), nullptr, st);
  u32* ikeys = S.alloc<u32>(bound + 1);
  u32* ievs = S.alloc<u32>(bound + 1);
  cudaEventRecord(c->ev[14], st);
  launch_expand(recs, g, page_bits, page_rank, shared_base, ub_off, ikeys, ievs, err, st);
  cudaEventRecord(c->ev[15], st);
  cudaEventRecord(c->ev[5], st);
  // ---- K5: stable radix sort by granule key; the first pass drops the never-written slots
  u64* n_items_dev = cnt + C_ITEMS;
  u32* ik2 = S.alloc<u32>(bound + 1);
  u32* iv2 = S.alloc<u32>(bound + 1);
  int kbits = bits_for(n_keys ? n_keys - 1 : 0);
  void* rtmp = S.alloc<char>(rs_temp_bytes(bound));
  cudaEventRecord(c->ev[12], st);
  alt = radix_sort_pairs(ikeys, ievs, ik2, iv2, bound, 2, 2 + kbits, rtmp, st, nullptr, n_items_dev, true);
  cudaEventRecord(c->ev[13], st);
  u32* skey = alt ? ik2 : ikeys;
  u32* sev = alt ? iv2 : ievs;
  cudaEventRecord(c->ev[6], st);
  // ---- K7: shadow check
  u32 race_cap = (u32)std::min<u64>(std::max<u64>(1u << 16, bound / 16), 1u << 30);
  uint4* rbuf = nullptr;
  u32* rcnt = reinterpret_cast<u32*>(cnt + C_RACES);
  u64* segc = cnt + C_SEGMENTS;  // [0] segments, [1] clock snapshot gathers (C_GATHERS)
  void* cstatus = S.alloc<char>(check_status_bytes(bound));
  u32 n_r = 0, nfind = 0;
  u64 n_items = 0;
  for (int attempt = 0; attempt < 2; ++attempt) {
    rbuf = S.alloc<uint4>(race_cap);
    cudaMemsetAsync(cnt + C_RACES, 0, 3 * sizeof(u64), st);  // races, segments, gathers
    cudaEventRecord(c->ev[10], st);
    launch_check(hc, skey, sev, n_items_dev, bound, cstatus, rbuf, rcnt, race_cap, segc, c->values, st);
    cudaEventRecord(c->ev[11], st);
    if (g.flags & BC_F_COUNT_GATHERS) launch_count_gathers(skey, n_items_dev, segc + 1, st);
    cudaMemcpyAsync(hcnt, cnt, C_N * sizeof(u64), cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "check");
    n_r = (u32)hcnt[C_RACES];
    herr = (u32)hcnt[C_ERR];
    sx.segments = hcnt[C_SEGMENTS];
    sx.clock_gathers = hcnt[C_GATHERS];
    n_items = hcnt[C_ITEMS];
    nfind = (u32)hcnt[C_FINDINGS];
    if (herr) break;
    if (n_r <= race_cap) break;
    race_cap = n_r;
  }
  if (herr & ERR_INFEASIBLE) return fail(c, BC_ERR_INFEASIBLE_TRACE, "infeasible trace");
  if (herr & ERR_OVERFLOW) return fail(c, BC_ERR_OVERFLOW, "index overflow / sync lookup step cap");
  sx.items = n_items;
  cudaEventRecord(c->ev[7], st);
  // ---- K8: finalize
  if (g.world > 1 && g.rank != 0) nfind = 0;  // findings come from the replicated replay: rank 0 reports them
  u64 total = (u64)n_r + nfind;
  if (total > c->races_cap) {
    if (c->races) cudaFree(c->races);
    c->races = nullptr;
    c->races_cap = 0;
    if (cudaMalloc(&c->races, std::max<u64>(total, 1) * sizeof(bc_race)) != cudaSuccess) {
      cudaGetLastError();
      return fail(c, BC_ERR_OOM, "race buffer");
    }
    c->races_cap = std::max<u64>(total, 1);
  }
  u32* page_num = S.alloc<u32>(n_pages + 1);
  if (n_r) launch_page_list(words, wl_prefix, page_bits, n_words, page_num, st);
  finalize_races(rbuf, n_r, find_blk, find_rec, nfind, g, snap, page_num, shared_base, (u32)n_keys, c->races, S, st);
  cudaEventRecord(c->ev[PH_N], st);
  if (cudaEventSynchronize(c->ev[PH_N]) != cudaSuccess) return cuda_check(c, "finalize");
  cs = cuda_check(c, "detect");
  if (cs) return cs;
  c->n_races = total;
  sx.races = n_r;
  sx.findings = nfind;
  cudaEventElapsedTime(&sx.ms_total, c->ev[0], c->ev[PH_N]);
  for (int i = 0; i < PH_N; ++i) {
    cudaEvent_t e1 = i + 1 < PH_N ? c->ev[i + 1] : c->ev[PH_N];
    cudaEventElapsedTime(&sx.ms_kernel[i], c->ev[i], e1);
  }
  // kernel-only timings of the three heavy kernels (no host gaps inside)
  if (n_items) {
    cudaEventElapsedTime(&sx.ms_kernel[PH_N + 0], c->ev[10], c->ev[11]);
    cudaEventElapsedTime(&sx.ms_kernel[PH_N + 1], c->ev[12], c->ev[13]);
  }
  cudaEventElapsedTime(&sx.ms_kernel[PH_N + 2], c->ev[14], c->ev[15]);
  sx.kernel_launches = g_launches - launches0;
  return BC_OK;
}

bc_status bc_load_values(bc_ctx* c, const uint64_t* values, uint64_t n, int on_device) {
  if (!c) return BC_ERR_INVALID_ARG;
  if (!c->loaded) return fail(c, BC_ERR_STATE, "bc_load_values before bc_load_trace");
  c->detected = false;
  c->values = nullptr;
  if (!values) return BC_OK;
  if (n != c->n_recs) return fail(c, BC_ERR_INVALID_ARG, "values: record count differs from the trace");
  if (n == 0) return BC_OK;
  cudaSetDevice(c->cfg.device);
  if (on_device) {
    if (((uintptr_t)values & 7) != 0) return fail(c, BC_ERR_INVALID_ARG, "values: misaligned device pointer");
    c->values = (const u64*)values;
    return BC_OK;
  }
  const size_t bytes = (size_t)n * 32 * sizeof(u64);
  if (c->values_cap < bytes) {
    if (c->values_owned) cudaFree(c->values_owned);
    c->values_owned = nullptr;
    c->values_cap = 0;
    if (cudaMalloc(&c->values_owned, bytes) != cudaSuccess) {
      cudaGetLastError();
      return fail(c, BC_ERR_OOM, "values buffer");
    }
    c->values_cap = bytes;
  }
  cudaMemcpyAsync(c->values_owned, values, bytes, cudaMemcpyHostToDevice, c->stream);
  if (cudaStreamSynchronize(c->stream) != cudaSuccess) return cuda_check(c, "values copy");
  c->values = c->values_owned;
  return BC_OK;
}

bc_status bc_detect(bc_ctx* c, bc_stats* out) {
  if (!c) return BC_ERR_INVALID_ARG;
  if (!c->loaded) return fail(c, BC_ERR_STATE, "bc_detect before bc_load_trace");
  cudaSetDevice(c->cfg.device);
  c->detected = false;
  c->err.clear();
  bc_status s;
  {
    Scratch S(c->stream, &c->arena);
    try {
      s = detect_impl(c, S);
    } catch (const std::bad_alloc&) {
      s = fail(c, BC_ERR_OOM, "scratch allocation");
    }
    S.release();
  }
  cudaStreamSynchronize(c->stream);
  if (s == BC_OK) {
    c->detected = true;
  } else {
    c->n_races = 0;
  }
  if (out) *out = c->stats;
  return s;
}

static bc_status races_copy(bc_ctx* c, bc_race* out, uint64_t cap, uint64_t* n_total, cudaMemcpyKind kind) {
  if (!c || !n_total) return BC_ERR_INVALID_ARG;
  if (!c->detected) return fail(c, BC_ERR_STATE, "bc_races before a successful bc_detect");
  *n_total = c->n_races;
  if (!out) return BC_OK;
  u64 k = std::min<u64>(cap, c->n_races);
  if (k) {
    cudaSetDevice(c->cfg.device);
    cudaMemcpyAsync(out, c->races, k * sizeof(bc_race), kind, c->stream);
    if (cudaStreamSynchronize(c->stream) != cudaSuccess) return cuda_check(c, "race copy");
  }
  return k < c->n_races ? BC_ERR_TRUNCATED : BC_OK;
}

bc_status bc_races(bc_ctx* c, bc_race* out, uint64_t cap, uint64_t* n_total) {
  return races_copy(c, out, cap, n_total, cudaMemcpyDeviceToHost);
}

bc_status bc_races_device(bc_ctx* c, bc_race* out, uint64_t cap, uint64_t* n_total) {
  return races_copy(c, out, cap, n_total, cudaMemcpyDeviceToDevice);
}

}  // extern "C"
