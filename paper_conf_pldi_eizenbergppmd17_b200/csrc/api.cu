// api.cu — the C ABI of include/bc.h: context, trace ownership and the bc_detect pipeline.
//
//   bc_detect = header (a1/a2) -> K1 warp partition (radix sort) -> K2 replay (a3) -> barrier
//               labels -> K3 sync skeleton (a4) -> K4 expansion (a5) -> K5 radix sort (a6)
//               -> K7 shadow check (a7) -> K8 finalize (a8/a9)
// all on cfg.stream; every phase is bracketed by cudaEvents for bc_stats.ms_kernel.
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <string>

#include "comm.cuh"
#include "common.cuh"
#include "kernels.cuh"

using namespace bc;

namespace bc {
std::atomic<u64> g_launches{0};  // kernels launched by this process (per-detect delta in bc_stats)
}

#include "ctx.cuh"

static const char* kPhase[] = {"header", "partition", "replay", "sync", "expand", "sort", "check", "finalize",
                               "k_check", "k_sort_items", "k_expand", nullptr};

void* ctx_buffer(bc_ctx* c, int slot, size_t bytes) {
  if (bytes <= c->xcap[slot]) return c->xbuf[slot];
  cudaStreamSynchronize(c->stream);
  c->da.free(c->xbuf[slot], c->xcap[slot]);
  c->xcap[slot] = 0;
  bytes = std::max<size_t>(bytes + bytes / 4, 4096);
  c->xbuf[slot] = c->da.alloc(bytes);
  if (c->xbuf[slot]) c->xcap[slot] = bytes;
  return c->xbuf[slot];
}

bc_status check_window(bc_ctx* c, CheckLaunch& L, u64 b, u64* cnt, u64& n_r, u64& pool_used, WindowOut& wo) {
  cudaStream_t st = c->stream;
  u64* const hcnt = c->hcnt;
  if (L.sh_out) {
    // every carried vector may be re-copied once and every item appended once
    const u64 need = 2 * pool_used + b + 1024;
    if (need >= (1ull << 32)) return fail(c, BC_ERR_OVERFLOW, "read-vector pool >= 2^32 entries");
    if (need > c->pool_cap) {
      uint2* np = (uint2*)c->da.alloc(need * sizeof(uint2));
      if (!np) return fail(c, BC_ERR_OOM, "read-vector pool");
      if (pool_used) cudaMemcpyAsync(np, c->pool, pool_used * sizeof(uint2), cudaMemcpyDeviceToDevice, st);
      cudaStreamSynchronize(st);
      c->da.free(c->pool, c->pool_cap * sizeof(uint2));
      c->pool = np;
      c->pool_cap = need;
    }
  }
  L.pool = c->pool;
  L.pool_cnt = reinterpret_cast<u32*>(cnt + C_POOL);
  L.pool_cap = (u32)std::min<u64>(c->pool_cap, 0xFFFFFFFFull);
  L.race_cnt = reinterpret_cast<u32*>(cnt + C_RACES);
  L.seg_cnt = cnt + C_SEGMENTS;
  u32 herr = 0;
  for (int attempt = 0; attempt < 3; ++attempt) {
    if (c->rbuf_cap < (1u << 16)) {
      c->da.free(c->rbuf, c->rbuf_cap * sizeof(uint4));
      c->rbuf_cap = 0;
      c->rbuf = (uint4*)c->da.alloc((1u << 16) * sizeof(uint4));
      if (!c->rbuf) return fail(c, BC_ERR_OOM, "race buffer");
      c->rbuf_cap = 1u << 16;
    }
    L.races = c->rbuf;
    L.race_cap = (u32)std::min<u64>(c->rbuf_cap, 0xFFFFFFFFull);
    // device counters: races so far, this window's segments / gathers, the carried pool size
    hcnt[C_RACES] = n_r;
    hcnt[C_SEGMENTS] = 0;
    hcnt[C_GATHERS] = 0;
    hcnt[C_POOL] = pool_used;
    cudaMemcpyAsync(cnt + C_RACES, hcnt + C_RACES, 4 * sizeof(u64), cudaMemcpyHostToDevice, st);
    cudaEventRecord(c->ev[10], st);
    launch_check(L, st);
    cudaEventRecord(c->ev[11], st);
    if (L.c.g.flags & BC_F_COUNT_GATHERS) launch_count_gathers(L.keys, L.n_dev, cnt + C_GATHERS, cnt + C_SEGMENTS, st);
    cudaMemcpyAsync(hcnt, cnt, C_N * sizeof(u64), cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "check");
    herr = (u32)hcnt[C_ERR];
    if (herr) break;
    const u64 tot = (u32)hcnt[C_RACES];
    if (tot <= c->rbuf_cap) break;
    // more races than room: grow (keeping the earlier windows' races) and check the window again
    // (idempotent: the shadow entries it writes are a function of the window, the pool is reset)
    const u64 cap2 = std::max<u64>(2 * c->rbuf_cap, tot + 1024);
    if (cap2 >= 0xFFFFFFFFull) return fail(c, BC_ERR_OVERFLOW, "2^32 or more races");
    uint4* nb2 = (uint4*)c->da.alloc(cap2 * sizeof(uint4));
    if (!nb2) return fail(c, BC_ERR_OOM, "race buffer");
    if (n_r) cudaMemcpyAsync(nb2, c->rbuf, n_r * sizeof(uint4), cudaMemcpyDeviceToDevice, st);
    cudaStreamSynchronize(st);
    c->da.free(c->rbuf, c->rbuf_cap * sizeof(uint4));
    c->rbuf = nb2;
    c->rbuf_cap = cap2;
  }
  if (herr & ERR_PAGES) return BC_RETRY_FULL_PAGES;  // the sampled page set missed a written page
  if (herr & ERR_INFEASIBLE) return fail(c, BC_ERR_INFEASIBLE_TRACE, "infeasible trace");
  if (herr & ERR_OVERFLOW) return fail(c, BC_ERR_OVERFLOW, "index overflow / sync lookup step cap");
  if (herr & ERR_UNDECLARED) return fail(c, BC_ERR_INVALID_ARG, "global access outside bc_config.global_ranges");
  n_r = (u32)hcnt[C_RACES];
  pool_used = (u32)hcnt[C_POOL];
  wo.items = hcnt[C_ITEMS];
  wo.segments = hcnt[C_SEGMENTS];
  wo.gathers = hcnt[C_GATHERS];
  cudaEventElapsedTime(&wo.ms_check, c->ev[10], c->ev[11]);
  return BC_OK;
}

// ---------------------------------------------------------------- streaming ingest (row f1)
// Queue header (bc.h): write_head, commit_head, read_head, capacity, error, pad[3]; ring after 64 B.
enum { Q_WRITE = 0, Q_COMMIT, Q_READ, Q_CAP, Q_ERROR, Q_HDR = 8 };

// Stand-in producer: one warp per record, persistent warps taking records in increasing order (so the
// warp that must commit before another is always resident).  Ticket t = the record's trace position:
// wait for ring room (read_head), write the 272-B record, fence, wait for commit_head == t, commit.
__global__ void __launch_bounds__(256) k_queue_push(u64* __restrict__ q, const bc_record* __restrict__ recs, u64 n) {
  const u64 w = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5, nw = ((u64)gridDim.x * blockDim.x) >> 5;
  const u32 lane = threadIdx.x & 31;
  volatile u64* vq = q;
  const u64 cap = vq[Q_CAP];
  bc_record* ring = reinterpret_cast<bc_record*>(q + Q_HDR);
  for (u64 t = w; t < n; t += nw) {
    if (lane == 0) atomicMax((unsigned long long*)&q[Q_WRITE], (unsigned long long)(t + 1));  // reservation
    const long long t0 = clock64();
    bool ok = true;
    while (t >= vq[Q_READ] + cap) {  // ring full: wait for the consumer
      if (vq[Q_ERROR] || clock64() - t0 > 20000000000ll) { ok = false; break; }
    }
    if (__any_sync(0xFFFFFFFFu, !ok)) {
      if (lane == 0) vq[Q_ERROR] = 1;
      return;
    }
    const u32* src = reinterpret_cast<const u32*>(recs + t);
    u32* dst = reinterpret_cast<u32*>(ring + t % cap);
    for (u32 i = lane; i < sizeof(bc_record) / 4; i += 32) dst[i] = __ldg(src + i);
    __threadfence();
    __syncwarp();
    if (lane == 0) {
      const long long t1 = clock64();
      while (vq[Q_COMMIT] != t) {  // commits in ticket order
        if (vq[Q_ERROR] || clock64() - t1 > 20000000000ll) {
          vq[Q_ERROR] = 1;
          break;
        }
      }
      __threadfence();
      vq[Q_COMMIT] = t + 1;
    }
    __syncwarp();
    if (vq[Q_ERROR]) return;
  }
}

// The session's drain thread (the consumer half of Fig. 6's queue).  It reads the heads, copies the
// newly committed records out of the ring into the trace buffer and then publishes the new read head,
// all with copy-engine transfers on its own stream: no SM is needed, so a producer that fills the GPU
// and waits on a full ring is always served, whatever the window checks are waiting for.
static void drain_loop(bc_ctx* c) {
  cudaSetDevice(c->cfg.device);
  cudaStream_t ds = c->dstream;
  u64* h = c->dhdr;
  const bc_record* ring = reinterpret_cast<const bc_record*>(c->queue + Q_HDR);
  const u64 cap = c->queue_cap;
  u64 done = 0;
  int idle = 0;
  while (!c->drain_stop.load(std::memory_order_acquire)) {
    cudaMemcpyAsync(h, c->queue, Q_HDR * sizeof(u64), cudaMemcpyDeviceToHost, ds);
    if (cudaStreamSynchronize(ds) != cudaSuccess) {
      c->drain_err.store(BC_ERR_CUDA);
      return;
    }
    if (h[Q_ERROR]) {
      c->drain_err.store(BC_ERR_INVALID_ARG);
      return;
    }
    const u64 committed = h[Q_COMMIT], w = h[Q_WRITE];
    if (committed > c->sbuf_cap) {
      c->drain_err.store(BC_ERR_TRUNCATED);
      h[Q_ERROR] = 1;  // stop the producer
      cudaMemcpyAsync(c->queue + Q_ERROR, h + Q_ERROR, sizeof(u64), cudaMemcpyHostToDevice, ds);
      cudaStreamSynchronize(ds);
      return;
    }
    if (committed > done) {
      for (u64 t = done; t < committed;) {  // two copies across the wrap
        const u64 slot = t % cap;
        const u64 m = std::min<u64>(committed - t, cap - slot);
        cudaMemcpyAsync(c->sbuf + t, ring + slot, m * sizeof(bc_record), cudaMemcpyDeviceToDevice, ds);
        t += m;
      }
      h[Q_HDR] = committed;  // the slots are free once the copies are done (stream order)
      cudaMemcpyAsync(c->queue + Q_READ, h + Q_HDR, sizeof(u64), cudaMemcpyHostToDevice, ds);
      if (cudaStreamSynchronize(ds) != cudaSuccess) {
        c->drain_err.store(BC_ERR_CUDA);
        return;
      }
      done = committed;
      c->drained.store(done, std::memory_order_release);
      idle = 0;
    } else if (++idle > 64) {
      std::this_thread::sleep_for(std::chrono::microseconds(50));
    }
    c->wseen.store(w, std::memory_order_release);
    c->dgen.fetch_add(1, std::memory_order_acq_rel);
  }
}

static void drain_stop(bc_ctx* c) {
  if (c->drainer.joinable()) {
    c->drain_stop.store(true, std::memory_order_release);
    c->drainer.join();
  }
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
  if (cfg->flags & ~(u32)(BC_F_RELEASE_OVERWRITE | BC_F_NO_SAME_VALUE_FILTER | BC_F_COUNT_GATHERS))
    return BC_ERR_INVALID_ARG;
  if ((cfg->dev_alloc == nullptr) != (cfg->dev_free == nullptr)) return BC_ERR_INVALID_ARG;
  if (cfg->world < 0 || cfg->world > 1024) return BC_ERR_INVALID_ARG;
  if (cfg->world > 1 && (cfg->rank < 0 || cfg->rank >= cfg->world)) return BC_ERR_INVALID_ARG;
  u64 nb = (u64)cfg->grid_dim[0] * cfg->grid_dim[1] * cfg->grid_dim[2];
  u64 tpb = (u64)cfg->block_dim[0] * cfg->block_dim[1] * cfg->block_dim[2];
  if (nb == 0 || tpb == 0 || tpb > 1024 || nb * tpb > 0xFFFFFFFFull) return BC_ERR_INVALID_ARG;
  u64 wpb = (tpb + ws - 1) / ws;
  // warps < 2^27: a thread id (warp << 5 | lane) is 32 bits (shadow entries, read-vector pool)
  if (nb * wpb >= (1ull << 27) || nb * wpb * wpb >= (1ull << 32)) return BC_ERR_INVALID_ARG;
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
  c->da.fa = cfg->dev_alloc;
  c->da.ff = cfg->dev_free;
  c->da.user = cfg->alloc_user;
  c->da.st = c->stream;
  c->arena.da = &c->da;
  if (cfg->world >= 1 && (cfg->nccl_unique_id || cfg->group)) {
    if (cfg->nccl_unique_id && cfg->group) {
      bc_destroy(c);
      return BC_ERR_INVALID_ARG;
    }
    int cs = BC_OK;
    c->comm = cfg->group ? make_local_comm(reinterpret_cast<LocalGroup*>(cfg->group), cfg->rank, cfg->device)
                         : make_nccl_comm(cfg->nccl_unique_id, cfg->rank, cfg->world, &cs);
    if (!c->comm) {
      bc_destroy(c);
      return (bc_status)cs;
    }
  }
  // keep pooled scratch memory cached between bc_detect calls
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, cfg->device) == cudaSuccess) {
    uint64_t thr = ~0ull;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  for (int i = 0; i < 18; ++i) cudaEventCreate(&c->ev[i]);
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
  drain_stop(c);
  if (c->stream) cudaStreamSynchronize(c->stream);
  c->da.free(c->owned, c->owned_cap);
  c->da.free(c->values_owned, c->values_cap);
  c->da.free(c->races, c->races_cap * sizeof(bc_race));
  c->da.free(c->rbuf, c->rbuf_cap * sizeof(uint4));
  c->da.free(c->pool, c->pool_cap * sizeof(uint2));
  c->da.free(c->gidx_owned, c->gidx_cap);
  for (int i = 0; i < 6; ++i) c->da.free(c->xbuf[i], c->xcap[i]);
  c->da.free(c->queue, c->queue_bytes);
  c->da.free(c->sbuf, c->sbuf_cap * sizeof(bc_record));
  c->da.free(c->granges, 2 * 64 * sizeof(u64));
  for (int q = 0; q < 2; ++q) c->da.free(c->sh[q], c->sh_bytes);
  c->arena.free_all();
  if (c->stream) cudaStreamSynchronize(c->stream);  // the stream-ordered frees
  delete c->comm;
  if (c->hcnt) cudaFreeHost(c->hcnt);
  if (c->dhdr) cudaFreeHost(c->dhdr);
  if (c->dstream) cudaStreamDestroy(c->dstream);
  for (int i = 0; i < 18; ++i)
    if (c->ev[i]) cudaEventDestroy(c->ev[i]);
  if (c->own_stream) cudaStreamDestroy(c->stream);
  delete c;
}

bc_status bc_load_trace(bc_ctx* c, const bc_record* recs, uint64_t n, int on_device) {
  if (!c) return BC_ERR_INVALID_ARG;
  if (n && !recs) return fail(c, BC_ERR_INVALID_ARG, "null trace");
  if (n >= 0xFFFFFFFFull) return fail(c, BC_ERR_OVERFLOW, "2^32 - 1 or more records (32-bit record indices)");
  cudaSetDevice(c->cfg.device);
  c->sharded = false;
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
      c->da.free(c->owned, c->owned_cap);
      c->owned_cap = 0;
      c->owned = (bc_record*)c->da.alloc(bytes);
      if (!c->owned) return fail(c, BC_ERR_OOM, "trace buffer");
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

// full_pages: k_header marks the page of every write address instead of a sample (the re-run after
// K4 found a write outside the sampled set, BC_RETRY_FULL_PAGES)
static bc_status detect_impl(bc_ctx* c, Scratch& S, const StreamWin* sw, bool full_pages = false) {
  cudaStream_t st = c->stream;
  Geo g = c->g;
  if (c->values) g.flags |= GEO_F_VALUES;
  if (sw) g.flags |= GEO_F_DECLARED;  // streaming: the page set is the declared allocations
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
  u32* rec_w = S.alloc<u32>(n);  // per record: window weight (item upper bound + REC_W)
  uint4* hdr16 = S.alloc<uint4>(n);  // compact record headers (K2 gathers them per warp)
  cudaMemsetAsync(cnt, 0, C_N * 8, st);
  cudaMemsetAsync(wcnt, 0, 3 * (size_t)(g.n_warps + 1) * 4, st);
  cudaMemsetAsync(page_bits, 0, nwords * 4, st);
  // ---- header pass; written pages ranked in address order from the list of non-zero bitmap words
  u32* word_list = S.alloc<u32>(nwords);
  u32* wl2 = S.alloc<u32>(nwords);
  launch_header(recs, g, wkey, wval, if_cnt, bar_cnt, sync_list, page_bits, word_list, cnt, rec_w, hdr16, rec_cnt, err, st,
                sw ? 0 : (full_pages ? 1 : 2));
  if (sw) launch_mark_ranges(c->granges, c->cfg.n_global_ranges, page_bits, word_list, cnt, err, st);
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
  launch_replay(hdr16, wrec, nullptr, warp_start, g, node_base, bar_base, snap, nodes, bar_rec, bar_next, find_blk,
                find_rec, find_cnt, err, st);
  launch_barriers(g, bar_cnt, bar_base, bar_rec, bar_next, blockR, err, st, sw && !sw->final);
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
  hc.e_off = hc.e_cnt = hc.e_arr = hc.e_key = hc.e_mask = hc.e_clk = nullptr;
  // ---- K3: sync skeleton
  if (hc_cnt[C_SYNC_RECS]) {
    u64 ne = 0;
    const u32 n_srec = (u32)hc_cnt[C_SYNC_RECS];
    bc_record* srecs = S.alloc<bc_record>(n_srec);
    gather_sync_records(recs, sync_list, n_srec, n, srecs, S, st);
    int rs = run_sync_skeleton(srecs, sync_list, n_srec, (u32)hc_cnt[C_SYNC_LANEOPS], (u32)hc_cnt[C_ACQ_RECS], hc, S, st,
                               &ne);
    if (rs) return fail(c, (bc_status)rs, "sync skeleton");
  }
  cudaEventRecord(c->ev[4], st);
  // ---- windows: consecutive record ranges of at most `we` weight (item upper bound +
  // REC_W per record: < 2^27 records, so window-local event ids are 32-bit); the per-granule shadow
  // state (Fig. 8) carries from one window to the next
  const u64 bound_all = hc_cnt[C_ITEM_BOUND];
  const u64 total_w = bound_all + (u64)REC_W * n;
  const u64 we = c->cfg.window_events ? std::min<u64>(c->cfg.window_events, WIN_MAX) : WIN_MAX;
  u64* cum = S.alloc<u64>(n + 1);
  exclusive_scan_u32_u64(rec_w, cum, n, S.alloc<char>(scan_temp_bytes(n)), cum + n, st);
  const u64 nwin64 = sw ? 1 : std::max<u64>(1, (total_w + we - 1) / we);
  if (nwin64 >= (1ull << 31)) return fail(c, BC_ERR_INVALID_ARG, "window_events too small for this trace");
  const u32 nwin = (u32)nwin64;
  std::vector<u64> wst(nwin + 1), wbd(nwin);
  if (sw) {  // streaming: the new records [R0, n) are the window
    u64 c01[2] = {0, 0};
    cudaMemcpyAsync(&c01[0], cum + sw->R0, 8, cudaMemcpyDeviceToHost, st);
    cudaMemcpyAsync(&c01[1], cum + n, 8, cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "windows");
    wst[0] = sw->R0;
    wst[1] = n;
    wbd[0] = (c01[1] - c01[0]) - (u64)REC_W * (n - sw->R0);
    if (n - sw->R0 >= (1ull << 27) || c01[1] - c01[0] > WIN_MAX)
      return fail(c, BC_ERR_OVERFLOW, "stream window too large: poll more often");
  } else if (nwin == 1) {
    wst[0] = 0;
    wst[1] = n;
    wbd[0] = bound_all;
  } else {
    u64* d_wst = S.alloc<u64>(nwin + 1);
    u64* d_wbd = S.alloc<u64>(nwin);
    launch_window_starts(cum, n, we, nwin, d_wst, d_wbd, st);
    cudaMemcpyAsync(wst.data(), d_wst, (nwin + 1) * sizeof(u64), cudaMemcpyDeviceToHost, st);
    cudaMemcpyAsync(wbd.data(), d_wbd, nwin * sizeof(u64), cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "windows");
  }
  u64 maxb = 0;
  int last_win = -1;
  for (u32 k = 0; k < nwin; ++k)
    if (wst[k + 1] > wst[k]) {
      maxb = std::max(maxb, wbd[k]);
      last_win = (int)k;
    }
  const bool multi = nwin > 1 || sw;
  u32* ikeys = S.alloc<u32>(maxb + 1);
  u32* ievs = S.alloc<u32>(maxb + 1);
  u32* ik2 = S.alloc<u32>(maxb + 1);
  u32* iv2 = S.alloc<u32>(maxb + 1);
  void* rtmp = S.alloc<char>(rs_temp_bytes(maxb));
  void* cstatus = S.alloc<char>(check_status_bytes(maxb));
  uint4* sh_cur = nullptr;  // the carried entries (current after every window)
  uint4* sh_nxt = nullptr;  // K7's output entries of the touched granules, committed into sh_cur
  bool have_state = false;
  if (sw) {  // a streaming session keeps its tables across polls (the declared page set fixes n_keys)
    const size_t bytes = 2 * n_keys * sizeof(uint4);
    if (!c->sh[0] || c->sh_bytes != bytes) {
      for (int q = 0; q < 2; ++q) {
        c->da.free(c->sh[q], c->sh_bytes);
        c->sh[q] = (uint4*)c->da.alloc(bytes);
        if (!c->sh[q]) return fail(c, BC_ERR_OOM, "stream shadow tables");
      }
      c->sh_bytes = bytes;
    }
    sh_cur = c->sh[0];
    sh_nxt = c->sh[1];
    have_state = c->have_state;
    if (sw->final) last_win = 0;
    else last_win = -2;  // the window writes entries for the next poll
  } else if (multi) {
    sh_cur = S.alloc<uint4>(2 * n_keys);
    sh_nxt = S.alloc<uint4>(2 * n_keys);
  }
  u64* n_items_dev = cnt + C_ITEMS;
  const int kbits = bits_for(n_keys ? n_keys - 1 : 0);
  u64 n_r = sw ? c->s_nr : 0, n_items = 0, pool_used = sw ? c->s_pool : 0;
  float ms_ex = 0, ms_sort = 0, ms_chk = 0;
  bool commit_pending = false;
  for (u32 k = 0; k < nwin; ++k) {
    const u64 R0 = wst[k], R1 = wst[k + 1], b = wbd[k];
    if (R0 == R1) continue;
    ++sx.windows;
    // ---- K4: expansion (static slots from the header's per-record upper bounds)
    cudaEventRecord(c->ev[14], st);
    launch_expand(recs, hdr16, g, page_bits, page_rank, shared_base, cum, R0, R1, nullptr, R0, ikeys, ievs, err, st);
    cudaEventRecord(c->ev[15], st);
    // ---- K5: stable radix sort by granule key; the first pass drops the never-written slots
    cudaEventRecord(c->ev[12], st);
    const bool alt = radix_sort_pairs(ikeys, ievs, ik2, iv2, b, 2, 2 + kbits, rtmp, st, nullptr, n_items_dev, true);
    cudaEventRecord(c->ev[13], st);
    u32* skey = alt ? ik2 : ikeys;
    u32* sev = alt ? iv2 : ievs;
    // ---- K7: shadow check of the window (carried entries in, entries for the next window out)
    uint4* sh_out = (multi && (int)k != last_win) ? sh_nxt : nullptr;
    // the first window that carries state: every entry starts empty (later windows update only the
    // entries of the granules they touch, k_shadow_commit)
    if (sh_out && !have_state) cudaMemsetAsync(sh_cur, 0, 2 * n_keys * sizeof(uint4), st);
    CheckLaunch L{};
    L.c = hc;
    L.keys = skey;
    L.evs = sev;
    L.n_dev = n_items_dev;
    L.n_max = b;
    L.R0 = (u32)R0;
    L.sh_in = have_state ? sh_cur : nullptr;
    L.sh_out = sh_out;
    L.values = c->values;
    L.status = cstatus;
    WindowOut wo;
    bc_status ws = check_window(c, L, b, cnt, n_r, pool_used, wo);
    if (ws) return ws;
    if (commit_pending) {  // the previous window's shadow commit is part of K7's time (the stream is synced)
      float tc = 0;
      cudaEventElapsedTime(&tc, c->ev[16], c->ev[17]);
      ms_chk += tc;
      commit_pending = false;
    }
    n_items += wo.items;
    sx.segments += wo.segments;
    sx.clock_gathers += wo.gathers;
    float t = 0;
    cudaEventElapsedTime(&t, c->ev[14], c->ev[15]);
    ms_ex += t;
    cudaEventElapsedTime(&t, c->ev[12], c->ev[13]);
    ms_sort += t;
    ms_chk += wo.ms_check;
    if (sh_out) {
      cudaEventRecord(c->ev[16], st);
      launch_shadow_commit(skey, n_items_dev, b, sh_nxt, sh_cur, st);
      cudaEventRecord(c->ev[17], st);
      commit_pending = true;
      have_state = true;
    }
  }
  if (sw) {  // the session's running totals
    c->have_state = have_state;
    c->s_nr = n_r;
    c->s_pool = pool_used;
    c->s_items += n_items;
    c->s_segs += sx.segments;
    c->s_windows += sx.windows;
    n_items = c->s_items;
    sx.segments = c->s_segs;
    sx.windows = c->s_windows;
  }
  u32 nfind = (u32)hcnt[C_FINDINGS];
  if (nwin == 1 && last_win < 0) {  // no records at all in the window loop (cannot happen for n > 0)
    nfind = 0;
  }
  sx.items = n_items;
  sx.vc_pool_entries = pool_used;
  cudaEventRecord(c->ev[7], st);
  if (sw && !sw->final) {  // more windows follow: no race list yet
    if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "stream window");
    sx.races = n_r;
    sx.kernel_launches = g_launches - launches0;
    return BC_OK;
  }
  // ---- K8: finalize
  if (g.world > 1 && g.rank != 0) nfind = 0;  // findings come from the replicated replay: rank 0 reports them
  u64 total = n_r + nfind;
  if (total > c->races_cap) {
    c->da.free(c->races, c->races_cap * sizeof(bc_race));
    c->races_cap = 0;
    c->races = (bc_race*)c->da.alloc(std::max<u64>(total, 1) * sizeof(bc_race));
    if (!c->races) return fail(c, BC_ERR_OOM, "race list");
    c->races_cap = std::max<u64>(total, 1);
  }
  u32* page_num = S.alloc<u32>(n_pages + 1);
  if (n_r) launch_page_list(words, wl_prefix, page_bits, n_words, page_num, st);
  finalize_races(c->rbuf, (u32)n_r, find_blk, find_rec, nfind, g, snap, page_num, shared_base, (u32)n_keys, c->races, S,
                 st);
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
    if (i == PH_EXPAND || i == PH_SORT || i == PH_CHECK) continue;
    cudaEventElapsedTime(&sx.ms_kernel[i], c->ev[i], e1);
  }
  // the window loop: per-kernel sums over the windows (expand / sort / check also as kernel-only times)
  sx.ms_kernel[PH_EXPAND] = ms_ex;
  sx.ms_kernel[PH_SORT] = ms_sort;
  sx.ms_kernel[PH_CHECK] = ms_chk;
  sx.ms_kernel[PH_N + 0] = ms_chk;
  sx.ms_kernel[PH_N + 1] = ms_sort;
  sx.ms_kernel[PH_N + 2] = ms_ex;
  sx.kernel_launches = g_launches - launches0;
  return BC_OK;
}

bc_status bc_load_trace_shard(bc_ctx* c, const bc_record* recs, const uint32_t* rec_index, uint64_t n_local,
                              uint64_t n_global, int on_device) {
  if (!c) return BC_ERR_INVALID_ARG;
  if (!c->comm) return fail(c, BC_ERR_STATE, "bc_load_trace_shard needs a transport (nccl_unique_id or group)");
  if (n_global >= 0xFFFFFFFFull) return fail(c, BC_ERR_OVERFLOW, "2^32 - 1 or more records");
  if (n_local > n_global || (n_local && !rec_index)) return fail(c, BC_ERR_INVALID_ARG, "shard indices");
  if (!on_device)
    for (u64 i = 0; i < n_local; ++i)
      if (rec_index[i] >= n_global || (i && rec_index[i] <= rec_index[i - 1]))
        return fail(c, BC_ERR_INVALID_ARG, "rec_index must increase and stay below n_global");
  bc_status s = bc_load_trace(c, recs, n_local, on_device);
  if (s) return s;
  c->loaded = false;
  if (n_local && (!on_device || ((uintptr_t)rec_index & 3))) {
    const size_t bytes = n_local * sizeof(u32);
    if (bytes > c->gidx_cap) {
      c->da.free(c->gidx_owned, c->gidx_cap);
      c->gidx_cap = 0;
      c->gidx_owned = (u32*)c->da.alloc(bytes);
      if (!c->gidx_owned) return fail(c, BC_ERR_OOM, "record index buffer");
      c->gidx_cap = bytes;
    }
    cudaMemcpyAsync(c->gidx_owned, rec_index, bytes, on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice,
                    c->stream);
    if (cudaStreamSynchronize(c->stream) != cudaSuccess) return cuda_check(c, "record index copy");
    c->gidx = c->gidx_owned;
  } else {
    c->gidx = rec_index;
  }
  c->sharded = true;
  c->n_global = n_global;
  c->loaded = true;
  return BC_OK;
}

bc_status bc_nccl_unique_id(void* out128) {
  if (!out128) return BC_ERR_INVALID_ARG;
  return (bc_status)nccl_unique_id(out128);
}

bc_status bc_group_create_local(int world, bc_group** out) {
  if (!out || world < 1 || world > 1024) return BC_ERR_INVALID_ARG;
  *out = reinterpret_cast<bc_group*>(local_group_create(world));
  return BC_OK;
}

void bc_group_destroy(bc_group* g) { local_group_destroy(reinterpret_cast<LocalGroup*>(g)); }

bc_status bc_load_values(bc_ctx* c, const uint64_t* values, uint64_t n, int on_device) {
  if (!c) return BC_ERR_INVALID_ARG;
  if (!c->loaded) return fail(c, BC_ERR_STATE, "bc_load_values before bc_load_trace");
  if (c->sharded && values) return fail(c, BC_ERR_INVALID_ARG, "store values with a sharded trace: not supported");
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
    c->da.free(c->values_owned, c->values_cap);
    c->values_cap = 0;
    c->values_owned = (u64*)c->da.alloc(bytes);
    if (!c->values_owned) return fail(c, BC_ERR_OOM, "values buffer");
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
      s = c->sharded ? detect_sharded(c, S) : detect_impl(c, S, nullptr);
      if (s == BC_RETRY_FULL_PAGES) {  // (internal) the sampled page set was incomplete: again, exactly
        c->err.clear();
        Scratch S2(c->stream, &c->arena);  // the same arena buffers, from the first again
        s = detect_impl(c, S2, nullptr, true);
      }
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

bc_status bc_stream_open(bc_ctx* c, uint64_t queue_records, uint64_t max_records, uint64_t min_window,
                         void** queue_dev) {
  if (!c || !queue_dev || queue_records == 0 || max_records == 0) return BC_ERR_INVALID_ARG;
  if (c->comm || c->cfg.world > 1) return fail(c, BC_ERR_INVALID_ARG, "streaming is single-GPU");
  if (c->cfg.n_global_ranges > 64) return fail(c, BC_ERR_INVALID_ARG, "at most 64 global ranges");
  if (max_records >= 0xFFFFFFFFull) return fail(c, BC_ERR_OVERFLOW, "2^32 - 1 or more records");
  cudaSetDevice(c->cfg.device);
  drain_stop(c);
  // every kernel a poll may launch is loaded now: under lazy loading a first launch waits for the
  // running kernels, i.e. for a producer that may be waiting for the queue to drain
  preload_sort();
  preload_check();
  preload_trace();
  preload_sync();
  preload_finalize();
  cudaStream_t st = c->stream;
  c->da.free(c->queue, c->queue_bytes);
  c->da.free(c->sbuf, c->sbuf_cap * sizeof(bc_record));
  c->queue = nullptr;
  c->sbuf = nullptr;
  c->queue_bytes = Q_HDR * sizeof(u64) + queue_records * sizeof(bc_record);
  c->queue = (u64*)c->da.alloc(c->queue_bytes);
  c->sbuf = (bc_record*)c->da.alloc(max_records * sizeof(bc_record));
  if (!c->granges) c->granges = (u64*)c->da.alloc(2 * 64 * sizeof(u64));
  if (!c->dstream) {  // highest priority: its copies are dispatched ahead of queued check kernels
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    cudaStreamCreateWithPriority(&c->dstream, cudaStreamNonBlocking, hi);
  }
  if (!c->dhdr) cudaMallocHost(&c->dhdr, (Q_HDR + 1) * sizeof(u64));
  if (!c->queue || !c->sbuf || !c->granges || !c->dstream || !c->dhdr) return fail(c, BC_ERR_OOM, "stream buffers");
  c->queue_cap = queue_records;
  c->sbuf_cap = max_records;
  u64* hdr = c->dhdr;
  memset(hdr, 0, Q_HDR * sizeof(u64));
  hdr[Q_CAP] = queue_records;
  cudaMemcpyAsync(c->queue, hdr, Q_HDR * sizeof(u64), cudaMemcpyHostToDevice, st);
  cudaMemcpyAsync(c->granges, c->cfg.global_ranges, 2 * 64 * sizeof(u64), cudaMemcpyHostToDevice, st);
  if (cudaStreamSynchronize(st) != cudaSuccess) return cuda_check(c, "stream open");
  c->checked = 0;
  c->drained.store(0);
  c->wseen.store(0);
  c->dgen.store(0);
  c->drain_err.store(0);
  c->drain_stop.store(false);
  c->min_window = std::max<u64>(min_window, 1);
  c->have_state = false;
  c->sh_cur = 0;
  c->s_nr = c->s_pool = c->s_items = c->s_segs = c->s_windows = 0;
  c->loaded = false;
  c->detected = false;
  c->values = nullptr;
  c->drainer = std::thread(drain_loop, c);
  c->streaming = true;
  *queue_dev = c->queue;
  return BC_OK;
}

bc_status bc_stream_poll(bc_ctx* c, int finish, bc_stats* out) {
  if (!c) return BC_ERR_INVALID_ARG;
  if (!c->streaming) return fail(c, BC_ERR_STATE, "bc_stream_poll without bc_stream_open");
  cudaSetDevice(c->cfg.device);
  cudaStream_t st = c->stream;
  auto stop_with = [&](bc_status s, const char* why) {
    drain_stop(c);
    c->streaming = false;
    return fail(c, s, why);
  };
  u64 avail = c->drained.load(std::memory_order_acquire);
  if (finish) {  // the producer has finished: one full drainer pass that began after this call sees the final heads
    const u64 g0 = c->dgen.load(std::memory_order_acquire);
    const auto t0 = std::chrono::steady_clock::now();
    while (!c->drain_err.load() && c->dgen.load(std::memory_order_acquire) < g0 + 2) {
      if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(30))
        return stop_with(BC_ERR_CUDA, "the drain thread stalled");
      std::this_thread::sleep_for(std::chrono::microseconds(20));
    }
    drain_stop(c);
    avail = c->drained.load(std::memory_order_acquire);
    if (!c->drain_err.load() && avail != c->wseen.load())
      return stop_with(BC_ERR_STATE, "finish before the producer committed everything");
  }
  if (int e = c->drain_err.load()) {
    return stop_with((bc_status)e, e == BC_ERR_TRUNCATED ? "more records than bc_stream_open's max_records"
                                                         : "the producer gave up (queue error flag)");
  }
  if (!finish && avail - c->checked < c->min_window) {
    if (out) *out = c->stats;
    return BC_OK;
  }
  // check the drained records as one window (clocks from the whole prefix)
  c->trace = c->sbuf;
  c->n_recs = avail;
  c->g.n_recs = avail;
  c->err.clear();
  StreamWin sw;
  sw.R0 = c->checked;
  sw.final = finish != 0;
  bc_status s;
  {
    Scratch S(st, &c->arena);
    try {
      s = detect_impl(c, S, &sw);
    } catch (const std::bad_alloc&) {
      s = fail(c, BC_ERR_OOM, "scratch allocation");
    }
  }
  cudaStreamSynchronize(st);
  if (out) *out = c->stats;
  if (s != BC_OK) {
    drain_stop(c);
    c->streaming = false;
    return s;
  }
  c->checked = avail;
  if (finish) {
    c->streaming = false;
    c->loaded = true;
    c->detected = true;
  }
  return BC_OK;
}

bc_status bc_queue_push(void* queue_dev, const bc_record* recs, uint64_t n, void* stream) {
  if (!queue_dev || (n && !recs)) return BC_ERR_INVALID_ARG;
  if (!n) return BC_OK;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  // persistent and co-resident (a warp may wait for an earlier ticket's warp): at most 2 CTAs per SM
  const u64 blocks = std::min<u64>((n + 7) / 8, (u64)sms * 2);
  // its SMs keep the full shared-memory split, so the session's check kernels can share them
  cudaFuncSetAttribute(k_queue_push, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  k_queue_push<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>((u64*)queue_dev, recs, n);
  ++g_launches;
  return cudaGetLastError() == cudaSuccess ? BC_OK : BC_ERR_CUDA;
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
