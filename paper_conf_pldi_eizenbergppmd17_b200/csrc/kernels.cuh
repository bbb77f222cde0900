// kernels.cuh — host-side launchers of the libbc kernels and the scratch allocator.
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <new>
#include <vector>

#include "common.cuh"

namespace bc {

// kernels launched by this process (bc_stats.kernel_launches is the delta over one bc_detect)
extern std::atomic<u64> g_launches;

// counters written by the kernels (u64 device array)
// (one u64 array, so that each host synchronisation reads every counter with ONE pinned copy; the u32
// words err / need_sort / races / findings live in the low half of their slot)
enum { C_LANE_EVENTS = 0, C_CONTROL_EVENTS, C_SYNC_RECS, C_ACQ_RECS, C_MEM_RECS, C_IFS, C_BARS, C_SYNC_LANEOPS,
       C_ITEMS, C_ITEM_BOUND, C_SEGMENTS_UNUSED, C_PAGE_WORDS, C_PAGES, C_ERR, C_NEED_SORT, C_FINDINGS,
       C_RACES, C_SEGMENTS, C_GATHERS, C_POOL, C_N };

// Device memory of a context: cudaMallocAsync / cudaFreeAsync on the context's stream, or the caller's allocator (bc_config.dev_alloc /
// dev_free, e.g. torch's caching allocator).
// Force-load kernels (CUDA lazy loading otherwise loads a kernel at its first launch, and that load
// waits for running kernels: a streaming session's consumer would wait for its spinning producer).
template <typename... K>
inline void preload(K... k) {
  cudaFuncAttributes a;
  (cudaFuncGetAttributes(&a, (const void*)k), ...);
}
void preload_sort();
void preload_check();
void preload_trace();
void preload_sync();
void preload_finalize();

struct DevAlloc {
  bc_dev_alloc_fn fa = nullptr;
  bc_dev_free_fn ff = nullptr;
  void* user = nullptr;
  cudaStream_t st = nullptr;
  void* alloc(size_t bytes) {
    if (fa) return fa(bytes, (void*)st, user);
    // stream-ordered: cudaFree would synchronise the whole device, which deadlocks a streaming
    // session whose producer kernel (another stream) waits for this context to drain the queue
    void* p = nullptr;
    if (cudaMallocAsync(&p, bytes ? bytes : 256, st) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    return p;
  }
  void free(void* p, size_t bytes) {
    if (!p) return;
    if (ff) ff(p, bytes, (void*)st, user);
    else cudaFreeAsync(p, st);
  }
};

// Per-context scratch arena.  A bc_detect allocates its scratch buffers in a fixed order; the i-th
// allocation reuses the i-th buffer of earlier calls when it is large enough, so repeated detects of
// one trace see identical pointers and allocate nothing.  Buffers are 256-B aligned and padded to a
// multiple of 256 B (the TMA bulk copies of the radix sort may read up to 12 B past an array's end).
// Freed at bc_destroy.
struct Arena {
  DevAlloc* da = nullptr;
  std::vector<std::pair<void*, size_t>> bufs;
  u64 gen = 0;  // bumped whenever a buffer is (re)allocated
  void free_all() {
    for (auto& b : bufs)
      if (b.first) da->free(b.first, b.second);
    bufs.clear();
    ++gen;
  }
};

class Scratch {
 public:
  Scratch(cudaStream_t st, Arena* ar) : st_(st), ar_(ar) {}
  template <typename T>
  T* alloc(size_t n) {
    size_t bytes = n * sizeof(T);
    if (bytes == 0) bytes = 16;
    bytes = (bytes + 255) & ~(size_t)255;
    const size_t i = next_++;
    if (i < ar_->bufs.size() && ar_->bufs[i].second >= bytes) return (T*)ar_->bufs[i].first;
    if (i < ar_->bufs.size()) {
      cudaStreamSynchronize(st_);  // the old buffer may still be read by queued work
      ar_->da->free(ar_->bufs[i].first, ar_->bufs[i].second);
      ar_->bufs[i] = {nullptr, 0};
    } else {
      ar_->bufs.push_back({nullptr, 0});
    }
    const size_t cap = bytes + ((bytes / 8 + 255) & ~(size_t)255);
    void* p = ar_->da->alloc(cap);
    if (!p) throw std::bad_alloc();
    ar_->bufs[i] = {p, cap};
    ++ar_->gen;
    return (T*)p;
  }
  void release() {}

 private:
  cudaStream_t st_;
  Arena* ar_;
  size_t next_ = 0;
};

// sort.cu
size_t rs_temp_bytes(u64 n);
bool radix_sort_pairs(u32* keys, u32* vals, u32* keys_alt, u32* vals_alt, u64 n, int bit_lo, int bit_hi, void* temp,
                      cudaStream_t st, const u64* n_dev = nullptr, u64* n_out_dev = nullptr, bool drop = false);
size_t scan_temp_bytes(u64 n);
void exclusive_scan_u32(const u32* in, u32* out, u64 n, void* temp, u64* total_dev, cudaStream_t st);
void exclusive_scan_u32_u64(const u32* in, u64* out, u64 n, void* temp, u64* total_dev, cudaStream_t st);

// trace.cu
// window weight of a record: its item upper bound + REC_W (DESIGN.md §7 "Windows"): a window of at
// most WIN_MAX weight holds < 2^27 records (32-bit window-local event ids) and < 2^30 items
constexpr u32 REC_W = 8;
constexpr u64 WIN_MAX = (1ull << 30) - 1024;
void launch_header(const bc_record* recs, const Geo& g, u32* wkey, u32* wval, u32* if_cnt, u32* bar_cnt,
                   u32* sync_list, u32* page_bits, u32* word_list, u64* cnt, u32* rec_w, uint4* hdr16,
                   u32* rec_cnt, u32* err, cudaStream_t st, int mark_pages = 1);  // 0 none, 1 every write address, 2 sampled
void launch_mark_ranges(const u64* ranges, u32 n_ranges, u32* page_bits, u32* word_list, u64* cnt, u32* err,
                        cudaStream_t st);
void launch_window_starts(const u64* cum, u64 n, u64 we, u32 nwin, u64* starts, u64* bounds, cudaStream_t st);
constexpr u32 WS_SMALL = 8192;  // n_warps up to which one CTA does the per-warp scans (launch_warp_scans)
void launch_warp_scans(const u32* rec_cnt, const u32* if_cnt, const u32* bar_cnt, u32 n_warps, u32* warp_start,
                       u32* node_base, u32* bar_base, cudaStream_t st);
void launch_page_rank(u32* words, const u64* n_words_dev, const u32* page_bits, u32* page_rank, u32* wl_prefix,
                      u64* n_pages_dev, u32* need_sort, int presorted, cudaStream_t st);
void launch_warp_start(const u32* skeys, u64 n, u32 n_warps, u32* warp_start, cudaStream_t st);
void launch_replay(const uint4* hdr16, const u32* wrec, const u32* gidx, const u32* warp_start, const Geo& g,
                   const u32* node_base, const u32* bar_base, uint4* snap, uint4* nodes, u32* bar_rec, u32* bar_next,
                   u32* find_blk, u32* find_rec, u32* find_cnt, u32* err, cudaStream_t st);
void launch_barriers(const Geo& g, const u32* bar_cnt, const u32* bar_base, const u32* bar_rec, const u32* bar_next,
                     u32* blockR, u32* err, cudaStream_t st, bool allow_pending = false);
void launch_snap_blab(uint4* snap, u64 n, u32 wpb, u32 n_warps, u64 n_bars, const u32* bar_base, const u32* blockR,
                      cudaStream_t st);
void launch_expand(const bc_record* recs, const uint4* hdr16, const Geo& g, const u32* page_bits, const u32* page_rank, u32 shared_base,
                   const u64* cum, u64 R0, u64 R1, const u32* gidx, u64 G0, u32* keys, u32* evs, u32* err,
                   cudaStream_t st);
void launch_node_base(const u32* if_excl, u32 n_warps, u32* node_base, cudaStream_t st);

// sync.cu
void sort_perm_by(u32* perm, const u32* f, u32 n, int bits, Scratch& S, cudaStream_t st);
void launch_iota(u32* p, u32 n, cudaStream_t st);
void launch_gather_u32(const u32* src, const u32* perm, u32 n, u32* dst, cudaStream_t st);
int run_sync_skeleton(const bc_record* srecs, const u32* sgidx, u32 n_srec, u32 n_lo, u32 n_acq, HbCtx& hc,
                      Scratch& S, cudaStream_t st, u64* n_entries_out);
void gather_sync_records(const bc_record* recs, u32* sync_list, u32 n, u64 n_recs, bc_record* srecs, Scratch& S,
                         cudaStream_t st);

// check.cu
size_t check_status_bytes(u64 n);
struct CheckLaunch {
  HbCtx c;
  const u32* keys;      // (granule key << 2) | op, sorted
  const u32* evs;       // (record - R0) << 5 | lane
  const u64* n_dev;     // item count (device)
  u64 n_max;            // upper bound of the item count
  u32 R0;               // first record of the window
  const uint4* sh_in;   // carried shadow entries (2 x uint4 per granule) or null (first window)
  uint4* sh_out;        // entries of the granules the window touches (others untouched), or null (last window)
  uint2* pool;          // append-only read-vector pool (record, warp << 5 | lane)
  u32* pool_cnt;
  u32 pool_cap;
  uint4* races;         // (key, cur rec, prior rec, cur lane | prior lane << 5 | kind << 10)
  u32* race_cnt;
  u32 race_cap;
  u64* seg_cnt;
  const u64* values;
  void* status;         // check_status_bytes() of scratch
};
void launch_check(const CheckLaunch& L, cudaStream_t st);

void launch_count_gathers(const u32* keys, const u64* n_dev, u64* out, u64* segs, cudaStream_t st);
// after K7 of a window: tab[k] = out[k] for every granule k the sorted items touch
void launch_shadow_commit(const u32* keys, const u64* n_dev, u64 n_max, const uint4* out, uint4* tab,
                          cudaStream_t st);

// finalize.cu
void launch_page_list(const u32* words, const u32* wl_prefix, const u32* page_bits, u64 n_words, u32* page_num,
                      cudaStream_t st);
void finalize_races(const uint4* races, u32 n_r, const u32* fblk, const u32* frec, u32 n_f, const Geo& g,
                    const uint4* snap, const u32* page_num, u32 shared_base, u32 n_keys, bc_race* out, Scratch& S,
                    cudaStream_t st);

}  // namespace bc
