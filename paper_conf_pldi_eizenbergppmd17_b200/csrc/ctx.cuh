// ctx.cuh — the context behind the opaque bc_ctx handle of include/bc.h (api.cu, shard.cu).
#pragma once
#include <atomic>
#include <string>
#include <thread>

#include "comm.cuh"
#include "common.cuh"
#include "kernels.cuh"

using namespace bc;

struct bc_ctx {
  bc_config cfg;
  Geo g;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  DevAlloc da;
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
  uint4* rbuf = nullptr;     // device, K7 race records of all windows (grown on demand)
  size_t rbuf_cap = 0;       // entries
  uint2* pool = nullptr;     // device, read-vector pool carried between windows (grown on demand)
  size_t pool_cap = 0;       // entries
  bc_stats stats{};
  Arena arena;  // scratch buffers, reused across bc_detect calls
  std::string err;
  cudaEvent_t ev[18] = {};
  u64* hcnt = nullptr;  // pinned host copy of the device counter array (one D2H copy per host sync)
  // block-sharded multi-GPU: this rank holds the records of blocks b % world == rank
  Comm* comm = nullptr;       // NCCL or in-process transport, null: single GPU / replicated trace
  bool sharded = false;       // loaded by bc_load_trace_shard
  const u32* gidx = nullptr;  // device, global record index of each local record (sharded)
  u32* gidx_owned = nullptr;
  size_t gidx_cap = 0;
  u64 n_global = 0;           // records of the whole trace (sharded)
  void* xbuf[6] = {};         // device exchange / scratch buffers (grown on demand)
  size_t xcap[6] = {};
  // streaming session (bc_stream_open)
  bool streaming = false;
  u64* queue = nullptr;       // device: 8 u64 header + ring
  size_t queue_bytes = 0;
  u64 queue_cap = 0;
  bc_record* sbuf = nullptr;  // device: the trace so far
  u64 sbuf_cap = 0;
  // the drain thread: copy-engine copies ring -> sbuf on its own stream, then the new read head; it
  // needs no SM, so a producer waiting on a full ring never waits for a window check
  std::thread drainer;
  std::atomic<bool> drain_stop{false};
  std::atomic<u64> drained{0};  // records in sbuf (published after the copies completed)
  std::atomic<u64> wseen{0};    // the write head the drainer last saw
  std::atomic<u64> dgen{0};     // completed drainer passes (header read, copies, publish)
  std::atomic<int> drain_err{0};
  cudaStream_t dstream = nullptr;
  u64* dhdr = nullptr;          // pinned: the header as last read, [Q_HDR] = the read head to write
  u64 checked = 0;            // records checked (the next window starts here)
  u64 min_window = 0;
  u64* granges = nullptr;     // device copy of bc_config.global_ranges
  uint4* sh[2] = {};          // shadow tables carried between polls
  size_t sh_bytes = 0;
  int sh_cur = 0;
  bool have_state = false;
  u64 s_nr = 0, s_pool = 0, s_items = 0, s_segs = 0, s_windows = 0;
};

// one window of a streaming session: records [R0, n) are new; earlier ones only feed the clocks
// internal status of detect_impl (never returned by the C ABI): re-run with every write page marked
constexpr bc_status BC_RETRY_FULL_PAGES = (bc_status)-100;

struct StreamWin {
  u64 R0 = 0;
  bool final = false;
};

enum { PH_HEADER = 0, PH_PARTITION, PH_REPLAY, PH_SYNC, PH_EXPAND, PH_SORT, PH_CHECK, PH_FINALIZE, PH_N };

inline bc_status fail(bc_ctx* c, bc_status s, const std::string& msg) {
  if (c) c->err = msg;
  return s;
}

inline bc_status cuda_check(bc_ctx* c, const char* where) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(c, BC_ERR_CUDA, std::string(where) + ": " + cudaGetErrorString(e));
  return BC_OK;
}

inline int bits_for(u64 maxval) {
  int b = 0;
  while (b < 64 && (maxval >> b)) ++b;
  return b;
}


// device buffer of the context that grows (contents not kept) to at least `bytes`
void* ctx_buffer(bc_ctx* c, int slot, size_t bytes);

// K7 over one window's sorted items: pool growth (when the window writes shadow entries), the race
// buffer retry, the counter round trip.  n_r / pool_used are cumulative; adds to the stats.
struct WindowOut {
  u64 items = 0, segments = 0, gathers = 0;
  float ms_check = 0;
};
bc_status check_window(bc_ctx* c, CheckLaunch& L, u64 window_bound, u64* cnt, u64& n_r, u64& pool_used,
                       WindowOut& wo);

bc_status detect_sharded(bc_ctx* c, Scratch& S);
