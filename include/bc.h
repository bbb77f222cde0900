/* bc.h — C ABI of the B200-native BARRACUDA race check.
 *
 * What this library computes (PAPER.md = /root/reference/PAPER.md, cited as P:Lnnn):
 *
 *   Input  — a *feasible* warp-granular trace of one kernel launch (§3.1) in the
 *            paper's fixed 272-byte queue record format (§4.2, Fig. 6), in
 *            global trace order, plus the traced launch geometry.
 *   Output — the race set the happens-before rules of Fig. 2 / Fig. 3 (§3.3)
 *            report on that trace: every failed epoch / vector-clock check is one race
 *            (prior event, current event) on a shadow granule, classified as in P:L1345-1347,
 *            plus barrier-divergence findings.  The set is bit-identical to the
 *            plain CPU oracle (oracle/oracle.cpp, test infrastructure) that interprets the
 *            same rules on uncompressed vector clocks.  Readings of garbled passages are
 *            listed in DESIGN.md §"Readings" (R1-R15) and are the same on both sides.
 *
 * Calls:
 *   bc_init -> bc_load_trace -> bc_detect -> bc_races -> bc_destroy
 *
 * Conventions:
 *   - One context per process / GPU.  Not thread-safe.  Every call is stream-ordered on
 *     cfg.stream and returns only after the work it needs has completed.
 *   - Errors are negative bc_status values; detail text via bc_last_error(ctx).
 *     Races and barrier-divergence findings are RESULTS, never errors.
 *   - There is no CPU fallback: bc_init fails with BC_ERR_CUDA if no sm_100 device is usable.
 */
#ifndef BC_H_
#define BC_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---------------------------------------------------------------- status codes */
typedef enum {
  BC_OK = 0,
  BC_ERR_INVALID_ARG = -1,      /* bad geometry / pointer / flag                                */
  BC_ERR_INFEASIBLE_TRACE = -2, /* trace violates P:L360-366 feasibility or R10 barrier rules   */
  BC_ERR_OOM = -3,              /* device allocation failed                                     */
  BC_ERR_CUDA = -4,             /* CUDA runtime error (no device, launch failure, ...)          */
  BC_ERR_NCCL = -5,             /* multi-GPU communicator error                                 */
  BC_ERR_STATE = -6,            /* call out of order (e.g. bc_detect before bc_load_trace)      */
  BC_ERR_TRUNCATED = -7,        /* bc_races: cap < number of races (cap entries were copied)    */
  BC_ERR_OVERFLOW = -8          /* an index space overflowed (records >= 2^32 - 1, shadow keys >= 2^30,
                                   sync-lookup step cap)                 */
} bc_status;

/* ------------------------------------------------------------- the trace record */
/* One warp-level instruction ("fields identifying the warp, the operation, a
 * 32-bit mask of active threads, and 32 entries for the addresses accessed by each thread
 * in the warp ... a fixed 16 + 8 x 32 = 272 bytes").  Little endian, 8-byte aligned. */
enum {
  BC_OP_LD = 0, BC_OP_ST = 1, BC_OP_ATOM = 2,                   /* rd / wr / atm   */
  BC_OP_ACQ_BLK = 3, BC_OP_ACQ_GLB = 4,                         /* acqBlk / acqGlb               */
  BC_OP_REL_BLK = 5, BC_OP_REL_GLB = 6,                         /* relBlk / relGlb               */
  BC_OP_AR_BLK = 7, BC_OP_AR_GLB = 8,                           /* arBlk  / arGlb                */
  BC_OP_FENCE = 9,                                              /* standalone fence: no-op (R14) */
  BC_OP_BAR = 10,                                               /* one warp's bar.sync arrival   */
  BC_OP_IF = 11, BC_OP_ELSE = 12, BC_OP_FI = 13                 /* if(w) else(w) fi(w) P:L290-306 */
};
enum { BC_SPACE_GLOBAL = 0, BC_SPACE_SHARED = 1, BC_SPACE_NONE = 2 };
enum { BC_REC_SAME_VALUE = 1 }; /* all active lanes store one value (reading R6) */

typedef struct bc_record {
  uint32_t warp;      /* global warp id = block_linear * warps_per_block + warp_in_block        */
  uint32_t mask;      /* bit i = lane i active; must equal the warp's SIMT-stack top */
  uint8_t op;         /* BC_OP_*                                                                */
  uint8_t space;      /* BC_SPACE_GLOBAL | BC_SPACE_SHARED (shared: byte offset in block smem)  */
  uint8_t size_log2;  /* access width 2^k bytes, k in 0..4; addresses naturally aligned        */
  uint8_t flags;      /* BC_REC_SAME_VALUE                                                      */
  uint32_t aux;       /* IF: then-lane mask (else = top & ~aux); otherwise 0                   */
  uint64_t addr[32];  /* per-lane byte address; inactive lanes ignored                          */
} bc_record;          /* 272 bytes */

/* ------------------------------------------------------------------ race record */
enum { BC_KIND_WW = 0, BC_KIND_WR, BC_KIND_RW, BC_KIND_WA, BC_KIND_AW, BC_KIND_RA, BC_KIND_AR,
       BC_KIND_NONE = 0xFF };                                   /* (prior, current) access type */
enum { BC_CLS_SAME_INSN = 0,          /* two lanes of one warp instruction         */
       BC_CLS_BRANCH = 1,             /* same warp, different instruction: branch ordering P:L591-630 */
       BC_CLS_INTRA_BLOCK = 2, BC_CLS_INTER_BLOCK = 3,
       BC_CLS_BARRIER_DIVERGENCE = 4 };                         /* finding          */

typedef struct bc_race {
  uint64_t addr;         /* granule start: global byte address, or byte offset in the block's smem */
  uint64_t prior_event;  /* (record_index << 5) | lane, record index in the whole trace; ~0 for findings */
  uint64_t cur_event;    /* (record_index << 5) | lane                                          */
  uint8_t kind, cls, space, pad;
  uint32_t block;        /* shared: owning block; global: block of the current event; finding: block */
} bc_race;               /* 32 bytes.  Canonical order: findings, then global races by address,
                            then shared races by (block, offset); ties by (cur_event, prior_event) */

/* ------------------------------------------------------------------ configuration */
enum {
  BC_F_RELEASE_OVERWRITE = 1u,    /* the printed release S_x := C_t (Fig. 3 RELBLOCK / RELGLOBAL,
                                     P:L754-758; ACQREL joins the slot before it
                                     writes it) instead of reading R1's join       */
  BC_F_NO_SAME_VALUE_FILTER = 2u, /* report intra-warp same-value WW races too (R6)           */
  BC_F_COUNT_GATHERS = 4u         /* statistics: fill bc_stats.clock_gathers and .segments (one extra pass) */
};

/* Optional device allocator ("PyTorch only for device memory"): every device buffer the
 * context owns (trace copy, scratch, shadow tables, race list) is obtained from dev_alloc and returned
 * to dev_free with the context's stream, e.g. torch's caching allocator.  NULL: cudaMallocAsync / cudaFreeAsync on the context stream.
 * dev_alloc returns NULL on failure (-> BC_ERR_OOM); returned memory must be 256-B aligned. */
typedef void* (*bc_dev_alloc_fn)(size_t bytes, void* stream, void* user);
typedef void (*bc_dev_free_fn)(void* ptr, size_t bytes, void* stream, void* user);

typedef struct bc_config {
  uint32_t grid_dim[3], block_dim[3]; /* traced launch geometry; x fastest          */
  uint32_t warp_size;                 /* 32, or 4 / 8 / 16: warp-size simulation (SURVEY row f4,
                                         P:L277-282): the trace's records describe warps of that
                                         many lanes (lanes >= warp_size inactive); see
                                         bc_split_warps() to produce such a trace from a 32-lane one */
  uint32_t granule_log2;              /* shadow granularity 2^G bytes, G in 0..4  */
  uint32_t smem_bytes_per_block;      /* shared-memory shadow size per block      */
  uint32_t flags;                     /* BC_F_*                                                  */
  int32_t device;                     /* CUDA device ordinal                                     */
  int32_t rank, world;                /* address sharding: world = 0 or
                                         1 checks every shadow granule.  world = W > 1 (W <= 1024,
                                         0 <= rank < W): every rank is given the SAME trace, derives
                                         the clocks (K1-K3) itself, and checks only the granules it
                                         owns, owner(g) = hash(g) mod W; barrier-divergence findings
                                         are reported by rank 0 only.  The W per-rank race lists are
                                         disjoint and their canonical merge is the world = 1 list
                                         (the caller gathers them, e.g. over torch.distributed). */
  void* stream;                       /* cudaStream_t (NULL = a stream owned by the context)     */
  uint64_t window_events;             /* trace window budget: records are checked in
                                         consecutive windows of at most this many items (granule x
                                         lane events) + 8 per record; the per-granule shadow state
                                         (Fig. 8) carries from one window to the next.
                                         0 = auto (one window up to 2^30 - 1024, else 2^28 each);
                                         larger values are clamped to 2^30 - 1024.                */
  bc_dev_alloc_fn dev_alloc;          /* optional, see above                                     */
  bc_dev_free_fn dev_free;
  void* alloc_user;
  /* Block-sharded multi-GPU: with world > 1 and a transport, every rank loads only the
   * records of the blocks b with b % world == rank (bc_load_trace_shard) and the ranks exchange what
   * the check needs (clock snapshots, sync records, per-window (granule, event) items to the granule's
   * owner, races to rank 0) over the transport.  Exactly one of:                                    */
  const void* nccl_unique_id;         /* 128 B from bc_nccl_unique_id() on rank 0, broadcast by the caller
                                         (e.g. torch.distributed): NCCL over NVLink / NVSwitch, one
                                         process per GPU; bc_init is collective                     */
  struct bc_group* group;             /* in-process transport: the ranks are contexts of this process,
                                         one host thread each (bc_group_create_local)              */
  /* Declared global allocations (the paper's global shadow page table):
   * (base, size) byte ranges.  Required for streaming (bc_stream_open): the page set, and with it every
   * shadow key, is then fixed before the first record arrives; a global access outside the ranges fails
   * the detect with BC_ERR_INVALID_ARG.  Ignored otherwise. */
  uint64_t global_ranges[2 * 64];
  uint32_t n_global_ranges;
} bc_config;

typedef struct bc_stats {
  uint64_t records, lane_events, control_events; /* SURVEY §8(d.1) units                         */
  uint64_t items;            /* (granule, lane event) pairs checked after the write-page filter   */
  uint64_t segments;         /* granule segments checked (summed over windows); 0 unless          
                                BC_F_COUNT_GATHERS                                                */
  uint64_t races, findings;  /* race records / barrier-divergence findings                       */
  uint64_t sync_ops;         /* acquire / release lane operations                                 */
  uint64_t written_pages;    /* 1-MB global pages with at least one write          */
  uint64_t kernel_launches;  /* libbc kernels launched by this bc_detect                          */
  uint64_t clock_gathers;    /* 16-B record clock snapshots the per-granule check reads (items that
                                some happens-before check needs); 0 unless BC_F_COUNT_GATHERS    */
  uint64_t windows;          /* trace windows checked (window_events)                             */
  uint64_t vc_pool_entries;  /* read-vector entries carried between windows                        */
  float ms_total;            /* device time of bc_detect (cudaEvents on the stream)               */
  float ms_kernel[12];       /* per phase, then kernel-only k_check / k_sort_items / k_expand;
                                see bc_phase_name()                                              */
} bc_stats;

/* ------------------------------------------------------------------------- calls */
typedef struct bc_ctx bc_ctx; /* opaque: one context per process / rank, not thread-safe          */

/* Create a context for one traced launch geometry. */
bc_status bc_init(const bc_config* cfg, struct bc_ctx** out);

/* Hand the trace to the context.  recs_on_device = 0: `recs` is host memory and is copied
 * (stream-ordered; the caller keeps ownership).  recs_on_device = 1: `recs` is device memory
 * on cfg.device, borrowed (not copied) until the next bc_load_trace / bc_destroy; the caller
 * must keep it alive and unmodified.  n_recs may be 0.  n_recs >= 2^32 - 1 -> BC_ERR_OVERFLOW. */
bc_status bc_load_trace(struct bc_ctx* ctx, const bc_record* recs, uint64_t n_recs, int recs_on_device);

/* Block-sharded trace (per-block partitioning of P:L1072-1084): this rank's records --
 * those of the traced blocks b with b % world == rank -- in trace order, with rec_index[i] = the
 * global record index of recs[i] (strictly increasing, < n_global), n_global = records of the whole
 * trace.  Ownership as bc_load_trace (recs_on_device applies to both arrays).  Needs a context with a
 * transport (nccl_unique_id or group).  bc_detect is then collective: every rank calls it; race
 * lists come back on rank 0 (bc_races on other ranks: 0 races).  Errors: BC_ERR_STATE (no transport),
 * BC_ERR_INVALID_ARG, BC_ERR_OVERFLOW (n_global >= 2^32 - 1), BC_ERR_OOM / BC_ERR_CUDA. */
bc_status bc_load_trace_shard(bc_ctx* ctx, const bc_record* recs, const uint32_t* rec_index, uint64_t n_local,
                              uint64_t n_global, int recs_on_device);

/* Warp-size simulation (reading R17 in DESIGN.md): re-split a trace recorded
 * with 32-lane warps (the geometry of ctx, whose warp_size must be 32) into virtual warps of ws lanes
 * (4, 8, 16; 32 copies it).  Record (warp w, mask m) becomes, in trace order, one record per virtual
 * warp j of w that executes it: warp (block, (w_in_block * 32 + j * ws) / ws), mask
 * (m >> j*ws) & (2^ws - 1), addresses addr[j*ws ...]; an IF none of whose lanes are in virtual warp j is
 * not executed by it, nor its ELSE / FI or anything nested.  recs, out, origin: DEVICE pointers on
 * ctx's device; origin[i] = (source record << 5) | first lane of out[i].  *n_out = records of the
 * split trace (out == NULL: count only); cap < *n_out -> cap records written, BC_ERR_TRUNCATED.  The
 * result is checked with a context of warp_size = ws and the same grid / block.  Stream-ordered on
 * ctx's stream, synchronizes before return. */
bc_status bc_split_warps(bc_ctx* ctx, const bc_record* recs, uint64_t n_recs, uint32_t ws, bc_record* out,
                         uint64_t* origin, uint64_t cap, uint64_t* n_out);

/* ---- streaming ingest (the device queue of Fig. 6) ----
 * The traced program pushes its records into a lock-free device queue while it runs; the context
 * consumes committed ranges as trace windows (row a5) while the producer keeps going, carrying every
 * granule's 32-B shadow state from window to window.  Queue layout (device memory, 8-B aligned):
 *   uint64_t write_head;   reservations: a producer takes ticket t = the record's trace position
 *   uint64_t commit_head;  records [0, commit_head) are complete; a producer commits ticket t (stores
 *                          t + 1) after writing its record, once commit_head == t (in ticket order)
 *   uint64_t read_head;    records [0, read_head) have been consumed; a producer waits while
 *                          t >= read_head + capacity (ring full)
 *   uint64_t capacity;     ring slots
 *   uint64_t error;        non-zero: a producer gave up (waited > ~10 s for room or its turn)
 *   uint64_t pad[3];
 *   bc_record ring[capacity];   record t lives in ring[t % capacity]
 * bc_stream_open: allocate the queue (queue_records slots; *queue_dev = its device address) and room for
 *   max_records records of trace; needs bc_config.global_ranges.  Starts the session's drain thread,
 *   which moves committed records from the ring into the trace and advances read_head with copy-engine
 *   transfers on its own (highest-priority) stream: the ring is served even while a window check waits
 *   for SMs the producer holds.  The trace so far is the context's loaded trace (bc_load_trace is not
 *   used in a streaming session).  Preloads every kernel a poll launches (CUDA lazy loading would
 *   otherwise make a first launch wait for the running producer).
 * bc_stream_poll: once at least min_window drained records are new (or finish = 1) check them as one
 *   window; returns BC_OK with nothing checked when too few are new.  finish = 1 is called after the
 *   producer has finished (e.g. its stream synchronised): it waits for the drain thread to take
 *   everything committed, checks the rest and makes the race list available to bc_races (the session
 *   ends).  Errors: as bc_detect, BC_ERR_STATE (no session / the producer reserved records it never
 *   committed), BC_ERR_TRUNCATED (more records than max_records), BC_ERR_INVALID_ARG (producer error,
 *   undeclared global access).  Any error ends the session.
 * bc_queue_push: a stand-in producer (the instrumented kernel of the paper): pushes records recs[0, n)
 *   (device memory, trace order) with tickets 0 .. n-1 through the protocol above, on `stream`
 *   (cudaStream_t), asynchronously; run it concurrently with bc_stream_poll. */
bc_status bc_stream_open(bc_ctx* ctx, uint64_t queue_records, uint64_t max_records, uint64_t min_window,
                         void** queue_dev);
bc_status bc_stream_poll(bc_ctx* ctx, int finish, bc_stats* out);
bc_status bc_queue_push(void* queue_dev, const bc_record* recs, uint64_t n_recs, void* stream);

/* 128-byte NCCL unique id for bc_config.nccl_unique_id (call on rank 0 only).  BC_ERR_NCCL if no NCCL
 * library can be loaded (libbc dlopens the libnccl.so.2 already in the process, else the system's). */
bc_status bc_nccl_unique_id(void* out128);

/* In-process group of `world` ranks for bc_config.group (tests, or several GPUs driven by one
 * process); destroy after every context of the group. */
typedef struct bc_group bc_group;
bc_status bc_group_create_local(int world, bc_group** out);
void bc_group_destroy(bc_group* group);

/* Optional per-lane store values (reading R6b in DESIGN.md).
 *   values[r * 32 + l] = the value lane l of store record r writes (8 B; a 64-bit digest for wider
 *   vector stores); entries of other records / inactive lanes are ignored.
 * With values loaded, the intra-warp same-value filter compares the two lanes' values (a
 * write-write race between two lanes of ONE record is filtered iff they store the same value)
 * instead of reading the BC_REC_SAME_VALUE flag.  n_recs must equal the loaded trace's record
 * count.  Host pointer: copied (caller keeps ownership); device pointer (values_on_device = 1,
 * 8-B aligned): borrowed until the next bc_load_trace / bc_load_values / bc_destroy.  values ==
 * NULL clears them.  bc_load_trace clears them too.  Errors: BC_ERR_STATE (no trace loaded),
 * BC_ERR_INVALID_ARG (count mismatch / misaligned device pointer), BC_ERR_OOM / BC_ERR_CUDA. */
bc_status bc_load_values(bc_ctx* ctx, const uint64_t* values, uint64_t n_recs, int values_on_device);

/* Run the race check on the loaded trace (all kernels on cfg.stream) and synchronize.
 * Infeasible trace -> BC_ERR_INFEASIBLE_TRACE (no races are kept).  `out` may be NULL.
 * Repeated calls on the same trace are idempotent. */
bc_status bc_detect(struct bc_ctx* ctx, bc_stats* out);

/* Copy the canonical race list (findings first) into host memory.  out == NULL: only
 * *n_total is written.  cap < *n_total: cap records are copied and BC_ERR_TRUNCATED returned. */
bc_status bc_races(struct bc_ctx* ctx, bc_race* out, uint64_t cap, uint64_t* n_total);

/* Same, into device memory (`out` is a device pointer on cfg.device). */
bc_status bc_races_device(struct bc_ctx* ctx, bc_race* out_dev, uint64_t cap, uint64_t* n_total);

void bc_destroy(struct bc_ctx* ctx);

const char* bc_status_string(bc_status s);
const char* bc_last_error(const struct bc_ctx* ctx);
const char* bc_phase_name(int i); /* names of bc_stats.ms_kernel[i]; NULL past the end */

#ifdef __cplusplus
}
#endif
#endif /* BC_H_ */
