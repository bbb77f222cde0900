// sync.cu — K3 sync skeleton: the ACQ / REL / ACQREL x BLOCK / GLOBAL
// rules of Fig. 3 and their scope semantics (§3.3.4) over the
// sync-location map S_x, reading R1 (release joins into S_x).
//
// S_x is kept as append-only arrays of entries instead of materialised vector clocks:
//   array G_x          (id = xid)            : what global-scope releases put in every S_x[b]
//   array B_{x,b}      (id = nx + bid)       : what block-scope releases of block b put in S_x[b]
//   array F_a          (id = nx + nB + a)    : the view acquire record a took
// A release lane-op at event e appends, at pos e, the releaser's structural clock (block-level
// barrier label, the warp's SIMT-stack levels) plus LINKs to the views of the acquires of its
// block it structurally knows (its foreign knowledge).  An acquire lane-op at event e records
// LINKs (G_x, bound e) and the block arrays it may read: S_x[b] = G_x ⊔ B_{x,b} (ACQ_BLK) or
// ⊔_b S_x[b] = G_x ⊔ ⊔_b B_{x,b} (ACQ_GLB).  Because a view is "entries with pos < bound",
// nothing has to be processed in trace order: every lane-op is independent (one thread each),
// and an AR chain (threadFenceReduction's atomicInc ticket) costs O(1) entries per op instead of
// the O(n) vector-clock copy of the printed rules.
#include <cstdio>
#include <cstdlib>

#include "common.cuh"
#include "kernels.cuh"

namespace bc {

namespace {

__device__ __forceinline__ bool is_acq_op(u32 op) {
  return op == BC_OP_ACQ_BLK || op == BC_OP_ACQ_GLB || op == BC_OP_AR_BLK || op == BC_OP_AR_GLB;
}
__device__ __forceinline__ bool is_rel_op(u32 op) {
  return op == BC_OP_REL_BLK || op == BC_OP_REL_GLB || op == BC_OP_AR_BLK || op == BC_OP_AR_GLB;
}
__device__ __forceinline__ bool is_glb_op(u32 op) {
  return op == BC_OP_ACQ_GLB || op == BC_OP_REL_GLB || op == BC_OP_AR_GLB;
}

__global__ void k_popc_recs(const bc_record* __restrict__ srecs, u32 n, u32* __restrict__ out) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) out[i] = __popc(__ldg(&srecs[i].mask));
}

// lane-ops: global record, lane, sync position, 64-bit location key (split), index
__global__ void k_laneops(const bc_record* __restrict__ srecs, const u32* __restrict__ sgidx, u32 n,
                          const u32* __restrict__ off, Geo g, u32* __restrict__ lo_rec, u32* __restrict__ lo_lane,
                          u32* __restrict__ lo_sp, u32* __restrict__ xk_lo, u32* __restrict__ xk_hi,
                          u32* __restrict__ lo_idx, u32* __restrict__ err) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  u32 r = sgidx[i];
  const bc_record& rc = srecs[i];
  u32 m = rc.mask, o = off[i];
  u32 w = rc.warp;
  while (m) {
    int l = __ffs(m) - 1;
    m &= m - 1;
    u64 a = rc.addr[l];
    u64 xk;
    if (rc.space == BC_SPACE_SHARED) {
      xk = (1ull << 63) | ((u64)(w / g.wpb) << 32) | (u64)(a >> g.G);
    } else {
      xk = a >> g.G;
      if (xk >> 63) set_err(err, ERR_OVERFLOW);
    }
    lo_rec[o] = r;
    lo_lane[o] = (u32)l;
    lo_sp[o] = i;
    xk_lo[o] = (u32)xk;
    xk_hi[o] = (u32)(xk >> 32);
    lo_idx[o] = o;
    ++o;
  }
}

// flags of the first occurrence of each distinct (hi, lo) in sorted order
__global__ void k_uniq_flags2(const u32* __restrict__ hi, const u32* __restrict__ lo, const u32* __restrict__ perm,
                              u32 n, u32* __restrict__ flag) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  u32 p = perm[i];
  u32 f = 1;
  if (i > 0) {
    u32 q = perm[i - 1];
    f = (hi[p] != hi[q] || lo[p] != lo[q]) ? 1u : 0u;
  }
  flag[i] = f;
}

// xid[perm[i]] = (inclusive flag scan)[i] - 1 ; here `ex` is the exclusive scan of flags
__global__ void k_assign_ids(const u32* __restrict__ perm, const u32* __restrict__ flag, const u32* __restrict__ ex,
                             u32 n, u32* __restrict__ id) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  id[perm[i]] = ex[i] + flag[i] - 1;
}

// candidate (xid, block) pairs of block-scope releases
__global__ void k_bpairs(const bc_record* __restrict__ srecs, const u32* __restrict__ lo_sp, const u32* __restrict__ xid,
                         u32 n, Geo g, u32* __restrict__ pk_hi, u32* __restrict__ pk_lo, u32* __restrict__ cnt) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const bc_record& rc = srecs[lo_sp[i]];
  u32 op = rc.op;
  if (op == BC_OP_REL_BLK || op == BC_OP_AR_BLK) {
    u32 at = atomicAdd(cnt, 1u);
    pk_hi[at] = xid[i];
    pk_lo[at] = rc.warp / g.wpb;
  }
}

// compact unique sorted pairs
__global__ void k_compact_pairs(const u32* __restrict__ hi, const u32* __restrict__ lo, const u32* __restrict__ perm,
                                const u32* __restrict__ flag, const u32* __restrict__ ex, u32 n,
                                u32* __restrict__ ohi, u32* __restrict__ olo) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n || !flag[i]) return;
  u32 p = perm[i];
  ohi[ex[i]] = hi[p];
  olo[ex[i]] = lo[p];
}

struct K3In {
  HbCtx hc;
  const bc_record* srecs;  // sync records, trace order
  u32 n_lo;
  const u32 *lo_rec, *lo_lane, *lo_sp, *xid;
  u32 nx, nB;
  const u32 *bp_x, *bp_b;  // unique sorted (xid, block) pairs, bid = index
  const u32* acq_idx_of_rec_sorted;  // unused
  // BC_F_RELEASE_OVERWRITE: the writer lane-ops of each array G_x / B_{x,b}, ascending
  bool ow;
  const u32* wr_pos;    // lane-op indices grouped by array
  const u32* wr_start;  // [nx + nB + 1]
};

__device__ __forceinline__ u32 pair_lower(const K3In& k, u32 x, u32 b) {
  u32 lo = 0, hi = k.nB;
  while (lo < hi) {
    u32 m = (lo + hi) >> 1;
    if (k.bp_x[m] < x || (k.bp_x[m] == x && k.bp_b[m] < b)) lo = m + 1; else hi = m;
  }
  return lo;
}
__device__ __forceinline__ u32 find_bid(const K3In& k, u32 x, u32 b) {
  u32 i = pair_lower(k, x, b);
  return (i < k.nB && k.bp_x[i] == x && k.bp_b[i] == b) ? i : NONE;
}

// index of acquire record r in the (block, rec)-sorted acquire list
__device__ __forceinline__ u32 acq_index(const HbCtx& c, u32 b, u32 r) {
  u32 lo = c.acq_block_start[b], hi = c.acq_block_start[b + 1];
  while (lo < hi) {
    u32 m = (lo + hi) >> 1;
    if (c.acq_rec[m] < r) lo = m + 1; else hi = m;
  }
  return lo;
}

// the latest writer lane-op of array a before lane-op ev (NONE: none)
__device__ __forceinline__ u32 last_writer(const K3In& k, u32 a, u32 ev) {
  u32 lo = k.wr_start[a], hi = k.wr_start[a + 1];
  const u32 base = lo;
  while (lo < hi) {
    u32 m = (lo + hi) >> 1;
    if (k.wr_pos[m] < ev) lo = m + 1; else hi = m;
  }
  return lo > base ? k.wr_pos[lo - 1] : NONE;
}

// Emit (or count, when out == nullptr) the entries of lane-op i.
struct EntOut {
  u32 *arr, *key, *pos, *mask, *clk;
};

__device__ __forceinline__ void put(const EntOut* o, u32& n, u32 arr, u32 key, u32 pos, u32 mask, u32 clk) {
  if (o) {
    o->arr[n] = arr;
    o->key[n] = key;
    o->pos[n] = pos;
    o->mask[n] = mask;
    o->clk[n] = clk;
  }
  ++n;
}

// Overwrite reading (the printed Fig. 3): what lane-op ev acquires from S_x is the content of its slot(s)
// as the latest writers left it -- window links to those writer lane-ops.  S_x[b] was last written by
// the later of G_x's and B_{x,b}'s latest writers; ⊔_b S_x[b] is G_x's latest writer plus every block
// writer after it.
__device__ void prev_links(const K3In& k, const EntOut* o, u32& n, u32 arr, u32 op, u32 x, u32 my_bid, u32 blo, u32 bhi,
                           u32 ev) {
  const u32 gp = last_writer(k, x, ev);
  if (is_glb_op(op)) {
    if (gp != NONE) put(o, n, arr, KEY_LINK | x, ev, LINK_WIN, gp);
    for (u32 j = blo; j < bhi; ++j) {
      const u32 p = last_writer(k, k.nx + j, ev);
      if (p != NONE && (gp == NONE || p > gp)) put(o, n, arr, KEY_LINK | (k.nx + j), ev, LINK_WIN, p);
    }
  } else {
    const u32 bp = my_bid != NONE ? last_writer(k, k.nx + my_bid, ev) : NONE;
    if (bp != NONE && (gp == NONE || bp > gp)) put(o, n, arr, KEY_LINK | (k.nx + my_bid), ev, LINK_WIN, bp);
    else if (gp != NONE) put(o, n, arr, KEY_LINK | x, ev, LINK_WIN, gp);
  }
}

__device__ u32 laneop_entries(const K3In& k, u32 i, const EntOut* o, u32 base) {
  const HbCtx& c = k.hc;
  u32 r = k.lo_rec[i], lane = k.lo_lane[i];
  u32 op = k.srecs[k.lo_sp[i]].op;
  u32 w = k.srecs[k.lo_sp[i]].warp;
  u32 b = w / c.g.wpb;
  u32 x = k.xid[i];
  // position of this lane-op = its rank among the sync lane-ops in trace order (record, then lane):
  // order-preserving, so "entries with pos < bound" is the trace-order view of Fig. 3, and 32 bits
  // suffice for any record count
  u32 ev = i;
  (void)lane;
  u32 n = base;
  // range of block arrays of x
  u32 blo = pair_lower(k, x, 0), bhi = pair_lower(k, x + 1, 0);
  u32 my_bid = find_bid(k, x, b);
  if (is_acq_op(op)) {
    u32 ai = acq_index(c, b, r);
    u32 farr = k.nx + k.nB + ai;
    if (k.ow) {
      prev_links(k, o, n, farr, op, x, my_bid, blo, bhi, ev);
    } else {
      put(o, n, farr, KEY_LINK | x, ev, 0u, ev);  // S_x global part
      if (is_glb_op(op)) {
        for (u32 j = blo; j < bhi; ++j) put(o, n, farr, KEY_LINK | (k.nx + j), ev, 0u, ev);
      } else if (my_bid != NONE) {
        put(o, n, farr, KEY_LINK | (k.nx + my_bid), ev, 0u, ev);
      }
    }
  }
  if (is_rel_op(op)) {
    u32 tarr = is_glb_op(op) ? x : (k.nx + my_bid);
    Snap s = load_snap(c.snap, r);
    // structural clock of the releaser (its block only)
    u32 bl = s.blab;
    if (bl) put(o, n, tarr, KEY_BLOCK | b, ev, 0xFFFFFFFFu, bl);
    if (s.node < c.n_nodes) {
      uint4 nd = c.nodes[s.node];
      if (s.ps) put(o, n, tarr, w, ev, nd.x, s.ps);
      for (int d = 0; d < 40 && nd.y < c.n_nodes; ++d) {
        uint4 pd = c.nodes[nd.y];
        if (nd.z) put(o, n, tarr, w, ev, pd.x, nd.z);
        nd = pd;
      }
    }
    // foreign knowledge: the acquires of this block it structurally knows
    for (u32 j = c.acq_block_start[b]; j < c.acq_block_start[b + 1]; ++j) {
      u32 ra = c.acq_rec[j];
      if (ra >= r) break;
      if (struct_knows(c, c.acq_warp[j], c.acq_lane[j], ra, s)) put(o, n, tarr, KEY_LINK | (k.nx + k.nB + j), ev, 0u, ev);
    }
    // ACQREL: the part of S_x it acquired that lives in another array (overwrite: the slot content
    // it joined before writing, since its own window shows only its own entries)
    if (k.ow) {
      if (op == BC_OP_AR_BLK || op == BC_OP_AR_GLB) prev_links(k, o, n, tarr, op, x, my_bid, blo, bhi, ev);
    } else if (op == BC_OP_AR_BLK) {
      put(o, n, tarr, KEY_LINK | x, ev, 0u, ev);
    } else if (op == BC_OP_AR_GLB) {
      for (u32 j = blo; j < bhi; ++j) put(o, n, tarr, KEY_LINK | (k.nx + j), ev, 0u, ev);
    }
  }
  return n - base;
}

// writer lists (overwrite reading): key = the array a release lane-op writes, or nx + nB for the rest
__global__ void k_wr_keys(K3In k, u32* __restrict__ key, u32* __restrict__ val) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= k.n_lo) return;
  const bc_record& rc = k.srecs[k.lo_sp[i]];
  const u32 op = rc.op;
  u32 a = k.nx + k.nB;
  if (is_rel_op(op)) a = is_glb_op(op) ? k.xid[i] : k.nx + find_bid(k, k.xid[i], rc.warp / k.hc.g.wpb);
  key[i] = a;
  val[i] = i;
}

__global__ void k_ent_count(K3In k, u32* __restrict__ out) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < k.n_lo) out[i] = laneop_entries(k, i, nullptr, 0);
}

__global__ void k_ent_fill(K3In k, const u32* __restrict__ off, EntOut o) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < k.n_lo) laneop_entries(k, i, &o, off[i]);
}

// acquire list: sync records (trace order) that acquire -> keys = block, vals = sync position
__global__ void k_acq_collect(const bc_record* __restrict__ srecs, u32 n, Geo g, u32* __restrict__ akey,
                              u32* __restrict__ aval, const u32* __restrict__ cnt) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  u32 op = srecs[i].op;
  // keep trace order: the slot is the rank among acquires (exclusive scan of the flags)
  if (is_acq_op(op)) {
    u32 at = cnt[i];
    akey[at] = srecs[i].warp / g.wpb;
    aval[at] = i;
  }
}
__global__ void k_acq_flags(const bc_record* __restrict__ srecs, u32 n, u32* __restrict__ flag) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) flag[i] = is_acq_op(srecs[i].op) ? 1u : 0u;
}
// acquire i (sorted by (block, record)): sync position -> global record, warp, a lane active in it
__global__ void k_acq_info(const bc_record* __restrict__ srecs, const u32* __restrict__ sgidx, u32* __restrict__ arec,
                           u32 n, u32* __restrict__ awarp, u32* __restrict__ alane) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const u32 sp = arec[i];
  awarp[i] = srecs[sp].warp;
  alane[i] = __ffs(srecs[sp].mask) - 1;
  arec[i] = sgidx[sp];
}
__global__ void k_block_start(const u32* __restrict__ sorted_blocks, u32 n, u32 n_blocks, u32* __restrict__ start) {
  u32 b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b > n_blocks) return;
  u32 lo = 0, hi = n;
  while (lo < hi) {
    u32 m = (lo + hi) >> 1;
    if (sorted_blocks[m] < b) lo = m + 1; else hi = m;
  }
  start[b] = lo;
}

__global__ void k_gather_u32(const u32* __restrict__ src, const u32* __restrict__ perm, u32 n, u32* __restrict__ dst) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) dst[i] = src[perm[i]];
}
__global__ void k_iota_add(u32* __restrict__ p, u32 n, u32 add) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] = i + add;
}
__global__ void k_iota(u32* __restrict__ p, u32 n) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] = i;
}
__global__ void k_make_ak(const u32* __restrict__ arr, const u32* __restrict__ key, const u32* __restrict__ pos,
                          const u32* __restrict__ mask, const u32* __restrict__ clk, const u32* __restrict__ perm,
                          u32 n, u64* __restrict__ ak, u32* __restrict__ opos, u32* __restrict__ omask,
                          u32* __restrict__ oclk) {
  u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  u32 p = perm[i];
  ak[i] = ((u64)arr[p] << 32) | key[p];
  opos[i] = pos[p];
  omask[i] = mask[p];
  oclk[i] = clk[p];
}

inline unsigned nb(u64 n) { return (unsigned)((n + 255) / 256); }

// compact copy of the sync records: dst[i] = recs[idx[i]] (one warp per record, 272 B)
__global__ void k_gather_records(const bc_record* __restrict__ recs, const u32* __restrict__ idx, u32 n,
                                 bc_record* __restrict__ dst) {
  const u32 i = (u32)(((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5), l = threadIdx.x & 31;
  if (i >= n) return;
  const u32* src = reinterpret_cast<const u32*>(recs + idx[i]);
  u32* d = reinterpret_cast<u32*>(dst + i);
  for (u32 q = l; q < sizeof(bc_record) / 4; q += 32) d[q] = src[q];
}

}  // namespace

// sync_list[0, n) (record indices, any order) -> sorted in place, srecs[i] = recs[sync_list[i]]
void gather_sync_records(const bc_record* recs, u32* sync_list, u32 n, u64 n_recs, bc_record* srecs, Scratch& S,
                         cudaStream_t st) {
  if (n == 0) return;
  u32* k2 = S.alloc<u32>(n);
  void* tmp = S.alloc<char>(rs_temp_bytes(n));
  int b = 0;
  while (b < 32 && (n_recs >> b)) ++b;
  const bool alt = radix_sort_pairs(sync_list, nullptr, k2, nullptr, n, 0, b, tmp, st);
  if (alt) cudaMemcpyAsync(sync_list, k2, (size_t)n * sizeof(u32), cudaMemcpyDeviceToDevice, st);
  k_gather_records<<<(unsigned)(((u64)n * 32 + 255) / 256), 256, 0, st>>>(recs, sync_list, n, srecs);
  ++g_launches;
}

// Sort a permutation `perm` (initially any order) stably by the 32-bit field `f` (bits [0, bits)).
void sort_perm_by(u32* perm, const u32* f, u32 n, int bits, Scratch& S, cudaStream_t st) {
  if (n <= 1) return;
  u32* k = S.alloc<u32>(n);
  u32* k2 = S.alloc<u32>(n);
  u32* p2 = S.alloc<u32>(n);
  void* tmp = S.alloc<char>(rs_temp_bytes(n));
  k_gather_u32<<<nb(n), 256, 0, st>>>(f, perm, n, k); ++g_launches;
  bool alt = radix_sort_pairs(k, perm, k2, p2, n, 0, bits, tmp, st);
  if (alt) cudaMemcpyAsync(perm, p2, n * sizeof(u32), cudaMemcpyDeviceToDevice, st);
}

void launch_iota(u32* p, u32 n, cudaStream_t st) {
  if (n) { k_iota<<<nb(n), 256, 0, st>>>(p, n); ++g_launches; }
}
void launch_gather_u32(const u32* src, const u32* perm, u32 n, u32* dst, cudaStream_t st) {
  if (n) { k_gather_u32<<<nb(n), 256, 0, st>>>(src, perm, n, dst); ++g_launches; }
}

static int bits_for(u64 maxval) {
  int b = 0;
  while (b < 32 && (maxval >> b)) ++b;
  return b;
}

// Runs K3 over the sync records srecs[0, n_srec) (ACQ / REL / AR records, 272 B each, in trace order)
// whose global record indices are sgidx[] (increasing).  Fills the foreign-knowledge fields of `hc`
// (acq_*, idx_*).  Returns 0 or a bc_status.
int run_sync_skeleton(const bc_record* srecs, const u32* sgidx, u32 n_srec, u32 n_lo, u32 n_acq, HbCtx& hc,
                      Scratch& S, cudaStream_t st, u64* n_entries_out) {
  const Geo& g = hc.g;
  *n_entries_out = 0;
  if (n_srec == 0) return 0;
  // 2. acquire list sorted by (block, rec)
  u32* aflag = S.alloc<u32>(n_srec);
  u32* aex = S.alloc<u32>(n_srec);
  u64* tot = S.alloc<u64>(1);
  k_acq_flags<<<nb(n_srec), 256, 0, st>>>(srecs, n_srec, aflag); ++g_launches;
  // (n_acq = the header's count of acquire records: no host round trip for it)
  exclusive_scan_u32(aflag, aex, n_srec, S.alloc<char>(scan_temp_bytes(n_srec)), tot, st);
  u32* acq_blk = S.alloc<u32>(n_acq + 1);
  u32* acq_rec = S.alloc<u32>(n_acq + 1);
  u32* acq_warp = S.alloc<u32>(n_acq + 1);
  u32* acq_lane = S.alloc<u32>(n_acq + 1);
  u32* acq_bstart = S.alloc<u32>(g.n_blocks + 1);
  if (n_acq) {
    k_acq_collect<<<nb(n_srec), 256, 0, st>>>(srecs, n_srec, g, acq_blk, acq_rec, aex); ++g_launches;
    u32* k2 = S.alloc<u32>(n_acq);
    u32* v2 = S.alloc<u32>(n_acq);
    void* tmp = S.alloc<char>(rs_temp_bytes(n_acq));
    bool alt = radix_sort_pairs(acq_blk, acq_rec, k2, v2, n_acq, 0, bits_for(g.n_blocks), tmp, st);
    if (alt) {
      cudaMemcpyAsync(acq_blk, k2, n_acq * 4, cudaMemcpyDeviceToDevice, st);
      cudaMemcpyAsync(acq_rec, v2, n_acq * 4, cudaMemcpyDeviceToDevice, st);
    }
    k_acq_info<<<nb(n_acq), 256, 0, st>>>(srecs, sgidx, acq_rec, n_acq, acq_warp, acq_lane); ++g_launches;
  }
  k_block_start<<<nb(g.n_blocks + 1), 256, 0, st>>>(acq_blk, n_acq, g.n_blocks, acq_bstart); ++g_launches;
  hc.n_acq = n_acq;
  hc.acq_block_start = acq_bstart;
  hc.acq_rec = acq_rec;
  hc.acq_warp = acq_warp;
  hc.acq_lane = acq_lane;

  // 3. lane-ops and dense sync-location ids
  u32* cnt = S.alloc<u32>(n_srec);
  u32* off = S.alloc<u32>(n_srec);
  k_popc_recs<<<nb(n_srec), 256, 0, st>>>(srecs, n_srec, cnt); ++g_launches;
  exclusive_scan_u32(cnt, off, n_srec, S.alloc<char>(scan_temp_bytes(n_srec)), nullptr, st);
  u32* lo_rec = S.alloc<u32>(n_lo);
  u32* lo_lane = S.alloc<u32>(n_lo);
  u32* lo_sp = S.alloc<u32>(n_lo);
  u32* xk_lo = S.alloc<u32>(n_lo);
  u32* xk_hi = S.alloc<u32>(n_lo);
  u32* perm = S.alloc<u32>(n_lo);
  k_laneops<<<nb(n_srec), 256, 0, st>>>(srecs, sgidx, n_srec, off, g, lo_rec, lo_lane, lo_sp, xk_lo, xk_hi, perm,
                                        hc.err);
  ++g_launches;
  sort_perm_by(perm, xk_lo, n_lo, 32, S, st);
  sort_perm_by(perm, xk_hi, n_lo, 32, S, st);
  u32* flag = S.alloc<u32>(n_lo);
  u32* ex = S.alloc<u32>(n_lo);
  u32* xid = S.alloc<u32>(n_lo);
  k_uniq_flags2<<<nb(n_lo), 256, 0, st>>>(xk_hi, xk_lo, perm, n_lo, flag); ++g_launches;
  exclusive_scan_u32(flag, ex, n_lo, S.alloc<char>(scan_temp_bytes(n_lo)), tot, st);
  k_assign_ids<<<nb(n_lo), 256, 0, st>>>(perm, flag, ex, n_lo, xid); ++g_launches;
  u64 nx64 = 0;
  cudaMemcpyAsync(&nx64, tot, 8, cudaMemcpyDeviceToHost, st);
  // 4. block arrays B_{x,b}
  u32* pk_hi = S.alloc<u32>(n_lo);
  u32* pk_lo = S.alloc<u32>(n_lo);
  u32* pcnt = S.alloc<u32>(1);
  cudaMemsetAsync(pcnt, 0, 4, st);
  k_bpairs<<<nb(n_lo), 256, 0, st>>>(srecs, lo_sp, xid, n_lo, g, pk_hi, pk_lo, pcnt); ++g_launches;
  u32 np = 0;
  cudaMemcpyAsync(&np, pcnt, 4, cudaMemcpyDeviceToHost, st);
  if (cudaStreamSynchronize(st) != cudaSuccess) return BC_ERR_CUDA;
  u32 nx = (u32)nx64;
  u32 nB = 0;
  u32* bp_x = S.alloc<u32>(np + 1);
  u32* bp_b = S.alloc<u32>(np + 1);
  if (np) {
    u32* pp = S.alloc<u32>(np);
    launch_iota(pp, np, st);
    sort_perm_by(pp, pk_lo, np, 32, S, st);
    sort_perm_by(pp, pk_hi, np, 32, S, st);
    u32* pf = S.alloc<u32>(np);
    u32* pe = S.alloc<u32>(np);
    k_uniq_flags2<<<nb(np), 256, 0, st>>>(pk_hi, pk_lo, pp, np, pf); ++g_launches;
    exclusive_scan_u32(pf, pe, np, S.alloc<char>(scan_temp_bytes(np)), tot, st);
    k_compact_pairs<<<nb(np), 256, 0, st>>>(pk_hi, pk_lo, pp, pf, pe, np, bp_x, bp_b); ++g_launches;
    u64 nb64 = 0;
    cudaMemcpyAsync(&nb64, tot, 8, cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return BC_ERR_CUDA;
    nB = (u32)nb64;
  }
  if (getenv("BC_DEBUG"))
    fprintf(stderr, "[bc] K3: n_srec=%u n_lo=%u n_acq=%u nx=%u np=%u nB=%u\n", n_srec, n_lo, n_acq, nx, np, nB);
  if ((u64)nx + nB + n_acq >= (1ull << 30)) return BC_ERR_OVERFLOW;
  hc.acq_arr = nullptr;
  // arrF ids are nx + nB + acquire index; expose them for K7
  {
    u32* acq_arr = S.alloc<u32>(n_acq + 1);
    if (n_acq) { k_iota_add<<<nb(n_acq), 256, 0, st>>>(acq_arr, n_acq, nx + nB); ++g_launches; }
    hc.acq_arr = acq_arr;
  }
  // 5. entries
  K3In k;
  k.hc = hc;
  k.srecs = srecs;
  k.lo_sp = lo_sp;
  k.n_lo = n_lo;
  k.lo_rec = lo_rec;
  k.lo_lane = lo_lane;
  k.xid = xid;
  k.nx = nx;
  k.nB = nB;
  k.bp_x = bp_x;
  k.bp_b = bp_b;
  k.acq_idx_of_rec_sorted = nullptr;
  k.ow = (g.flags & BC_F_RELEASE_OVERWRITE) != 0;
  k.wr_pos = nullptr;
  k.wr_start = nullptr;
  if (k.ow) {  // writer lane-ops per array, ascending (stable sort of lane-op order by array)
    u32* wk = S.alloc<u32>(n_lo);
    u32* wv = S.alloc<u32>(n_lo);
    u32* wk2 = S.alloc<u32>(n_lo);
    u32* wv2 = S.alloc<u32>(n_lo);
    u32* wstart = S.alloc<u32>((size_t)nx + nB + 2);
    k_wr_keys<<<nb(n_lo), 256, 0, st>>>(k, wk, wv); ++g_launches;
    const bool alt = radix_sort_pairs(wk, wv, wk2, wv2, n_lo, 0, bits_for((u64)nx + nB), S.alloc<char>(rs_temp_bytes(n_lo)),
                                      st);
    const u32* sk = alt ? wk2 : wk;
    k.wr_pos = alt ? wv2 : wv;
    k_block_start<<<nb((u64)nx + nB + 1), 256, 0, st>>>(sk, n_lo, nx + nB, wstart); ++g_launches;
    k.wr_start = wstart;
  }
  u32* ecnt = S.alloc<u32>(n_lo);
  u32* eoff = S.alloc<u32>(n_lo);
  k_ent_count<<<nb(n_lo), 256, 0, st>>>(k, ecnt); ++g_launches;
  exclusive_scan_u32(ecnt, eoff, n_lo, S.alloc<char>(scan_temp_bytes(n_lo)), tot, st);
  u64 ne64 = 0;
  cudaMemcpyAsync(&ne64, tot, 8, cudaMemcpyDeviceToHost, st);
  if (cudaStreamSynchronize(st) != cudaSuccess) return BC_ERR_CUDA;
  if (getenv("BC_DEBUG")) fprintf(stderr, "[bc] K3: entries=%llu\n", (unsigned long long)ne64);
  if (ne64 >= (1ull << 31)) return BC_ERR_OVERFLOW;
  u32 ne = (u32)ne64;
  *n_entries_out = ne;
  EntOut eo;
  eo.arr = S.alloc<u32>(ne + 1);
  eo.key = S.alloc<u32>(ne + 1);
  eo.pos = S.alloc<u32>(ne + 1);
  eo.mask = S.alloc<u32>(ne + 1);
  eo.clk = S.alloc<u32>(ne + 1);
  k_ent_fill<<<nb(n_lo), 256, 0, st>>>(k, eoff, eo); ++g_launches;
  // 6. index sorted by (arr, key, pos)
  u32* ep = S.alloc<u32>(ne + 1);
  launch_iota(ep, ne, st);
  sort_perm_by(ep, eo.pos, ne, 32, S, st);
  sort_perm_by(ep, eo.key, ne, 32, S, st);
  sort_perm_by(ep, eo.arr, ne, bits_for((u64)nx + nB + n_acq), S, st);
  u64* ak = S.alloc<u64>(ne + 1);
  u32* ipos = S.alloc<u32>(ne + 1);
  u32* imask = S.alloc<u32>(ne + 1);
  u32* iclk = S.alloc<u32>(ne + 1);
  if (ne) { k_make_ak<<<nb(ne), 256, 0, st>>>(eo.arr, eo.key, eo.pos, eo.mask, eo.clk, ep, ne, ak, ipos, imask, iclk); ++g_launches; }
  hc.n_idx = ne;
  hc.e_off = eoff;
  hc.e_cnt = ecnt;
  hc.e_arr = eo.arr;
  hc.e_key = eo.key;
  hc.e_mask = eo.mask;
  hc.e_clk = eo.clk;
  hc.lo_rec = lo_rec;
  hc.f_base = nx + nB;
  hc.idx_ak = ak;
  hc.idx_pos = ipos;
  hc.idx_mask = imask;
  hc.idx_clk = iclk;
  return 0;
}

void preload_sync() {
  preload(k_acq_collect, k_acq_flags, k_acq_info, k_assign_ids, k_block_start, k_bpairs, k_compact_pairs,
          k_ent_count, k_ent_fill, k_gather_records, k_gather_u32, k_iota, k_iota_add, k_laneops, k_make_ak, k_popc_recs,
          k_uniq_flags2, k_wr_keys);
}

}  // namespace bc
