// common.cuh — device-side types and helpers shared by the sm_100a kernels of libbc.
//
// Nothing here is shared with the oracle (oracle/oracle.cpp); see DESIGN.md "Parity".
//
// Clock representation (DESIGN.md §"Record-index clocks"): every step of a thread (an
// endi / if / else / fi / bar join-fork) is labelled with
// (trace record index + 1).  The labels along one thread's timeline are strictly increasing,
// so "t knows u's step labelled L" is a lossless stand-in for the paper's epoch comparison
// c@u ⪯ C_t: the access of u in record r1 happened before t's current point iff
// know_t(u) >= r1 + 1.  know_t(u) is never materialised as a vector; it is evaluated from
//   - the barrier label of t's block phase (§4.3.2 block max),
//   - the warp's SIMT-stack node chain (the PTVC warp part, Fig. 7),
//   - foreign knowledge through acquire/release views (the SPARSEVC part).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "bc.h"

namespace bc {

typedef uint32_t u32;
typedef uint64_t u64;

constexpr u32 NONE = 0xFFFFFFFFu;
constexpr int WARP = 32;

// error flags (device word) -> bc_status
constexpr u32 ERR_INFEASIBLE = 1u;
constexpr u32 ERR_OVERFLOW = 2u;
constexpr u32 ERR_UNDECLARED = 8u;  // streaming: a global access outside the declared allocations
constexpr u32 ERR_PAGES = 16u;      // K4 met a global write whose page the sampled page set lacks (re-run)

// item op codes (2 low bits of an item's key word)
constexpr u32 IOP_LD = 0, IOP_ST = 1, IOP_ST_SV = 2, IOP_ATOM = 3;
// item key of a dropped slot (never-written global page); removed by the first radix pass
constexpr u32 KEY_DROP = 0xFFFFFFFFu;

// sync-index key space (K3)
constexpr u32 KEY_BLOCK = 0x80000000u;  // block-level entry: key = KEY_BLOCK | block
constexpr u32 KEY_LINK = 0xC0000000u;   // link entry:        key = KEY_LINK | target array
constexpr u32 SYNC_LOOKUP_CAP = 1u << 16;  // step cap of one foreign lookup
// internal Geo.flags bit: per-lane store values are loaded (row f3, reading R6b): every store item
// is a same-value filter candidate and K7 compares the two lanes' values
constexpr u32 GEO_F_VALUES = 0x80000000u;
// internal Geo.flags bit: the global page set is the declared allocations (streaming, row f1)
constexpr u32 GEO_F_DECLARED = 0x40000000u;

struct Geo {
  u32 n_blocks, tpb, wpb, n_warps;
  u32 ws;          // warp size: 32, or 4 / 8 / 16 for warp-size simulation
  u32 wpb_m;       // ceil(2^32 / wpb), 0 when wpb == 1: block of warp w = umulhi(w, wpb_m) (exact: n_warps * wpb < 2^32)
  u32 rank, world; // address sharding: this context checks the granules g with shard_of(g) == rank
  u32 G;           // granule_log2
  u32 smem;        // bytes per block
  u32 smem_gran;   // granules per block
  u32 flags;
  u64 n_recs;
};

// owner rank of dense shadow key k (every rank derives the same dense keys from the same trace):
// a murmur3 finaliser spreads neighbouring granules, then a multiply-shift maps to [0, world)
__device__ __forceinline__ u32 shard_of(u32 k, u32 world) {
  k ^= k >> 16;
  k *= 0x85EBCA6Bu;
  k ^= k >> 13;
  k *= 0xC2B2AE35u;
  k ^= k >> 16;
  return (u32)(((u64)k * world) >> 32);
}

// traced block of traced warp w without an integer division
__device__ __forceinline__ u32 blk_of(const Geo& g, u32 w) { return g.wpb_m ? __umulhi(w, g.wpb_m) : w; }

__host__ __device__ inline u32 init_mask(const Geo& g, u32 w) {
  u32 wib = w % g.wpb;
  u32 lanes = g.tpb - wib * g.ws;
  if (lanes > g.ws) lanes = g.ws;
  return lanes >= 32u ? 0xFFFFFFFFu : ((1u << lanes) - 1u);
}

// 16-byte record header as loaded from the 272-byte record
struct Hdr {
  u32 warp, mask, aux;
  u32 op, space, size_log2, flags;
};
__device__ __forceinline__ Hdr load_hdr(const bc_record* recs, u64 r) {
  uint4 v = __ldg(reinterpret_cast<const uint4*>(recs + r));
  Hdr h;
  h.warp = v.x;
  h.mask = v.y;
  h.op = v.z & 0xFFu;
  h.space = (v.z >> 8) & 0xFFu;
  h.size_log2 = (v.z >> 16) & 0xFFu;
  h.flags = (v.z >> 24) & 0xFFu;
  h.aux = v.w;
  return h;
}

__device__ __forceinline__ void set_err(u32* err, u32 bits) { atomicOr(err, bits); }

__device__ __forceinline__ u32 lanemask_lt() {
  u32 m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// ---------------------------------------------------------------- per-record snapshot
// K2 output, one per record (16 B): the compressed clock of the record's active lanes.
//   warp : traced warp id
//   ps   : label of the warp's last step before this record (0 = none)
//   node : SIMT-stack node the record executes in (its mask == the record's mask); node == warp
//          is the warp's root (converged) node
//   blab : label of the last completed barrier of the block (0 = none); K2 writes the barrier
//          phase here and k_snap_blab replaces it by the label once all warps are replayed
struct Snap {
  u32 warp, ps, node, blab;
};
__device__ __forceinline__ Snap load_snap(const uint4* snap, u32 r) {
  uint4 v = __ldg(snap + r);
  return Snap{v.x, v.y, v.z, v.w};
}
__device__ __forceinline__ Snap to_snap(uint4 v) { return Snap{v.x, v.y, v.z, v.w}; }

// SIMT-stack node (16 B): mask, parent node, popen = label of the warp's last step before the
// IF that opened this node's branch (what the lanes outside it last shared with it).
struct Node {
  u32 mask, parent, popen, pad;
};

// ------------------------------------------------------------ read-only analysis state
// Everything the happens-before query needs; passed by value to K3/K7/K8.
struct HbCtx {
  Geo g;
  const uint4* snap;      // [n_recs]
  const uint4* nodes;     // [n_nodes]
  u32 n_nodes;
  // foreign knowledge (K3); n_acq == 0 => none
  u32 n_acq;
  const u32* acq_block_start;  // [n_blocks + 1] ranges into acq_*
  const u32* acq_rec;          // acquire records sorted by (block, rec)
  const u32* acq_warp;
  const u32* acq_lane;         // a lane active in the acquire record
  const u32* acq_arr;          // its arrF array id
  u32 n_idx;
  const u64* idx_ak;           // (arr << 32 | key), sorted with idx_pos
  const u32* idx_pos;
  const u32* idx_mask;
  const u32* idx_clk;
  // BC_F_RELEASE_OVERWRITE (the printed S_x := C_t): the K3 entries in emission order, lane-op p's at
  // [e_off[p], e_off[p] + e_cnt[p]) -- a window link names one writer lane-op of G_x / B_{x,b}
  const u32* e_off;
  const u32* e_cnt;
  const u32* e_arr;
  const u32* e_key;
  const u32* e_mask;
  const u32* e_clk;
  const u32* lo_rec;  // lane-op -> global record
  u32 f_base;         // acquire views F_a have array ids f_base + a
  u32* err;
};

// know_t(u) for u = lane `ul` of t's own warp, t executing a record with snapshot s (intra-warp
// part only; the PTVC CONVERGED / DIVERGED / NESTEDDIVERGED lookup of Fig. 7).
static __device__ __noinline__ u32 intra_walk(const uint4* __restrict__ nodes, u32 n_nodes, u32 node, u32 ps, u32 ul) {
  if (node >= n_nodes) return 0;  // only after an infeasible replay (result discarded)
  uint4 nd = __ldg(nodes + node);
  if ((nd.x >> ul) & 1u) return ps;
  // walk up the branch tree to the lowest ancestor whose mask holds ul
  for (int d = 0; d < 40; ++d) {
    u32 p = nd.y;
    if (p >= n_nodes) return 0;  // NONE: cannot happen for a valid lane (root mask = init mask)
    uint4 pd = __ldg(nodes + p);
    if ((pd.x >> ul) & 1u) return nd.z;
    nd = pd;
  }
  return 0;
}
__device__ __forceinline__ u32 intra_know(const HbCtx& c, const Snap& s, u32 ul) {
  if (s.node == s.warp) return s.ps;  // converged: every lane of the warp is in the root node
  return intra_walk(c.nodes, c.n_nodes, s.node, s.ps, ul);
}

// structural happens-before: does t (executing record r2 with snapshot s2) know the step of
// (warp w1, lane l1) at record r1?  Same block only; no same-thread shortcut (callers do it).
__device__ __forceinline__ bool struct_knows(const HbCtx& c, u32 w1, u32 l1, u32 r1, const Snap& s2) {
  if (blk_of(c.g, w1) != blk_of(c.g, s2.warp)) return false;
  if (r1 + 1u <= s2.blab) return true;
  if (w1 == s2.warp && intra_know(c, s2, l1) >= r1 + 1u) return true;
  return false;
}

// ------------------------------------------------------- foreign knowledge (K3 output)
// The sync index holds, per array (S_x global part, S_x[b] block part, or an acquire record's
// view), entries sorted by (arr, key, pos):
//   key = KEY_BLOCK|b : the releaser knew all of block b up to label clk
//   key = warp w      : the releaser knew lanes `mask` of warp w up to label clk
//   key = KEY_LINK|a  : the releaser / acquirer also knew array a's entries with pos < clk
// pos = (record << 5 | lane) of the release that appended the entry; a view (arr, bound)
// sees the entries with pos < bound (S_x as it stood when the acquire ran, Fig. 3).
__device__ __forceinline__ u32 idx_lower_bound(const HbCtx& c, u64 ak) {
  u32 lo = 0, hi = c.n_idx;
  while (lo < hi) {
    u32 mid = (lo + hi) >> 1;
    if (c.idx_ak[mid] < ak) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// does view (arr, bound) know the step of (warp uw, lane ul) at record r1?  Depth-first over
// the link DAG; an array already visited with a bound >= the new one is skipped (its entries
// are a superset), which keeps chains of releases linear.
static __device__ __noinline__ bool view_knows(const HbCtx c, u32 uw, u32 ul, u32 r1, u32 arr, u32 bound) {
  constexpr int STK = 256, VIS = 256;
  u32 st_arr[STK], st_bd[STK];
  u32 vis_arr[VIS], vis_bd[VIS];
  int sp = 0, nv = 0;
  st_arr[sp] = arr;
  st_bd[sp++] = bound;
  u32 steps = 0;
  const u32 need = r1 + 1u;
  const u32 ub = uw / c.g.wpb;
  while (sp > 0) {
    --sp;
    const u32 a = st_arr[sp], bd = st_bd[sp];
    bool skip = false;
    for (int q = 0; q < nv; ++q)
      if (vis_arr[q] == a) {
        if (vis_bd[q] >= bd) skip = true; else vis_bd[q] = bd;
        break;
      }
    if (skip) continue;
    if (nv < VIS) {
      bool found = false;
      for (int q = 0; q < nv; ++q) found |= vis_arr[q] == a;
      if (!found) { vis_arr[nv] = a; vis_bd[nv++] = bd; }
    }
    if (++steps > SYNC_LOOKUP_CAP) {
      set_err(c.err, ERR_OVERFLOW);
      return false;
    }
    // once any lookup has overflowed the whole detect fails (BC_ERR_OVERFLOW): stop early instead of
    // finishing every other long walk (lock-heavy traces)
    if ((steps & 255u) == 0u && (*(volatile u32*)c.err & ERR_OVERFLOW)) return false;
    // block-level entries
    u64 ak = ((u64)a << 32) | (KEY_BLOCK | ub);
    for (u32 i = idx_lower_bound(c, ak); i < c.n_idx && c.idx_ak[i] == ak && c.idx_pos[i] < bd; ++i)
      if (c.idx_clk[i] >= need) return true;
    // warp-level entries
    ak = ((u64)a << 32) | uw;
    for (u32 i = idx_lower_bound(c, ak); i < c.n_idx && c.idx_ak[i] == ak && c.idx_pos[i] < bd; ++i)
      if (((c.idx_mask[i] >> ul) & 1u) && c.idx_clk[i] >= need) return true;
    // links: per target, the last entry with pos < bd carries the largest bound
    u64 lk = ((u64)a << 32) | KEY_LINK;
    u64 end = ((u64)a << 32) | 0xFFFFFFFFull;
    u32 i = idx_lower_bound(c, lk);
    while (i < c.n_idx && c.idx_ak[i] <= end) {
      u64 key = c.idx_ak[i];
      u32 best = 0;
      bool any = false;
      for (; i < c.n_idx && c.idx_ak[i] == key; ++i)
        if (c.idx_pos[i] < bd) {
          u32 b2 = c.idx_clk[i] < bd ? c.idx_clk[i] : bd;
          if (!any || b2 > best) best = b2;
          any = true;
        }
      if (any) {
        u32 tgt = (u32)(key & 0x3FFFFFFFull);
        bool seen = false;
        for (int q = 0; q < nv; ++q)
          if (vis_arr[q] == tgt && vis_bd[q] >= best) seen = true;
        // already waiting on the stack: keep one entry with the larger bound (lock chains reach the
        // same views along many paths)
        for (int q = 0; q < sp && !seen; ++q)
          if (st_arr[q] == tgt) {
            if (st_bd[q] < best) st_bd[q] = best;
            seen = true;
          }
        if (seen) continue;
        if (sp >= STK) {
          set_err(c.err, ERR_OVERFLOW);
          return false;
        }
        st_arr[sp] = tgt;
        st_bd[sp++] = best;
      }
    }
  }
  return false;
}

// The same question under BC_F_RELEASE_OVERWRITE.  There, S_x[b] holds only what its latest writer
// put there (an ACQREL writer joins the previous content first, Fig. 3), so K3 links an
// acquire (and an ACQREL's release) to a *window*: the entries of exactly one writer lane-op p
// (link mask LINK_WIN, clk = p), read in emission order.  An acquire's own view F_a is still reached
// as a prefix (entries with pos < bound).  Stack items: (array | WIN_BIT, lane-op) or (array, bound).
constexpr u32 LINK_WIN = 1u;
constexpr u32 WIN_BIT = 0x80000000u;
static __device__ __noinline__ bool view_knows_ow(const HbCtx c, u32 uw, u32 ul, u32 r1, u32 arr, u32 bound) {
  constexpr int STK = 256, VIS = 256;
  u32 st_a[STK], st_v[STK];
  u32 vis_a[VIS], vis_v[VIS];
  int sp = 0, nv = 0;
  st_a[sp] = arr;
  st_v[sp++] = bound;
  u32 steps = 0;
  const u32 need = r1 + 1u;
  const u32 kb = KEY_BLOCK | (uw / c.g.wpb);
  bool ovf = false;
  // push a link target unless an item that sees at least as much is already visited or waiting
  auto push = [&](u32 a, u32 v) {
    const bool win = a & WIN_BIT;
    for (int q = 0; q < nv; ++q)
      if (vis_a[q] == a && (win ? vis_v[q] == v : vis_v[q] >= v)) return;
    for (int q = 0; q < sp; ++q)
      if (st_a[q] == a) {
        if (win) {
          if (st_v[q] == v) return;
        } else {
          if (st_v[q] < v) st_v[q] = v;
          return;
        }
      }
    if (sp >= STK) {
      ovf = true;
      return;
    }
    st_a[sp] = a;
    st_v[sp++] = v;
  };
  // Everything reachable from a writer window or an acquire view happened before that writer's /
  // acquirer's record, so one older than r1 cannot know the step at r1: not pushed.
  auto link = [&](u32 key, u32 mask, u32 clk, u32 cap) {
    const u32 tgt = key & 0x3FFFFFFFu;
    if (mask == LINK_WIN) {
      if (c.lo_rec[clk] > r1) push(tgt | WIN_BIT, clk);
    } else if (tgt < c.f_base || c.acq_rec[tgt - c.f_base] > r1) {
      push(tgt, clk < cap ? clk : cap);
    }
  };
  while (sp > 0) {
    --sp;
    const u32 a = st_a[sp], v = st_v[sp];
    const bool win = a & WIN_BIT;
    bool skip = false, found = false;
    for (int q = 0; q < nv; ++q) {
      if (vis_a[q] != a) continue;
      if (win) {
        if (vis_v[q] == v) {
          skip = true;
          break;
        }
      } else {  // one visited record per prefix array, with the largest bound walked so far
        found = true;
        if (vis_v[q] >= v) skip = true;
        else vis_v[q] = v;
        break;
      }
    }
    if (skip) continue;
    if (!found && nv < VIS) {
      vis_a[nv] = a;
      vis_v[nv++] = v;
    }
    if (++steps > SYNC_LOOKUP_CAP || ovf) {
      set_err(c.err, ERR_OVERFLOW);
      return false;
    }
    if (win) {  // the entries writer lane-op v put into array a
      const u32 aid = a & ~WIN_BIT, e0 = c.e_off[v], e1 = e0 + c.e_cnt[v];
      for (u32 e = e0; e < e1; ++e) {
        if (c.e_arr[e] != aid) continue;
        const u32 key = c.e_key[e], top = key & KEY_LINK;
        if (top == KEY_LINK) link(key, c.e_mask[e], c.e_clk[e], NONE);
        else if (key == kb) {
          if (c.e_clk[e] >= need) return true;
        } else if (top == 0 && key == uw) {
          if (((c.e_mask[e] >> ul) & 1u) && c.e_clk[e] >= need) return true;
        }
      }
    } else {  // prefix view of array a: entries with pos < v
      u64 ak = ((u64)a << 32) | kb;
      for (u32 i = idx_lower_bound(c, ak); i < c.n_idx && c.idx_ak[i] == ak && c.idx_pos[i] < v; ++i)
        if (c.idx_clk[i] >= need) return true;
      ak = ((u64)a << 32) | uw;
      for (u32 i = idx_lower_bound(c, ak); i < c.n_idx && c.idx_ak[i] == ak && c.idx_pos[i] < v; ++i)
        if (((c.idx_mask[i] >> ul) & 1u) && c.idx_clk[i] >= need) return true;
      const u64 end = ((u64)a << 32) | 0xFFFFFFFFull;
      for (u32 i = idx_lower_bound(c, ((u64)a << 32) | KEY_LINK); i < c.n_idx && c.idx_ak[i] <= end; ++i)
        if (c.idx_pos[i] < v) link((u32)c.idx_ak[i], c.idx_mask[i], c.idx_clk[i], v);
    }
  }
  if (ovf) set_err(c.err, ERR_OVERFLOW);
  return false;
}

// foreign part of know_t(u) >= r1+1 for t executing record r2 (snapshot s2): through the
// views of the acquires of t's block that t structurally knows (every release->acquire path
// into t's block ends at one of them).
// The acquires are tried newest first: in lock-based code the acquire that orders an access is almost
// always the latest one t knows (the critical section it is in), and its view holds the previous
// holder's release directly -- an oldest-first search would walk the views of every earlier critical
// section of the block first (the lock-heavy programs of SURVEY row f2).
static __device__ __noinline__ bool foreign_knows(const HbCtx c, u32 w1, u32 l1, u32 r1, u32 r2, const Snap s2) {
  u32 b2 = s2.warp / c.g.wpb;
  u32 lo = c.acq_block_start[b2], hi = c.acq_block_start[b2 + 1];
  while (lo < hi) {  // first acquire of the block at or after r2
    const u32 m = (lo + hi) >> 1;
    if (c.acq_rec[m] < r2) lo = m + 1; else hi = m;
  }
  for (u32 i = lo; i-- > c.acq_block_start[b2];) {
    const u32 ra = c.acq_rec[i];
    if (ra < r1) break;  // an acquire before the access cannot order it (view entries are older than ra)
    if (!struct_knows(c, c.acq_warp[i], c.acq_lane[i], ra, s2)) continue;
    if ((c.g.flags & BC_F_RELEASE_OVERWRITE) ? view_knows_ow(c, w1, l1, r1, c.acq_arr[i], NONE)
                                             : view_knows(c, w1, l1, r1, c.acq_arr[i], NONE))
      return true;
  }
  return false;
}

// e1 = (record r1, lane l1, warp w1) happened before e2 = (record r2, lane l2, snapshot s2)?
// r1 <= r2 in trace order.
__device__ __forceinline__ bool hb(const HbCtx& c, u32 r1, u32 l1, u32 w1, u32 r2, u32 l2, const Snap& s2) {
  if (r1 == r2) return l1 == l2;               // lanes of one instruction are concurrent
  if (w1 == s2.warp && l1 == l2) return true;  // same thread: program order
  if (struct_knows(c, w1, l1, r1, s2)) return true;
  if (c.n_acq == 0) return false;
  u32 b2 = s2.warp / c.g.wpb;
  if (c.acq_block_start[b2] == c.acq_block_start[b2 + 1]) return false;
  return foreign_knows(c, w1, l1, r1, r2, s2);
}

// ------------------------------------------------------------------ warp primitives
template <typename T>
__device__ __forceinline__ T warp_incl_sum(T v) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T n = __shfl_up_sync(0xFFFFFFFFu, v, o);
    if ((threadIdx.x & 31) >= o) v += n;
  }
  return v;
}

// ------------------------------------------------ TMA 1-D bulk copies + mbarriers (sm_90+)
__device__ __forceinline__ u32 smem_u32(const void* p) { return (u32)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(u64* bar, u32 count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(u64* bar, u32 bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, u32 bytes, u64* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(u64* bar, u32 phase) {
  u32 done = 0;
  while (!done) {
    asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
                 : "=r"(done) : "r"(smem_u32(bar)), "r"(phase) : "memory");
  }
}

}  // namespace bc
