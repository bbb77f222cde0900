// bcgen — seeded synthetic trace generators for SURVEY.md §8(d.2) configs C2-C5.
//
// Input fixtures only: this file holds no race-detection arithmetic and is
// shared by the oracle tests and the CUDA path.  It emits traces in the
// paper's 272-byte record format (§4.2) in a global
// interleaving produced by a small scheduler: resident waves of up to
// `max_resident` blocks, seeded round-robin with random bursts across resident
// warps; a warp at BAR waits until every warp of its block has arrived.
//
// Programs (per warp):
//   C2 stencil      1-D 3-point stencil with shared-memory double buffering; injected variant
//                   (inject = 1): in `inj_scale` (default 8) seeded blocks, one iteration's barrier
//                   interval holds an unsynchronised exchange -- warp 0 stores scratch[lane], warp 1
//                   loads scratch[lane] with no barrier between them (the missing BAR of SURVEY §8(d.2))
//   C3 tfr          threadFenceReduction: 40 grid-stride loads, shared tree,
//                   tid0 {st part[b]; AR_GLB count}, last block reduces part[]; injected variant
//                   (inject = 1): block 0 takes its ticket with a plain atomicInc (no fence: an ATOM,
//                   no release), so its part[0] store and its ticket are unordered with the last
//                   block's read of part[0] and its final store count = 0
//   C4 bfs          BFS-like frontier expansion with divergent neighbour loops,
//                   atomics on cost/mask, Zipf(0.8) neighbour ids, injected races
//   C5 scale        C4 shape with 16384 blocks, N = 2^26, 10 nodes/thread and a
//                   BAR after every node iteration
//   C6 hashtable    lock-heavy GPU-TM-style hashtable:
//                   every thread inserts `iters` keys; the lanes of a warp take turns
//                   (IF lane), each locks its bucket (atomicCAS + fence = ACQ_GLB), reads
//                   and writes the bucket head, writes its node, and unlocks (fence +
//                   atomicExch = REL_GLB).  `bug` reproduces the two bugs of §6.3: bit 0 =
//                   CAS without fence (a plain ATOM, no acquire), bit 1 = unlock by a plain
//                   store without fence (ST, no release).  The scheduler keeps the locks
//                   mutually exclusive (an acquire of a held lock waits).
#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <vector>

namespace {

enum Op : uint8_t { LD = 0, ST, ATOM, ACQ_BLK, ACQ_GLB, REL_BLK, REL_GLB, AR_BLK, AR_GLB,
                    FENCE, BAR, IF, ELSE, FI, DYN = 0xEE };
enum Space : uint8_t { GLOBAL = 0, SHARED = 1 };

struct Rec {  // 272 B output record (format: bcgen/format.py)
  uint32_t warp, mask;
  uint8_t op, space, size_log2, flags;
  uint32_t aux;
  uint64_t addr[32];
};
static_assert(sizeof(Rec) == 272, "record layout");

struct CRec {  // compact record: header + an address "role" evaluated at fill time
  uint32_t warp, mask;
  uint8_t op, space, size_log2, flags;
  uint32_t aux;
  uint16_t role, p16;
  uint32_t p32;
  uint64_t p64;
};

static inline uint64_t splitmix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

struct Rng {
  uint64_t s;
  explicit Rng(uint64_t seed) : s(seed) {}
  uint64_t next() { s += 0x9E3779B97F4A7C15ull; return splitmix64(s); }
  uint32_t below(uint32_t n) { return (uint32_t)(next() % n); }
};

constexpr uint64_t GB = 0x7F0000000000ull;  // global base (format.py GLOBAL_BASE)
constexpr uint64_t REGION = 1ull << 34;     // 16 GiB between arrays

enum Role : uint16_t {
  R_NONE = 0,
  // C2
  R2_IN, R2_TILE, R2_HALO_IN, R2_HALO_TILE, R2_OUT,
  // C3
  R3_IN, R3_SD, R3_SD_PLUS, R3_PART, R3_COUNT, R3_AMLAST, R3_PART_READ, R3_RESULT,
  // injected variants of C2 / C3 (ground truth: bcgen_truth_list)
  R2_INJ_ST, R2_INJ_LD, R3_INJ_PART, R3_INJ_COUNT, R3_FINAL_COUNT,
  // C4/C5
  R4_FRONTIER, R4_RP, R4_COL, R4_COST, R4_MASK, R4_INJ_INTER, R4_INJ_BR_ST, R4_INJ_BR_LD,
  R4_INJ_ATM,
  // C6
  R6_KEYS, R6_LOCK, R6_HEAD, R6_NODE,
};

struct Params {
  int32_t config;        // 2..5
  uint32_t n_blocks;     // 0 = config default
  uint32_t tpb;          // 0 = default 256
  uint32_t iters;        // C2 iterations (default 36); C3 loads/thread (default 40)
  uint32_t log2_nodes;   // C4/C5 graph size (0 = default)
  uint32_t nodes_per_thread;
  uint32_t max_resident; // blocks resident at once (0 = 148*8)
  uint32_t inject;       // C4/C5: 1 = inject races (default 1)
  uint32_t inj_scale;    // number of warp pairs per injected kind (0 = default)
  uint32_t deg_lo, deg_hi;
  uint32_t bar_per_node; // C5 style barrier after each node iteration
  uint64_t seed;
  uint32_t bug;          // C6: bit 0 = CAS without fence, bit 1 = unlock by plain store
  uint32_t log2_buckets; // C6: hashtable buckets (0 = default 2^12)
};

struct Gen {
  Params p;
  uint32_t nb, tpb, wpb, nw, nthreads;
  uint32_t smem = 0;
  // C4
  uint32_t N = 0, K = 0;
  std::vector<uint32_t> rowptr;
  double zipf_a = 0, zipf_e = 0;
  // dynamic state
  uint32_t ticket = 0;
  std::vector<uint8_t> is_last;
  std::vector<uint8_t> inj_kind;  // per warp: 0 none, 1 inter, 2 branch, 3 atm-A, 4 atm-L
  std::vector<uint32_t> inj_slot; // per warp: slot index

  std::vector<CRec> out;

  uint32_t init_mask(uint32_t w) const {
    uint32_t wib = w % wpb;
    uint32_t lanes = std::min<uint32_t>(32, tpb - wib * 32);
    return lanes == 32 ? 0xFFFFFFFFu : ((1u << lanes) - 1);
  }
  uint32_t tib(uint32_t w, int lane) const { return (w % wpb) * 32 + lane; }
  uint32_t gtid(uint32_t w, int lane) const { return (w / wpb) * tpb + tib(w, lane); }

  // ------------------------------------------------------------- C4 graph
  uint32_t deg(uint32_t v) const {
    return p.deg_lo + (uint32_t)(splitmix64(p.seed * 31 + v) % (p.deg_hi - p.deg_lo + 1));
  }
  bool frontier(uint32_t v) const { return (splitmix64(p.seed * 131 + v * 7 + 3) >> 17) & 1; }
  uint32_t col(uint64_t e) const {
    // Zipf(0.8) over N via the continuous inverse CDF, then a bijective
    // scatter (odd multiplier mod 2^k) so hot nodes are spread out.
    double u = (double)(splitmix64(p.seed * 977 + e) >> 11) * (1.0 / 9007199254740992.0);
    double r = std::pow(zipf_a * u + 1.0, zipf_e);
    uint64_t rank = (uint64_t)r;
    if (rank < 1) rank = 1;
    if (rank > N) rank = N;
    return (uint32_t)(((rank - 1) * 0x9E3779B1ull) & (N - 1));
  }

  // C6: bucket of the key inserted by thread g in iteration it
  uint32_t bucket(uint32_t g, uint32_t it) const {
    return (uint32_t)(splitmix64(p.seed * 7919 + (uint64_t)g * 64 + it) & ((1u << p.log2_buckets) - 1));
  }

  uint64_t addr(const CRec& c, int lane) const {
    uint32_t w = c.warp, t = tib(w, lane), b = w / wpb, g = gtid(w, lane);
    switch (c.role) {
      case R2_IN: return GB + 4ull * g;
      case R2_TILE: return 4ull * (c.p16 * 258u + t + c.p32);
      case R2_HALO_IN: {
        uint64_t i = (t == 0) ? (uint64_t)b * tpb + nthreads - 1 : (uint64_t)b * tpb + tpb;
        return GB + 4ull * (i % nthreads);
      }
      case R2_HALO_TILE: return 4ull * (c.p16 * 258u + (t == 0 ? 0u : 257u));
      case R2_OUT: return GB + REGION + 4ull * g;
      case R3_IN: return GB + 4ull * ((uint64_t)g + (uint64_t)c.p32 * nthreads);
      case R3_SD: return 4ull * t;
      case R3_SD_PLUS: return 4ull * (t + c.p32);
      case R3_PART: return GB + REGION + 4ull * b;
      case R3_COUNT: return GB + 2 * REGION;
      case R3_AMLAST: return 4ull * tpb;
      case R3_PART_READ: return GB + REGION + 4ull * (t + c.p32 * tpb);
      case R3_RESULT: return GB + 2 * REGION + 64;
      case R2_INJ_ST: case R2_INJ_LD: return 4ull * (2u * 258u + (uint32_t)lane);
      case R3_INJ_PART: return GB + REGION + 4ull * b;
      case R3_INJ_COUNT: case R3_FINAL_COUNT: return GB + 2 * REGION;
      case R4_FRONTIER: return GB + 4ull * ((uint64_t)g + (uint64_t)c.p32 * nthreads);
      case R4_RP: return GB + REGION + 4ull * ((uint64_t)g + (uint64_t)c.p32 * nthreads + c.p16);
      case R4_COL: {
        uint32_t v = g + c.p32 * nthreads;
        return GB + 2 * REGION + 4ull * ((uint64_t)rowptr[v] + c.p16);
      }
      case R4_COST: case R4_MASK: {
        uint32_t v = g + c.p32 * nthreads;
        uint32_t n = col((uint64_t)rowptr[v] + c.p16);
        return GB + (c.role == R4_COST ? 3 : 4) * REGION + 4ull * n;
      }
      case R4_INJ_INTER: return GB + 5 * REGION + 4ull * (32ull * c.p32 + lane);
      case R4_INJ_BR_ST: return GB + 6 * REGION + 4ull * (32ull * c.p32 + lane);
      case R4_INJ_BR_LD: return GB + 6 * REGION + 4ull * (32ull * c.p32 + (lane ^ 1));
      case R4_INJ_ATM: return GB + 7 * REGION + 4ull * (32ull * c.p32 + lane);
      case R6_KEYS: return GB + 4ull * ((uint64_t)g * p.iters + c.p32);
      case R6_LOCK: return GB + REGION + 4ull * bucket(g, c.p32);
      case R6_HEAD: return GB + 2 * REGION + 4ull * bucket(g, c.p32);
      case R6_NODE: return GB + 3 * REGION + 8ull * ((uint64_t)g * p.iters + c.p32);
      default: return 0;
    }
  }

  // ------------------------------------------------------------ programs
  static CRec mk(uint32_t w, uint32_t mask, uint8_t op, uint8_t space = 0, uint16_t role = 0,
                 uint16_t p16 = 0, uint32_t p32 = 0, uint32_t aux = 0, uint8_t flags = 0) {
    CRec c;
    c.warp = w; c.mask = mask; c.op = op; c.space = space; c.size_log2 = 2; c.flags = flags;
    c.aux = aux; c.role = role; c.p16 = p16; c.p32 = p32; c.p64 = 0;
    return c;
  }

  // Branch helper: IF(then) {body} ELSE {} FI with body emitted only if the
  // then-mask is non-empty (an empty path issues no instructions).
  template <class F>
  void branch(std::vector<CRec>& v, uint32_t w, uint32_t top, uint32_t then, F body) {
    then &= top;
    v.push_back(mk(w, top, IF, 0, 0, 0, 0, then));
    if (then) body(then);
    v.push_back(mk(w, then, ELSE));
    v.push_back(mk(w, top & ~then, FI));
  }

  void prog_c2(uint32_t w, std::vector<CRec>& v) {
    uint32_t m = init_mask(w), wib = w % wpb;
    v.push_back(mk(w, m, LD, GLOBAL, R2_IN));
    v.push_back(mk(w, m, ST, SHARED, R2_TILE, 0, 1));
    v.push_back(mk(w, m, ST, SHARED, R2_TILE, 1, 1));
    uint32_t halo = 0;
    if (wib == 0) halo |= 1u;
    if (wib == wpb - 1) halo |= 1u << ((tpb - 1) % 32);
    branch(v, w, m, halo, [&](uint32_t tm) {
      v.push_back(mk(w, tm, LD, GLOBAL, R2_HALO_IN));
      v.push_back(mk(w, tm, ST, SHARED, R2_HALO_TILE, 0));
      v.push_back(mk(w, tm, ST, SHARED, R2_HALO_TILE, 1));
    });
    uint32_t cur = 0;
    const uint32_t b = w / wpb;
    for (uint32_t it = 0; it < p.iters; ++it) {
      v.push_back(mk(w, m, BAR));
      if (inj_kind[w] && it == inj_slot[w]) {  // the unsynchronised exchange of the injected variant
        if (wib == 0) v.push_back(mk(w, m, ST, SHARED, R2_INJ_ST));
        if (wib == 1) v.push_back(mk(w, m, LD, SHARED, R2_INJ_LD));
      }
      for (uint32_t off = 0; off < 3; ++off) v.push_back(mk(w, m, LD, SHARED, R2_TILE, cur, off));
      v.push_back(mk(w, m, ST, SHARED, R2_TILE, cur ^ 1, 1));
      cur ^= 1;
    }
    (void)b;
    v.push_back(mk(w, m, BAR));
    v.push_back(mk(w, m, ST, GLOBAL, R2_OUT));
  }

  uint32_t lanes_below(uint32_t w, uint32_t s) const {  // lanes with tid_in_block < s
    uint32_t base = (w % wpb) * 32, m = init_mask(w);
    if (s <= base) return 0;
    if (s >= base + 32) return m;
    return m & ((1u << (s - base)) - 1);
  }

  void tree(std::vector<CRec>& v, uint32_t w, uint32_t m) {
    for (uint32_t s = tpb / 2; s >= 1; s >>= 1) {
      branch(v, w, m, lanes_below(w, s), [&](uint32_t tm) {
        v.push_back(mk(w, tm, LD, SHARED, R3_SD));
        v.push_back(mk(w, tm, LD, SHARED, R3_SD_PLUS, 0, s));
        v.push_back(mk(w, tm, ST, SHARED, R3_SD));
      });
      v.push_back(mk(w, m, BAR));
    }
  }

  void prog_c3(uint32_t w, std::vector<CRec>& v) {
    uint32_t m = init_mask(w);
    for (uint32_t k = 0; k < p.iters; ++k) v.push_back(mk(w, m, LD, GLOBAL, R3_IN, 0, k));
    v.push_back(mk(w, m, ST, SHARED, R3_SD));
    v.push_back(mk(w, m, BAR));
    tree(v, w, m);
    const bool inj = inj_kind[w] != 0;
    branch(v, w, m, lanes_below(w, 1), [&](uint32_t tm) {
      v.push_back(mk(w, tm, ST, GLOBAL, inj ? R3_INJ_PART : R3_PART));
      if (inj) v.push_back(mk(w, tm, ATOM, GLOBAL, R3_INJ_COUNT));  // atomicInc without the fence
      else v.push_back(mk(w, tm, AR_GLB, GLOBAL, R3_COUNT));        // __threadfence + atomicInc (amb. 12)
      v.push_back(mk(w, tm, ST, SHARED, R3_AMLAST));
    });
    v.push_back(mk(w, m, BAR));
    v.push_back(mk(w, m, LD, SHARED, R3_AMLAST));
    v.push_back(mk(w, m, DYN));
  }

  void prog_c3_tail(uint32_t w, std::vector<CRec>& v) {
    uint32_t m = init_mask(w), b = w / wpb;
    uint32_t then = is_last[b] ? m : 0;
    branch(v, w, m, then, [&](uint32_t tm) {
      for (uint32_t k = 0; k * tpb < nb; ++k) {
        uint32_t lm = lanes_below(w, std::min<uint32_t>(tpb, nb - k * tpb));
        branch(v, w, tm, lm, [&](uint32_t lm2) { v.push_back(mk(w, lm2, LD, GLOBAL, R3_PART_READ, 0, k)); });
      }
      v.push_back(mk(w, tm, ST, SHARED, R3_SD));
      v.push_back(mk(w, tm, BAR));
      tree(v, w, tm);
      branch(v, w, tm, lanes_below(w, 1), [&](uint32_t t0) {
        v.push_back(mk(w, t0, ST, GLOBAL, R3_RESULT));
        v.push_back(mk(w, t0, ST, GLOBAL, R3_FINAL_COUNT));  // plain store count = 0
      });
    });
  }

  void prog_c4(uint32_t w, std::vector<CRec>& v) {
    uint32_t m = init_mask(w);
    for (uint32_t k = 0; k < K; ++k) {
      v.push_back(mk(w, m, LD, GLOBAL, R4_FRONTIER, 0, k));
      uint32_t fm = 0, maxd = 0;
      uint32_t dg[32];
      for (int l = 0; l < 32; ++l) {
        if (!((m >> l) & 1)) continue;
        uint32_t vtx = gtid(w, l) + k * nthreads;
        if (frontier(vtx)) { fm |= 1u << l; dg[l] = deg(vtx); maxd = std::max(maxd, dg[l]); }
      }
      branch(v, w, m, fm, [&](uint32_t tm) {
        v.push_back(mk(w, tm, LD, GLOBAL, R4_RP, 0, k));
        v.push_back(mk(w, tm, LD, GLOBAL, R4_RP, 1, k));
        for (uint32_t j = 0; j < maxd; ++j) {
          uint32_t dm = 0;
          for (int l = 0; l < 32; ++l) if (((tm >> l) & 1) && dg[l] > j) dm |= 1u << l;
          branch(v, w, tm, dm, [&](uint32_t jm) {
            v.push_back(mk(w, jm, LD, GLOBAL, R4_COL, (uint16_t)j, k));
            v.push_back(mk(w, jm, ATOM, GLOBAL, R4_COST, (uint16_t)j, k));
            v.push_back(mk(w, jm, ATOM, GLOBAL, R4_MASK, (uint16_t)j, k));
          });
        }
      });
      if (p.bar_per_node) v.push_back(mk(w, m, BAR));
    }
    switch (inj_kind[w]) {
      case 1: v.push_back(mk(w, m, ST, GLOBAL, R4_INJ_INTER, 0, inj_slot[w])); break;
      case 2: {
        uint32_t even = m & 0x55555555u;
        v.push_back(mk(w, m, IF, 0, 0, 0, 0, even));
        if (even) v.push_back(mk(w, even, ST, GLOBAL, R4_INJ_BR_ST, 0, inj_slot[w]));
        v.push_back(mk(w, even, ELSE));
        if (m & ~even) v.push_back(mk(w, m & ~even, LD, GLOBAL, R4_INJ_BR_LD, 0, inj_slot[w]));
        v.push_back(mk(w, m & ~even, FI));
        break;
      }
      case 3: v.push_back(mk(w, m, ATOM, GLOBAL, R4_INJ_ATM, 0, inj_slot[w])); break;
      case 4: v.push_back(mk(w, m, LD, GLOBAL, R4_INJ_ATM, 0, inj_slot[w])); break;
      default: break;
    }
  }

  void prog_c6(uint32_t w, std::vector<CRec>& v) {
    const uint32_t m = init_mask(w);
    const bool cas_nofence = p.bug & 1u, unlock_plain = p.bug & 2u;
    for (uint32_t it = 0; it < p.iters; ++it) {
      v.push_back(mk(w, m, LD, GLOBAL, R6_KEYS, 0, it));
      for (int l = 0; l < 32; ++l) {  // the lanes take turns: one lock holder per warp at a time
        if (!((m >> l) & 1u)) continue;
        branch(v, w, m, 1u << l, [&](uint32_t tm) {
          v.push_back(mk(w, tm, cas_nofence ? ATOM : ACQ_GLB, GLOBAL, R6_LOCK, (uint16_t)l, it));
          v.push_back(mk(w, tm, LD, GLOBAL, R6_HEAD, (uint16_t)l, it));
          v.push_back(mk(w, tm, ST, GLOBAL, R6_NODE, (uint16_t)l, it));
          v.push_back(mk(w, tm, ST, GLOBAL, R6_HEAD, (uint16_t)l, it));
          v.push_back(mk(w, tm, unlock_plain ? ST : REL_GLB, GLOBAL, R6_LOCK, (uint16_t)(l | 0x100), it));
        });
      }
    }
  }

  void setup() {
    int c = p.config;
    tpb = p.tpb ? p.tpb : 256;
    wpb = (tpb + 31) / 32;
    if (c == 2) {
      nb = p.n_blocks ? p.n_blocks : 256;
      if (!p.iters) p.iters = 36;
      smem = 2 * 258 * 4 + (p.inject ? 32 * 4 : 0);
    } else if (c == 3) {
      nb = p.n_blocks ? p.n_blocks : 4096;
      if (!p.iters) p.iters = 40;
      smem = tpb * 4 + 16;
    } else if (c == 6) {
      tpb = p.tpb ? p.tpb : 128;
      wpb = (tpb + 31) / 32;
      nb = p.n_blocks ? p.n_blocks : 256;
      if (!p.iters) p.iters = 2;
      if (!p.log2_buckets) p.log2_buckets = 12;
      smem = 16;
    } else {
      nb = p.n_blocks ? p.n_blocks : (c == 5 ? 16384 : 4096);
      uint32_t ln = p.log2_nodes ? p.log2_nodes : (c == 5 ? 26 : 24);
      N = 1u << ln;
      K = p.nodes_per_thread ? p.nodes_per_thread : (c == 5 ? 10 : 8);
      if (!p.deg_lo) { p.deg_lo = 8; p.deg_hi = 24; }
      if (c == 5) p.bar_per_node = 1;
      smem = 16;
    }
    nw = nb * wpb;
    nthreads = nb * tpb;
    is_last.assign(nb, 0);
    inj_kind.assign(nw, 0);
    inj_slot.assign(nw, 0);
    if (c == 2 && p.inject && wpb >= 2) {  // warps 0 and 1 of `scale` seeded blocks, one iteration each
      const uint32_t scale = std::min<uint32_t>(p.inj_scale ? p.inj_scale : 8, nb);
      for (uint32_t q = 0; q < scale; ++q) {
        uint32_t blk = (uint32_t)(splitmix64(p.seed * 7 + q) % nb);
        while (inj_kind[blk * wpb]) blk = (blk + 1) % nb;
        const uint32_t it = (uint32_t)(splitmix64(p.seed * 13 + q) % p.iters);
        for (uint32_t i = 0; i < 2; ++i) {
          inj_kind[blk * wpb + i] = 1;
          inj_slot[blk * wpb + i] = it;
        }
      }
    }
    if (c == 3 && p.inject) inj_kind[0] = 1;  // block 0, warp 0 (its tid 0 takes the ticket)
    if (c == 4 || c == 5) {
      if ((uint64_t)nthreads * K > N) { N = 1u; while ((uint64_t)N < (uint64_t)nthreads * K) N <<= 1; }
      rowptr.resize((size_t)N + 1);
      rowptr[0] = 0;
      for (uint32_t v = 0; v < N; ++v) rowptr[v + 1] = rowptr[v] + deg(v);
      double s = 0.8;
      zipf_a = std::pow((double)N, 1.0 - s) - 1.0;
      zipf_e = 1.0 / (1.0 - s);
      if (p.inject) {
        uint32_t scale = p.inj_scale ? p.inj_scale : (c == 5 ? 128 : 32);
        uint32_t n_inter = scale, n_br = 2 * scale, n_atm = std::max<uint32_t>(1, scale / 4);
        auto wsel = [&](uint32_t blk, uint32_t wib) { return (blk % nb) * wpb + (wib % wpb); };
        for (uint32_t q = 0; q < n_inter; ++q) {
          uint32_t b1 = (q * 7) % nb, b2 = (q * 7 + nb / 2 + 1) % nb;
          if (b2 == b1) b2 = (b1 + 1) % nb;
          uint32_t a = wsel(b1, 1), bb = wsel(b2, 1);
          if (nb < 2 || inj_kind[a] || inj_kind[bb]) continue;
          inj_kind[a] = inj_kind[bb] = 1; inj_slot[a] = inj_slot[bb] = q;
        }
        for (uint32_t q = 0; q < n_br; ++q) {
          uint32_t a = wsel((q * 13 + 5) % nb, 2);
          if (inj_kind[a]) continue;
          inj_kind[a] = 2; inj_slot[a] = q;
        }
        for (uint32_t q = 0; q < n_atm; ++q) {
          uint32_t b1 = (q * 11 + 3) % nb, b2 = (q * 11 + 3 + nb / 3 + 1) % nb;
          if (b2 == b1) b2 = (b1 + 1) % nb;
          uint32_t a = wsel(b1, 3), bb = wsel(b2, 3);
          if (nb < 2 || inj_kind[a] || inj_kind[bb]) continue;
          inj_kind[a] = 3; inj_kind[bb] = 4; inj_slot[a] = inj_slot[bb] = q;
        }
      }
    }
  }

  void program(uint32_t w, std::vector<CRec>& v) {
    switch (p.config) {
      case 2: prog_c2(w, v); break;
      case 3: prog_c3(w, v); break;
      case 6: prog_c6(w, v); break;
      default: prog_c4(w, v); break;
    }
  }

  // ----------------------------------------------------------- scheduler
  void schedule() {
    Rng rng(splitmix64(p.seed ^ 0xC0FFEEull) + (uint64_t)p.config);
    uint32_t max_res = p.max_resident ? p.max_resident : 148 * 8;
    std::vector<std::vector<CRec>> prog(nw);
    std::vector<uint32_t> pc(nw, 0);
    std::vector<uint8_t> waiting(nw, 0);
    std::vector<uint32_t> arrived(nb, 0), live(nb, 0);
    std::vector<uint32_t> active;  // resident warps
    std::vector<uint32_t> holder;  // C6: lock holder (warp + 1) per bucket, 0 = free
    if (p.config == 6) holder.assign(1u << p.log2_buckets, 0);
    uint32_t next_block = 0, resident = 0, done_blocks = 0;
    out.clear();
    while (done_blocks < nb) {
      while (resident < max_res && next_block < nb) {
        uint32_t b = next_block++;
        ++resident;
        live[b] = wpb;
        for (uint32_t i = 0; i < wpb; ++i) {
          uint32_t w = b * wpb + i;
          program(w, prog[w]);
          active.push_back(w);
        }
      }
      // one round in a seeded random order
      for (size_t i = active.size(); i > 1; --i) std::swap(active[i - 1], active[rng.below((uint32_t)i)]);
      std::vector<uint32_t> keep;
      keep.reserve(active.size());
      for (uint32_t w : active) {
        uint32_t b = w / wpb;
        if (!waiting[w]) {
          uint32_t burst = 1 + rng.below(3);
          for (uint32_t k = 0; k < burst && pc[w] < prog[w].size(); ++k) {
            if (!holder.empty() && prog[w][pc[w]].role == R6_LOCK) {
              const CRec& lc = prog[w][pc[w]];
              const uint32_t bk = bucket(gtid(w, lc.p16 & 0xFF), lc.p32);
              if (!(lc.p16 & 0x100)) {  // lock: wait while another thread holds the bucket
                if (holder[bk]) break;
                holder[bk] = w + 1;
              } else {
                holder[bk] = 0;
              }
            }
            CRec c = prog[w][pc[w]++];
            if (c.op == DYN) { prog_c3_tail(w, prog[w]); --k; continue; }
            if ((c.op == AR_GLB && c.role == R3_COUNT) || c.role == R3_INJ_COUNT) {
              if (ticket == nb - 1) is_last[b] = 1;
              ++ticket;
            }
            out.push_back(c);
            if (c.op == BAR) {
              waiting[w] = 1;
              if (++arrived[b] == wpb) {
                arrived[b] = 0;
                for (uint32_t j = 0; j < wpb; ++j) waiting[b * wpb + j] = 0;
              }
              break;
            }
          }
        }
        if (pc[w] >= prog[w].size() && !waiting[w]) {
          std::vector<CRec>().swap(prog[w]);
          if (--live[b] == 0) { --resident; ++done_blocks; }
        } else {
          keep.push_back(w);
        }
      }
      active.swap(keep);
    }
  }

  void fill(Rec* dst, uint64_t begin, uint64_t end) const {
    for (uint64_t i = begin; i < end; ++i) {
      const CRec& c = out[i];
      Rec& r = dst[i - begin];  // (dst points at record `begin`)
      r.warp = c.warp; r.mask = c.mask; r.op = c.op; r.space = c.space;
      r.size_log2 = c.size_log2; r.flags = c.flags; r.aux = c.aux;
      bool has_addr = c.op <= AR_GLB;
      for (int l = 0; l < 32; ++l)
        r.addr[l] = (has_addr && ((c.mask >> l) & 1)) ? addr(c, l) : 0;
    }
  }
};

}  // namespace

extern "C" {

struct bcgen_info {
  uint64_t n_records;
  uint32_t grid_x, tpb, smem_bytes, n_truth;
};

struct bcgen_truth {  // one expected race (same 32-B layout as a race record)
  uint64_t addr, prior_event, cur_event;
  uint8_t kind, cls, space, pad;
  uint32_t block;
};

void* bcgen_plan(const Params* p, bcgen_info* info) {
  Gen* g = new Gen();
  g->p = *p;
  g->setup();
  g->schedule();
  info->n_records = g->out.size();
  info->grid_x = g->nb;
  info->tpb = g->tpb;
  info->smem_bytes = g->smem;
  info->n_truth = 0;
  return g;
}

// Fill records [begin, end) into dst (272 B each) using `threads` host threads.
void bcgen_fill(void* h, void* dst, uint64_t begin, uint64_t end, int threads) {
  Gen* g = (Gen*)h;
  if (end > g->out.size()) end = g->out.size();
  if (begin >= end) return;
  if (threads < 1) threads = 1;
  uint64_t n = end - begin, chunk = (n + threads - 1) / threads;
  std::vector<std::thread> ts;
  for (int t = 0; t < threads; ++t) {
    uint64_t b = begin + t * chunk, e = std::min(end, b + chunk);
    if (b >= e) break;
    ts.emplace_back([=] { g->fill((Rec*)dst + (b - begin), b, e); });
  }
  for (auto& t : ts) t.join();
}

// Block shard: the records of the traced blocks b with b % world == rank, in trace
// order, and their global indices.  dst == NULL: only the count.
uint64_t bcgen_fill_shard(void* h, void* dst, uint32_t* idx, uint32_t rank, uint32_t world, int threads) {
  Gen* g = (Gen*)h;
  const uint64_t n = g->out.size();
  if (threads < 1) threads = 1;
  const uint64_t chunk = (n + threads - 1) / threads;
  std::vector<uint64_t> cnt(threads + 1, 0);
  auto mine = [&](uint64_t i) { return (g->out[i].warp / g->wpb) % world == rank; };
  {
    std::vector<std::thread> ts;
    for (int t = 0; t < threads; ++t)
      ts.emplace_back([&, t] {
        uint64_t c = 0;
        for (uint64_t i = t * chunk; i < std::min(n, (t + 1) * chunk); ++i) c += mine(i);
        cnt[t + 1] = c;
      });
    for (auto& t : ts) t.join();
  }
  for (int t = 0; t < threads; ++t) cnt[t + 1] += cnt[t];
  if (!dst) return cnt[threads];
  std::vector<std::thread> ts;
  for (int t = 0; t < threads; ++t)
    ts.emplace_back([&, t] {
      uint64_t o = cnt[t];
      for (uint64_t i = t * chunk; i < std::min(n, (t + 1) * chunk); ++i)
        if (mine(i)) {
          g->fill((Rec*)dst + o, i, i + 1);
          idx[o] = (uint32_t)i;
          ++o;
        }
    });
  for (auto& t : ts) t.join();
  return cnt[threads];
}

// Ground truth for the injected races (C4/C5): every injected granule is
// touched by exactly two conflicting, unsynchronised accesses, so the race is
// (earlier access, later access) by construction.  Returns the count; writes
// up to `cap` entries (unsorted).  Classification: kind from the two access
// types, cls from the two warps/blocks, space GLOBAL.
uint64_t bcgen_truth_list(void* h, bcgen_truth* out, uint64_t cap, uint32_t granule_log2) {
  Gen* g = (Gen*)h;
  struct Acc { uint64_t gran; uint64_t ev; uint8_t type; uint32_t warp; uint8_t space; uint64_t addr; };
  std::vector<Acc> acc;
  auto injected = [&](const CRec& c) {
    if (c.op > ATOM) return false;
    if (c.role >= R4_INJ_INTER && c.role <= R4_INJ_ATM) return true;
    if (c.role == R2_INJ_ST || c.role == R2_INJ_LD) return true;
    // C3: block 0's part store and ticket, every read of part[] by the last block, the final count store
    if (g->p.inject && (c.role == R3_INJ_PART || c.role == R3_INJ_COUNT || c.role == R3_PART_READ ||
                        c.role == R3_FINAL_COUNT)) return true;
    return false;
  };
  for (uint64_t i = 0; i < g->out.size(); ++i) {
    const CRec& c = g->out[i];
    if (!injected(c)) continue;
    for (int l = 0; l < 32; ++l) {
      if (!((c.mask >> l) & 1)) continue;
      uint8_t ty = c.op == LD ? 0 : (c.op == ST ? 1 : 2);
      const uint64_t a = g->addr(c, l);
      // a shared location is (block, offset)
      const uint64_t gran = c.space == SHARED ? (((uint64_t)(c.warp / g->wpb) + 1) << 44) | (a >> granule_log2)
                                              : a >> granule_log2;
      acc.push_back({gran, (i << 5) | (uint64_t)l, ty, c.warp, c.space, (a >> granule_log2) << granule_log2});
    }
  }
  std::stable_sort(acc.begin(), acc.end(), [](const Acc& a, const Acc& b) {
    return a.gran != b.gran ? a.gran < b.gran : a.ev < b.ev;
  });
  uint64_t n = 0;
  for (size_t i = 0; i + 1 < acc.size(); ++i) {
    if (acc[i].gran != acc[i + 1].gran) continue;
    const Acc &a = acc[i], &b = acc[i + 1];
    // kind encoding (format.py): WW WR RW WA AW RA AR
    static const uint8_t kind_tab[3][3] = {{0xFF, 2, 5}, {1, 0, 3}, {6, 4, 0xFF}};
    uint8_t kind = kind_tab[a.type][b.type];
    if (kind == 0xFF) continue;  // two reads / two atomics: not a conflict
    uint8_t cls;
    if ((a.ev >> 5) == (b.ev >> 5)) cls = 0;
    else if (a.warp == b.warp) cls = 1;
    else if (a.warp / g->wpb == b.warp / g->wpb) cls = 2;
    else cls = 3;
    if (n < cap) {
      out[n].addr = a.addr;
      out[n].prior_event = a.ev;
      out[n].cur_event = b.ev;
      out[n].kind = kind; out[n].cls = cls; out[n].space = a.space; out[n].pad = 0;
      out[n].block = a.space == SHARED ? a.warp / g->wpb : b.warp / g->wpb;
    }
    ++n;
  }
  return n;
}

void bcgen_free(void* h) { delete (Gen*)h; }

}  // extern "C"
