// oracle.cpp — TEST INFRASTRUCTURE ONLY.
//
// A plain, slow, single-threaded CPU implementation of the BARRACUDA
// happens-before race check, written from the paper (Eizenberg et al.,
// PLDI'17; /root/reference/PAPER.md, cited below as P:Lnnn).  It interprets a
// trace of warp-level records in trace order with the operational rules of
// Fig. 2 and Fig. 3 on UNCOMPRESSED per-thread vector clocks (one full VC per
// thread, stored sparsely: zero entries omitted).  It exists only to be the
// parity reference for the CUDA path and shares no code, header, table or
// helper with it.  Only tests/, __graft_entry__.smoke() and bench.py's
// cpu_baseline / --impl reference legs may load it.
//
// Readings of garbled or ambiguous passages follow SURVEY.md §8(c.4) and are
// listed in DESIGN.md §"Readings":
//   R1  release joins into S_x (S_x[b] := S_x[b] ⊔ C_t) instead of the printed
//       overwrite; ORACLE_F_RELEASE_OVERWRITE reproduces the printed text.
//   R2  acquire/release ops do not check or update R_x / W_x.
//   R3  the printed atomic rules are kept (atomics never check a previous
//       atomic write).
//   R4  after a failed check the race is reported and the rule's update is
//       applied unchanged (continue after race).
//   R5  lanes of a record are processed in ascending lane order, granules in
//       ascending order; event id = (record index << 5) | lane.
//   R6  SAME_VALUE record flag suppresses write-write races between two lanes
//       of that same record.  R6b: when per-lane
//       store values are supplied (values[record * 32 + lane]), the filter
//       compares them instead of the flag: a write-write race between two lanes
//       of one record is filtered iff the two lanes store the same value.
//   R7  an access of 2^k bytes at a (naturally aligned) address covers the
//       granules [addr >> G, (addr + size - 1) >> G].
//   R8  reported pairs are exactly the failed checks of the rules (FastTrack
//       style), sorted canonically.
//   R9  race class from the two event ids: SAME_INSN, BRANCH, INTRA_BLOCK,
//       INTER_BLOCK.
//   R10 a BAR record is its warp's arrival; bar(b) applies when the last warp
//       of b arrives; a BAR record whose active mask is not the warp's initial
//       mask is a BARRIER_DIVERGENCE finding and the barrier
//       still completes; a warp that issues a record while waiting, or a
//       barrier still incomplete at the end of the trace, is infeasible.
//   R11 shared locations are (block, offset); global locations are addresses.
//   R14 FENCE records are no-ops; warp size 32; x-fastest linearisation.
#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <tuple>
#include <unordered_map>
#include <utility>
#include <vector>

namespace {

// ---- input record (the paper's 272-B queue record) ----------
struct Record {
  uint32_t warp;
  uint32_t mask;
  uint8_t op, space, size_log2, flags;
  uint32_t aux;
  uint64_t addr[32];
};
static_assert(sizeof(Record) == 272, "272-byte record (P:L1070)");

enum Op { LD = 0, ST, ATOM, ACQ_BLK, ACQ_GLB, REL_BLK, REL_GLB, AR_BLK, AR_GLB, FENCE, BAR, IF_,
          ELSE_, FI_ };
enum Space { GLOBAL = 0, SHARED = 1, NOSPACE = 2 };
enum Kind { WW = 0, WR, RW, WA, AW, RA, AR };
enum Cls { SAME_INSN = 0, BRANCH, INTRA_BLOCK, INTER_BLOCK, BARRIER_DIVERGENCE };
constexpr uint32_t F_RELEASE_OVERWRITE = 1u, F_NO_SAME_VALUE_FILTER = 2u, F_CHECK_INVARIANT = 0x100u;
constexpr uint64_t NO_EVENT = ~0ull;
constexpr int MAX_OPEN_IFS = 32;  // format limit, include/bc.h

// ---- vector clocks --------------------------------------------
// A vector clock maps every thread to a timestamp; entries not stored are 0.
struct VC {
  std::vector<std::pair<uint32_t, uint32_t>> e;  // (thread, clock > 0), sorted by thread

  uint32_t get(uint32_t t) const {
    auto it = std::lower_bound(e.begin(), e.end(), std::make_pair(t, 0u));
    return (it != e.end() && it->first == t) ? it->second : 0;
  }
  void set(uint32_t t, uint32_t c) {
    auto it = std::lower_bound(e.begin(), e.end(), std::make_pair(t, 0u));
    if (it != e.end() && it->first == t) {
      if (c) it->second = c; else e.erase(it);
    } else if (c) {
      e.insert(it, {t, c});
    }
  }
  // V ⊔ V' = λt. max(V(t), V'(t))
  void join(const VC& o) {
    std::vector<std::pair<uint32_t, uint32_t>> r;
    r.reserve(e.size() + o.e.size());
    size_t i = 0, j = 0;
    while (i < e.size() || j < o.e.size()) {
      if (j == o.e.size() || (i < e.size() && e[i].first < o.e[j].first)) r.push_back(e[i++]);
      else if (i == e.size() || o.e[j].first < e[i].first) r.push_back(o.e[j++]);
      else { r.push_back({e[i].first, std::max(e[i].second, o.e[j].second)}); ++i; ++j; }
    }
    e.swap(r);
  }
};
// inc_t(V) = λu. if u = t then V(u) + 1 else V(u)
static VC inc(const VC& v, uint32_t t) {
  VC r = v;
  r.set(t, v.get(t) + 1);
  return r;
}

// An epoch c@t, remembering the event that produced it so that
// a failed check can name both racing accesses.  ⊥_e = 0@t0 (no event).
struct Epoch {
  uint32_t c = 0, t = 0;
  uint64_t ev = NO_EVENT;
  bool bottom() const { return ev == NO_EVENT; }
};
// c@t ⪯ V  iff  c <= V(t)
static bool epoch_leq(const Epoch& a, const VC& V) { return a.c <= V.get(a.t); }

// Per-location metadata: W_x = (write epoch, atomic bit),
// R_x = epoch or vector clock.
struct Shadow {
  Epoch W;
  bool W_atomic = false;
  bool R_is_vc = false;
  Epoch R;
  std::map<uint32_t, Epoch> Rvc;  // thread -> (clock, event) when R_x is a VC
};

struct Race {
  uint64_t addr, prior_event, cur_event;
  uint8_t kind, cls, space, pad;
  uint32_t block;
};
static_assert(sizeof(Race) == 32, "race record");

struct LocKey {
  uint8_t space;
  uint32_t block;
  uint64_t granule;
  bool operator==(const LocKey& o) const { return space == o.space && block == o.block && granule == o.granule; }
  bool operator<(const LocKey& o) const {
    return std::tie(space, block, granule) < std::tie(o.space, o.block, o.granule);
  }
};
struct LocHash {
  size_t operator()(const LocKey& k) const {
    uint64_t h = k.granule * 0x9E3779B97F4A7C15ull ^ ((uint64_t)k.block << 8) ^ k.space;
    return (size_t)(h ^ (h >> 29));
  }
};

// ws = warp size: 32, or 4 / 8 / 16 when simulating smaller warps:
// warp w of a block holds threads (w % wpb) * ws ... + ws - 1 of it in lanes 0 .. ws-1.
struct Geom {
  uint32_t n_blocks, tpb, wpb, n_warps, n_threads, G, smem, ws;
  uint32_t init_mask(uint32_t w) const {
    uint32_t lanes = std::min<uint32_t>(ws, tpb - (w % wpb) * ws);
    return lanes == 32 ? 0xFFFFFFFFu : ((1u << lanes) - 1);
  }
  uint32_t block_of_warp(uint32_t w) const { return w / wpb; }
  uint32_t tid(uint32_t w, int lane) const { return (w / wpb) * tpb + (w % wpb) * ws + lane; }
};

enum EntryKind { ROOT, ELSE_ENTRY, THEN_ENTRY };

struct Oracle {
  const Record* recs;
  const uint64_t* values = nullptr;  // R6b: per-lane store values, nullable
  uint64_t n;
  Geom g;
  uint32_t flags;

  std::vector<VC> C;                                   // C_t per thread
  std::vector<std::vector<uint32_t>> K;                // K_w: stack of active masks
  std::vector<std::vector<uint8_t>> Kkind;             // bookkeeping for if/else/fi feasibility
  std::map<LocKey, std::map<uint32_t, VC>> S;          // S_x: block -> VC
  std::unordered_map<LocKey, Shadow, LocHash> shadow;  // R_x, W_x
  std::vector<uint32_t> arrived;                       // per block: warps at the barrier
  std::vector<uint8_t> waiting;                        // per warp
  std::vector<Race> races;
  uint64_t lane_events = 0, control_events = 0;

  // ---------------------------------------------------------------- helpers
  uint32_t tid_block(uint32_t t) const { return t / g.tpb; }

  uint8_t classify(uint64_t prior_ev, uint64_t cur_ev) const {  // P:L1345-1347 (R9)
    uint64_t pr = prior_ev >> 5, cr = cur_ev >> 5;
    if (pr == cr) return SAME_INSN;
    uint32_t pw = recs[pr].warp, cw = recs[cr].warp;
    if (pw == cw) return BRANCH;
    if (g.block_of_warp(pw) == g.block_of_warp(cw)) return INTRA_BLOCK;
    return INTER_BLOCK;
  }

  void report(const LocKey& x, const Epoch& prior, uint64_t ev, uint8_t kind) {
    Race r;
    r.addr = x.granule << g.G;
    r.prior_event = prior.ev;
    r.cur_event = ev;
    r.kind = kind;
    r.cls = classify(prior.ev, ev);
    r.space = x.space;
    r.pad = 0;
    r.block = x.space == SHARED ? x.block : g.block_of_warp(recs[ev >> 5].warp);
    races.push_back(r);
  }

  Epoch E(uint32_t t, uint64_t ev) const {  // E(t) = C_t(t)@t
    Epoch e;
    e.c = C[t].get(t);
    e.t = t;
    e.ev = ev;
    return e;
  }

  // ---- Fig. 2: reads (READSHARED / READEXCL / READINFLATE) ----
  void rd(uint32_t t, const LocKey& x, uint64_t ev) {
    Shadow& s = shadow[x];
    const VC& Ct = C[t];
    if (!epoch_leq(s.W, Ct))  // every read rule requires W_x ⪯ C_t
      report(x, s.W, ev, s.W_atomic ? AR : WR);
    if (s.R_is_vc) {                                   // READSHARED: R' = R_x[t := C_t(t)]
      s.Rvc[t] = E(t, ev);
    } else if (epoch_leq(s.R, Ct)) {                   // READEXCL: R' = E(t)
      s.R = E(t, ev);
    } else {                                           // READINFLATE: ⊥_V[t := C_t(t), t' := clock]
      s.R_is_vc = true;
      s.Rvc.clear();
      s.Rvc[s.R.t] = s.R;
      s.Rvc[t] = E(t, ev);
    }
  }

  // R_x ⪯ C_t (epoch) or R_x ⊑ C_t (vector clock); one race per failing entry.
  void check_reads(Shadow& s, const LocKey& x, uint32_t t, uint64_t ev, uint8_t kind) {
    const VC& Ct = C[t];
    if (!s.R_is_vc) {
      if (!epoch_leq(s.R, Ct)) report(x, s.R, ev, kind);
    } else {
      for (auto& kv : s.Rvc)  // ascending thread order
        if (!(kv.second.c <= Ct.get(kv.first))) report(x, kv.second, ev, kind);
    }
  }

  // ---- Fig. 2: writes (WRITEEXCL / WRITESHARED) ----------------
  void wr(uint32_t t, const LocKey& x, uint64_t ev, bool same_value_rec) {
    Shadow& s = shadow[x];
    if (!epoch_leq(s.W, C[t])) {
      uint8_t kind = s.W_atomic ? AW : WW;
      const bool same_value = values ? values[s.W.ev] == values[ev] : same_value_rec;  // R6 / R6b
      bool filtered = kind == WW && same_value && !(flags & F_NO_SAME_VALUE_FILTER) &&
                      (s.W.ev >> 5) == (ev >> 5);  // intra-warp same-value store
      if (!filtered) report(x, s.W, ev, kind);
    }
    check_reads(s, x, t, ev, RW);
    s.R_is_vc = false;  // R' = R[x := ⊥]
    s.Rvc.clear();
    s.R = Epoch();
    s.W = E(t, ev);     // W' = W[x := (E(t), false)]
    s.W_atomic = false;
  }

  // ---- Fig. 3: atomics (INITATOMEXCL/SHRD, ATOMEXCL/SHARED) ----
  void atm(uint32_t t, const LocKey& x, uint64_t ev) {
    Shadow& s = shadow[x];
    if (!s.W_atomic) {  // INITATOM*: previous write non-atomic, W_x ⪯ C_t checked
      if (!epoch_leq(s.W, C[t])) report(x, s.W, ev, WA);
    }                   // ATOM*: check of the previous atomic write elided
    check_reads(s, x, t, ev, RA);
    s.R_is_vc = false;
    s.Rvc.clear();
    s.R = Epoch();
    s.W = E(t, ev);     // W' = W[x := (E(t), true)]
    s.W_atomic = true;
  }

  // ---- Fig. 3: synchronisation (§3.3.4) ------------
  void release_into(VC& slot, const VC& v) {
    if (flags & F_RELEASE_OVERWRITE) slot = v;  // printed text
    else slot.join(v);                           // reading R1
  }
  void sync_op(uint8_t op, uint32_t t, const LocKey& x) {
    uint32_t b = tid_block(t);
    auto& Sx = S[x];
    switch (op) {
      case ACQ_BLK:  // C' = C[t := C_t ⊔ S_x[block(t)]]
        C[t].join(Sx[b]);
        break;
      case REL_BLK:  // S' = S_x[block(t) := C_t]; C' = C[t := inc_t(C_t)]
        release_into(Sx[b], C[t]);
        C[t] = inc(C[t], t);
        break;
      case AR_BLK: {  // C'_t = C_t ⊔ S_x[block(t)]; S_x[block(t)] := C'_t; C''_t = inc_t(C'_t)
        VC cp = C[t];
        cp.join(Sx[b]);
        release_into(Sx[b], cp);
        C[t] = inc(cp, t);
        break;
      }
      case ACQ_GLB: {  // C' = C[t := C_t ⊔ ⊔_{b ∈ grid} S_x[b]]
        VC vc;
        for (auto& kv : Sx) vc.join(kv.second);
        C[t].join(vc);
        break;
      }
      case REL_GLB: {  // ∀b ∈ grid. S'_x[b] = C_t; C' = C[t := inc_t(C_t)]
        for (uint32_t bb = 0; bb < g.n_blocks; ++bb) release_into(Sx[bb], C[t]);
        C[t] = inc(C[t], t);
        break;
      }
      case AR_GLB: {  // vc = ⊔_b S_x[b]; C' = C_t ⊔ vc; ∀b S'_x[b] = C'; C'' = inc_t(C')
        VC vc;
        for (auto& kv : Sx) vc.join(kv.second);
        VC cp = C[t];
        cp.join(vc);
        for (uint32_t bb = 0; bb < g.n_blocks; ++bb) release_into(Sx[bb], cp);
        C[t] = inc(cp, t);
        break;
      }
    }
  }

  // ---- Fig. 2: ENDINSN / IF / ELSEENDIF; Fig. 3: BAR ----------------------
  // join the given threads, then fork them: ∀t ∈ set. C'_t = inc_t(⊔_{u ∈ set} C_u)
  void join_fork(const std::vector<uint32_t>& ts) {
    if (ts.empty()) return;
    VC vc;
    for (uint32_t t : ts) vc.join(C[t]);
    for (uint32_t t : ts) C[t] = inc(vc, t);
  }
  std::vector<uint32_t> threads_of(uint32_t w, uint32_t mask) const {
    std::vector<uint32_t> v;
    for (int l = 0; l < 32; ++l)
      if ((mask >> l) & 1) v.push_back(g.tid(w, l));
    return v;
  }
  void endinsn(uint32_t w) { join_fork(threads_of(w, K[w].back())); }  // amask = K_w.peek()

  // ---------------------------------------------------------------- driver
  int run() {
    uint32_t nt = g.n_threads;
    C.assign(nt, VC());
    for (uint32_t t = 0; t < nt; ++t) C[t].set(t, 1);  // σ0: C_t = inc_t(⊥_V)
    K.assign(g.n_warps, {});
    Kkind.assign(g.n_warps, {});
    for (uint32_t w = 0; w < g.n_warps; ++w) { K[w].push_back(g.init_mask(w)); Kkind[w].push_back(ROOT); }
    arrived.assign(g.n_blocks, 0);
    waiting.assign(g.n_warps, 0);
    const int INF = -2;

    for (uint64_t r = 0; r < n; ++r) {
      const Record& rec = recs[r];
      uint32_t w = rec.warp;
      if (w >= g.n_warps || rec.op > FI_) return INF;
      if (waiting[w]) return INF;                       // R10
      if (rec.mask & ~g.init_mask(w)) return INF;
      if (rec.mask != K[w].back()) return INF;          // feasibility
      uint32_t b = g.block_of_warp(w);
      uint8_t op = rec.op;
      if (op <= AR_GLB) {
        if (rec.mask == 0 || rec.size_log2 > 4 || rec.space > SHARED) return INF;
        uint64_t size = 1ull << rec.size_log2;
        for (int l = 0; l < 32; ++l) {
          if (!((rec.mask >> l) & 1)) continue;
          uint64_t a = rec.addr[l];
          if (a % size) return INF;                               // natural alignment
          if (rec.space == SHARED && a + size > g.smem) return INF;
        }
        for (int l = 0; l < 32; ++l) {  // ascending lane order (R5)
          if (!((rec.mask >> l) & 1)) continue;
          ++lane_events;
          uint32_t t = g.tid(w, l);
          uint64_t ev = (r << 5) | (uint64_t)l;
          uint64_t a = rec.addr[l];
          if (op <= ATOM) {
            for (uint64_t gr = a >> g.G; gr <= (a + size - 1) >> g.G; ++gr) {
              LocKey x{rec.space, rec.space == SHARED ? b : 0u, gr};
              if (op == LD) rd(t, x, ev);
              else if (op == ST) wr(t, x, ev, rec.flags & 1);
              else atm(t, x, ev);
            }
          } else {
            LocKey x{rec.space, rec.space == SHARED ? b : 0u, a >> g.G};
            sync_op(op, t, x);
          }
        }
        endinsn(w);
      } else {
        ++control_events;
        switch (op) {
          case FENCE:
            if (rec.mask == 0) return INF;
            break;
          case IF_: {
            if (rec.mask == 0 || (rec.aux & ~rec.mask)) return INF;
            int open = 0;  // each open if keeps exactly one else-entry until its fi
            for (uint8_t k : Kkind[w]) open += (k == ELSE_ENTRY);
            if (open >= MAX_OPEN_IFS) return INF;
            uint32_t top = K[w].back();
            uint32_t then = top & rec.aux, els = top & ~rec.aux;  // splitActive
            K[w].push_back(els); Kkind[w].push_back(ELSE_ENTRY);  // else path pushed first
            K[w].push_back(then); Kkind[w].push_back(THEN_ENTRY); // then path runs first
            join_fork(threads_of(w, then));
            break;
          }
          case ELSE_:
            if (Kkind[w].back() != THEN_ENTRY) return INF;
            K[w].pop_back(); Kkind[w].pop_back();
            endinsn(w);  // ELSEENDIF: pop, join and fork the new top
            break;
          case FI_:
            if (Kkind[w].back() != ELSE_ENTRY) return INF;
            K[w].pop_back(); Kkind[w].pop_back();
            endinsn(w);
            break;
          case BAR: {
            if (rec.mask == 0) return INF;
            if (rec.mask != g.init_mask(w)) {  // barrier divergence
              Race d;
              d.addr = 0; d.prior_event = NO_EVENT; d.cur_event = r << 5;
              d.kind = 0xFF; d.cls = BARRIER_DIVERGENCE; d.space = NOSPACE; d.pad = 0; d.block = b;
              races.push_back(d);
            }
            waiting[w] = 1;
            if (++arrived[b] == g.wpb) {  // bar(b): ∀t ∈ b. C'_t = inc_t(⊔_{u ∈ b} C_u)
              arrived[b] = 0;
              std::vector<uint32_t> ts;
              for (uint32_t i = 0; i < g.tpb; ++i) ts.push_back(b * g.tpb + i);
              join_fork(ts);
              for (uint32_t i = 0; i < g.wpb; ++i) waiting[b * g.wpb + i] = 0;
            }
            break;
          }
        }
      }
      if ((flags & F_CHECK_INVARIANT) && !invariant_holds()) return -100;
    }
    for (uint32_t bb = 0; bb < g.n_blocks; ++bb)
      if (arrived[bb]) return INF;  // barrier incomplete at end of trace (R10)
    canonical_sort();
    return 0;
  }

  // FastTrack-style invariant: C_t(t) > C_u(t) for u != t, and
  // R_x(t), W_x(t), S_x(t) <= C_t(t).  Debug mode, tiny traces only.
  bool invariant_holds() const {
    uint32_t nt = g.n_threads;
    for (uint32_t u = 0; u < nt; ++u)
      for (auto& kv : C[u].e)
        if (kv.first != u && !(kv.second < C[kv.first].get(kv.first))) return false;
    for (auto& kv : shadow) {
      const Shadow& s = kv.second;
      if (!s.W.bottom() && s.W.c > C[s.W.t].get(s.W.t)) return false;
      if (!s.R_is_vc && !s.R.bottom() && s.R.c > C[s.R.t].get(s.R.t)) return false;
      for (auto& e : s.Rvc) if (e.second.c > C[e.first].get(e.first)) return false;
    }
    for (auto& kv : S)
      for (auto& bv : kv.second)
        for (auto& e : bv.second.e)
          if (e.second > C[e.first].get(e.first)) return false;
    return true;
  }

  // Canonical order (include/bc.h): (space rank: findings, global, shared;
  // block for shared/findings; addr; cur_event; prior_event).
  void canonical_sort() {
    auto rank = [](uint8_t sp) { return sp == NOSPACE ? 0 : (sp == GLOBAL ? 1 : 2); };
    std::sort(races.begin(), races.end(), [&](const Race& a, const Race& b) {
      uint32_t ba = a.space == GLOBAL ? 0 : a.block, bb = b.space == GLOBAL ? 0 : b.block;
      return std::make_tuple(rank(a.space), ba, a.addr, a.cur_event, a.prior_event) <
             std::make_tuple(rank(b.space), bb, b.addr, b.cur_event, b.prior_event);
    });
  }
};

}  // namespace

extern "C" {

struct oracle_geom {
  uint32_t grid[3], block[3], warp_size, granule_log2, smem_bytes, flags;
};

struct oracle_result {
  void* races;  // Race[n_races], free with oracle_free
  uint64_t n_races, lane_events, control_events;
};

int oracle_detect_values(const void* recs, uint64_t n_recs, const oracle_geom* gm, const uint64_t* values,
                         oracle_result* res);
int oracle_detect(const void* recs, uint64_t n_recs, const oracle_geom* gm, oracle_result* res) {
  return oracle_detect_values(recs, n_recs, gm, nullptr, res);
}

// values: nullable, values[record * 32 + lane] = the value lane `lane` of store record `record`
// writes (R6b); other entries are ignored
int oracle_detect_values(const void* recs, uint64_t n_recs, const oracle_geom* gm, const uint64_t* values,
                         oracle_result* res) {
  if (!gm || !res || (n_recs && !recs)) return -1;
  const uint32_t ws = gm->warp_size;
  if ((ws != 4 && ws != 8 && ws != 16 && ws != 32) || gm->granule_log2 > 4) return -1;
  Oracle o;
  o.recs = (const Record*)recs;
  o.values = values;
  o.n = n_recs;
  o.flags = gm->flags;
  uint64_t nb = (uint64_t)gm->grid[0] * gm->grid[1] * gm->grid[2];
  uint64_t tpb = (uint64_t)gm->block[0] * gm->block[1] * gm->block[2];
  if (nb == 0 || tpb == 0 || tpb > 1024 || nb * tpb > 0xFFFFFFFFull) return -1;
  o.g.n_blocks = (uint32_t)nb;
  o.g.tpb = (uint32_t)tpb;
  o.g.ws = ws;
  o.g.wpb = (uint32_t)((tpb + ws - 1) / ws);
  o.g.n_warps = o.g.n_blocks * o.g.wpb;
  o.g.n_threads = (uint32_t)(nb * tpb);
  o.g.G = gm->granule_log2;
  o.g.smem = gm->smem_bytes;
  int st = o.run();
  res->n_races = 0;
  res->races = nullptr;
  res->lane_events = o.lane_events;
  res->control_events = o.control_events;
  if (st != 0) return st;
  res->n_races = o.races.size();
  if (!o.races.empty()) {
    res->races = std::malloc(o.races.size() * sizeof(Race));
    std::memcpy(res->races, o.races.data(), o.races.size() * sizeof(Race));
  }
  return 0;
}

void oracle_free(void* p) { std::free(p); }

}  // extern "C"
