// apps.cuh -- relax policies of the two edge-relax applications.
#pragma once
#include <cooperative_groups.h>

#include "device.cuh"

namespace atos {

// ------------------------------------------------------------------- BFS
// Speculative BFS relax (Alg.2, Listing 4):
//   pop v, d = depth[v]; for each neighbour w: old = atomicMin(depth+w, d+1);
//   if d+1 < old: push w.
// B200 additions:
//   * shadow depth: a u8 copy min(depth, 254) with 255 = "unvisited or >= 255",
//     n bytes (67 MB at scale 26) -- small enough to stay in the 126 MB L2
//     (loads evict_last, the col stream evict_first), so the per-edge
//     prefilter almost never touches HBM.  Written after a successful update;
//     concurrent writers can only leave a value depth[w] once held, so it
//     stays an upper bound and `shadow <= d+1` safely skips the edge;
//   * dedupe (default): the "queued" flag lives in bit 31 of the depth word
//     (word = depth | INQ; 0xFFFFFFFF = unreached).  The activator improves
//     depth and sets INQ in ONE CAS and pushes only if INQ was clear; the
//     popper clears INQ with an acquire RMW that also returns the current
//     depth -- one location, so every improvement after the pop re-queues v
//     and no update is lost, without release fences or a separate bitmap.
//     At termination every queued vertex was popped, so all INQ bits are 0.
//   * two-phase relax (pre: prefilter load, post: decision + atomics) so the
//     engine can keep several edges' loads in flight per thread.
#ifndef ATOS_FUSED_BEGIN
#define ATOS_FUSED_BEGIN 1
#endif
#ifndef ATOS_DEFER_CAS
#define ATOS_DEFER_CAS 1
#endif
constexpr uint32_t kInq = 0x80000000u;
constexpr uint32_t kDepthMask = 0x7FFFFFFFu;

// Partition view (S10).  Queue items, row_ptr and the
// per-vertex state are LOCAL (id - vb); col holds GLOBAL ids.  A neighbour
// outside [vb, vb+nl) is combined into the n-sized ghost array (min for BFS,
// sum for PageRank) and listed once per round in `touched`, to be shipped to
// its owner by the exchange.  ghost == nullptr: single partition, all local.
struct GhostView {
  uint32_t vb, nl;
  void* ghost;
  uint32_t* touched;
  unsigned long long* ntouched;
  __device__ __forceinline__ bool remote_dyn(uint32_t w) const { return ghost != nullptr && (w - vb) >= nl; }
  // warp-aggregated: one atomicAdd on the list counter per group of lanes touching together
  __device__ __forceinline__ void touch(uint32_t w) const {
    namespace cg = cooperative_groups;
    const cg::coalesced_group grp = cg::coalesced_threads();
    unsigned long long base = 0;
    if (grp.thread_rank() == 0) base = atomicAdd(ntouched, (unsigned long long)grp.size());
    base = grp.shfl(base, 0);
    touched[base + grp.thread_rank()] = w;
  }
};

// PART (compile time): partitioned run (ghosts, local ids); false = single
// partition, where every neighbour is local and vb == 0.
// ACQ: acquire pops.  Needed only by the paper-literal mode (dedupe = 0), which
// reads depth[v] with a plain load; the dedupe mode reads it through its RMW.
template <bool PART, bool ACQ = true>
struct BfsAppT {
  static constexpr bool kAcquirePop = ACQ;
  static constexpr bool kPfCta = false;  // CTA workers other than the (256,5) build: direct col loads
  // fused consume + begin (engine.cuh consume_slot_fused): begin() only clears the queued flag / reads the
  // depth, so a speculative begin on a slot lost to a lapping producer can at worst cause a duplicate push
  static constexpr bool kFusedBegin = ATOS_FUSED_BEGIN != 0 && !PART;
  // CAS first (the low-degree PF builds, engine.cuh): no prefilter load -- the CAS guesses "unvisited" and
  // a visited target fails it, returning the word the prefilter would have read.  On a high-diameter graph
  // the prefilter costs one round trip per hop, two past depth 254 (the u8 shadow saturates there and the
  // depth word is read as well).
#ifndef ATOS_CAS_FIRST
#define ATOS_CAS_FIRST 1
#endif
  static constexpr bool kCasFirst = ATOS_CAS_FIRST != 0 && !PART;
  static constexpr uint32_t kBlind = 0xFFFFFFFFu;  // the token that means "no prefilter read"
  using Payload = uint32_t;  // d + 1
  using Token = uint32_t;    // prefilter value (shadow byte, or depth word)
  const uint32_t* __restrict__ row_ptr;
  const uint32_t* __restrict__ col;
  uint32_t* depth;
  int dedupe;         // 0 -> paper-literal push on every improvement (atomicMin)
  uint8_t* shadow;    // nullptr -> prefilter on depth[] itself
  unsigned long long pol_first, pol_last;
  GhostView gv;

  __device__ __forceinline__ bool remote(uint32_t w) const { return PART && gv.remote_dyn(w); }
  __device__ __forceinline__ uint32_t neighbor(uint32_t e) const { return ld_stream(col + e, pol_first); }
  __device__ __forceinline__ void prepare() {
    pol_first = policy_evict_first();
    pol_last = policy_evict_last();
  }

  __device__ __forceinline__ bool begin(uint32_t v, uint32_t& start, uint32_t& deg, Payload& p) const {
    start = __ldg(row_ptr + v);
    const uint32_t end = __ldg(row_ptr + v + 1);
    uint32_t d;
    if (dedupe) d = (ACQ ? atom_and_acquire(depth + v, ~kInq) : atomicAnd(depth + v, ~kInq)) & kDepthMask;
    else d = ld_relaxed(depth + v);  // coherent read (L2): the value that caused the push
    deg = end - start;
    p = d + 1;
    return deg != 0;
  }

  __device__ __forceinline__ Token pre_local(uint32_t lw) const {
    if (shadow) return ld_u8_hint(shadow + lw, pol_last);
    uint32_t cur;
    asm volatile("ld.global.u32 %0, [%1];" : "=r"(cur) : "l"(depth + lw));
    return cur;
  }

  __device__ __forceinline__ Token pre(const Payload nd, uint32_t w) const {
    if (remote(w)) return 0u;
    return pre_local(PART ? w - gv.vb : w);
  }

  // relax local vertex lw with candidate depth nd; true -> enqueue lw
  __device__ __forceinline__ bool relax_local(const Payload nd, uint32_t lw, Token tok, uint32_t& out) const {
    uint32_t expect = 0xFFFFFFFFu;  // guess: unvisited
    if (shadow && tok != kBlind) {
      if (tok != 255u && tok <= nd) return false;
      if (nd >= 255u) {  // shadow carries no information at this depth: prefilter on the word
        asm volatile("ld.global.u32 %0, [%1];" : "=r"(expect) : "l"(depth + lw));
        if (expect != 0xFFFFFFFFu && (expect & kDepthMask) <= nd) return false;
      }
    } else {
      expect = tok;
      if (expect != 0xFFFFFFFFu && (expect & kDepthMask) <= nd) return false;
    }
    bool pushed;
    if (dedupe) {
      while (true) {
        const uint32_t old = atomicCAS(depth + lw, expect, nd | kInq);
        if (old == expect) {
          pushed = (old == 0xFFFFFFFFu) || !(old & kInq);
          break;
        }
        if (old != 0xFFFFFFFFu && (old & kDepthMask) <= nd) return false;
        expect = old;
      }
    } else {
      if (atomicMin(depth + lw, nd) <= nd) return false;
      pushed = true;
    }
    if (shadow) st_u8_hint(shadow + lw, nd < 255u ? nd : 255u, pol_last);
    out = lw;
    return pushed;
  }

  __device__ __forceinline__ bool post(const Payload nd, uint32_t w, Token tok, uint32_t& out) const {
    if (remote(w)) {
      // remote relaxation: min-combine into the ghost, list it on first touch this round
      uint32_t* g = (uint32_t*)gv.ghost + w;
      if (ld_relaxed(g) <= nd) return false;
      if (atomicMin(g, nd) == 0xFFFFFFFFu) gv.touch(w);
      return false;
    }
    return relax_local(nd, PART ? w - gv.vb : w, tok, out);
  }

  __device__ __forceinline__ bool relax(const Payload nd, uint32_t w, uint32_t& out) const {
    return post(nd, w, pre(nd, w), out);
  }
  // an inbound (owner-local) relaxation from the exchange
  __device__ __forceinline__ bool apply(const Payload nd, uint32_t lw, uint32_t& out) const {
    return relax_local(nd, lw, pre_local(lw), out);
  }
};

// ------------------------------------------------------ BFS, byte state
// Byte-state BFS: while depths stay below 126 the
// whole per-vertex state is ONE byte -- bit 7 the queued flag, bits 0-6 the
// depth, 126 = unreached -- so the state of a scale-26 graph is 67 MB and
// stays in the 126 MB L2: the pop-time flag clear, the per-edge prefilter and
// the improving CAS all hit L2 instead of a 268 MB u32 array in HBM.  Same
// protocol as BfsAppT's dedupe mode (one CAS improves the depth and sets the
// flag; the popper clears the flag with an acquire RMW that returns the
// depth), on the aligned 32-bit word that holds the byte.  A pop at depth 125
// cannot relax (126 is not encodable): it raises kStatusDeep and the host
// re-runs the traversal with the u32 state (high-diameter graphs).
constexpr uint32_t kBUnreached = 126u, kBMaxDepth = 125u, kBInq = 0x80u;

template <bool PART>
struct BfsByteAppT {
  // Acquire pops: the slot load must synchronise with the pusher's release so that the
  // popper's AND is ordered after the pusher's CAS on the same word (the PTX model gives no
  // ordering through the address dependency alone); the AND itself can then stay relaxed.
  static constexpr bool kAcquirePop = true;
  static constexpr bool kPfCta = false;
  static constexpr bool kFusedBegin = ATOS_FUSED_BEGIN != 0 && !PART;  // consume_slot_fused (engine.cuh)
  static constexpr bool kDeferCas = ATOS_DEFER_CAS != 0 && !PART;       // post_d / resolve (engine.cuh)
  using Payload = uint32_t;  // d + 1
  using Token = uint32_t;    // the 32-bit word holding w's state byte (prefilter and CAS guess)
  // A lane's deferred discovery CAS: issued in one expand iteration, its result consumed in the next (after
  // that iteration's col loads and state gathers are in flight), so the CAS round trip leaves the chain.
  struct Pend {
    uint32_t res, exp, w, nd;
    bool on;
  };
  const uint32_t* __restrict__ row_ptr;
  const uint32_t* __restrict__ col;
  uint8_t* state;            // n bytes, padded to a multiple of 4
  uint32_t* status;          // queue control block status word
  unsigned long long pol_first, pol_last;
  GhostView gv;              // PART: ghost = n_global bytes, bits 0-6 the best depth sent or pending for the
                             // remote vertex (kBUnreached = none), bit 7 = improved this round (the pack
                             // scans the ghost bytes for it: no list append, no extra atomic in the relax).
                             // The depth survives the pack (only bit 7 is cleared), so a remote vertex is
                             // re-sent only when its depth improves -- the ghost filters across rounds.

  __device__ __forceinline__ uint32_t neighbor(uint32_t e) const { return ld_stream(col + e, pol_first); }
  __device__ __forceinline__ void prepare() {
    pol_first = policy_evict_first();
    pol_last = policy_evict_last();
  }
  __device__ __forceinline__ uint32_t* word_of(uint32_t v) const { return (uint32_t*)(state + (v & ~3u)); }
  __device__ __forceinline__ bool remote(uint32_t w) const { return PART && gv.remote_dyn(w); }
  __device__ __forceinline__ uint32_t* ghost_word(uint32_t w) const {
    return (uint32_t*)((uint8_t*)gv.ghost + (w & ~3u));
  }

  __device__ __forceinline__ bool begin(uint32_t v, uint32_t& start, uint32_t& deg, Payload& p) const {
    start = __ldg(row_ptr + v);
    const uint32_t end = __ldg(row_ptr + v + 1);
    const uint32_t sh = (v & 3u) * 8u;
    // relaxed RMW: the acquire slot load already ordered it after the pusher's CAS
    const uint32_t d = (atomicAnd(word_of(v), ~(kBInq << sh)) >> sh) & 0x7Fu;
    deg = end - start;
    p = d + 1;
    if (deg != 0 && d >= kBMaxDepth) {
      atomicOr(status, kStatusDeep);
      return false;
    }
    return deg != 0;
  }
  __device__ __forceinline__ Token pre(const Payload, uint32_t w) const {
    uint32_t word;
#ifdef ATOS_EXP_SKIP_REMOTE
    if (remote(w)) return 0u;
#endif
    const uint32_t* a = remote(w) ? ghost_word(w) : word_of(PART ? w - gv.vb : w);
    asm volatile("ld.global.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(word) : "l"(a), "l"(pol_last) : "memory");
    return word;
  }
  // A stale word only over-states depths (they only decrease), so skipping on it is safe;
  // the CAS decides everything else.
  __device__ __forceinline__ bool post(const Payload nd, uint32_t w, Token word, uint32_t& out) const {
    if (remote(w)) {
#ifdef ATOS_EXP_SKIP_REMOTE
      return false;
#endif
      // remote relaxation (S10): min-combine into the ghost byte; list w on its first touch this round
      const uint32_t sh = (w & 3u) * 8u;
      uint32_t* gp = ghost_word(w);
      while (true) {
        const uint32_t b = (word >> sh) & 0xFFu;
        if ((b & 0x7Fu) <= nd) return false;  // kBUnreached (126) > every encodable nd
        const uint32_t old = atomicCAS(gp, word, (word & ~(0xFFu << sh)) | ((nd | kBInq) << sh));
        if (old == word) return false;  // bit 7 marks w for the pack's ghost scan (no list append here)
        word = old;
      }
    }
    return relax_local(nd, PART ? w - gv.vb : w, word, out);
  }
  // an inbound (owner-local) relaxation from the exchange
  __device__ __forceinline__ bool apply(const Payload nd, uint32_t lw, uint32_t& out) const {
    uint32_t word;
    asm volatile("ld.global.u32 %0, [%1];" : "=r"(word) : "l"(word_of(lw)) : "memory");
    return relax_local(nd, lw, word, out);
  }
  __device__ __forceinline__ bool relax_local(const Payload nd, uint32_t w, Token word, uint32_t& out) const {
    const uint32_t sh = (w & 3u) * 8u;
    uint32_t* wp = word_of(w);
    while (true) {
      const uint32_t b = (word >> sh) & 0xFFu;
      const uint32_t D = b & 0x7Fu;
      if (D != kBUnreached && D <= nd) return false;
      const uint32_t nw = (word & ~(0xFFu << sh)) | ((nd | kBInq) << sh);
      const uint32_t old = atomicCAS(wp, word, nw);
      if (old == word) {
        out = w;
        return !(b & kBInq);  // queue w unless it is already queued (dedupe)
      }
      word = old;
    }
  }
  __device__ __forceinline__ bool relax(const Payload nd, uint32_t w, uint32_t& out) const {
    return post(nd, w, pre(nd, w), out);
  }
  // post() with the lane's first improving CAS deferred (at most one pending per lane; others run inline)
  __device__ __forceinline__ bool post_d(const Payload nd, uint32_t w, Token word, uint32_t& out, Pend& pd) const {
    if (PART || pd.on) return post(nd, w, word, out);
    const uint32_t sh = (w & 3u) * 8u;
    const uint32_t D = (word >> sh) & 0x7Fu;
    if (D != kBUnreached && D <= nd) return false;
    pd.res = atomicCAS(word_of(w), word, (word & ~(0xFFu << sh)) | ((nd | kBInq) << sh));
    pd.exp = word;
    pd.w = w;
    pd.nd = nd;
    pd.on = true;
    return false;
  }
  // the pending CAS's outcome: won -> queue w unless it was queued; lost -> the ordinary retry loop
  __device__ __forceinline__ bool resolve(Pend& pd, uint32_t& out) const {
    if (!pd.on) return false;
    pd.on = false;
    if (pd.res == pd.exp) {
      out = pd.w;
      return !((pd.exp >> ((pd.w & 3u) * 8u)) & kBInq);
    }
    return relax_local(pd.nd, pd.w, pd.res, out);
  }
};

// -------------------------------------------------------------- PageRank
// Asynchronous push PageRank relax (Alg.4):
//   res = atomicExch(residue+v, 0); atomicAdd(rank+v, res);
//   res = res*lambda/deg(v); for each neighbour: atomicAdd(residue+w, res)
// Activation (DESIGN.md R-PR-6): w is pushed iff its residue crosses eps from
// below (old <= eps < old + delta, evaluated in the same fp64 rounding as the
// atomic), which keeps "residue[v] > eps  =>  v queued or in flight".
// Residue slot of vertex v (single-partition PageRank on a degree-layout graph, rs_log = log2 T > 0): the
// 16T highest-degree vertices are spread as (v mod T) * 16 + v / T so that each of the T hottest owns a whole
// 128-byte line of the f64 residue array -- same-line atomics serialise in the L2 atomic unit -- while the ids
// themselves stay packed by degree (what the BFS byte state wants).  A bijection on [0, n) (16T <= n).
__host__ __device__ __forceinline__ uint32_t res_slot(uint32_t v, uint32_t rs_log) {
  if (rs_log == 0 || v >= (16u << rs_log)) return v;
  return ((v & ((1u << rs_log) - 1u)) << 4) | (v >> rs_log);
}

template <bool PART>
struct PrAppT {
  static constexpr bool kAcquirePop = true;  // atomicExch must follow the pusher's crossing add
#ifndef ATOS_PF_PR
#define ATOS_PF_PR 1
#endif
  static constexpr bool kPfCta = ATOS_PF_PR != 0 && !PART;  // cp.async col prefetch (C3: 65.3 -> 63.6 ms)
  static constexpr bool kFusedBegin = false;  // begin() takes the residue: not speculatable
  using Payload = double;  // delta = alpha * rho / deg(v)
  using Token = double;    // residue before our atomicAdd
  const uint32_t* __restrict__ row_ptr;
  const uint32_t* __restrict__ col;
  unsigned long long pol_first;
  double* rank;
  double* res;
  double alpha, eps;
  int activate;          // 1: crossing activation (default); 0: sweep-only (Check_Size variant)
  uint32_t* dbg_expand;  // debug: per-vertex count of expanding pops
  GhostView gv;
  double defer = 0.0;    // partitioned schedule only: a popped vertex with deg > 32 and residue < defer * deg
                         // keeps its residue (not expanded) until a later, lower threshold re-seeds it
  unsigned long long pol_last = 0;  // single partition: residue atomics evict_last, rank reductions evict_first
  uint32_t rs_log = 0;              // single partition on a degree-layout graph: residue and rank slots (res_slot)

  __device__ __forceinline__ bool remote(uint32_t w) const { return PART && gv.remote_dyn(w); }
  __device__ __forceinline__ uint32_t neighbor(uint32_t e) const { return ld_stream(col + e, pol_first); }
  __device__ __forceinline__ void prepare() {
    pol_first = policy_evict_first();
    pol_last = policy_evict_last();
  }

  __device__ __forceinline__ bool begin(uint32_t v, uint32_t& start, uint32_t& deg, Payload& p) const {
    const double rho = __longlong_as_double(
        (long long)atomicExch((unsigned long long*)(res + (PART ? v : res_slot(v, rs_log))), 0ull));
    start = __ldg(row_ptr + v);
    deg = __ldg(row_ptr + v + 1) - start;
    if (PART && defer > 0.0 && deg > 32 && rho < defer * (double)deg) {
      // hub with too little residue for its edge count: hand it back; re-seeded at a lower threshold
      if (rho != 0.0) red_add_f64(res + v, rho);
      return false;
    }
    if (rho != 0.0) {
      if (!PART)
        asm volatile("red.global.add.L2::cache_hint.f64 [%0], %1, %2;" ::"l"(rank + res_slot(v, rs_log)), "d"(rho),
                     "l"(pol_first)
                     : "memory");
      else
        red_add_f64(rank + v, rho);
    }
    if (deg == 0 || rho == 0.0) return false;  // dangling: absorb (R-PR-3)
    if (dbg_expand) atomicAdd(dbg_expand + v, 1u);
    p = alpha * rho / (double)deg;
    return true;
  }

  __device__ __forceinline__ Token pre(const Payload delta, uint32_t w) const {
    if (remote(w)) return 0.0;
    const uint32_t lw = PART ? w - gv.vb : w;
    if (!PART) {
      // residue atomics keep their lines in L2 (evict_last) against the col stream and the rank reductions
      // (C5: residue 537 MB > L2; 1.24 -> 1.17 s, profiles/r02_ab_pr_l2_hints.txt)
      double old;
      asm volatile("atom.global.add.L2::cache_hint.f64 %0, [%1], %2, %3;"
                   : "=d"(old) : "l"(res + res_slot(lw, rs_log)), "d"(delta), "l"(pol_last) : "memory");
      return old;
    }
    return atomicAdd(res + lw, delta);
  }
  __device__ __forceinline__ bool crossing(const Payload delta, uint32_t lw, Token old, uint32_t& out) const {
    if (activate && old <= eps && old + delta > eps) {
      out = lw;
      return true;
    }
    return false;
  }
  __device__ __forceinline__ bool post(const Payload delta, uint32_t w, Token old, uint32_t& out) const {
    if (remote(w)) {
      // remote mass: sum into the ghost (red, no return); the pack lists non-zero ghosts
      red_add_f64((double*)gv.ghost + w, delta);
      return false;
    }
    return crossing(delta, PART ? w - gv.vb : w, old, out);
  }
  __device__ __forceinline__ bool relax(const Payload delta, uint32_t w, uint32_t& out) const {
    return post(delta, w, pre(delta, w), out);
  }
  __device__ __forceinline__ bool apply(const Payload delta, uint32_t lw, uint32_t& out) const {
    return crossing(delta, lw, atomicAdd(res + lw, delta), out);
  }
};

using BfsByteApp = BfsByteAppT<false>;
using BfsBytePartApp = BfsByteAppT<true>;
using BfsApp = BfsAppT<false>;
using BfsDedupeApp = BfsAppT<false, true>;  // u32 state, dedupe mode (acquire pops, see BfsByteApp)
using BfsPartApp = BfsAppT<true>;
using PrApp = PrAppT<false>;
using PrPartApp = PrAppT<true>;

}  // namespace atos
