// engine.cuh -- the Atos worker loop (Listing 2) for edge-relax apps
// (BFS, PageRank), B200-first.
//
// One kernel template covers the paper's design space (Sec.3):
//   * kernel strategy: PERSIST=true  -> persistent kernel, CTAs loop on the
//                                       shared queue until global termination;
//                      PERSIST=false -> discrete kernel over one frontier
//                                       [h0, t0) of the same ring;
//   * worker size:     MODE_CTA    -> the whole CTA is one worker; the fetched
//                                     vertices' edges are flattened with a
//                                     block scan and redistributed to threads
//                                     (load-balancing search, P:459-468,
//                                     P:877-884);
//                      MODE_WARP   -> a warp is one worker and strides one
//                                     vertex's neighbours at a time (Listing 4
//                                     BFSWarp);
//                      MODE_THREAD -> each thread is a worker, walking its own
//                                     vertices' rows serially;
//   * FETCH_SIZE: items claimed by one worker per pop.
//
// App interface (all __device__, const):
//   using Payload = ...;
//   bool begin(uint32_t item, uint32_t& start, uint32_t& deg, Payload& p);
//        called once per consumed item by the consuming thread; false -> no
//        edges to relax (task still counts as done);
//   bool relax(const Payload& p, uint32_t w, uint32_t& out);
//        one neighbour; true -> enqueue `out`;
//   const uint32_t* col;  (neighbour array)
//   bool sweep(...) hooks are app-specific and live in the app files.
#pragma once
#include <type_traits>

#include "device.cuh"

namespace atos {

enum { MODE_CTA = 0, MODE_WARP = 1, MODE_THREAD = 2 };
#ifndef ATOS_KU
#define ATOS_KU 4
#endif
constexpr int kU = ATOS_KU;  // edges in flight per thread per expand iteration
constexpr uint32_t kCown = 2048;  // CTA mode: per-batch owner table of 32*kU-edge chunks
#ifndef ATOS_MINB
#define ATOS_MINB 1
#endif
#ifndef ATOS_MIN_CLAIM
#define ATOS_MIN_CLAIM 16
#endif
constexpr unsigned long long kMinClaim = ATOS_MIN_CLAIM;  // smallest fair-share claim (items)
#ifndef ATOS_BACKOFF_MAX
#define ATOS_BACKOFF_MAX 1024  // idle poll backoff cap (ns)
#endif

// ------------------------------------------------------------ big-task assist
// A popped vertex whose degree exceeds big_threshold is not expanded by the
// worker that popped it: it is registered in a small global table and its
// edge list is split into big_chunk-edge chunks that ANY worker claims with
// one atomicAdd -- busy workers check the table before fetching new items and
// idle workers are sent there first.  This extends the paper's CTA-internal
// data-parallel balancing across CTAs for hubs, which otherwise
// pin one worker for milliseconds on scale-free graphs.  The
// popped item counts as done only when its last chunk finishes, so the
// queue's termination rule is unchanged.  (DESIGN.md "Big-task assist".)
struct __align__(64) BigTask {
  unsigned long long ctr;      // gen:24 | nchunks:20 | next:20 -- one word, so a claim's validity
                               // (next < nchunks of the same generation) comes from ONE atomic
  unsigned long long payload;  // Payload bits
  uint32_t state;              // 0 free, 1 filling, 2 active (gates registration; a hint for claimers)
  uint32_t start, deg, chunk, finished;
  uint32_t pad[9];
};
constexpr uint32_t kBigNextBits = 20, kBigChunkBits = 20;

// Debug edge counters (build with -DATOS_DEBUG_COUNTS; runtime-enabled by ATOS_DEBUG_EDGES).
#ifdef ATOS_DEBUG_COUNTS
#define ATOS_DBG_EDGE(P, e) \
  do {                      \
    if ((P).dbg_edge) atomicAdd((P).dbg_edge + (e), 1u); \
  } while (0)
#else
#define ATOS_DBG_EDGE(P, e) \
  do {                      \
  } while (0)
#endif
// Phase profile (tools only: build with -DATOS_PHASE_PROF): thread 0 of each CTA
// worker accumulates clock64() per phase of the batch loop; the host prints the
// totals after the launch when ATOS_PHASE is set.
#ifdef ATOS_PHASE_PROF
enum { PH_BIG = 0, PH_CLAIM, PH_GATHER, PH_IDLE, PH_BEGIN, PH_SCAN, PH_EXPAND, PH_COMPLETE, PH_NB_LO, PH_NB_HI,
       PH_EXP_LO, PH_EXP_HI, PH_EDGES_LO, PH_EDGES_HI, PH_N };
static __device__ unsigned long long g_phase[PH_N];
#define ATOS_PH_DECL unsigned long long ph_last, ph_acc[PH_N];
#define ATOS_PH(i)                                                   \
  do {                                                               \
    if (threadIdx.x == 0) {                                          \
      const unsigned long long _n = clock64();                       \
      ph_acc[i] += _n - ph_last;                                     \
      ph_last = _n;                                                  \
    }                                                                \
  } while (0)
#define ATOS_PH_FLUSH()                                                  \
  do {                                                                   \
    if (threadIdx.x == 0)                                                \
      for (int _i = 0; _i < PH_N; ++_i) atomicAdd(&g_phase[_i], ph_acc[_i]); \
  } while (0)
#else
#define ATOS_PH_DECL
#define ATOS_PH(i) do {} while (0)
#define ATOS_PH_FLUSH() do {} while (0)
#endif

__host__ __device__ constexpr unsigned long long big_pack(uint32_t gen, uint32_t nchunks, uint32_t next) {
  return ((unsigned long long)(gen & 0xFFFFFFu) << 40) | ((unsigned long long)nchunks << 20) | next;
}
__host__ __device__ constexpr uint32_t big_gen(unsigned long long c) { return (uint32_t)(c >> 40); }
__host__ __device__ constexpr uint32_t big_nchunks(unsigned long long c) { return (uint32_t)(c >> 20) & 0xFFFFFu; }
__host__ __device__ constexpr uint32_t big_next(unsigned long long c) { return (uint32_t)c & 0xFFFFFu; }

struct EngineParams {
  Ring q;
  uint32_t fetch;                   // items per claim per worker (per lane for THREAD)
  unsigned long long watchdog_ns;   // spin budget before the watchdog trips
  unsigned long long h0, t0;        // discrete mode: the frontier [h0, t0)
  BigTask* big;                     // nullptr: no assist
  uint32_t nbig, big_threshold, big_chunk;
  unsigned long long* tl;           // progress timeline (nullptr: off)
  uint32_t tl_cap, tl_interval_ns;
  unsigned long long timeout_ns;    // cfg.timeout_s as a device deadline (0: none) -- catches livelock
  uint32_t* dbg_edge;               // debug (ATOS_DEBUG_EDGES): per-edge relaxation counts
  uint32_t* dbg_claim;              // debug: last gen that claimed (slot, chunk), 64 x 4096
  uint32_t min_claim = kMinClaim;   // smallest fair-share claim (items); the host sets it per app
};

// Progress sample (globaltimer, done, tail, head) at most every tl_interval_ns,
// taken by whichever worker first notices the sampling time has passed.
__device__ __forceinline__ void tl_sample(const EngineParams& P) {
  if (!P.tl) return;
  QueueCtl* c = P.q.ctl;
  const unsigned long long now = globaltimer();
  const unsigned long long nxt = ld_relaxed(&c->tl_next.v);
  if (now < nxt) return;
  if (atomicCAS(&c->tl_next.v, nxt, now + P.tl_interval_ns) != nxt) return;
  const unsigned long long k = atomicAdd(&c->tl_count.v, 1ull);
  if (k >= P.tl_cap) return;
  unsigned long long* e = P.tl + 4 * k;
  e[0] = now;
  e[1] = ld_relaxed(&c->done.v);
  e[2] = ld_relaxed(&c->tail.v);
  e[3] = ld_relaxed(&c->head.v);
}

// The closing sample: the first worker that observes global termination records one last row (the run's
// final done / tail), then parks the sampling clock at +inf so no later row is written.
__device__ __forceinline__ void tl_final(const EngineParams& P) {
  if (!P.tl) return;
  QueueCtl* c = P.q.ctl;
  if (atomicExch(&c->tl_next.v, ~0ull) == ~0ull) return;
  const unsigned long long k = atomicAdd(&c->tl_count.v, 1ull);
  if (k >= P.tl_cap) return;
  unsigned long long* e = P.tl + 4 * k;
  e[0] = globaltimer();
  e[1] = ld_relaxed(&c->done.v);
  e[2] = ld_relaxed(&c->tail.v);
  e[3] = ld_relaxed(&c->head.v);
}

constexpr uint32_t kGoBig = 0xFFFFFFFFu;

// ---------------------------------------------------------- col prefetch (cp.async)
// PF (kernel template flag): the CTA worker's expand loop stages the NEXT iteration's neighbour ids into a
// per-warp shared-memory double buffer with cp.async (no registers held across the iteration), so the col
// load's latency overlaps the current iteration's state gathers and atomics instead of adding to them.
// Measured (tools/ab.py, profiles/r02_ab_*): mesh / road-like BFS and PageRank faster, scale-free BFS
// slower (its hub spans are already one coalesced load per lane) -- the launcher picks it per graph.
constexpr uint32_t kPfKU = 4;                              // buffer sized for up to 4 edges per lane
constexpr uint32_t kPfWarpBytes = 2u * 32u * kPfKU * 6u;   // 2 stages x (u32 id + u16 owner) per edge slot

__device__ __forceinline__ void cp_async4(void* smem, const void* gmem, unsigned long long pol) {
  const uint32_t sa = (uint32_t)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 4, %2;" ::"r"(sa), "l"(gmem), "l"(pol)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }

template <class Payload>
__device__ __forceinline__ unsigned long long payload_bits(const Payload& p) {
  static_assert(sizeof(Payload) <= 8, "payload must fit 8 bytes");
  unsigned long long b = 0;
  memcpy(&b, &p, sizeof(Payload));
  return b;
}
template <class Payload>
__device__ __forceinline__ Payload payload_from(unsigned long long b) {
  Payload p;
  memcpy(&p, &b, sizeof(Payload));
  return p;
}

__device__ __forceinline__ unsigned long long atom_add_acquire(unsigned long long* p, unsigned long long v) {
  unsigned long long old;
  asm volatile("atom.acquire.gpu.global.add.u64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
  return old;
}
__device__ __forceinline__ unsigned long long atom_exch_release(unsigned long long* p, unsigned long long v) {
  unsigned long long old;
  asm volatile("atom.release.gpu.global.exch.b64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
  return old;
}

// Register item v (row [start, start+deg), payload p) as a big task.  False
// when the chosen slot is busy (the caller expands the vertex itself).
// The fields and `finished` are written first; ONE release exchange then
// publishes (gen+1, nchunks, next=0) in the counter word.  Chunk size is
// raised if needed so nchunks < 2^19 (the counter's 20-bit field keeps room
// for stale over-claims).
template <class Payload>
__device__ __forceinline__ bool register_big(const EngineParams& P, uint32_t v, uint32_t start, uint32_t deg,
                                             const Payload& p) {
  const uint32_t slot = (uint32_t)(atomicAdd(&P.q.ctl->big_rr.v, 1ull) % P.nbig);
  BigTask* t = P.big + slot;
  if (atomicCAS(&t->state, 0u, 1u) != 0u) return false;
  fence_acq_rel_gpu();  // the previous instance's retirement happens-before our writes
  uint32_t chunk = P.big_chunk;
  const uint32_t minchunk = (deg + (1u << 19) - 1) >> 19;
  if (chunk < minchunk) chunk = minchunk;
  const uint32_t nchunks = (deg + chunk - 1) / chunk;
  t->start = start;
  t->deg = deg;
  t->chunk = chunk;
  t->finished = 0;
  t->payload = payload_bits(p);
  const uint32_t gen = big_gen(ld_relaxed(&t->ctr)) + 1u;  // we own the slot: only `next` moves meanwhile
  atom_exch_release(&t->ctr, big_pack(gen, nchunks, 0));
  st_release(&t->state, 2u);
  atomicAdd(&P.q.ctl->big_count.v, 1ull);
  return true;
}

// Warp-collective: claim one chunk of an active big task.  Returns the slot
// (or -1) and sets chunk; every lane gets the same answer.  When a chunk is
// claimed, lane 0 writes out[0..5] = start, deg, payload lo, payload hi,
// nchunks, chunk size (shared memory).  A claim is valid iff the counter value
// returned by the acquire RMW has next < nchunks: a valid chunk keeps its
// task instance alive (it cannot retire before the chunk finishes), so the
// fields read after the acquire are that instance's; stale over-claims on a
// retired or refilling slot see next >= nchunks and are dropped.
__device__ __forceinline__ int claim_big_warp(const EngineParams& P, uint32_t& chunk, uint32_t* out) {
  if (ld_relaxed(&P.q.ctl->big_count.v) == 0) return -1;
  for (uint32_t base = 0; base < P.nbig; base += 32) {
    const uint32_t i = base + lane_id();
    bool act = false;
    if (i < P.nbig) {
      BigTask* t = P.big + i;
      const unsigned long long c = ld_relaxed(&t->ctr);
      act = ld_relaxed(&t->state) == 2u && big_next(c) < big_nchunks(c);
    }
    unsigned m = __ballot_sync(0xffffffffu, act);
    while (m) {
      const uint32_t L = __ffs(m) - 1;
      m &= m - 1;
      BigTask* t = P.big + base + L;
      int ok = 0;
      uint32_t c = 0;
      if (lane_id() == 0) {
        const unsigned long long old = atom_add_acquire(&t->ctr, 1ull);
        c = big_next(old);
        if (c < big_nchunks(old)) {
          ok = 1;
          out[0] = ld_relaxed(&t->start);
          out[1] = ld_relaxed(&t->deg);
          const unsigned long long pb = ld_relaxed(&t->payload);
          out[2] = (uint32_t)pb;
          out[3] = (uint32_t)(pb >> 32);
          out[4] = big_nchunks(old);
          out[5] = ld_relaxed(&t->chunk);
          if (P.dbg_claim && c < 4096) {
            const uint32_t prev = atomicExch(P.dbg_claim + (base + L) * 4096 + c, big_gen(old));
            if (prev == big_gen(old))
              printf("DUP claim slot %u gen %u chunk %u\n", base + L, big_gen(old), c);
          }
        }
      }
      ok = __shfl_sync(0xffffffffu, ok, 0);
      c = __shfl_sync(0xffffffffu, c, 0);
      if (ok) {
        chunk = c;
        return (int)(base + L);
      }
    }
  }
  return -1;
}

// A chunk is finished (its pushes published): the last finisher retires the
// task and counts the original item as done.  `nchunks` is the value from the
// claim: once our increment lands the slot may be retired and refilled, so
// nothing of the slot is re-read after it.
__device__ __forceinline__ void finish_big_chunk(const EngineParams& P, int slot, uint32_t nchunks) {
  BigTask* t = P.big + slot;
  fence_acq_rel_gpu();
  const uint32_t f = atomicAdd(&t->finished, 1u);
  if (P.dbg_claim && f >= nchunks) printf("OVERFINISH slot %d f %u nchunks %u\n", slot, f, nchunks);
  if (f + 1 == nchunks) {
    fence_acq_rel_gpu();
    st_release(&t->state, 0u);
    atomicAdd(&P.q.ctl->big_count.v, (unsigned long long)-1ll);
    atom_add_release(&P.q.ctl->done.v, 1ull);
  }
}

// apps whose discovery CAS result can be consumed one expand iteration later (BfsByteAppT::kDeferCas)
template <class A, class = void>
struct has_defer_cas : std::false_type {};
template <class A>
struct has_defer_cas<A, std::void_t<decltype(A::kDeferCas)>> : std::bool_constant<A::kDeferCas> {};
template <class A, bool ON = has_defer_cas<A>::value>
struct PendOf {
  struct type {};
};
template <class A>
struct PendOf<A, true> {
  using type = typename A::Pend;
};

// apps whose relax can start with the CAS instead of a prefilter read (BfsAppT::kCasFirst, token kBlind)
template <class A, class = void>
struct has_cas_first : std::false_type {};
template <class A>
struct has_cas_first<A, std::void_t<decltype(A::kCasFirst)>> : std::bool_constant<A::kCasFirst> {};

// Per-group shared-memory arena.  K = items a group may hold at once.
template <class Payload>
struct GroupSmem {
  uint32_t* item;
  uint32_t* start;
  uint32_t* off;      // degree, then exclusive prefix
  Payload* pay;
  unsigned long long* pend;
  unsigned long long* pend2;
  uint32_t* ctr;      // [0] nready [1] npend [2] npend_new [3] exit [4] claim_cnt [5] spare
                      // [6..7] claim_base (u64, 8-byte aligned) [8..40] scan scratch
};

template <class Payload>
__host__ __device__ constexpr size_t group_smem_bytes(uint32_t K) {
  // 3 u32 arrays, payload array, two u64 pending arrays, 56 u32 counters
  return ((size_t)K * (3 * sizeof(uint32_t)) + 15) / 16 * 16 + ((size_t)K * sizeof(Payload) + 15) / 16 * 16 +
         (size_t)K * 16 + 56 * sizeof(uint32_t);
}

template <class Payload>
__device__ __forceinline__ GroupSmem<Payload> carve(unsigned char* base, uint32_t K) {
  GroupSmem<Payload> s;
  size_t o = 0;
  s.item = (uint32_t*)(base + o); o += K * 4;
  s.start = (uint32_t*)(base + o); o += K * 4;
  s.off = (uint32_t*)(base + o); o += K * 4;
  o = (o + 15) / 16 * 16;
  s.pay = (Payload*)(base + o); o += ((size_t)K * sizeof(Payload) + 15) / 16 * 16;
  s.pend = (unsigned long long*)(base + o); o += K * 8;
  s.pend2 = (unsigned long long*)(base + o); o += K * 8;
  s.ctr = (uint32_t*)(base + o);
  return s;
}

template <int MODE>
__device__ __forceinline__ void group_sync() {
  if (MODE == MODE_CTA) __syncthreads(); else __syncwarp();
}

template <int MODE>
__device__ __forceinline__ uint32_t group_rank() {
  return MODE == MODE_CTA ? threadIdx.x : lane_id();
}
template <int MODE>
__device__ __forceinline__ uint32_t group_size() {
  return MODE == MODE_CTA ? blockDim.x : 32u;
}

// Try to consume index `idx`: on success the item goes to s.item[] (slot freed
// for the next lap); otherwise idx is appended to the new pending list.
template <bool ACQ, class Payload>
__device__ __forceinline__ void consume_slot(const Ring& q, const GroupSmem<Payload>& s,
                                             unsigned long long idx) {
  uint32_t v;
  const int rc = try_consume<ACQ>(q, idx, &v);
  if (rc == 0) {
    uint32_t k = atomicAdd(&s.ctr[2], 1u);
    s.pend2[k] = idx;
  } else if (rc > 0) {
    uint32_t k = atomicAdd(&s.ctr[0], 1u);
    s.item[k] = v;
  }
}

// Fused consume + begin (apps with kFusedBegin, the byte-state BFS): after the acquire load has shown the
// slot published, the slot-freeing CAS (relaxed: the acquire load already synchronised with the
// producer's release) and the app's begin (row_ptr loads, the state RMW) are issued together, so a pop
// costs two dependent round trips instead of three.  If the CAS loses (a lapping producer stole the item,
// which the default capacity makes impossible in practice) the item is dropped; the speculative begin is
// then harmless for BFS: clearing the queued flag early can only cause a duplicate push of the vertex,
// and BFS is label-correcting.
template <class App>
__device__ __forceinline__ void consume_slot_fused(const Ring& q, const GroupSmem<typename App::Payload>& s,
                                                   unsigned long long idx, const App& app) {
  unsigned long long* slot = q.slots + (idx & q.mask);
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(slot) : "memory");
  const int32_t d = (int32_t)((uint32_t)(v >> 32) - (uint32_t)(idx + 1));
  if (d < 0) {
    const uint32_t k = atomicAdd(&s.ctr[2], 1u);
    s.pend2[k] = idx;
    return;
  }
  if (d > 0) return;
  const uint32_t item = (uint32_t)v;
  const unsigned long long freed = make_slot(idx + q.mask + 1, 0u);
  const unsigned long long old = atomicCAS(slot, v, freed);
  uint32_t st = 0, dg = 0;
  typename App::Payload p{};
  if (!app.begin(item, st, dg, p)) dg = 0;
  if (old != v) return;
  const uint32_t k = atomicAdd(&s.ctr[0], 1u);
  s.item[k] = item;
  s.start[k] = st;
  s.off[k] = dg;
  s.pay[k] = p;
}

// ------------------------------------------------------------ worker group
// One worker (a CTA, a warp, or -- for MODE_THREAD -- a warp of 32 thread
// workers that share one claim) and its queue protocol: claim / gather /
// idle-with-termination (acquire) and completion (complete).
template <int MODE, bool PERSIST, class Payload, bool ACQ = true>
struct Worker {
  GroupSmem<Payload> s;
  uint32_t r, G, K;
  unsigned long long ggid;
  bool first;
  unsigned backoff;
  unsigned long long idle_since;
  unsigned long long deadline;
  unsigned long long maxocc;  // leader only: largest visible backlog (tail - head) seen at a claim
  ATOS_PH_DECL

  __device__ __forceinline__ void init(unsigned char* arena, const EngineParams& P) {
    const uint32_t nwarps = blockDim.x >> 5;
    K = (MODE == MODE_THREAD) ? 32u * P.fetch : P.fetch;
    const uint32_t gid = (MODE == MODE_CTA) ? 0 : warp_id();
    s = carve<Payload>(arena + group_smem_bytes<Payload>(K) * gid, K);
    r = group_rank<MODE>();
    G = group_size<MODE>();
    const unsigned long long groups_per_block = (MODE == MODE_CTA) ? 1 : nwarps;
    ggid = (unsigned long long)blockIdx.x * groups_per_block + gid;
    first = true;
    backoff = 32;
    idle_since = 0;
    maxocc = 0;
    deadline = P.timeout_ns ? globaltimer() + P.timeout_ns : 0;
    if (r == 0) s.ctr[1] = 0;
#ifdef ATOS_PHASE_PROF
    ph_last = clock64();
    for (int i = 0; i < PH_N; ++i) ph_acc[i] = 0;
#endif
    group_sync<MODE>();
  }

  // Returns the number of ready items now in s.item[0..n), or 0 when the
  // worker must exit (global termination, watchdog, or end of a discrete chunk).
  // With a fused app (kFusedBegin) the items' begin() results are already in s.start / s.off / s.pay.
  template <class FusedApp = void>
  __device__ __forceinline__ uint32_t acquire(const EngineParams& P, const FusedApp* fapp = nullptr) {
    const Ring& q = P.q;
    while (true) {
      // ------------------------------------------------------ 1. claim
      if (r == 0) {
        s.ctr[0] = 0; s.ctr[2] = 0; s.ctr[3] = 0; s.ctr[4] = 0; s.ctr[5] = 0;
        *(unsigned long long*)&s.ctr[6] = 0;
        if (deadline && globaltimer() > deadline) {
          // busy past cfg.timeout_s (e.g. a livelocking policy): stop everyone
          atomicOr((unsigned int*)&q.ctl->status.v, kStatusTimeout);
          s.ctr[3] = 1;
        } else if (!PERSIST) {
          if (!first) {
            s.ctr[3] = 1;
          } else {
            const unsigned long long b = P.h0 + ggid * K;
            const unsigned long long e = b + K < P.t0 ? b + K : P.t0;
            if (b >= P.t0) s.ctr[3] = 1;
            else { *(unsigned long long*)&s.ctr[6] = b; s.ctr[4] = (uint32_t)(e - b); }
          }
        } else if (s.ctr[1] == 0) {
          // Claim.  Plenty of published work (>= 2K visible): one atomicAdd of K
          // (a concurrent over-claim past the tail is filled by the ongoing pushes).
          // Sparse queue: an exact CAS claim of what is visible, so no index past
          // the tail is ever parked in a sleeping worker's pending list (that made
          // late improvement cascades crawl one backoff period per item).
          // Claim size: K, or -- when the visible work is thin relative to the
          // number of workers (a high-diameter frontier) -- the fair share
          // visible / workers, at least kMinClaim, so one worker does not
          // serialise a whole small frontier while the others idle.
          unsigned long long h = ctr_ld(&q.ctl->head.v);
          const unsigned long long t = ctr_ld(&q.ctl->tail.v);
          if (h < t) {
            if (t - h > maxocc) maxocc = t - h;
            const unsigned long long nworkers =
                (unsigned long long)gridDim.x * (MODE == MODE_CTA ? 1u : (blockDim.x >> 5));
            unsigned long long want = (t - h) / nworkers;
            const unsigned long long lo = K < P.min_claim ? K : P.min_claim;
            want = want < lo ? lo : (want > K ? K : want);
            if (t - h >= 2ull * want) {
              const unsigned long long b = ctr_add(&q.ctl->head.v, want);
              *(unsigned long long*)&s.ctr[6] = b;
              s.ctr[4] = (uint32_t)want;
            } else {
              for (int tries = 0; tries < 4 && h < t; ++tries) {
                const unsigned long long amt = t - h < want ? t - h : want;
                const unsigned long long old = atomicCAS(&q.ctl->head.v, h, h + amt);
                if (old == h) {
                  *(unsigned long long*)&s.ctr[6] = h;
                  s.ctr[4] = (uint32_t)amt;
                  break;
                }
                h = old;
              }
            }
          }
        }
      }
      first = false;
      group_sync<MODE>();
      ATOS_PH(PH_CLAIM);
      if (s.ctr[3]) return 0;
      // ------------------------------------------------------ 2. gather
      {
        const unsigned long long cb = *(unsigned long long*)&s.ctr[6];
        const uint32_t cc = s.ctr[4], np = s.ctr[1];
        if constexpr (!std::is_void<FusedApp>::value) {
          for (uint32_t i = r; i < cc; i += G) consume_slot_fused(q, s, cb + i, *fapp);
          for (uint32_t i = r; i < np; i += G) consume_slot_fused(q, s, s.pend[i], *fapp);
        } else {
          for (uint32_t i = r; i < cc; i += G) consume_slot<ACQ>(q, s, cb + i);
          for (uint32_t i = r; i < np; i += G) consume_slot<ACQ>(q, s, s.pend[i]);
        }
      }
      group_sync<MODE>();
      const uint32_t nready = s.ctr[0];
      const uint32_t npn = s.ctr[2];
      for (uint32_t i = r; i < npn; i += G) s.pend[i] = s.pend2[i];
      group_sync<MODE>();
      ATOS_PH(PH_GATHER);
      if (nready) {
        if (r == 0) s.ctr[1] = npn;
        idle_since = 0;
        backoff = 32;
        group_sync<MODE>();
        return nready;
      }
      // ------------------------------------------------------ 3. idle (f2)
      if (r == 0) {
        s.ctr[1] = npn;
        // poll with plain relaxed loads (hundreds of idle workers' RMWs on the done / tail lines queued in
        // front of the pushers' and completers' atomics: mesh -1.8 %, road-like -2.7 %, colouring -1 %,
        // profiles/r02_ab_poll_backoff.txt); an apparent quiescence is confirmed with the RMW reads, which
        // return the latest values in coherence order (done first, then tail: the termination argument)
        unsigned long long d = ctr_ld(&q.ctl->done.v);
        unsigned long long t = ctr_ld(&q.ctl->tail.v);
        if (d == t) {
          d = ctr_read_acquire(&q.ctl->done.v);
          t = ctr_read_acquire(&q.ctl->tail.v);
        }
        const uint32_t st = *(volatile uint32_t*)&q.ctl->status.v;
        if (d == t || st != 0) {
          if (PERSIST && d == t) tl_final(P);
          s.ctr[3] = 1;
        } else if (PERSIST && P.nbig && ld_relaxed(&q.ctl->big_count.v) != 0) {
          tl_sample(P);
          s.ctr[3] = 2;  // go help with big tasks
        } else {
          const unsigned long long now = globaltimer();
          if (idle_since == 0) idle_since = now;
          else if (now - idle_since > P.watchdog_ns) {
            atomicOr((unsigned int*)&q.ctl->status.v, kStatusTimeout);
            s.ctr[3] = 1;
          }
          tl_sample(P);
          __nanosleep(backoff);
          backoff = backoff < ATOS_BACKOFF_MAX ? backoff * 2 : ATOS_BACKOFF_MAX;
        }
      }
      group_sync<MODE>();
      ATOS_PH(PH_IDLE);
      if (s.ctr[3] == 2) return kGoBig;
      if (s.ctr[3]) return 0;
      // every member has read s.ctr[3] before the group leader resets it for the next claim
      // (compute-sanitizer racecheck: WAR on s.ctr[3] across the loop back-edge)
      group_sync<MODE>();
    }
  }

  // kernel exit: the leader folds its largest observed backlog into the control block
  __device__ __forceinline__ void flush_occ(const EngineParams& P) const {
    if (r == 0 && maxocc) atomicMax(&P.q.ctl->stat_maxocc.v, maxocc);
  }

  // All pushes of the batch are published (every warp flushed before this):
  // count the batch as done with release semantics.
  // LEAN (the latency-bound PF builds): no trailing barrier -- the batch's shared state is dead after the
  // first one, and the next claim's barrier waits for the leader anyway
  template <bool LEAN = false>
  __device__ __forceinline__ void complete(const EngineParams& P, uint32_t nready) {
    group_sync<MODE>();
    if (PERSIST && r == 0 && nready) {
      // release reduction, no return value to wait for: the barrier above orders every warp's pushes
      // before the leader's release (cumulative), and nobody needs the old count (C5 BFS -1 %)
      ctr_red_release(&P.q.ctl->done.v, (unsigned long long)nready);
    }
    if (r == 0) tl_sample(P);
    if (!LEAN) group_sync<MODE>();
  }
};

__device__ __forceinline__ void flush_stats(const Ring& q, unsigned long long pops, unsigned long long edges,
                                            unsigned long long pushes_lane0) {
  for (int o = 16; o; o >>= 1) {
    pops += __shfl_xor_sync(0xffffffffu, pops, o);
    edges += __shfl_xor_sync(0xffffffffu, edges, o);
  }
  if (lane_id() == 0) {
    if (pops) atomicAdd(&q.ctl->stat_pops.v, pops);
    if (edges) atomicAdd(&q.ctl->stat_edges.v, edges);
    if (pushes_lane0) atomicAdd(&q.ctl->stat_pushes.v, pushes_lane0);
  }
}

// ------------------------------------------------------------------- kernel
// KU: edges in flight per thread per expand iteration.  MINB > 1: a variant for
// 256-thread CTA workers with __launch_bounds__(256, MINB) -- fewer registers,
// MINB resident CTAs per SM (the host picks it, see launch_relax_mode).
#ifndef ATOS_MAXT
#define ATOS_MAXT 1024
#endif
template <class App, int MODE, bool PERSIST, int KU = kU, int MINB = ATOS_MINB, bool PF = false>
__global__ void __launch_bounds__(MINB == 1 ? ATOS_MAXT : 256, MINB) k_relax_worker(App app, EngineParams P) {
  using Payload = typename App::Payload;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t nwarps = blockDim.x >> 5;
  // push rings first (kPushBuf u32 per warp), then one arena per group
  uint32_t* pushbuf = (uint32_t*)smem_raw;
  Worker<MODE, PERSIST, Payload, App::kAcquirePop> wk;
  wk.init(smem_raw + (size_t)nwarps * kPushBuf * 4, P);
  const GroupSmem<Payload>& s = wk.s;
  const uint32_t r = wk.r, G = wk.G;
  // low-degree (PF) builds are latency-bound: single-CAS publishes and the small-batch scan below
  auto pusher = make_pusher<PF>(pushbuf);
  // CTA mode: owner table after the group arena
  uint32_t* cown = (uint32_t*)(smem_raw + (size_t)nwarps * kPushBuf * 4 + group_smem_bytes<Payload>(wk.K));
  unsigned long long my_pops = 0, my_edges = 0;
  const Ring& q = P.q;
  app.prepare();
  constexpr bool kAssist = PERSIST && MODE != MODE_THREAD;
  const bool assist = kAssist && P.nbig != 0;
#ifdef ATOS_PHASE_PROF
  auto& ph_acc = wk.ph_acc;
  auto& ph_last = wk.ph_last;
  unsigned long long ph_exp0 = 0;
  uint32_t ph_total = 0;
#endif

  while (true) {
    // ---------------------------------------------------------- 0. big-task chunks first
    if (assist) {
      if (MODE == MODE_CTA) {
        if (warp_id() == 0) {
          uint32_t c = 0;
          const int slot = claim_big_warp(P, c, s.ctr + 43);
          if (lane_id() == 0) { s.ctr[41] = (uint32_t)slot; s.ctr[42] = c; }
        }
        __syncthreads();
      } else {
        uint32_t c = 0;
        const int slot = claim_big_warp(P, c, s.ctr + 43);
        if (lane_id() == 0) { s.ctr[41] = (uint32_t)slot; s.ctr[42] = c; }
        __syncwarp();
      }
      const int slot = (int)s.ctr[41];
      if (slot >= 0) {
        const uint32_t c = s.ctr[42];
        const uint32_t b0 = c * s.ctr[48];
        const uint32_t len = min(s.ctr[48], s.ctr[44] - b0);
        const uint32_t st0 = s.ctr[43] + b0;
        const Payload p = payload_from<Payload>(((unsigned long long)s.ctr[46] << 32) | s.ctr[45]);
        my_edges += (r == 0) ? len : 0;
        for (uint32_t base = 0; base < len; base += G * KU) {
          // strided lanes (k * G + r): coalesced loads
          uint32_t w[KU];
          typename App::Token tk[KU];
#pragma unroll
          for (int k = 0; k < KU; ++k)
            if (base + k * G + r < len) {
              w[k] = app.neighbor(st0 + base + k * G + r);
              ATOS_DBG_EDGE(P, st0 + base + k * G + r);
            }
#pragma unroll
          for (int k = 0; k < KU; ++k)
            if (base + k * G + r < len) tk[k] = app.pre(p, w[k]);
          bool want[KU];
          uint32_t out[KU];
#pragma unroll
          for (int k = 0; k < KU; ++k) {
            want[k] = false;
            out[k] = 0;
            if (base + k * G + r < len) want[k] = app.post(p, w[k], tk[k], out[k]);
          }
          pusher.push_n<KU>(q, want, out, P.watchdog_ns);
        }
        pusher.flush(q, P.watchdog_ns);
        group_sync<MODE>();
        if (r == 0) finish_big_chunk(P, slot, s.ctr[47]);
        group_sync<MODE>();
        ATOS_PH(PH_BIG);
        continue;
      }
      group_sync<MODE>();
      ATOS_PH(PH_BIG);
    }
    constexpr bool kFused = App::kFusedBegin && MODE == MODE_CTA;
    const uint32_t nready = kFused ? wk.acquire(P, &app) : wk.acquire(P);
    if (nready == kGoBig) continue;
    if (nready == 0) break;
    // ---------------------------------------------------------- begin (per item)
    // (PF builds, fused pops, no assist: the pass below would only copy the gather's results in place)
    const bool skip_begin = PF && kFused && !assist;
    if (!skip_begin) {
    for (uint32_t k = r; k < nready; k += G) {
      uint32_t st = 0, dg = 0;
      Payload p{};
      if (kFused) {
        st = s.start[k];
        dg = s.off[k];
        p = s.pay[k];
      } else if (!app.begin(s.item[k], st, dg, p)) {
        dg = 0;
      }
      if (assist && dg > P.big_threshold && register_big(P, s.item[k], st, dg, p)) {
        dg = 0;  // expanded by the assist chunks; counted done by the last chunk
        atomicAdd(&s.ctr[5], 1u);
      }
      s.start[k] = st;
      s.off[k] = dg;
      s.pay[k] = p;
    }
    group_sync<MODE>();
    }
    ATOS_PH(PH_BEGIN);
    my_pops += (r == 0) ? nready : 0;
    const uint32_t deferred = s.ctr[5];

    // ---------------------------------------------------------- expand + relax
    if (MODE == MODE_CTA) {
      // load-balancing search over the flattened edge list of the batch
      uint32_t total = 0;
      if (PF && nready <= 32u) {
        // small batch (thin frontiers): warp 0 scans, one barrier instead of the block scan's four
        if (r < 32u) {
          const uint32_t d = r < nready ? s.off[r] : 0u;
          uint32_t incl = d;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
            if (r >= (uint32_t)o) incl += y;
          }
          if (r < nready) s.off[r] = incl - d;
          if (r == 31u) s.ctr[40] = incl;
        }
        __syncthreads();
        total = s.ctr[40];
      } else {
      uint32_t mydeg = 0;
      const uint32_t per = (nready + G - 1) / G;
      const uint32_t i0 = min(r * per, nready), i1 = min(i0 + per, nready);
      for (uint32_t i = i0; i < i1; ++i) mydeg += s.off[i];
      uint32_t excl = block_exclusive_scan(mydeg, s.ctr + 8, &total);
      for (uint32_t i = i0; i < i1; ++i) { const uint32_t d = s.off[i]; s.off[i] = excl; excl += d; }
      __syncthreads();
      }
      my_edges += (r == 0) ? total : 0;
      // KU CONSECUTIVE edges per lane per iteration (a warp covers 32*KU
      // consecutive flattened edges, so col reads stay coalesced).  Owners:
      // lanes 0/1 binary-search the owners of the warp's first/last edge over
      // the whole batch, then every lane searches only that narrow range and
      // walks forward over its KU edges.  All col loads, then all prefilter
      // loads, then the decisions/atomics: KU memory chains in flight per lane.
      const uint32_t wspan = 32u * KU;
      // owner of every wspan-edge chunk start, once per batch (a warp's span is
      // one chunk, so its owner range comes from two table reads)
      const uint32_t nchunk = (total + wspan - 1) / wspan;
      // (PF builds: a batch of at most 8 chunks skips the table and its barrier; lanes 0/1 search instead)
      const bool table = nchunk <= kCown && (!PF || nchunk > 8u);
      if (table) {
        for (uint32_t c = r; c < nchunk; c += G) {
          const uint32_t e = c * wspan;
          uint32_t l = 0, h = nready;
          while (h - l > 1) {
            const uint32_t mid = (l + h) >> 1;
            if (s.off[mid] <= e) l = mid; else h = mid;
          }
          cown[c] = l;
        }
        __syncthreads();
      }
      ATOS_PH(PH_SCAN);
#ifdef ATOS_PHASE_PROF
      ph_exp0 = ph_last;
      ph_total = total;
#endif
      if constexpr (PF) {
        // per-warp double buffer after the owner table: [stage][KU*32] u32 ids, then [stage][KU*32] u16 owners
        uint32_t* pf_id = (uint32_t*)((unsigned char*)(cown + kCown) + (size_t)warp_id() * kPfWarpBytes);
        uint16_t* pf_own = (uint16_t*)(pf_id + 2 * 32 * kPfKU);
        const uint32_t step = G * KU;
        // stage: the owners of this warp's span of iteration `base` and cp.async of its neighbour ids
        auto stage = [&](uint32_t base, uint32_t buf) {
          const uint32_t wfirst = base + (r & ~31u) * KU;
          uint16_t* ob_ = pf_own + buf * 32 * kPfKU;
          uint32_t* ib_ = pf_id + buf * 32 * kPfKU;
          if (wfirst >= total) {
#pragma unroll
            for (int k = 0; k < KU; ++k) ob_[k * 32 + lane_id()] = 0xFFFFu;
            return;
          }
          const uint32_t wlast = min(wfirst + wspan, total) - 1;
          uint32_t ob = 0;
          if (table) {
            const uint32_t c = wfirst / wspan;
            ob = lane_id() == 0 ? cown[c] : (c + 1 < nchunk ? cown[c + 1] : nready - 1);
          } else if (lane_id() < 2) {
            const uint32_t e = lane_id() == 0 ? wfirst : wlast;
            uint32_t l = 0, h = nready;
            while (h - l > 1) {
              const uint32_t mid = (l + h) >> 1;
              if (s.off[mid] <= e) l = mid; else h = mid;
            }
            ob = l;
          }
          const uint32_t olo = __shfl_sync(0xffffffffu, ob, 0), ohi = __shfl_sync(0xffffffffu, ob, 1);
          // lane-strided edges e = wfirst + k*32 + lane: every cp.async instruction covers 32 consecutive
          // flattened edges; owners by binary search over [olo, ohi], monotone in k
          uint32_t o = olo;
#pragma unroll
          for (int k = 0; k < KU; ++k) {
            const uint32_t e = wfirst + k * 32 + lane_id();
            uint16_t own = 0xFFFFu;
            if (e <= wlast) {
              uint32_t l = o, h = ohi + 1;
              while (h - l > 1) {
                const uint32_t mid = (l + h) >> 1;
                if (s.off[mid] <= e) l = mid; else h = mid;
              }
              o = l;
              own = (uint16_t)l;
              cp_async4(ib_ + k * 32 + lane_id(), app.col + s.start[l] + (e - s.off[l]), app.pol_first);
              ATOS_DBG_EDGE(P, s.start[l] + (e - s.off[l]));
            }
            ob_[k * 32 + lane_id()] = own;
          }
        };
        stage(0, 0);
        cp_async_commit();
        uint32_t buf = 0;
        for (uint32_t base = 0; base < total; base += step, buf ^= 1u) {
          stage(base + step, buf ^ 1u);
          cp_async_commit();
          cp_async_wait1();  // this iteration's group has landed
          __syncwarp();
          const uint32_t wfirst = base + (r & ~31u) * KU;
          if (wfirst >= total) continue;  // warp-uniform
          const uint16_t* ob_ = pf_own + buf * 32 * kPfKU;
          const uint32_t* ib_ = pf_id + buf * 32 * kPfKU;
          uint32_t w[KU], own[KU];
          typename App::Token tk[KU];
          bool want[KU];
          uint32_t out[KU];
#pragma unroll
          for (int k = 0; k < KU; ++k) {
            own[k] = ob_[k * 32 + lane_id()];
            if (own[k] != 0xFFFFu) w[k] = ib_[k * 32 + lane_id()];
          }
#pragma unroll
          for (int k = 0; k < KU; ++k)
            if (own[k] != 0xFFFFu) {
              if constexpr (has_cas_first<App>::value) tk[k] = App::kBlind;
              else tk[k] = app.pre(s.pay[own[k]], w[k]);
            }
#pragma unroll
          for (int k = 0; k < KU; ++k) {
            want[k] = false;
            out[k] = 0;
            if (own[k] != 0xFFFFu) want[k] = app.post(s.pay[own[k]], w[k], tk[k], out[k]);
          }
          pusher.push_n<KU>(q, want, out, P.watchdog_ns);
        }
        asm volatile("cp.async.wait_all;" ::: "memory");
        __syncwarp();
      } else {
      constexpr bool kDefer = has_defer_cas<App>::value;
      typename PendOf<App>::type pd{};
      for (uint32_t base = 0; base < total; base += G * KU) {
        const uint32_t wfirst = base + (r & ~31u) * KU;
        if (wfirst >= total) continue;  // warp-uniform; no collective below is skipped by part of a warp
        const uint32_t wlast = min(wfirst + wspan, total) - 1;
        uint32_t ob = 0;
        if (table) {
          const uint32_t c = wfirst / wspan;
          ob = lane_id() == 0 ? cown[c] : (c + 1 < nchunk ? cown[c + 1] : nready - 1);
        } else if (lane_id() < 2) {
          const uint32_t e = lane_id() == 0 ? wfirst : wlast;
          uint32_t l = 0, h = nready;
          while (h - l > 1) {
            const uint32_t mid = (l + h) >> 1;
            if (s.off[mid] <= e) l = mid; else h = mid;
          }
          ob = l;
        }
        const uint32_t olo = __shfl_sync(0xffffffffu, ob, 0), ohi = __shfl_sync(0xffffffffu, ob, 1);
        uint32_t w[KU];
        typename App::Token tk[KU];
        bool want[KU];
        uint32_t out[KU];
        if (olo == ohi) {
          // fast path (warp-uniform): the warp's span lies in ONE row -- no owner search,
          // strided lanes so every load instruction is one coalesced 128-byte access
          const uint32_t st0 = s.start[olo] + (wfirst - s.off[olo]);
          const uint32_t len = wlast - wfirst + 1;
          const Payload p = s.pay[olo];
#pragma unroll
          for (int k = 0; k < KU; ++k)
            if (k * 32 + lane_id() < len) {
              w[k] = app.neighbor(st0 + k * 32 + lane_id());
              ATOS_DBG_EDGE(P, st0 + k * 32 + lane_id());
            }
#pragma unroll
          for (int k = 0; k < KU; ++k)
            if (k * 32 + lane_id() < len) tk[k] = app.pre(p, w[k]);
          if constexpr (kDefer) {
            uint32_t po = 0;
            const bool pw = app.resolve(pd, po);
            pusher.push(q, pw, po, P.watchdog_ns);
          }
#pragma unroll
          for (int k = 0; k < KU; ++k) {
            want[k] = false;
            out[k] = 0;
            if (k * 32 + lane_id() < len) {
              if constexpr (kDefer) want[k] = app.post_d(p, w[k], tk[k], out[k], pd);
              else want[k] = app.post(p, w[k], tk[k], out[k]);
            }
          }
          pusher.push_n<KU>(q, want, out, P.watchdog_ns);
          continue;
        }
        uint32_t own[KU];
        bool val[KU];
#ifdef ATOS_LBS_STRIDED
        // lane-strided: edge wfirst + k*32 + lane (each col load instruction covers 32 consecutive
        // flattened edges); owners by binary search over [olo, ohi], monotone in k
        uint32_t o = olo;
#pragma unroll
        for (int k = 0; k < KU; ++k) {
          const uint32_t e = wfirst + k * 32 + lane_id();
          val[k] = e <= wlast;
          if (val[k]) {
            uint32_t l = o, h = ohi + 1;
            while (h - l > 1) {
              const uint32_t mid = (l + h) >> 1;
              if (s.off[mid] <= e) l = mid; else h = mid;
            }
            o = l;
            own[k] = l;
            const uint32_t ce = s.start[l] + (e - s.off[l]);
            w[k] = app.neighbor(ce);
            ATOS_DBG_EDGE(P, ce);
          }
        }
#else
        const uint32_t e0 = wfirst + lane_id() * KU;
#ifndef ATOS_OWN_FILL
#define ATOS_OWN_FILL 1
#endif
        if (ATOS_OWN_FILL && KU * 32u <= 128u && nchunk + 32u * nwarps <= kCown && ohi - olo >= 8u &&
            ohi - olo < 255u) {
          // a span over many short rows (warp-uniform): instead of a binary search plus a walk per lane, the
          // lanes write each row's owner offset over its edges into a per-warp byte map (the owner table's
          // unused tail: 128 B = 32 words per warp) -- rows are disjoint, so every byte has one writer -- and every lane
          // reads its KU owners back with one shared-memory load each
          uint8_t* own_s = (uint8_t*)(cown + kCown - 32u * nwarps) + warp_id() * 128u;
          __syncwarp();  // the previous span's reads are done
          for (uint32_t it = olo + lane_id(); it <= ohi; it += 32u) {
            const uint32_t a = max(s.off[it], wfirst);
            const uint32_t b = min(it + 1u < nready ? s.off[it + 1u] : total, wfirst + wspan);
            for (uint32_t e = a; e < b; ++e) own_s[e - wfirst] = (uint8_t)(it - olo);
          }
          __syncwarp();
#pragma unroll
          for (int k = 0; k < KU; ++k) {
            const uint32_t e = e0 + k;
            val[k] = e < total;
            if (val[k]) {
              const uint32_t o = olo + own_s[e - wfirst];
              own[k] = o;
              const uint32_t ce = s.start[o] + (e - s.off[o]);
              w[k] = app.neighbor(ce);
              ATOS_DBG_EDGE(P, ce);
            }
          }
        } else {
        uint32_t o = olo;
        {
          uint32_t l = olo, h = ohi + 1;
          while (h - l > 1) {
            const uint32_t mid = (l + h) >> 1;
            if (s.off[mid] <= e0) l = mid; else h = mid;
          }
          o = l;
        }
#pragma unroll
        for (int k = 0; k < KU; ++k) {
          const uint32_t e = e0 + k;
          val[k] = e < total;
          if (val[k]) {
            while (o < ohi && s.off[o + 1] <= e) ++o;
            own[k] = o;
            const uint32_t ce = s.start[o] + (e - s.off[o]);
            w[k] = app.neighbor(ce);
            ATOS_DBG_EDGE(P, ce);
          }
        }
        }
#endif
#pragma unroll
        for (int k = 0; k < KU; ++k)
          if (val[k]) tk[k] = app.pre(s.pay[own[k]], w[k]);
        if constexpr (kDefer) {
          uint32_t po = 0;
          const bool pw = app.resolve(pd, po);
          pusher.push(q, pw, po, P.watchdog_ns);
        }
#pragma unroll
        for (int k = 0; k < KU; ++k) {
          want[k] = false;
          out[k] = 0;
          if (val[k]) {
            if constexpr (kDefer) want[k] = app.post_d(s.pay[own[k]], w[k], tk[k], out[k], pd);
            else want[k] = app.post(s.pay[own[k]], w[k], tk[k], out[k]);
          }
        }
        pusher.push_n<KU>(q, want, out, P.watchdog_ns);
      }
      if constexpr (kDefer) {
        // the last iteration's pending CAS (every lane of the warp reaches here together)
        uint32_t po = 0;
        const bool pw = app.resolve(pd, po);
        pusher.push(q, pw, po, P.watchdog_ns);
      }
      }  // !PF
    } else if (MODE == MODE_WARP) {
      for (uint32_t k = 0; k < nready; ++k) {
        const uint32_t st = s.start[k], dg = s.off[k];
        const Payload p = s.pay[k];
        my_edges += (r == 0) ? dg : 0;
        for (uint32_t j = 0; j < dg; j += 32 * KU) {
          // strided lanes: each load instruction is one coalesced access
          uint32_t w[KU];
          typename App::Token tk[KU];
#pragma unroll
          for (int k = 0; k < KU; ++k)
            if (j + k * 32 + r < dg) {
              w[k] = app.neighbor(st + j + k * 32 + r);
              ATOS_DBG_EDGE(P, st + j + k * 32 + r);
            }
#pragma unroll
          for (int k = 0; k < KU; ++k)
            if (j + k * 32 + r < dg) tk[k] = app.pre(p, w[k]);
          bool want[KU];
          uint32_t out[KU];
#pragma unroll
          for (int k = 0; k < KU; ++k) {
            want[k] = false;
            out[k] = 0;
            if (j + k * 32 + r < dg) want[k] = app.post(p, w[k], tk[k], out[k]);
          }
          pusher.push_n<KU>(q, want, out, P.watchdog_ns);
        }
      }
    } else {
      // THREAD: lane r walks items r, r+32, ... serially; lanes advance in lock step
      uint32_t k = r, st = 0, dg = 0, j = 0;
      Payload p{};
      if (k < nready) { st = s.start[k]; dg = s.off[k]; p = s.pay[k]; }
      while (true) {
        while (k < nready && j >= dg) {
          k += 32;
          j = 0;
          if (k < nready) { st = s.start[k]; dg = s.off[k]; p = s.pay[k]; }
        }
        const bool active = k < nready;
        if (__ballot_sync(0xffffffffu, active) == 0) break;
        bool want = false;
        uint32_t out = 0;
        if (active) {
          const uint32_t w = app.neighbor(st + j);
          ++j;
          ++my_edges;
          want = app.relax(p, w, out);
        }
        pusher.push(q, want, out, P.watchdog_ns);
      }
    }
    pusher.flush(q, P.watchdog_ns);
#ifdef ATOS_PHASE_PROF
    if (MODE == MODE_CTA) __syncthreads();
    ATOS_PH(PH_EXPAND);
    if (MODE == MODE_CTA && threadIdx.x == 0) {
      const bool lo = ph_total < 8192;
      ph_acc[lo ? PH_NB_LO : PH_NB_HI] += 1;
      ph_acc[lo ? PH_EXP_LO : PH_EXP_HI] += ph_last - ph_exp0;
      ph_acc[lo ? PH_EDGES_LO : PH_EDGES_HI] += ph_total;
    }
#endif
    wk.template complete<PF>(P, nready - deferred);
    ATOS_PH(PH_COMPLETE);
  }
  ATOS_PH_FLUSH();
  wk.flush_occ(P);
  flush_stats(q, my_pops, my_edges, lane_id() == 0 ? pusher.total : 0);
}

// Host-side helper: dynamic shared memory for a launch.
template <class Payload>
inline size_t relax_worker_smem(int mode, uint32_t block, uint32_t fetch, bool pf = false) {
  uint32_t nwarps = block / 32;
  uint32_t K = mode == MODE_THREAD ? 32u * fetch : fetch;
  uint32_t groups = mode == MODE_CTA ? 1u : nwarps;
  return (size_t)nwarps * kPushBuf * 4 + group_smem_bytes<Payload>(K) * groups +
         (mode == MODE_CTA ? kCown * 4 + (pf ? (size_t)nwarps * kPfWarpBytes : 0) : 0);
}

}  // namespace atos
