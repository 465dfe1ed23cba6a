// color.cu -- asynchronous speculative greedy colouring (Alg.6) as
// an uberkernel: one queue carries two task types,
//   assign(v)  (item = v):            forbidden set of neighbours' colours ->
//                                     smallest free colour, store,
//                                     fence.sc.gpu, enqueue check(v);
//   check(v)   (item = v | 0x80000000, R-GC-1 -- the paper's sign trick cannot
//              encode vertex 0):      for every neighbour w != v with
//                                     color[w] == color[v] enqueue assign of
//                                     the LOSER of (v, w) (R-GC-2), or -- paper
//                                     literal policy -- assign(v).
// Correctness argument: for two adjacent
// vertices whose final assignments carry the same colour, the SC fences of the
// two assigns are totally ordered, so the check that runs after the later
// fence reads the other colour and re-queues the loser -- no conflict survives
// quiescence.  Forbidden sets are windowed (R-GC-4): only colours in
// [base, base+window) are marked; a full window moves to the next one, so
// colour <= deg(v) always.
#include <algorithm>
#include <cstdlib>
#include <vector>

#include "internal.h"

namespace atos {

constexpr uint32_t kCheck = 0x80000000u;
constexpr uint32_t kWin = 1024;  // colours per forbidden-set window (warp/CTA workers)

#ifndef ATOS_GC_KU
#define ATOS_GC_KU 4
#endif
constexpr int kUc = ATOS_GC_KU;  // CTA worker: edges in flight per thread per expand iteration

// Tools only (build with -DATOS_GC_COUNTS, run with ATOS_GC_COUNTS=<file>): per-vertex counts of
// assign and check tasks, written as u32 pairs [v][assign, check] to <file> after the run.
#ifdef ATOS_GC_COUNTS
static __device__ uint32_t* g_gc_counts;
#define ATOS_GC_COUNT(v, chk) do { if (g_gc_counts) atomicAdd(g_gc_counts + 2 * (v) + ((chk) ? 1 : 0), 1u); } while (0)
#else
#define ATOS_GC_COUNT(v, chk) do {} while (0)
#endif

struct ColorCtx {
  const uint32_t* __restrict__ row_ptr;
  const uint32_t* __restrict__ col;
  int32_t* color;
  uint32_t* inq;            // assign-task dedupe bitmap (always on for colouring)
  uint8_t* att;             // recolours per vertex so far (saturating; a heuristic, races are harmless)
  uint32_t spread;          // cfg.recolor_spread (CTA worker): 1 = Alg.6's smallest free colour on every assign
  unsigned long long seed;
  int literal;              // 1: paper-literal self-recolour policy
  int hash_only;            // 1: conflict priority by hash only (conflict_policy 2)

  // true when x loses against y (R-GC-2): by default the lower-DEGREE endpoint
  // recolours (largest-degree-first, so hubs -- whose assign tasks cost a
  // whole neighbour scan -- are not recoloured for every low-degree neighbour
  // they collide with), then lower priority splitmix64(seed ^ id), then id.
  // conflict_policy 2: hash priority only.
  __device__ __forceinline__ bool loses(uint32_t x, uint32_t y) const {
    if (!hash_only) {
      const uint32_t dx = __ldg(row_ptr + x + 1) - __ldg(row_ptr + x);
      const uint32_t dy = __ldg(row_ptr + y + 1) - __ldg(row_ptr + y);
      if (dx != dy) return dx < dy;
    }
    const unsigned long long px = splitmix64(seed ^ x), py = splitmix64(seed ^ y);
    return px < py || (px == py && x < y);
  }
  // assign(x) may be enqueued once at a time (bit set by the enqueuer, cleared by the popper)
  __device__ __forceinline__ bool claim_assign(uint32_t x) const {
    const uint32_t bit = 1u << (x & 31);
    return !(atom_or_release(inq + (x >> 5), bit) & bit);
  }

};

// ---------------------------------------------------------------- warp worker
// The warp strides one vertex's neighbours at a time (the paper's persist-warp
// variant, its best colouring configuration on scale-free graphs).
__device__ __forceinline__ void color_item_warp(const ColorCtx& c, uint32_t item, uint32_t* bm,
                                                WarpPusher& pusher, const Ring& q,
                                                unsigned long long wd, unsigned long long& edges) {
  const uint32_t lane = lane_id();
  const uint32_t v = item & ~kCheck;
  const uint32_t st = __ldg(c.row_ptr + v), deg = __ldg(c.row_ptr + v + 1) - st;
  if (!(item & kCheck)) {
    // assign(v): clear the dedupe bit first (acquire), then read neighbours' colours
    atom_and_acquire(c.inq + (v >> 5), ~(1u << (v & 31)));
    uint32_t base = 0;
    int32_t chosen = -1;
    while (chosen < 0) {
      bm[lane] = 0;
      __syncwarp();
      for (uint32_t j = lane; j < deg; j += 32) {
        const uint32_t w = __ldg(c.col + st + j);
        if (w == v) continue;
        const int32_t cw = ld_relaxed(c.color + w);
        if (cw >= (int32_t)base && cw < (int32_t)(base + kWin)) {
          const uint32_t o = (uint32_t)cw - base;
          atomicOr(bm + (o >> 5), 1u << (o & 31));
        }
      }
      __syncwarp();
      const uint32_t freebits = ~bm[lane];
      const unsigned m = __ballot_sync(0xffffffffu, freebits != 0);
      if (m) {
        const uint32_t L = __ffs(m) - 1;
        const uint32_t fb = __shfl_sync(0xffffffffu, freebits, L);
        chosen = (int32_t)(base + L * 32 + (__ffs(fb) - 1));
      } else {
        base += kWin;
      }
      __syncwarp();
    }
    edges += deg;
    if (lane == 0) {
      st_relaxed(c.color + v, chosen);
      fence_sc_gpu();
    }
    __syncwarp();
    pusher.push(q, lane == 0, v | kCheck, wd);
  } else {
    // check(v)
    const int32_t cv = ld_relaxed(c.color + v);
    bool self = false;
    for (uint32_t j0 = 0; j0 < deg; j0 += 32) {
      const uint32_t j = j0 + lane;
      bool want = false;
      uint32_t out = 0;
      if (j < deg) {
        const uint32_t w = __ldg(c.col + st + j);
        if (w != v && ld_relaxed(c.color + w) == cv) {
          if (c.literal || c.loses(v, w)) self = true;
          else if (c.claim_assign(w)) { want = true; out = w; }
        }
      }
      pusher.push(q, want, out, wd);
    }
    edges += deg;
    const bool any_self = __ballot_sync(0xffffffffu, self) != 0;
    bool want = false;
    if (any_self && lane == 0) want = c.claim_assign(v);
    pusher.push(q, want, v, wd);
  }
}

template <bool PERSIST>
__global__ void __launch_bounds__(1024) k_color_warp(ColorCtx c, EngineParams P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t nwarps = blockDim.x >> 5;
  uint32_t* pushbuf = (uint32_t*)smem_raw;
  uint32_t* bms = pushbuf + nwarps * kPushBuf;  // 32 words per warp
  Worker<MODE_WARP, PERSIST, uint32_t> wk;
  wk.init((unsigned char*)(bms + nwarps * 32), P);
  WarpPusher pusher = make_pusher(pushbuf);
  unsigned long long pops = 0, edges = 0;
  while (true) {
    const uint32_t nready = wk.acquire(P);
    if (!nready) break;
    for (uint32_t k = 0; k < nready; ++k)
      color_item_warp(c, wk.s.item[k], bms + warp_id() * 32, pusher, P.q, P.watchdog_ns, edges);
    pops += lane_id() == 0 ? nready : 0;
    pusher.flush(P.q, P.watchdog_ns);
    wk.complete(P, nready);
  }
  wk.flush_occ(P);
  flush_stats(P.q, pops, lane_id() == 0 ? edges : 0, lane_id() == 0 ? pusher.total : 0);
}

// ----------------------------------------------------------------- CTA worker
// The CTA fetches a batch, flattens all items' edges (load-balancing search)
// and marks per-item forbidden windows in shared memory; then one warp per
// assign item picks its colour.  Items whose first window is full fall back to
// the warp routine for the next windows.
template <bool PERSIST>
__global__ void __launch_bounds__(1024) k_color_cta(ColorCtx c, EngineParams P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t nwarps = blockDim.x >> 5;
  const uint32_t F = P.fetch;
  uint32_t* pushbuf = (uint32_t*)smem_raw;
  uint32_t* wbm = pushbuf + nwarps * kPushBuf;   // 32 words per warp (fallback windows)
  uint32_t* ibm = wbm + nwarps * 32;       // 32 words per item
  uint32_t* flag = ibm + F * 32;           // per item: check found a self-conflict
  int32_t* cval = (int32_t*)(flag + F);    // per item: colour of v (check items)
  Worker<MODE_CTA, PERSIST, uint32_t> wk;
  wk.init((unsigned char*)(cval + F), P);
  const GroupSmem<uint32_t>& s = wk.s;
  WarpPusher pusher = make_pusher(pushbuf);
  unsigned long long pops = 0, edges = 0;
  const uint32_t tid = threadIdx.x, B = blockDim.x;
  while (true) {
    const uint32_t nready = wk.acquire(P);
    if (!nready) break;
    for (uint32_t k = tid; k < nready; k += B) {
      const uint32_t item = s.item[k], v = item & ~kCheck;
      ATOS_GC_COUNT(v, item & kCheck);
      const uint32_t st = __ldg(c.row_ptr + v);
      s.start[k] = st;
      s.off[k] = __ldg(c.row_ptr + v + 1) - st;
      flag[k] = 0;
      if (item & kCheck) {
        cval[k] = ld_relaxed(c.color + v);
      } else {
        atom_and_acquire(c.inq + (v >> 5), ~(1u << (v & 31)));
        // a recolour (v already holds a colour: it lost a conflict) may spread its choice (see finalize):
        // flag[k] = the spread for this attempt, doubling with every recolour of v
        cval[k] = c.spread > 1 ? ld_relaxed(c.color + v) : -1;
        if (cval[k] >= 0 && !c.literal) {
          const uint32_t a = c.att[v];
          flag[k] = min(1u << min(a, 15u), c.spread);
          c.att[v] = (uint8_t)min(a + 1, 15u);
        }
      }
    }
    for (uint32_t i = tid; i < nready * 32; i += B) ibm[i] = 0;
    __syncthreads();
    uint32_t total = 0, mydeg = 0;
    const uint32_t per = (nready + B - 1) / B;
    const uint32_t i0 = min(tid * per, nready), i1 = min(i0 + per, nready);
    for (uint32_t i = i0; i < i1; ++i) mydeg += s.off[i];
    uint32_t excl = block_exclusive_scan(mydeg, s.ctr + 8, &total);
    for (uint32_t i = i0; i < i1; ++i) { const uint32_t d = s.off[i]; s.off[i] = excl; excl += d; }
    __syncthreads();
    edges += tid == 0 ? total : 0;
    // kUc CONSECUTIVE flattened edges per thread per iteration: one owner search per thread, all col
    // loads, then all colour loads, then the forbidden-set marks / conflict checks -- kUc independent
    // memory chains in flight per thread instead of one.
    for (uint32_t base = 0; base < total; base += B * kUc) {
      const uint32_t e0 = base + tid * kUc;
      uint32_t o = 0;
      if (e0 < total) {
        uint32_t lo = 0, hi = nready;
        while (hi - lo > 1) {
          const uint32_t mid = (lo + hi) >> 1;
          if (s.off[mid] <= e0) lo = mid; else hi = mid;
        }
        o = lo;
      }
      uint32_t w[kUc], own[kUc];
      int32_t cw[kUc];
      bool val[kUc], want[kUc];
      uint32_t out[kUc];
#pragma unroll
      for (int k = 0; k < kUc; ++k) {
        const uint32_t e = e0 + k;
        val[k] = e < total;
        if (val[k]) {
          while (o + 1 < nready && s.off[o + 1] <= e) ++o;
          own[k] = o;
          w[k] = __ldg(c.col + s.start[o] + (e - s.off[o]));
        }
      }
#pragma unroll
      for (int k = 0; k < kUc; ++k) {
        cw[k] = -1;
        if (val[k]) {
          val[k] = w[k] != (s.item[own[k]] & ~kCheck);
          if (val[k]) cw[k] = ld_relaxed(c.color + w[k]);
        }
      }
#pragma unroll
      for (int k = 0; k < kUc; ++k) {
        want[k] = false;
        out[k] = 0;
        if (!val[k]) continue;
        const uint32_t item = s.item[own[k]];
        if (!(item & kCheck)) {
          if (cw[k] >= 0 && cw[k] < (int32_t)kWin)
            atomicOr(ibm + own[k] * 32 + (cw[k] >> 5), 1u << (cw[k] & 31));
        } else if (cw[k] == cval[own[k]]) {
          if (c.literal || c.loses(item & ~kCheck, w[k])) flag[own[k]] = 1;
          else if (c.claim_assign(w[k])) { want[k] = true; out[k] = w[k]; }
        }
      }
      pusher.push_n<kUc>(P.q, want, out, P.watchdog_ns);
    }
    __syncthreads();
    // finalize: one warp per item
    for (uint32_t k0 = 0; k0 < nready; k0 += nwarps) {
      const uint32_t k = k0 + warp_id();
      bool want = false;
      uint32_t out = 0;
      if (k < nready) {
        const uint32_t item = s.item[k], v = item & ~kCheck;
        if (!(item & kCheck)) {
          int32_t chosen = -1;
          // free colours of the first window, limited to [0, deg(v)] so that colour <= deg(v) holds for
          // every choice (at most deg(v) of those deg(v)+1 colours are taken, so one is always free)
          const uint32_t dv = (k + 1 < nready ? s.off[k + 1] : total) - s.off[k];
          const uint32_t lo_c = lane_id() * 32;
          const uint32_t lim = dv >= lo_c + 31 ? 0xFFFFFFFFu : (dv < lo_c ? 0u : (0xFFFFFFFFu >> (31 - (dv - lo_c))));
          const uint32_t freebits = ~ibm[k * 32 + lane_id()] & lim;
          // Recolour spread: the vertices that keep losing in the dense core of a scale-free graph share
          // most of their neighbourhoods, so when several recolour concurrently they all find the SAME
          // smallest free colour and collide again (measured at C4: ranks 128..8192 by degree were
          // re-assigned 8-16x and took 80 % of the edge visits).  The a-th recolour of v takes the j-th
          // smallest free colour of the first window, j = splitmix64(seed ^ v ^ old colour) mod
          // min(2^(a-1), cfg.recolor_spread): the first assign and the first recolour keep Alg.6's smallest
          // free colour, and only vertices caught in a repeated collision spread out (R-GC-10).
          // Off by default (recolor_spread = 1): it trades colours for time (C4: 8.7 ms / 690 colours at 1,
          // 7.1 / 818 at 4, 6.7 / 910 at 8, 6.3 / 1017 at 16 -- DESIGN.md section 6).
          uint32_t j = 0;
          if (flag[k] > 1)
            j = (uint32_t)(splitmix64(c.seed ^ v ^ ((unsigned long long)(uint32_t)cval[k] << 32)) % flag[k]);
          const uint32_t cnt = __popc(freebits);
          uint32_t incl = cnt;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane_id() >= (uint32_t)o) incl += y;
          }
          const uint32_t nfree = __shfl_sync(0xffffffffu, incl, 31);
          if (nfree) {
            if (j >= nfree) j = nfree - 1;
            // the lane holding the j-th free bit picks it
            const bool mine = incl > j && incl - cnt <= j;
            const unsigned who = __ballot_sync(0xffffffffu, mine);
            const uint32_t L = __ffs(who) - 1;
            uint32_t fb = __shfl_sync(0xffffffffu, freebits, L);
            const uint32_t skip = j - (__shfl_sync(0xffffffffu, incl - cnt, L));
            for (uint32_t t = 0; t < skip; ++t) fb &= fb - 1;  // drop the lowest `skip` free bits
            chosen = (int32_t)(L * 32 + (__ffs(fb) - 1));
          } else {
            // window [0, 1024) is full: scan further windows with the warp
            const uint32_t st = __ldg(c.row_ptr + v), deg = __ldg(c.row_ptr + v + 1) - st;
            uint32_t* bm = wbm + warp_id() * 32;
            uint32_t wbase = kWin;
            while (chosen < 0) {
              bm[lane_id()] = 0;
              __syncwarp();
              for (uint32_t j = lane_id(); j < deg; j += 32) {
                const uint32_t w = __ldg(c.col + st + j);
                if (w == v) continue;
                const int32_t cw = ld_relaxed(c.color + w);
                if (cw >= (int32_t)wbase && cw < (int32_t)(wbase + kWin)) {
                  const uint32_t o = (uint32_t)cw - wbase;
                  atomicOr(bm + (o >> 5), 1u << (o & 31));
                }
              }
              __syncwarp();
              const uint32_t fb2 = ~bm[lane_id()];
              const unsigned m2 = __ballot_sync(0xffffffffu, fb2 != 0);
              if (m2) {
                const uint32_t L = __ffs(m2) - 1;
                const uint32_t f = __shfl_sync(0xffffffffu, fb2, L);
                chosen = (int32_t)(wbase + L * 32 + (__ffs(f) - 1));
              } else {
                wbase += kWin;
              }
              __syncwarp();
            }
          }
          if (lane_id() == 0) {
            st_relaxed(c.color + v, chosen);
            fence_sc_gpu();
          }
          __syncwarp();
          want = lane_id() == 0;
          out = v | kCheck;
        } else if (flag[k]) {
          want = lane_id() == 0 && c.claim_assign(v);
          out = v;
        }
      }
      pusher.push(P.q, want, out, P.watchdog_ns);
    }
    pops += tid == 0 ? nready : 0;
    pusher.flush(P.q, P.watchdog_ns);
    wk.complete(P, nready);
  }
  wk.flush_occ(P);
  flush_stats(P.q, pops, edges, lane_id() == 0 ? pusher.total : 0);
}

// -------------------------------------------------------------- thread worker
// Each lane colours its own vertices serially with a 64-colour register
// window; lanes advance in lock step so pushes stay warp-aggregated.
template <bool PERSIST>
__global__ void __launch_bounds__(1024) k_color_thread(ColorCtx c, EngineParams P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const uint32_t nwarps = blockDim.x >> 5;
  uint32_t* pushbuf = (uint32_t*)smem_raw;
  Worker<MODE_THREAD, PERSIST, uint32_t> wk;
  wk.init((unsigned char*)(pushbuf + nwarps * kPushBuf), P);
  const GroupSmem<uint32_t>& s = wk.s;
  WarpPusher pusher = make_pusher(pushbuf);
  unsigned long long pops = 0, edges = 0;
  const uint32_t lane = lane_id();
  while (true) {
    const uint32_t nready = wk.acquire(P);
    if (!nready) break;
    // per-lane state machine over items lane, lane+32, ...
    uint32_t k = lane, v = 0, item = 0, st = 0, deg = 0, j = 0, base = 0;
    unsigned long long used = 0;
    int32_t cv = 0;
    bool self = false, loaded = false;
    while (true) {
      bool want = false;
      uint32_t out = 0;
      if (k < nready && !loaded) {
        item = s.item[k];
        v = item & ~kCheck;
        st = __ldg(c.row_ptr + v);
        deg = __ldg(c.row_ptr + v + 1) - st;
        j = 0; base = 0; used = 0; self = false; loaded = true;
        if (item & kCheck) cv = ld_relaxed(c.color + v);
        else atom_and_acquire(c.inq + (v >> 5), ~(1u << (v & 31)));
      }
      const bool active = k < nready;
      if (__ballot_sync(0xffffffffu, active) == 0) break;
      if (active) {
        if (j < deg) {
          const uint32_t w = __ldg(c.col + st + j);
          ++j;
          ++edges;
          if (w != v) {
            const int32_t cw = ld_relaxed(c.color + w);
            if (!(item & kCheck)) {
              if (cw >= (int32_t)base && cw < (int32_t)(base + 64)) used |= 1ull << (cw - (int32_t)base);
            } else if (cw == cv) {
              if (c.literal || c.loses(v, w)) self = true;
              else if (c.claim_assign(w)) { want = true; out = w; }
            }
          }
        } else {
          // end of row
          if (!(item & kCheck)) {
            if (~used) {
              const int32_t chosen = (int32_t)(base + __ffsll((long long)~used) - 1);
              st_relaxed(c.color + v, chosen);
              fence_sc_gpu();
              want = true;
              out = v | kCheck;
              k += 32; loaded = false;
            } else {
              base += 64; used = 0; j = 0;  // next window: rescan the row
            }
          } else {
            if (self && c.claim_assign(v)) { want = true; out = v; }
            k += 32; loaded = false;
          }
        }
      }
      pusher.push(P.q, want, out, P.watchdog_ns);
    }
    pops += lane == 0 ? nready : 0;
    pusher.flush(P.q, P.watchdog_ns);
    wk.complete(P, nready);
  }
  wk.flush_occ(P);
  flush_stats(P.q, pops, edges, lane == 0 ? pusher.total : 0);
}

// ------------------------------------------------------------ init / finalize
// Seeded bijection on [0, 2^bits) (odd multiplies and xorshifts are each
// invertible modulo 2^bits), cycle-walked into [0, n): the seeded initial
// queue order of permute_init.
__device__ __forceinline__ uint32_t permute_index(uint32_t i, uint32_t n, uint32_t bits, unsigned long long seed) {
  const unsigned long long mask = (bits >= 32) ? 0xFFFFFFFFull : ((1ull << bits) - 1);
  const unsigned long long k = splitmix64(seed);
  const unsigned long long a1 = (k | 1ull) & mask, b1 = (k >> 32) & mask;
  const unsigned long long a2 = (splitmix64(k) | 1ull) & mask, b2 = (splitmix64(k) >> 32) & mask;
  const uint32_t sh = bits / 2 ? bits / 2 : 1;
  unsigned long long x = i;
  do {
    x = (x * a1 + b1) & mask;
    x ^= x >> sh;
    x = (x * a2 + b2) & mask;
    x ^= x >> sh;
  } while (x >= n);
  return (uint32_t)x;
}

// color = -1, every vertex queued as an assign task (Alg.6 line 1
// "same initialization as Algorithm 5"), in ID order or a seeded permutation.
// o2n (degree layout, layout.cu): the queue is seeded in the CALLER's vertex-id
// order (R-GC-6) -- entry i is the internal id of caller vertex i (or of the
// seeded permutation's i-th vertex).
__global__ void k_color_init(int32_t* color, uint32_t* inq, Ring q, uint32_t n,
                             int permute, uint32_t bits, unsigned long long seed, unsigned long long wd,
                             const uint32_t* __restrict__ o2n) {
  const unsigned long long t0 = q.ctl->done.v;  // set to the run's start index by k_color_begin
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    color[i] = -1;
    uint32_t v = permute ? permute_index(i, n, bits, seed) : i;
    if (o2n) v = o2n[v];
    publish_one(q, t0 + i, v, wd);
  }
  const uint32_t words = (n + 31) / 32;
  for (uint32_t w = blockIdx.x * blockDim.x + threadIdx.x; w < words; w += gridDim.x * blockDim.x) {
    const uint32_t lo = w * 32;
    inq[w] = (n - lo >= 32) ? 0xFFFFFFFFu : ((1u << (n - lo)) - 1u);
  }
}

__global__ void k_color_begin(QueueCtl* ctl, unsigned long long n) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    const unsigned long long t = ctl->tail.v;
    ctl->head.v = t;
    ctl->done.v = t;
    ctl->tail.v = t + n;  // the init kernel publishes indices [t, t+n)
    ctl->status.v = 0;
    ctl->stat_pops.v = 0;
    ctl->stat_pushes.v = n;
    ctl->stat_edges.v = 0;
    ctl->stat_maxocc.v = 0;
    ctl->misc.v = 0;
    ctl->tl_next.v = 0;
    ctl->tl_count.v = 0;
  }
}

__global__ void k_color_max(const int32_t* color, uint32_t n, unsigned long long* mx, unsigned* bad) {
  int32_t best = -1;
  for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
    const int32_t c = color[v];
    best = max(best, c);
    if (c < 0) atomicOr(bad, 1u);
  }
  for (int o = 16; o; o >>= 1) best = max(best, __shfl_xor_sync(0xffffffffu, best, o));
  if (lane_id() == 0 && best >= 0) atomicMax(mx, (unsigned long long)best);
}

// symmetry check (cfg.validate): every edge (u,w), u != w, has its reverse.
__global__ void k_check_symmetric(const uint32_t* __restrict__ row_ptr, const uint32_t* __restrict__ col,
                                  uint32_t n, unsigned* bad) {
  for (uint32_t u = blockIdx.x * (blockDim.x / 32) + warp_id(); u < n; u += gridDim.x * (blockDim.x / 32)) {
    const uint32_t a = row_ptr[u], b = row_ptr[u + 1];
    for (uint32_t e = a + lane_id(); e < b; e += 32) {
      const uint32_t w = col[e];
      if (w == u) continue;
      const uint32_t wa = row_ptr[w], wb = row_ptr[w + 1];
      // binary search (rows sorted), then a linear scan for unsorted rows
      uint32_t lo = wa, hi = wb;
      while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (col[mid] < u) lo = mid + 1; else hi = mid;
      }
      bool found = lo < wb && col[lo] == u;
      for (uint32_t f = wa; f < wb && !found; ++f) found = col[f] == u;
      if (!found) atomicOr(bad, 1u);
    }
  }
}

// ------------------------------------------------------------------ launcher
static inline uint64_t pow2_ceil(uint64_t x) {
  uint64_t c = 1;
  while (c < x) c <<= 1;
  return c;
}

template <class K>
static int launch_color_kernel(K kern_p, K kern_d, const ColorCtx& c, EngineParams P, const Resolved& r,
                               int block, size_t smem, uint64_t items_per_block, Part& p, atos_stats* st) {
  cudaStream_t s = r.stream;
  if (smem > 227 * 1024) {
    set_error("colouring: fetch_size %d with worker %d needs %zu B of shared memory", r.fetch, r.worker, smem);
    return ATOS_ERR_INVALID_ARG;
  }
  if (r.persistent) {
    const void* fn = (const void*)kern_p;
    if (smem > 48 * 1024) ATOS_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int grid = 0;
    ATOS_TRY(persistent_grid(fn, block, smem, &grid));
    if (r.num_blocks > 0) grid = std::min(grid, r.num_blocks);
    void* args[] = {(void*)&c, (void*)&P};
    ATOS_CUDA(cudaLaunchCooperativeKernel(fn, grid, block, args, smem, s));
    g_launches++;
    if (st) st->rounds += 1;
    return ATOS_OK;
  }
  const void* fn = (const void*)kern_d;
  if (smem > 48 * 1024) ATOS_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  unsigned long long* h = (unsigned long long*)p.host_pinned;
  QueueCtl* ctl = P.q.ctl;
  ATOS_CUDA(cudaMemcpyAsync(h, &ctl->head.v, 256, cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  uint64_t h0 = h[0], t0 = h[16];
  while (h0 < t0) {
    P.h0 = h0;
    P.t0 = t0;
    uint64_t grid = (t0 - h0 + items_per_block - 1) / items_per_block;
    void* args[] = {(void*)&c, (void*)&P};
    ATOS_CUDA(cudaLaunchKernel(fn, dim3((unsigned)std::min<uint64_t>(grid, 0x7FFFFFFF)), dim3(block), args, smem, s));
    g_launches++;
    if (st) st->rounds += 1;
    ATOS_CUDA(cudaMemcpyAsync(h, &ctl->tail.v, 8, cudaMemcpyDeviceToHost, s));
    ATOS_TRY(stream_wait(s, r.timeout_s));
    h0 = t0;
    t0 = h[0];
    if (t0 - h0 > p.ring_cap) {
      p.ring_clean = false;
      set_error("discrete colouring frontier exceeds the ring capacity");
      return ATOS_ERR_QUEUE_OVERFLOW;
    }
  }
  ATOS_CUDA(cudaMemcpyAsync(&ctl->head.v, &ctl->tail.v, 8, cudaMemcpyDeviceToDevice, s));
  ATOS_CUDA(cudaMemcpyAsync(&ctl->done.v, &ctl->tail.v, 8, cudaMemcpyDeviceToDevice, s));
  return ATOS_OK;
}

// cfg.validate: reject a non-symmetric CSR (R-GC-8).  Shared with the BSP baseline (bsp.cu).
int check_symmetric_if(Part& p, const Resolved& r) {
  if (!r.validate) return ATOS_OK;
  cudaStream_t s = r.stream;
  unsigned* bad = nullptr;
  ATOS_CUDA(cudaMalloc(&bad, 4));
  ATOS_CUDA(cudaMemsetAsync(bad, 0, 4, s));
  k_check_symmetric<<<1184, 256, 0, s>>>(p.row_ptr, p.col, (uint32_t)p.n_local, bad);
  g_launches++;
  unsigned hb = 0;
  ATOS_CUDA(cudaMemcpyAsync(&hb, bad, 4, cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  cudaFree(bad);
  if (hb) {
    set_error("atos_color: CSR is not symmetric");
    return ATOS_ERR_NOT_SYMMETRIC;
  }
  return ATOS_OK;
}

// colours used (max + 1); fails if a vertex is left uncoloured.
int color_count(Part& p, const int32_t* color, int64_t* used, cudaStream_t s) {
  const uint32_t n = (uint32_t)p.n_local;
  ATOS_TRY(p.scratch.ensure(64));
  unsigned long long* mx = p.scratch.as<unsigned long long>();
  unsigned* bad = (unsigned*)(mx + 1);
  ATOS_CUDA(cudaMemsetAsync(mx, 0, 16, s));
  k_color_max<<<592, 256, 0, s>>>(color, n, mx, bad);
  g_launches++;
  unsigned long long hm[2] = {0, 0};
  ATOS_CUDA(cudaMemcpyAsync(hm, mx, 16, cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  if ((unsigned)hm[1]) {
    set_error("colouring left a vertex uncoloured");
    return ATOS_ERR_CUDA;
  }
  *used = n ? (int64_t)hm[0] + 1 : 0;
  return ATOS_OK;
}

int color_single(atos_csr* g, Part& p, uint64_t seed, int32_t* color, const Resolved& r, atos_stats* st) {
  cudaStream_t s = r.stream;
  const uint32_t n = (uint32_t)p.n_local;
  ATOS_TRY(check_symmetric_if(p, r));
  // assign and check tasks of one vertex can both be queued: 2n outstanding + slack
  const uint64_t want = r.queue_capacity ? r.queue_capacity : std::max<uint64_t>(4ull * n, 4096);
  ATOS_TRY(ensure_queue(p, pow2_ceil(want), s));
  const size_t words = ((size_t)n + 31) / 32;
  ATOS_TRY(p.bitmap.ensure(words * 4 + ((size_t)n + 15) / 16 * 16));  // dedupe bits, then recolour counts
  ATOS_TRY(p.scratch.ensure(64));
  Ring q;
  q.slots = p.ring.as<unsigned long long>();
  q.mask = p.ring_cap - 1;
  q.ctl = p.ctl.as<QueueCtl>();
  ColorCtx c{p.row_ptr, p.col, color, p.bitmap.as<uint32_t>(), (uint8_t*)(p.bitmap.as<uint32_t>() + words),
             (uint32_t)std::max(1, r.recolor_spread), seed, r.conflict_policy == 1 ? 1 : 0,
             r.conflict_policy == 2 ? 1 : 0};
  if (c.spread > 1) ATOS_CUDA(cudaMemsetAsync(c.att, 0, (size_t)n, s));
  // init: reserve [t, t+n) then publish every vertex
  k_color_begin<<<1, 32, 0, s>>>(q.ctl, n);
  g_launches++;
  uint32_t bits = 1;
  while ((1ull << bits) < n) ++bits;
  if (bits < 2) bits = 2;
  k_color_init<<<1184, 256, 0, s>>>(color, c.inq, q, n, r.permute_init, bits, seed, r.watchdog_ns,
                                    g->relabeled ? g->o2n.as<uint32_t>() : nullptr);
  g_launches++;
  ATOS_CUDA(cudaGetLastError());
  p.ring_clean = false;
  EngineParams P;
  P.q = q;
  P.fetch = (uint32_t)r.fetch;
  P.watchdog_ns = r.watchdog_ns;
  P.h0 = P.t0 = 0;
  P.timeout_ns = r.timeout_s > 0 ? (unsigned long long)(r.timeout_s * 1e9) : 0ull;
  P.dbg_edge = nullptr;
  P.dbg_claim = nullptr;
  P.tl = r.timeline;
  P.tl_cap = r.timeline_cap;
  P.tl_interval_ns = r.timeline_interval_ns;
  P.big = nullptr;
  P.nbig = 0;
  P.big_threshold = 0xFFFFFFFFu;
  P.big_chunk = 1;
  // colouring claims down to 2 vertices when the visible queue is thin: fewer concurrently (re)assigned
  // dense-core vertices pick the same colour, so fewer recolour cascades (C4: 8.7 -> 7.8 ms, edge visits
  // 11.4 -> 10.0 per m, same colour count; profiles/r02_ab_min_claim.txt)
  P.min_claim = min_claim_for(2);
  const int mode = mode_of(r.worker);
  int rc;
#ifdef ATOS_GC_COUNTS
  uint32_t* dcounts = nullptr;
  const char* gc_out = getenv("ATOS_GC_COUNTS");
  if (gc_out) {
    ATOS_CUDA(cudaMalloc(&dcounts, (size_t)n * 8));
    ATOS_CUDA(cudaMemset(dcounts, 0, (size_t)n * 8));
  }
  ATOS_CUDA(cudaMemcpyToSymbol(g_gc_counts, &dcounts, sizeof(dcounts)));
#endif
  WorkerTimer wt;
  wt.start(s);
  if (mode == MODE_WARP) {
    const int block = r.block_threads, nw = block / 32;
    const size_t smem = (size_t)nw * kPushBuf * 4 + (size_t)nw * 32 * 4 + group_smem_bytes<uint32_t>(r.fetch) * nw;
    rc = launch_color_kernel(k_color_warp<true>, k_color_warp<false>, c, P, r, block, smem,
                             (uint64_t)r.fetch * nw, p, st);
  } else if (mode == MODE_CTA) {
    const int block = r.worker, nw = block / 32;
    const size_t smem = (size_t)nw * kPushBuf * 4 + (size_t)nw * 32 * 4 + (size_t)r.fetch * 32 * 4 +
                        (size_t)r.fetch * 8 + group_smem_bytes<uint32_t>(r.fetch);
    rc = launch_color_kernel(k_color_cta<true>, k_color_cta<false>, c, P, r, block, smem, (uint64_t)r.fetch, p, st);
  } else {
    const int block = r.block_threads, nw = block / 32;
    const size_t smem = (size_t)nw * kPushBuf * 4 + group_smem_bytes<uint32_t>(32u * r.fetch) * nw;
    rc = launch_color_kernel(k_color_thread<true>, k_color_thread<false>, c, P, r, block, smem,
                             (uint64_t)r.fetch * 32 * nw, p, st);
  }
  wt.stop(s);
#ifdef ATOS_GC_COUNTS
  if (dcounts) {
    std::vector<uint32_t> h((size_t)n * 2);
    cudaDeviceSynchronize();
    cudaMemcpy(h.data(), dcounts, (size_t)n * 8, cudaMemcpyDeviceToHost);
    if (FILE* f = fopen(gc_out, "wb")) {
      fwrite(h.data(), 4, h.size(), f);
      fclose(f);
    }
    cudaFree(dcounts);
    dcounts = nullptr;
    cudaMemcpyToSymbol(g_gc_counts, &dcounts, sizeof(dcounts));
  }
#endif
  if (rc != ATOS_OK) return rc;
  if (st) st->worker_ms += wt.elapsed();
  rc = finish_queue(p, s, st, "color");
  if (rc != ATOS_OK) return rc;
  int64_t used = 0;
  ATOS_TRY(color_count(p, color, &used, s));
  if (st) st->colors_used = used;
  return ATOS_OK;
}

}  // namespace atos
