// device.cuh -- memory-order helpers, warp utilities, the ring queue and the
// per-warp push buffer shared by every Atos worker kernel (sm_100a).
//
// Queue design (ours; the paper specifies only "concurrent_pop / concurrent_push"
// on a single shared queue, and push_warp):
//   * ring of C 64-bit slots (C a power of two), slot = (seq << 32) | item,
//     a per-slot sequence number in the style of Vyukov's bounded MPMC queue:
//       slot idx&mask is free for the producer of index idx  iff seq == idx,
//       it holds the item of index idx                         iff seq == idx+1,
//     (seq compared modulo 2^32);
//   * 64-bit monotone counters head (claims), tail (reservations), done
//     (completed tasks), each on its own 128-byte line; they persist across
//     runs (a run starts with head = done = tail), so the ring never needs
//     re-initialisation between calls;
//   * a producer reserves [t, t+k) with ONE atomicAdd per warp-batch and
//     publishes each slot with one st.release of (idx+1, item); a consumer
//     claims [h, h+k) with ONE atomicAdd per worker, waits (without blocking
//     its ready work) for seq == idx+1, takes the item and frees the slot for
//     the next lap with seq = idx + C.  Over-claimed indices (>= tail) are
//     therefore never confused with another lap's item;
//   * termination: done == tail read after an acquire of done (DESIGN.md
//     "Termination"): every reserved slot has been processed, so no task is in
//     flight and none can be produced.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace atos {

constexpr uint32_t kEmpty = 0xFFFFFFFFu;
constexpr uint32_t kUnreached = 0xFFFFFFFFu;

// status bits written by the device watchdog
constexpr uint32_t kStatusOverflow = 1u;
constexpr uint32_t kStatusTimeout = 2u;
constexpr uint32_t kStatusDeep = 4u;     // byte-state BFS met a depth it cannot encode (host re-runs)

struct __align__(128) Line64 {
  unsigned long long v;
  unsigned long long pad[15];
};

// Control block of one queue (device memory).  Statistics counters are
// accumulated per CTA and flushed once per CTA at kernel exit.
struct QueueCtl {
  Line64 head;
  Line64 tail;
  Line64 done;
  Line64 status;      // watchdog / overflow flags (u32 in .v)
  Line64 check;       // PageRank Check_Size sweep cursor
  Line64 stat_pops;
  Line64 stat_pushes;
  Line64 stat_edges;
  Line64 misc;        // app scratch (e.g. colouring: max colour)
  Line64 big_count;   // active big tasks (hub assist)
  Line64 big_rr;      // round-robin slot cursor for big-task registration
  Line64 tl_next;     // timeline: globaltimer of the next sample
  Line64 tl_count;    // timeline: samples taken
  Line64 stat_maxocc; // largest tail - head a worker saw at a claim (atos_stats.max_queue_occupancy)
};

struct Ring {
  unsigned long long* slots;  // C slots of (seq << 32 | item)
  unsigned long long mask;    // C - 1
  QueueCtl* ctl;
};

__device__ __forceinline__ unsigned long long make_slot(unsigned long long seq, uint32_t item) {
  return ((unsigned long long)(uint32_t)seq << 32) | item;
}

// ---------------------------------------------------------------- memory order
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_relaxed(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int32_t ld_relaxed(const int32_t* p) {
  int32_t v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ double ld_relaxed(const double* p) {
  double v;
  asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_acquire(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_release(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed(int32_t* p, int32_t v) {
  asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t atom_or_release(uint32_t* p, uint32_t v) {
  uint32_t old;
  asm volatile("atom.release.gpu.global.or.b32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  return old;
}
__device__ __forceinline__ uint32_t atom_and_acquire(uint32_t* p, uint32_t v) {
  uint32_t old;
  asm volatile("atom.acquire.gpu.global.and.b32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  return old;
}
__device__ __forceinline__ unsigned long long atom_add_release(unsigned long long* p, unsigned long long v) {
  unsigned long long old;
  asm volatile("atom.release.gpu.global.add.u64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
  return old;
}
__device__ __forceinline__ unsigned long long atom_read(unsigned long long* p) {
  // an RMW returns the latest value in the location's coherence order
  unsigned long long old;
  asm volatile("atom.acquire.gpu.global.or.b64 %0, [%1], 0;" : "=l"(old) : "l"(p) : "memory");
  return old;
}
__device__ __forceinline__ void red_add_f64(double* p, double v) {
  asm volatile("red.relaxed.gpu.global.add.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}
// L2 eviction-priority policies (createpolicy) and hinted loads: graph
// streams (col) are evict_first so they do not push the small hot state
// (shadow depth, bitmaps) out of the 126 MB L2.
__device__ __forceinline__ unsigned long long policy_evict_first() {
  unsigned long long p;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ unsigned long long policy_evict_last() {
  unsigned long long p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint32_t ld_stream(const uint32_t* a, unsigned long long pol) {
  uint32_t v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(a), "l"(pol));
  return v;
}
__device__ __forceinline__ uint32_t ld_u8_hint(const uint8_t* a, unsigned long long pol) {
  uint16_t v;
  asm volatile("ld.global.L2::cache_hint.u8 %0, [%1], %2;" : "=h"(v) : "l"(a), "l"(pol) : "memory");
  return v;
}
__device__ __forceinline__ void st_u8_hint(uint8_t* a, uint32_t v, unsigned long long pol) {
  asm volatile("st.global.L2::cache_hint.u8 [%0], %1, %2;" ::"l"(a), "h"((uint16_t)v), "l"(pol) : "memory");
}

// Queue counters (head / tail / done): every access carries an L2 evict_last cache-policy hint (the
// north_star's "L2 persistence hints on the queue counters"), so the few hot counter lines are the last
// candidates for eviction while the col stream (evict_first) and the state gathers churn through L2.
// (The stream's access-policy window -- cfg.l2_persist -- is spent on the per-vertex state instead.)
__device__ __forceinline__ unsigned long long ctr_policy() {
  unsigned long long p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ unsigned long long ctr_ld(const unsigned long long* a) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(a), "l"(ctr_policy()) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ctr_add(unsigned long long* a, unsigned long long x) {
  unsigned long long old;
  asm volatile("atom.relaxed.gpu.global.add.L2::cache_hint.u64 %0, [%1], %2, %3;"
               : "=l"(old) : "l"(a), "l"(x), "l"(ctr_policy()) : "memory");
  return old;
}
__device__ __forceinline__ void ctr_red_release(unsigned long long* a, unsigned long long x) {
  asm volatile("red.release.gpu.global.add.L2::cache_hint.u64 [%0], %1, %2;" ::"l"(a), "l"(x), "l"(ctr_policy())
               : "memory");
}
__device__ __forceinline__ unsigned long long ctr_read_acquire(unsigned long long* a) {
  // an RMW returns the latest value in the location's coherence order
  unsigned long long old;
  asm volatile("atom.acquire.gpu.global.or.L2::cache_hint.b64 %0, [%1], 0, %2;"
               : "=l"(old) : "l"(a), "l"(ctr_policy()) : "memory");
  return old;
}

__device__ __forceinline__ void fence_sc_gpu() { asm volatile("fence.sc.gpu;" ::: "memory"); }
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31u; }
__device__ __forceinline__ uint32_t warp_id() { return threadIdx.x >> 5; }
__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

// splitmix64 (Steele, Lea, Flood 2014): colouring priority pi(v) = splitmix64(seed ^ v).
// Implemented here independently of the oracle (shared only by name and constants).
__device__ __forceinline__ unsigned long long splitmix64(unsigned long long x) {
  unsigned long long z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// -------------------------------------------------------------------- pushing
__device__ __forceinline__ unsigned long long atom_cas_acq_rel(unsigned long long* p, unsigned long long cmp,
                                                           unsigned long long val) {
  unsigned long long old;
  asm volatile("atom.acq_rel.gpu.global.cas.b64 %0, [%1], %2, %3;"
               : "=l"(old) : "l"(p), "l"(cmp), "l"(val) : "memory");
  return old;
}

// Publish `item` at reserved index idx.  Normally the slot is free for this
// lap (seq == idx) and one release store publishes (idx+1, item).  If the slot
// still holds the previous lap's item (seq == idx-C+1) because its claimant is
// busy, the producer STEALS it with one CAS that publishes its own item in the
// same step, then re-publishes the stolen item at a freshly reserved index and
// counts the stolen index as done (after the re-publication, so termination
// can never be observed early).  The claimant sees the slot's seq past its
// index and drops the claim.  Producers therefore never wait on a busy
// consumer; they only wait (bounded, watchdog) for a previous-lap producer
// that reserved but has not yet written.
// CAS_PUB (latency-bound workers, see WarpPusherT): try the common case first -- the slot is free for this
// lap (seq == idx, item 0: exactly what the consumer's CAS left, or the initial state) -- with ONE release
// CAS instead of a read of the slot followed by a release store (one round trip less per publish; a thin
// high-diameter frontier pays it on every hop).  Throughput-bound workers keep the read + store (the CAS
// goes through the L2 atomic unit the relax atomics already load: C5 BFS +1 %).
template <bool CAS_PUB = false>
__device__ __forceinline__ void publish_one(const Ring& q, unsigned long long idx, uint32_t item,
                                            unsigned long long watchdog_ns) {
  const unsigned long long C = q.mask + 1;
  unsigned long long stolen = 0, t0 = 0;
  if (CAS_PUB &&
      atom_cas_acq_rel(q.slots + (idx & q.mask), make_slot(idx, 0u), make_slot(idx + 1, item)) == make_slot(idx, 0u))
    return;
  while (true) {
    unsigned long long* slot = q.slots + (idx & q.mask);
    const unsigned long long v = ld_relaxed(slot);
    const uint32_t seq = (uint32_t)(v >> 32);
    if (seq == (uint32_t)idx) {
      st_release(slot, make_slot(idx + 1, item));
      break;
    }
    if (seq == (uint32_t)(idx - C + 1)) {
      // previous lap's item still unconsumed: swap ours in, take it along
      if (atom_cas_acq_rel(slot, v, make_slot(idx + 1, item)) == v) {
        item = (uint32_t)v;
        ++stolen;
        idx = atomicAdd(&q.ctl->tail.v, 1ull);
        t0 = 0;
      }
      continue;
    }
    // the previous lap's producer has reserved but not yet written: wait, bounded
    if (t0 == 0) t0 = globaltimer();
    else if (globaltimer() - t0 > watchdog_ns) {
      atomicOr((unsigned int*)&q.ctl->status.v, kStatusOverflow);
      break;
    }
    __nanosleep(64);
  }
  if (stolen) atom_add_release(&q.ctl->done.v, stolen);
}

// Try to take the item of index idx: 1 = taken (*item set, slot freed for the
// next lap), 0 = not published yet, -1 = the item was stolen by a lap-blocked
// producer (drop the claim).
// ACQ = false: relaxed load and CAS (no CCTL.IVALL / MEMBAR per consumed item).
// Only valid for an app that reads nothing the pusher wrote before publishing:
// without the acquire, the PTX model does not order the consumer's later RMWs
// after the pusher's writes (every app in this library uses ACQ = true).
template <bool ACQ = true>
__device__ __forceinline__ int try_consume(const Ring& q, unsigned long long idx, uint32_t* item) {
  unsigned long long* slot = q.slots + (idx & q.mask);
  unsigned long long v;
  if (ACQ) asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(slot) : "memory");
  else asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(slot) : "memory");
  const int32_t d = (int32_t)((uint32_t)(v >> 32) - (uint32_t)(idx + 1));
  if (d < 0) return 0;
  if (d > 0) return -1;
  const unsigned long long freed = make_slot(idx + q.mask + 1, 0u);
  if ((ACQ ? atom_cas_acq_rel(slot, v, freed) : atomicCAS(slot, v, freed)) != v) return -1;
  *item = (uint32_t)v;
  return 1;
}

// Per-warp staging ring in shared memory (kPushBuf entries).  push_n() is
// warp-collective (all 32 lanes call it, each with up to N candidate items);
// entries accumulate and are published 32 at a time: one atomicAdd on tail
// per 32 pushes and one coalesced release store per lane.  flush() publishes
// the remainder.  (The paper's push_warp, aggregated to whole lines.)
constexpr uint32_t kPushBuf = 256;

template <bool CAS_PUB = false>
struct WarpPusherT {
  uint32_t* buf;      // kPushBuf entries of shared memory owned by this warp
  uint32_t head;      // warp-uniform ring head
  uint32_t cnt;       // warp-uniform fill level (< 32 between calls)
  uint32_t total;     // warp-uniform number of pushes issued (stats)

  __device__ __forceinline__ void publish(const Ring& q, uint32_t k, unsigned long long watchdog_ns) {
    // k <= 32 entries at buf[head .. head+k)
    unsigned long long base = 0;
    if (lane_id() == 0) base = ctr_add(&q.ctl->tail.v, (unsigned long long)k);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (lane_id() < k)
      publish_one<CAS_PUB>(q, base + lane_id(), buf[(head + lane_id()) & (kPushBuf - 1)], watchdog_ns);
    head = (head + k) & (kPushBuf - 1);
    cnt -= k;
    total += k;
  }

  template <int N>
  __device__ __forceinline__ void push_n(const Ring& q, const bool (&want)[N], const uint32_t (&item)[N],
                                         unsigned long long watchdog_ns) {
    uint32_t c = 0;
#pragma unroll
    for (int k = 0; k < N; ++k) c += want[k] ? 1u : 0u;
    if (!__any_sync(0xffffffffu, c != 0)) return;  // common case late in a run: nothing to push
    uint32_t incl = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane_id() >= (uint32_t)o) incl += y;
    }
    const uint32_t sum = __shfl_sync(0xffffffffu, incl, 31);
    if (sum == 0) return;
    uint32_t pos = head + cnt + incl - c;
#pragma unroll
    for (int k = 0; k < N; ++k)
      if (want[k]) buf[(pos++) & (kPushBuf - 1)] = item[k];
    cnt += sum;
    __syncwarp();
    while (cnt >= 32) {
      publish(q, 32, watchdog_ns);
      __syncwarp();
    }
  }

  __device__ __forceinline__ void push(const Ring& q, bool want, uint32_t item, unsigned long long watchdog_ns) {
    const bool w[1] = {want};
    const uint32_t it[1] = {item};
    push_n<1>(q, w, it, watchdog_ns);
  }

  __device__ __forceinline__ void flush(const Ring& q, unsigned long long watchdog_ns) {
    if (cnt) publish(q, cnt, watchdog_ns);
    __syncwarp();
  }
};

// the calling warp's pusher over a per-block array of kPushBuf-entry rings
using WarpPusher = WarpPusherT<false>;
template <bool CAS_PUB = false>
__device__ __forceinline__ WarpPusherT<CAS_PUB> make_pusher(uint32_t* bufs) {
  return WarpPusherT<CAS_PUB>{bufs + warp_id() * kPushBuf, 0u, 0u, 0u};
}

// -------------------------------------------------------- block-wide helpers
// exclusive scan of one value per thread; returns the exclusive prefix and
// writes the block total to *total.  tmp: shared scratch of >= 32 words.
__device__ __forceinline__ uint32_t block_exclusive_scan(uint32_t x, uint32_t* tmp, uint32_t* total) {
  uint32_t lane = lane_id(), wid = warp_id(), nw = (blockDim.x + 31) >> 5;
  uint32_t incl = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= (uint32_t)o) incl += y;
  }
  if (lane == 31) tmp[wid] = incl;
  __syncthreads();
  if (wid == 0) {
    uint32_t w = lane < nw ? tmp[lane] : 0;
    uint32_t wi = w;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, wi, o);
      if (lane >= (uint32_t)o) wi += y;
    }
    if (lane < nw) tmp[lane] = wi - w;   // exclusive warp offsets
    if (lane == nw - 1) tmp[32] = wi;    // total
  }
  __syncthreads();
  uint32_t r = tmp[wid] + incl - x;
  *total = tmp[32];
  __syncthreads();
  return r;
}

}  // namespace atos
