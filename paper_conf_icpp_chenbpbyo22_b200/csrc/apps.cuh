// apps.cuh -- relax policies of the two edge-relax applications.
#pragma once
#include "device.cuh"

namespace atos {

// ------------------------------------------------------------------- BFS
// Speculative BFS relax (Alg.2, Listing 4):
//   pop v, d = depth[v]; for each neighbour w: old = atomicMin(depth+w, d+1);
//   if d+1 < old: push w.
// B200 additions:
//   * prefilter: a plain load of depth[w] first; depth only decreases, so a
//     stale value is an upper bound and `cur <= d+1` safely skips the atomic;
//   * dedupe (optional): in-queue bitmap; the activator sets the bit with a
//     release RMW after its atomicMin and pushes only if the bit was clear;
//     the popper clears it with an acquire RMW BEFORE reading depth[v], so
//     every improvement after that read re-queues v (no update is lost).
//   * shadow depth (B200 addition): a u8 copy
//     min(depth, 254) with 255 = "unvisited or >= 255", n bytes (67 MB at
//     scale 26) -- small enough to stay in the 126 MB L2 (loads evict_last,
//     the col stream evict_first), so the per-edge prefilter almost never
//     touches HBM.  Written after a successful atomicMin; concurrent writers
//     can only leave a value depth[w] once held, so it stays an upper bound.
struct BfsApp {
  using Payload = uint32_t;  // d + 1
  const uint32_t* __restrict__ row_ptr;
  const uint32_t* __restrict__ col;
  uint32_t* depth;
  uint32_t* inq;      // nullptr -> paper-literal push on every improvement
  uint8_t* shadow;    // nullptr -> prefilter on depth[] itself
  unsigned long long pol_first, pol_last;

  __device__ __forceinline__ uint32_t neighbor(uint32_t e) const { return ld_stream(col + e, pol_first); }
  __device__ __forceinline__ void prepare() {
    pol_first = policy_evict_first();
    pol_last = policy_evict_last();
  }

  __device__ __forceinline__ bool begin(uint32_t v, uint32_t& start, uint32_t& deg, Payload& p) const {
    if (inq) atom_and_acquire(inq + (v >> 5), ~(1u << (v & 31)));
    const uint32_t d = ld_relaxed(depth + v);  // coherent read (L2): the value that caused the push
    start = __ldg(row_ptr + v);
    deg = __ldg(row_ptr + v + 1) - start;
    p = d + 1;
    return deg != 0;
  }

  __device__ __forceinline__ bool relax(const Payload nd, uint32_t w, uint32_t& out) const {
    bool need_depth_check = true;
    if (shadow) {
      const uint32_t sh = ld_u8_hint(shadow + w, pol_last);
      if (sh != 255u && sh <= nd) return false;
      need_depth_check = nd >= 255u;  // sh == 255 && nd < 255: unvisited or deeper -> must improve
    }
    if (need_depth_check) {
      uint32_t cur;
      asm volatile("ld.global.u32 %0, [%1];" : "=r"(cur) : "l"(depth + w));
      if (cur <= nd) return false;
    }
    const uint32_t old = atomicMin(depth + w, nd);
    if (old <= nd) return false;
    if (shadow) st_u8_hint(shadow + w, nd < 255u ? nd : 255u, pol_last);
    if (inq) {
      const uint32_t bit = 1u << (w & 31);
      if (atom_or_release(inq + (w >> 5), bit) & bit) return false;
    }
    out = w;
    return true;
  }
};

// -------------------------------------------------------------- PageRank
// Asynchronous push PageRank relax (Alg.4):
//   res = atomicExch(residue+v, 0); atomicAdd(rank+v, res);
//   res = res*lambda/deg(v); for each neighbour: atomicAdd(residue+w, res)
// Activation (DESIGN.md R-PR-6): w is pushed iff its residue crosses eps from
// below (old <= eps < old + delta, evaluated in the same fp64 rounding as the
// atomic), which keeps "residue[v] > eps  =>  v queued or in flight".
struct PrApp {
  using Payload = double;  // delta = alpha * rho / deg(v)
  const uint32_t* __restrict__ row_ptr;
  const uint32_t* __restrict__ col;
  unsigned long long pol_first;
  __device__ __forceinline__ uint32_t neighbor(uint32_t e) const { return ld_stream(col + e, pol_first); }
  __device__ __forceinline__ void prepare() { pol_first = policy_evict_first(); }
  double* rank;
  double* res;
  double alpha, eps;
  int activate;  // 1: crossing activation (default); 0: sweep-only (Check_Size variant)

  __device__ __forceinline__ bool begin(uint32_t v, uint32_t& start, uint32_t& deg, Payload& p) const {
    const double rho = __longlong_as_double(
        (long long)atomicExch((unsigned long long*)(res + v), 0ull));
    if (rho != 0.0) red_add_f64(rank + v, rho);
    start = __ldg(row_ptr + v);
    deg = __ldg(row_ptr + v + 1) - start;
    if (deg == 0 || rho == 0.0) return false;  // dangling: absorb (R-PR-3)
    p = alpha * rho / (double)deg;
    return true;
  }

  __device__ __forceinline__ bool relax(const Payload delta, uint32_t w, uint32_t& out) const {
    const double old = atomicAdd(res + w, delta);
    if (activate && old <= eps && old + delta > eps) {
      out = w;
      return true;
    }
    return false;
  }
};

}  // namespace atos
