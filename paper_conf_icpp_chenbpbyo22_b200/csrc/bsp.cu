// bsp.cu -- the bulk-synchronous (BSP) baselines the paper measures Atos
// against, on the same device, CSR and conventions:
//   * Alg.1 BFS: per level, advance the input frontier with
//                       atomicMin(dist, d+1) and append improved neighbours to
//                       the output frontier; host barrier; swap.
//   * Alg.3 PageRank: same init as the asynchronous version; per
//                       iteration push every frontier vertex's residue
//                       (atomicExch, rank += res, atomicAdd to neighbours),
//                       barrier, then rebuild the frontier as every vertex with
//                       residue > eps (a filter over all n), barrier.
//   * Alg.5 colouring: per iteration an assign kernel (smallest
//                       colour not used by a neighbour, forbidden sets windowed
//                       as R-GC-4) then, after a barrier, a conflict kernel
//                       whose conflicting vertices form the next frontier.
//                       Alg.5 appends BOTH endpoints of a conflict; read as
//                       R-GC-2 (the lower-priority endpoint, priority = degree,
//                       then splitmix64(seed ^ v)), literal policy as the knob
//                       conflict_policy = 1 (may livelock; honours timeout_s).
// The barrier is the host round trip of the paper's cudaDeviceSynchronize()
// (the frontier size is read back every iteration).
//
// B200 design (the baseline is given the same care as the Atos path, so the
// comparison measures scheduling, not implementation effort): frontier
// expansion is edge-balanced like Gunrock's LB advance -- a degree pass, a
// device-wide exclusive scan (CUB) and an advance kernel whose CTAs take
// 2048-edge tiles, stage the tile's owner range (offsets, rows) in shared
// memory and binary-search owners there; appends are warp-aggregated (one
// atomicAdd per warp).  Colouring uses a warp per vertex with a 1024-colour
// shared-memory window, like the asynchronous warp worker.
#include <cub/device/device_scan.cuh>

#include <algorithm>
#include <chrono>

#include "internal.h"

namespace atos {

namespace {

constexpr int kBT = 256;              // advance block
constexpr int kEPT = 8;               // edges per thread per tile
constexpr uint32_t kTile = kBT * kEPT;
constexpr uint32_t kOwnCap = kTile;   // owner range staged in smem when it fits
constexpr int kGrid = 148 * 8;        // grid-stride kernels: 8 CTAs per SM

// warp-aggregated append of `item` where want (one atomicAdd per warp)
__device__ __forceinline__ void append(uint32_t* out, unsigned long long* nout, bool want, uint32_t item) {
  const unsigned m = __ballot_sync(0xffffffffu, want);
  if (!m) return;
  unsigned long long base = 0;
  if (lane_id() == 0) base = atomicAdd(nout, (unsigned long long)__popc(m));
  base = __shfl_sync(0xffffffffu, base, 0);
  if (want) out[base + __popc(m & ((1u << lane_id()) - 1u))] = item;
}

// last index i in [lo, hi] with off[i] <= e (off non-decreasing, off[lo] <= e)
__device__ __forceinline__ uint32_t owner_of(const uint32_t* off, uint32_t lo, uint32_t hi, uint32_t e) {
  while (lo < hi) {
    const uint32_t mid = lo + ((hi - lo + 1) >> 1);
    if (off[mid] <= e) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// --------------------------------------------------------------- frontier prep
// BFS: deg[i] of frontier vertex i (deg[F] = 0 so the exclusive scan yields the total).
__global__ void k_bsp_degrees(const uint32_t* __restrict__ row_ptr, const uint32_t* __restrict__ front, uint32_t F,
                              uint32_t* deg) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i <= F; i += gridDim.x * blockDim.x) {
    uint32_t d = 0;
    if (i < F) {
      const uint32_t v = front[i];
      d = __ldg(row_ptr + v + 1) - __ldg(row_ptr + v);
    }
    deg[i] = d;
  }
}

// PageRank (Alg.3): res = atomicExch(residue[v], 0); rank[v] += res;
// delta = lambda * res / deg(v), kept per frontier slot for the advance.
// deg(v) = 0: the residue is absorbed and nothing is pushed (R-PR-3).
__global__ void k_bsp_pr_prep(const uint32_t* __restrict__ row_ptr, const uint32_t* __restrict__ front, uint32_t F,
                              double* rank, double* res, double alpha, uint32_t* deg, double* delta) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i <= F; i += gridDim.x * blockDim.x) {
    uint32_t d = 0;
    if (i < F) {
      const uint32_t v = front[i];
      const double rho = __longlong_as_double((long long)atomicExch((unsigned long long*)(res + v), 0ull));
      rank[v] += rho;  // a vertex is in the frontier once: plain add
      d = __ldg(row_ptr + v + 1) - __ldg(row_ptr + v);
      delta[i] = d ? alpha * rho / (double)d : 0.0;
    }
    deg[i] = d;
  }
}

// ------------------------------------------------------------------- advance
// Edge-balanced advance over the flattened edge list of the frontier:
// off[0..F] is the exclusive scan of the frontier degrees (off[F] = total).
// Op::edge(i, v, w, out) relaxes edge (v -> w) of frontier slot i and returns
// true to append `out` to the output frontier.
template <class Op>
__global__ void __launch_bounds__(kBT) k_bsp_advance(Op op, const uint32_t* __restrict__ row_ptr,
                                                     const uint32_t* __restrict__ col,
                                                     const uint32_t* __restrict__ front,
                                                     const uint32_t* __restrict__ off, uint32_t F, uint32_t* out,
                                                     unsigned long long* nout, unsigned long long* reset,
                                                     unsigned long long* stat_edges) {
  __shared__ uint32_t s_off[kOwnCap + 1];
  __shared__ uint32_t s_start[kOwnCap];
  __shared__ uint32_t s_v[kOwnCap];
  __shared__ uint32_t s_lohi[2];
  const uint32_t total = off[F];
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    if (reset) *reset = 0;  // the next iteration's append counter (read by the host last iteration)
    *stat_edges += total;
  }
  for (uint64_t t = blockIdx.x; t * kTile < total; t += gridDim.x) {
    const uint32_t e0 = (uint32_t)(t * kTile);
    const uint32_t e1 = (uint32_t)std::min<uint64_t>((uint64_t)e0 + kTile, total);
    if (threadIdx.x == 0) s_lohi[0] = owner_of(off, 0, F - 1, e0);
    if (threadIdx.x == 32) s_lohi[1] = owner_of(off, 0, F - 1, e1 - 1);
    __syncthreads();
    const uint32_t lo = s_lohi[0], hi = s_lohi[1];
    const uint32_t cnt = hi - lo + 1;
    const bool staged = cnt <= kOwnCap;
    if (staged) {
      for (uint32_t i = threadIdx.x; i < cnt; i += kBT) {
        const uint32_t v = front[lo + i];
        s_off[i] = off[lo + i];
        s_v[i] = v;
        s_start[i] = __ldg(row_ptr + v);
      }
    }
    __syncthreads();
#pragma unroll 2
    for (int k = 0; k < kEPT; ++k) {
      const uint32_t e = e0 + k * kBT + threadIdx.x;  // strided: each load instruction is coalesced
      bool want = false;
      uint32_t o = 0;
      if (e < e1) {
        uint32_t i, v, st, base;
        if (staged) {
          i = owner_of(s_off, 0, cnt - 1, e);
          v = s_v[i];
          st = s_start[i];
          base = s_off[i];
          i += lo;
        } else {
          i = owner_of(off, lo, hi, e);
          v = front[i];
          st = __ldg(row_ptr + v);
          base = off[i];
        }
        const uint32_t w = __ldg(col + st + (e - base));
        want = op.edge(i, v, w, o);
      }
      if (Op::kAppends) append(out, nout, want, o);
    }
    __syncthreads();
  }
}

struct BfsOp {
  static constexpr bool kAppends = true;
  uint32_t* depth;
  uint32_t nd;  // level + 1
  __device__ __forceinline__ bool edge(uint32_t, uint32_t, uint32_t w, uint32_t& out) const {
    if (ld_relaxed(depth + w) <= nd) return false;  // depth only decreases: a stale read is an upper bound
    const uint32_t old = atomicMin(depth + w, nd);  // Alg.1
    out = w;
    return old > nd;
  }
};

struct PrOp {
  static constexpr bool kAppends = false;
  double* res;
  const double* delta;
  __device__ __forceinline__ bool edge(uint32_t i, uint32_t, uint32_t w, uint32_t&) const {
    red_add_f64(res + w, delta[i]);  // Alg.3
    return false;
  }
};

__global__ void k_bsp_bfs_init(uint32_t* depth, uint32_t src, uint32_t* front) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    depth[src] = 0;
    front[0] = src;
  }
}

// Alg.3: frontier = every vertex with residue > eps.
__global__ void k_bsp_pr_filter(const double* __restrict__ res, uint32_t n, double eps, uint32_t* out,
                                unsigned long long* nout, unsigned long long* reset) {
  if (blockIdx.x == 0 && threadIdx.x == 0) *reset = 0;
  for (uint32_t b = blockIdx.x * blockDim.x; b < n; b += gridDim.x * blockDim.x) {
    const uint32_t v = b + threadIdx.x;
    append(out, nout, v < n && res[v] > eps, v);
  }
}

// ------------------------------------------------------------------ colouring
// R-GC-2, as the asynchronous path: lower degree loses, then lower hash priority, then lower id
// (policy 2: hash priority only)
__device__ __forceinline__ bool bsp_loses(const uint32_t* __restrict__ row_ptr, int hash_only,
                                          unsigned long long seed, uint32_t x, uint32_t y) {
  if (!hash_only) {
    const uint32_t dx = __ldg(row_ptr + x + 1) - __ldg(row_ptr + x);
    const uint32_t dy = __ldg(row_ptr + y + 1) - __ldg(row_ptr + y);
    if (dx != dy) return dx < dy;
  }
  const unsigned long long px = splitmix64(seed ^ x), py = splitmix64(seed ^ y);
  return px < py || (px == py && x < y);
}

constexpr uint32_t kWinB = 1024;

// Alg.5: a warp per frontier vertex; forbidden colours of the
// neighbours in a 1024-colour window (next window when full, so colour <= deg).
__global__ void __launch_bounds__(256) k_bsp_color_assign(const uint32_t* __restrict__ row_ptr,
                                                          const uint32_t* __restrict__ col, int32_t* color,
                                                          const uint32_t* __restrict__ front, uint32_t F,
                                                          unsigned long long* edges) {
  __shared__ uint32_t s_bm[8][32];
  uint32_t* bm = s_bm[warp_id()];
  const uint32_t lane = lane_id();
  unsigned long long my_edges = 0;
  for (uint32_t i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < F; i += (gridDim.x * blockDim.x) >> 5) {
    const uint32_t v = front[i];
    const uint32_t st = __ldg(row_ptr + v), deg = __ldg(row_ptr + v + 1) - st;
    uint32_t base = 0;
    int32_t chosen = -1;
    while (chosen < 0) {
      bm[lane] = 0;
      __syncwarp();
      for (uint32_t j = lane; j < deg; j += 32) {
        const uint32_t w = __ldg(col + st + j);
        if (w == v) continue;  // R-GC-7
        const int32_t cw = ld_relaxed(color + w);
        if (cw >= (int32_t)base && cw < (int32_t)(base + kWinB)) {
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
        base += kWinB;
      }
      __syncwarp();
    }
    if (lane == 0) {
      st_relaxed(color + v, chosen);
      my_edges += deg;
    }
  }
  if (lane == 0 && my_edges) atomicAdd(edges, my_edges);
}

// Alg.5: conflicting frontier vertices form the next frontier.
__global__ void __launch_bounds__(256) k_bsp_color_conflicts(const uint32_t* __restrict__ row_ptr,
                                                             const uint32_t* __restrict__ col,
                                                             const int32_t* __restrict__ color,
                                                             const uint32_t* __restrict__ front, uint32_t F,
                                                             unsigned long long seed, int literal /* conflict_policy */, uint32_t* out,
                                                             unsigned long long* nout, unsigned long long* reset,
                                                             unsigned long long* edges) {
  if (blockIdx.x == 0 && threadIdx.x == 0) *reset = 0;
  const uint32_t lane = lane_id();
  unsigned long long my_edges = 0;
  for (uint32_t i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < F; i += (gridDim.x * blockDim.x) >> 5) {
    const uint32_t v = front[i];
    const uint32_t st = __ldg(row_ptr + v), deg = __ldg(row_ptr + v + 1) - st;
    const int32_t cv = color[v];
    bool bad = false;
    for (uint32_t j = lane; j < deg && !bad; j += 32) {
      const uint32_t w = __ldg(col + st + j);
      if (w != v && color[w] == cv && (literal == 1 || bsp_loses(row_ptr, literal == 2, seed, v, w))) bad = true;
    }
    const bool any = __ballot_sync(0xffffffffu, bad) != 0;
    if (lane == 0) {
      my_edges += deg;
      if (any) out[atomicAdd(nout, 1ull)] = v;
    }
  }
  if (lane == 0 && my_edges) atomicAdd(edges, my_edges);
}

__global__ void k_bsp_iota(uint32_t* front, uint32_t n) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) front[i] = i;
}

// ------------------------------------------------------------------ host side
struct BspBufs {
  uint32_t *fa, *fb, *off;
  unsigned long long* ctr;  // [0] / [2] append counters of even / odd iterations, [1] edges
  void* cub_tmp;
  size_t cub_bytes;
};

int bsp_buffers(Part& p, uint64_t n, bool need_off, BspBufs* b, cudaStream_t s) {
  ATOS_TRY(p.bsp_fa.ensure((size_t)std::max<uint64_t>(n, 1) * 4));
  ATOS_TRY(p.bsp_fb.ensure((size_t)std::max<uint64_t>(n, 1) * 4));
  ATOS_TRY(p.bsp_ctr.ensure(64));
  b->fa = p.bsp_fa.as<uint32_t>();
  b->fb = p.bsp_fb.as<uint32_t>();
  b->ctr = p.bsp_ctr.as<unsigned long long>();
  b->off = nullptr;
  b->cub_tmp = nullptr;
  b->cub_bytes = 0;
  if (need_off) {
    ATOS_TRY(p.bsp_off.ensure((size_t)(n + 1) * 4));
    b->off = p.bsp_off.as<uint32_t>();
    size_t bytes = 0;
    ATOS_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, bytes, b->off, b->off, (int)(n + 1), s));
    ATOS_TRY(p.bsp_tmp.ensure(std::max<size_t>(bytes, 16)));
    b->cub_tmp = p.bsp_tmp.p;
    b->cub_bytes = bytes;
  }
  if (!p.host_pinned) ATOS_TRY(pinned_page(&p.host_pinned));
  ATOS_CUDA(cudaMemsetAsync(b->ctr, 0, 64, s));
  return ATOS_OK;
}

// one iteration's barrier: read the output frontier size (the kernels of the next
// iteration zero the counter after next, so no memset sits on the critical path)
int bsp_barrier(Part& p, unsigned long long* ctr, uint64_t* nout, const Resolved& r,
                std::chrono::steady_clock::time_point t_start) {
  unsigned long long* h = (unsigned long long*)p.host_pinned;
  ATOS_CUDA(cudaMemcpyAsync(h, ctr, 8, cudaMemcpyDeviceToHost, r.stream));
  ATOS_TRY(stream_wait(r.stream, r.timeout_s));
  *nout = h[0];
  if (r.timeout_s > 0 &&
      std::chrono::duration<double>(std::chrono::steady_clock::now() - t_start).count() > r.timeout_s) {
    set_error("BSP iteration did not converge within timeout_s=%.3f", r.timeout_s);
    return ATOS_ERR_TIMEOUT;
  }
  return ATOS_OK;
}

inline int grid_for(uint64_t items, int per_block) {
  return (int)std::max<uint64_t>(1, std::min<uint64_t>((items + per_block - 1) / per_block, kGrid));
}

int read_edges(Part& p, unsigned long long* ctr, atos_stats* st, cudaStream_t s) {
  if (!st) return ATOS_OK;
  unsigned long long* h = (unsigned long long*)p.host_pinned;
  ATOS_CUDA(cudaMemcpyAsync(h, ctr + 1, 8, cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  st->edges += h[0];
  return ATOS_OK;
}

}  // namespace

int bfs_bsp_single(atos_csr* g, Part& p, int64_t src, uint32_t* depth, const Resolved& r, atos_stats* st) {
  cudaStream_t s = r.stream;
  const uint64_t n = (uint64_t)p.n_local;
  BspBufs b;
  ATOS_TRY(bsp_buffers(p, n, true, &b, s));
  ATOS_CUDA(cudaMemsetAsync(depth, 0xFF, n * 4, s));  // Alg.1
  k_bsp_bfs_init<<<1, 32, 0, s>>>(depth, (uint32_t)src, b.fa);
  g_launches++;
  WorkerTimer wt;
  wt.start(s);
  const auto t0 = std::chrono::steady_clock::now();
  uint64_t F = 1;
  uint32_t level = 0;
  while (F > 0) {
    k_bsp_degrees<<<grid_for(F + 1, 256), 256, 0, s>>>(p.row_ptr, b.fa, (uint32_t)F, b.off);
    ATOS_CUDA(cub::DeviceScan::ExclusiveSum(b.cub_tmp, b.cub_bytes, b.off, b.off, (int)(F + 1), s));
    unsigned long long* cnt = b.ctr + 2 * (level & 1);
    k_bsp_advance<BfsOp><<<kGrid, kBT, 0, s>>>(BfsOp{depth, level + 1}, p.row_ptr, p.col, b.fa, b.off,
                                                (uint32_t)F, b.fb, cnt, b.ctr + 2 * ((level + 1) & 1), b.ctr + 1);
    g_launches += 4;  // degrees, CUB scan (init + scan), advance
    ATOS_CUDA(cudaGetLastError());
    if (st) { st->pops += F; st->rounds += 1; }
    uint64_t nf = 0;
    ATOS_TRY(bsp_barrier(p, cnt, &nf, r, t0));  // cudaDeviceSynchronize()
    if (st) st->pushes += nf;
    std::swap(b.fa, b.fb);
    F = nf;
    ++level;
  }
  wt.stop(s);
  ATOS_TRY(read_edges(p, b.ctr, st, s));
  if (st) st->worker_ms += wt.elapsed();
  return ATOS_OK;
}

int pagerank_bsp_single(atos_csr* g, Part& p, double alpha, double eps, double* rank, const Resolved& r,
                        atos_stats* st) {
  cudaStream_t s = r.stream;
  const uint64_t n = (uint64_t)p.n_local;
  BspBufs b;
  ATOS_TRY(bsp_buffers(p, n, true, &b, s));
  ATOS_TRY(p.vbuf_a.ensure(n * 8));
  ATOS_TRY(p.vbuf_b.ensure((n + 1) * 8));
  ATOS_TRY(p.scratch.ensure(64));
  double* res = p.vbuf_a.as<double>();
  double* delta = p.vbuf_b.as<double>();
  ATOS_TRY(pr_init_state(p, alpha, rank, res, s));  // Alg.3 P:761-767 (R-PR-init), shared with Alg.4
  WorkerTimer wt;
  wt.start(s);
  const auto t0 = std::chrono::steady_clock::now();
  // initial frontier: every vertex with residue > eps (R-PR-7)
  k_bsp_pr_filter<<<kGrid, 256, 0, s>>>(res, (uint32_t)n, eps, b.fa, b.ctr, b.ctr + 2);
  g_launches++;
  uint64_t F = 0;
  ATOS_TRY(bsp_barrier(p, b.ctr, &F, r, t0));
  uint32_t it = 1;
  if (st) st->pushes += F;
  while (F > 0) {
    k_bsp_pr_prep<<<grid_for(F + 1, 256), 256, 0, s>>>(p.row_ptr, b.fa, (uint32_t)F, rank, res, alpha, b.off,
                                                         delta);
    ATOS_CUDA(cub::DeviceScan::ExclusiveSum(b.cub_tmp, b.cub_bytes, b.off, b.off, (int)(F + 1), s));
    k_bsp_advance<PrOp><<<kGrid, kBT, 0, s>>>(PrOp{res, delta}, p.row_ptr, p.col, b.fa, b.off, (uint32_t)F,
                                               nullptr, nullptr, nullptr, b.ctr + 1);
    // barrier, then the frontier filter over all vertices
    unsigned long long* cnt = b.ctr + 2 * (it & 1);
    k_bsp_pr_filter<<<kGrid, 256, 0, s>>>(res, (uint32_t)n, eps, b.fb, cnt, b.ctr + 2 * ((it + 1) & 1));
    ++it;
    g_launches += 5;  // prep, CUB scan (init + scan), advance, filter
    ATOS_CUDA(cudaGetLastError());
    if (st) { st->pops += F; st->rounds += 1; }
    uint64_t nf = 0;
    ATOS_TRY(bsp_barrier(p, cnt, &nf, r, t0));
    if (st) st->pushes += nf;
    std::swap(b.fa, b.fb);
    F = nf;
  }
  wt.stop(s);
  ATOS_TRY(read_edges(p, b.ctr, st, s));
  if (st) st->worker_ms += wt.elapsed();
  double h_sum = 0;
  ATOS_TRY(pr_finalize(p, rank, res, &h_sum, s));  // rank_out = x / n (R-PR-4)
  if (st) st->residual_sum = h_sum;
  return ATOS_OK;
}

int color_bsp_single(atos_csr* g, Part& p, uint64_t seed, int32_t* color, const Resolved& r, atos_stats* st) {
  cudaStream_t s = r.stream;
  const uint64_t n = (uint64_t)p.n_local;
  ATOS_TRY(check_symmetric_if(p, r));
  BspBufs b;
  ATOS_TRY(bsp_buffers(p, n, false, &b, s));
  ATOS_CUDA(cudaMemsetAsync(color, 0xFF, n * 4, s));  // Alg.5: colour = -1
  k_bsp_iota<<<kGrid, 256, 0, s>>>(b.fa, (uint32_t)n);    // in_frontier = all vertices, ID order
  g_launches += 1;
  WorkerTimer wt;
  wt.start(s);
  const auto t0 = std::chrono::steady_clock::now();
  uint64_t F = n;
  for (uint32_t it = 0; F > 0; ++it) {
    const int grid = grid_for(F * 32, 256);
    unsigned long long* cnt = b.ctr + 2 * (it & 1);
    k_bsp_color_assign<<<grid, 256, 0, s>>>(p.row_ptr, p.col, color, b.fa, (uint32_t)F, b.ctr + 1);
    // barrier, then conflict detection
    k_bsp_color_conflicts<<<grid, 256, 0, s>>>(p.row_ptr, p.col, color, b.fa, (uint32_t)F, seed,
                                                r.conflict_policy, b.fb, cnt,
                                                b.ctr + 2 * ((it + 1) & 1), b.ctr + 1);
    g_launches += 2;
    ATOS_CUDA(cudaGetLastError());
    if (st) { st->pops += 2 * F; st->rounds += 1; }
    uint64_t nf = 0;
    ATOS_TRY(bsp_barrier(p, cnt, &nf, r, t0));
    if (st) st->pushes += nf;
    std::swap(b.fa, b.fb);
    F = nf;
  }
  wt.stop(s);
  ATOS_TRY(read_edges(p, b.ctr, st, s));
  if (st) st->worker_ms += wt.elapsed();
  int64_t used = 0;
  ATOS_TRY(color_count(p, color, &used, s));
  if (st) st->colors_used = used;
  return ATOS_OK;
}

}  // namespace atos
