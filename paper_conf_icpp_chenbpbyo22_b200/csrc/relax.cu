// relax.cu -- single-partition BFS and PageRank: init kernels, launchers
// (persistent and discrete), finalisation.
#include <algorithm>
#include <cstdlib>
#include <vector>

#include "internal.h"
#include "apps.cuh"

namespace atos {

static uint32_t* g_dbg_edge = nullptr;  // debug (ATOS_DEBUG_EDGES): per-edge relaxation counts
static uint32_t* g_dbg_claim = nullptr;

// ------------------------------------------------------------- init kernels
// Start of a run on a persistent ring: abandon stale over-claims (head = tail),
// done = tail, clear status and per-run statistics.
__device__ __forceinline__ void run_begin(QueueCtl* ctl) {
  const unsigned long long t = ctl->tail.v;
  ctl->head.v = t;
  ctl->done.v = t;
  ctl->status.v = 0;
  ctl->check.v = 0;
  ctl->stat_pops.v = 0;
  ctl->stat_pushes.v = 0;
  ctl->stat_edges.v = 0;
  ctl->misc.v = 0;
  ctl->tl_next.v = 0;
  ctl->tl_count.v = 0;
  ctl->stat_maxocc.v = 0;
}

// Before every persistent launch: over-claims abandoned by a previous kernel
// of the same run are dropped.  Between launches nothing is in flight and the
// previous kernel consumed everything below `done`, so the unconsumed items
// are exactly [done, tail).
__global__ void k_sync_head(QueueCtl* ctl) {
  if (threadIdx.x == 0 && blockIdx.x == 0) ctl->head.v = ctl->done.v;
}

__global__ void k_run_begin(QueueCtl* ctl) {
  if (threadIdx.x == 0 && blockIdx.x == 0) run_begin(ctl);
}

// BFS init (Alg.1 P:721-725 "vertex.dist = MAX_UINT32", frontier = [source];
// source depth 0, R-BFS-1).  depth[] was memset to 0xFF on the stream.
__global__ void k_bfs_init(uint32_t* depth, int dedupe, uint8_t* shadow, Ring q, uint32_t src,
                           unsigned long long wd) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    run_begin(q.ctl);
    depth[src] = dedupe ? kInq : 0u;  // depth 0, queued
    if (shadow) shadow[src] = 0;
    const unsigned long long idx = q.ctl->tail.v;
    q.ctl->tail.v = idx + 1;
    publish_one(q, idx, src, wd);
  }
}

// Byte-state BFS init: state[] was memset to kBUnreached; source depth 0, queued.
__global__ void k_bfs_byte_init(uint8_t* state, Ring q, uint32_t src, unsigned long long wd) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    run_begin(q.ctl);
    state[src] = (uint8_t)kBInq;
    const unsigned long long idx = q.ctl->tail.v;
    q.ctl->tail.v = idx + 1;
    publish_one(q, idx, src, wd);
  }
}

// Degree layout: depth_out in the CALLER's ids, gathered (coalesced writes, state bytes read from L2).
__global__ void k_bfs_byte_output_mapped(const uint8_t* __restrict__ state, const uint32_t* __restrict__ o2n,
                                         uint32_t* depth, int64_t n) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t D = state[o2n[j]] & 0x7Fu;
    depth[j] = D == kBUnreached ? 0xFFFFFFFFu : D;
  }
}

// depth_out from the byte state (kBUnreached -> 0xFFFFFFFF), 4 vertices per thread.
__global__ void k_bfs_byte_output(const uint8_t* __restrict__ state, uint32_t* depth, int64_t n) {
  const int64_t nw = (n + 3) / 4;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nw; i += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t word = ((const uint32_t*)state)[i];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int64_t v = 4 * i + k;
      if (v < n) {
        const uint32_t D = (word >> (8 * k)) & 0x7Fu;
        depth[v] = D == kBUnreached ? 0xFFFFFFFFu : D;
      }
    }
  }
}

// PageRank vertex init (Alg.3): rank = 1 - lambda, residue = 0.
__global__ void k_pr_init_vertices(double* rank, double* res, int64_t n, double one_minus_alpha) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    rank[v] = one_minus_alpha;
    res[v] = 0.0;
  }
}

// Row owning edge e: largest r in [lo, hi] with row_ptr[r] <= e.
__device__ __forceinline__ uint32_t row_of(const uint32_t* __restrict__ row_ptr, uint32_t lo, uint32_t hi,
                                           uint32_t e) {
  while (lo < hi) {
    uint32_t mid = lo + ((hi - lo + 1) >> 1);
    if (__ldg(row_ptr + mid) <= e) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// PageRank residue init, read as R-PR-init (garbled P:766): for every vertex v
// and every out-neighbour w, residue[w] += (1-lambda)*lambda/deg(v).
// Edge-parallel over tiles of blockDim edges: two global searches per tile
// bound the tile's rows, then each thread searches only that (L1-resident)
// row range -- load-balanced regardless of hub degrees.
__global__ void k_pr_init_edges(const uint32_t* __restrict__ row_ptr, const uint32_t* __restrict__ col,
                                double* res, uint32_t n, uint32_t m, double c, uint32_t rs_log = 0) {
  __shared__ uint32_t s_r[2];
  for (uint64_t t0 = (uint64_t)blockIdx.x * blockDim.x; t0 < m; t0 += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t e0 = (uint32_t)t0;
    const uint64_t tend = t0 + blockDim.x < (uint64_t)m ? t0 + blockDim.x : (uint64_t)m;
    const uint32_t e1 = (uint32_t)(tend - 1);
    if (threadIdx.x == 0) s_r[0] = row_of(row_ptr, 0, n - 1, e0);
    if (threadIdx.x == 32 || (blockDim.x <= 32 && threadIdx.x == 0)) s_r[1] = row_of(row_ptr, 0, n - 1, e1);
    __syncthreads();
    const uint32_t e = e0 + threadIdx.x;
    if (e <= e1) {
      const uint32_t v = row_of(row_ptr, s_r[0], s_r[1], e);
      const uint32_t deg = __ldg(row_ptr + v + 1) - __ldg(row_ptr + v);
      red_add_f64(res + res_slot(__ldg(col + e), rs_log), c / (double)deg);
    }
    __syncthreads();
  }
}

// Initial frontier (R-PR-7): every vertex with residue > eps, warp-aggregated pushes.
__global__ void k_pr_seed(const double* res, int64_t n, double eps, Ring q, unsigned long long wd,
                          uint32_t rs_log = 0) {
  __shared__ uint32_t bufs[32 * kPushBuf];
  WarpPusher pusher = make_pusher(bufs);
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
    const int64_t v = base + threadIdx.x;
    const bool want = v < n && res[res_slot((uint32_t)v, rs_log)] > eps;
    pusher.push(q, want, (uint32_t)v, wd);
  }
  pusher.flush(q, wd);
  if (lane_id() == 0) atomicAdd(&q.ctl->stat_pushes.v, (unsigned long long)pusher.total);
}

// Slot-addressed accumulation (res_slot, rs_log > 0): rank_out[v] = acc[slot(v)] / n, residual sum as below.
__global__ void k_pr_finalize_slots(const double* acc, double* rank, const double* res, int64_t n, double n_global,
                                    uint32_t rs_log, double* sum) {
  double a = 0.0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    rank[v] = acc[res_slot((uint32_t)v, rs_log)] / n_global;
    a += res[v];
  }
  for (int o = 16; o; o >>= 1) a += __shfl_xor_sync(0xffffffffu, a, o);
  if (lane_id() == 0 && a != 0.0) atomicAdd(sum, a);
}

// rank_out = rank / n_global (R-PR-4); residual sum into *sum (conservation check).
__global__ void k_pr_finalize_n(double* rank, const double* res, int64_t n, double n_global, double* sum) {
  double acc = 0.0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    rank[v] = rank[v] / n_global;
    acc += res[v];
  }
  for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if (lane_id() == 0 && acc != 0.0) atomicAdd(sum, acc);
}

// Check_Size sweep (paper's Alg.4), run by a
// separate single-CTA-per-SM kernel between persistent drains: reserve
// Check_Size ids with one atomicAdd on the check cursor and enqueue those with
// residue > eps.  (The sweep variant drives activation; see pagerank_single.)
__global__ void k_pr_sweep(const double* res, int64_t n, double eps, Ring q, uint32_t check_size,
                           unsigned long long wd, uint32_t rs_log = 0) {
  __shared__ uint32_t bufs[32 * kPushBuf];
  __shared__ unsigned long long s_c;
  WarpPusher pusher = make_pusher(bufs);
  // each CTA sweeps chunks until the cursor passed n ids since kernel start
  while (true) {
    if (threadIdx.x == 0) s_c = atomicAdd(&q.ctl->check.v, (unsigned long long)check_size);
    __syncthreads();
    const unsigned long long c = s_c;
    __syncthreads();
    if (c >= (unsigned long long)n) break;
    for (uint32_t i = 0; i < check_size; i += blockDim.x) {
      const unsigned long long id = c + i + threadIdx.x;
      const bool want = (i + threadIdx.x) < check_size && id < (unsigned long long)n &&
                        res[res_slot((uint32_t)id, rs_log)] > eps;
      pusher.push(q, want, (uint32_t)id, wd);
    }
  }
  pusher.flush(q, wd);
  if (lane_id() == 0) atomicAdd(&q.ctl->stat_pushes.v, (unsigned long long)pusher.total);
}

// -------------------------------------------------------------- launchers
#ifndef ATOS_PF_LOWDEG
#define ATOS_PF_LOWDEG 1
#endif
constexpr bool kPfLowDegree = ATOS_PF_LOWDEG != 0;
#ifndef ATOS_HD_KU
#define ATOS_HD_KU 4    // high-degree graphs: edges in flight per thread of the (256, MINB) build
#endif
#ifndef ATOS_HD_MINB
#define ATOS_HD_MINB 5  // resident 256-thread CTAs per SM the register budget is sized for
#endif

static inline uint64_t pow2_at_least(uint64_t x) {
  uint64_t c = 1;
  while (c < x) c <<= 1;
  return c;
}

template <class App, int MODE, int KU = kU, int MINB = ATOS_MINB, bool PF = false>
static int launch_relax_mode(const App& app, EngineParams P, const Resolved& r, int block,
                             Part& p, atos_stats* st) {
  using Payload = typename App::Payload;
  cudaStream_t s = r.stream;
  const size_t smem = relax_worker_smem<Payload>(MODE, block, P.fetch, PF && MODE == MODE_CTA);
  if (smem > 227 * 1024) {
    set_error("fetch_size %d with worker %d needs %zu B of shared memory (> 227 KB)", r.fetch, r.worker, smem);
    return ATOS_ERR_INVALID_ARG;
  }
  if (r.persistent) {
    const void* fn = (const void*)k_relax_worker<App, MODE, true, KU, MINB, PF>;
    if (smem > 48 * 1024) ATOS_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int grid = 0;
    ATOS_TRY(persistent_grid(fn, block, smem, &grid));
    if (r.num_blocks > 0) grid = std::min(grid, r.num_blocks);
    k_sync_head<<<1, 32, 0, s>>>(P.q.ctl);
    g_launches++;
    void* args[] = {(void*)&app, (void*)&P};
    ATOS_CUDA(cudaLaunchCooperativeKernel(fn, grid, block, args, smem, s));
    g_launches++;
    if (st) st->rounds += 1;
    return ATOS_OK;
  }
  // discrete: one launch per frontier [h0, t0); the host reads the
  // tail after each launch -- the per-frontier host round trip the paper measures.
  const void* fn = (const void*)k_relax_worker<App, MODE, false, KU, MINB, PF>;
  if (smem > 48 * 1024) ATOS_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const uint64_t K = MODE == MODE_THREAD ? 32ull * P.fetch : P.fetch;
  const uint64_t groups_per_block = MODE == MODE_CTA ? 1 : block / 32;
  const uint64_t items_per_block = K * groups_per_block;
  unsigned long long* h_ctl = (unsigned long long*)p.host_pinned;
  QueueCtl* ctl = P.q.ctl;
  ATOS_CUDA(cudaMemcpyAsync(h_ctl, &ctl->head.v, 16 * 8 * 2, cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  // head line then tail line (Line64 = 16 words)
  uint64_t h0 = h_ctl[0], t0 = h_ctl[16];
  // the discrete frontier is consumed in order, so head follows h0
  while (h0 < t0) {
    P.h0 = h0;
    P.t0 = t0;
    if (st && t0 - h0 > st->max_queue_occupancy) st->max_queue_occupancy = t0 - h0;
    uint64_t grid = (t0 - h0 + items_per_block - 1) / items_per_block;
    if (grid > 0x7FFFFFFFull) grid = 0x7FFFFFFFull;
    void* args[] = {(void*)&app, (void*)&P};
    ATOS_CUDA(cudaLaunchKernel(fn, dim3((unsigned)grid), dim3(block), args, smem, s));
    g_launches++;
    if (st) st->rounds += 1;
    ATOS_CUDA(cudaMemcpyAsync(h_ctl, &ctl->tail.v, 8, cudaMemcpyDeviceToHost, s));
    ATOS_TRY(stream_wait(s, r.timeout_s));
    h0 = t0;
    t0 = h_ctl[0];
    if (t0 - h0 > p.ring_cap) {
      set_error("discrete frontier of %llu items exceeds the ring capacity %llu",
                (unsigned long long)(t0 - h0), (unsigned long long)p.ring_cap);
      p.ring_clean = false;
      return ATOS_ERR_QUEUE_OVERFLOW;
    }
  }
  // mirror the persistent bookkeeping so finish_queue sees a drained queue
  ATOS_CUDA(cudaMemcpyAsync(&ctl->head.v, &ctl->tail.v, 8, cudaMemcpyDeviceToDevice, s));
  ATOS_CUDA(cudaMemcpyAsync(&ctl->done.v, &ctl->tail.v, 8, cudaMemcpyDeviceToDevice, s));
  return ATOS_OK;
}

template <class App>
static int launch_relax_inner(const App& app, const Ring& q, const Resolved& r, Part& p, atos_stats* st);

template <class App>
static int launch_relax(const App& app, const Ring& q, const Resolved& r, Part& p, atos_stats* st) {
  WorkerTimer wt;
  wt.start(r.stream);
  const int rc = launch_relax_inner(app, q, r, p, st);
  wt.stop(r.stream);
  if (rc == ATOS_OK && st) st->worker_ms += wt.elapsed();
#ifdef ATOS_PHASE_PROF
  if (getenv("ATOS_PHASE")) {
    unsigned long long h[PH_N] = {};
    cudaStreamSynchronize(r.stream);
    cudaMemcpyFromSymbol(h, g_phase, sizeof(h));
    static const char* nm[PH_N] = {"big", "claim", "gather", "idle", "begin", "scan", "expand", "complete",
                                   "nb_lo", "nb_hi", "exp_lo", "exp_hi", "edges_lo", "edges_hi"};
    fprintf(stderr, "[phase]");
    for (int i = 0; i < PH_N; ++i) fprintf(stderr, " %s=%llu", nm[i], h[i]);
    fprintf(stderr, "\n");
    unsigned long long z[PH_N] = {};
    cudaMemcpyToSymbol(g_phase, z, sizeof(z));
  }
#endif
  return rc;
}

template <class App>
static int launch_relax_inner(const App& app, const Ring& q, const Resolved& r, Part& p, atos_stats* st) {
  EngineParams P;
  P.q = q;
  P.fetch = (uint32_t)r.fetch;
  P.watchdog_ns = r.watchdog_ns;
  P.h0 = P.t0 = 0;
  // smallest fair-share claim: 24 items on low-degree graphs (m < 8n: meshes / road-like, whose thin
  // frontiers are chains of small batches -- C2 mesh 30.1 -> 28.7 ms, road-like 42.4 -> 40.4 ms vs 16,
  // profiles/r02_ab_min_claim.txt), 16 otherwise
  P.min_claim = min_claim_for(p.n_local > 0 && p.m_local < 8 * p.n_local ? 24u : (uint32_t)kMinClaim);
  const int mode = mode_of(r.worker);
  const int block = mode == MODE_CTA ? r.worker : r.block_threads;
  // hub assist (persistent CTA / warp workers): auto threshold = 32 edges per
  // worker thread, chunks of 8 edges per worker thread (>= 1024)
  P.timeout_ns = r.timeout_s > 0 ? (unsigned long long)(r.timeout_s * 1e9) : 0ull;
  P.dbg_edge = g_dbg_edge;
  P.dbg_claim = g_dbg_claim;
  P.tl = r.timeline;
  P.tl_cap = r.timeline_cap;
  P.tl_interval_ns = r.timeline_interval_ns;
  P.big = nullptr;
  P.nbig = 0;
  P.big_threshold = 0xFFFFFFFFu;
  P.big_chunk = 1;
  if (r.persistent && mode != MODE_THREAD && r.big_threshold >= 0 && p.big.p) {
    const uint32_t wsz = mode == MODE_CTA ? (uint32_t)r.worker : 32u;
    P.big = p.big.as<BigTask>();
    P.nbig = kBigSlots;
    P.big_threshold = r.big_threshold > 0 ? (uint32_t)r.big_threshold : std::max(4096u, 32u * wsz);
    P.big_chunk = r.big_chunk > 0 ? (uint32_t)r.big_chunk : std::max(1024u, 8u * wsz);
    // no row can become a big task (known maximum degree below the threshold): no assist, so the worker
    // loop skips the per-batch big-task check (one L2 round trip and a barrier per batch -- ~7 % of a
    // hop on high-diameter meshes, tools/hop_latency.py)
    if (p.max_deg <= P.big_threshold) {
      P.big = nullptr;
      P.nbig = 0;
      P.big_threshold = 0xFFFFFFFFu;
    }
  }
  if (mode == MODE_CTA) {
    // 256-thread CTA workers: the (256, 5) register budget (48 regs, 40 warps per SM); kU = 2 edges
    // in flight per thread on low-degree graphs (meshes / road-like: m/n < 8), 4 otherwise.  Measured
    // (tools/sweep.py, one B200): C5 BFS 15.25 -> 14.8 ms, C2 mesh 58 -> 47 ms, road 68 -> 52 ms.
    // Low-degree graphs also stage the next iteration's col loads with cp.async (PF): their LBS spans cross
    // many short rows, so the col load is a full extra round trip per iteration (mesh 48.5 -> 46.8 ms, road
    // 55 -> 49.6 ms); scale-free BFS keeps the direct loads (13.4 -> 15.9 ms with PF).
    if (block == 256 && r.persistent && r.engine_variant != 1) {
      const bool low_degree = p.n_local > 0 && p.m_local < 8 * p.n_local;
      if (low_degree) return launch_relax_mode<App, MODE_CTA, 2, 5, kPfLowDegree>(app, P, r, block, p, st);
      return launch_relax_mode<App, MODE_CTA, ATOS_HD_KU, ATOS_HD_MINB>(app, P, r, block, p, st);
    }
    if (App::kPfCta && r.persistent && r.engine_variant != 1)
      return launch_relax_mode<App, MODE_CTA, kU, ATOS_MINB, true>(app, P, r, block, p, st);
    return launch_relax_mode<App, MODE_CTA>(app, P, r, block, p, st);
  }
  if (mode == MODE_WARP) return launch_relax_mode<App, MODE_WARP>(app, P, r, block, p, st);
  return launch_relax_mode<App, MODE_THREAD>(app, P, r, block, p, st);
}

static Ring ring_of(Part& p) {
  Ring q;
  q.slots = p.ring.as<unsigned long long>();
  q.mask = p.ring_cap - 1;
  q.ctl = p.ctl.as<QueueCtl>();
  return q;
}

// --------------------------------------------------------------------- BFS
// Byte-state traversal (BfsByteApp).  *deep = true when a depth >= 126 was met
// (nothing is written to depth then; the caller re-runs with the u32 state).
static int bfs_single_bytes(Part& p, int64_t src, uint32_t* depth, const Resolved& r, atos_stats* st, bool* deep) {
  cudaStream_t s = r.stream;
  const int64_t n = p.n_local;
  *deep = false;
  const size_t nb = (size_t)(n + 3) / 4 * 4;
  ATOS_TRY(p.shadow.ensure(nb));
  uint8_t* state = p.shadow.as<uint8_t>();
  ATOS_CUDA(cudaMemsetAsync(state, (int)kBUnreached, nb, s));
  trace_mark("bfs: state", true);
  Ring q = ring_of(p);
  k_bfs_byte_init<<<1, 32, 0, s>>>(state, q, (uint32_t)src, r.watchdog_ns);
  g_launches++;
  ATOS_CUDA(cudaGetLastError());
  if (r.l2_persist) set_l2_window(s, state, nb, true);
  BfsByteApp app{p.row_ptr, p.col, state, (uint32_t*)&q.ctl->status.v, 0ull, 0ull};
  p.ring_clean = false;
  int rc = launch_relax(app, q, r, p, st);
  trace_mark("bfs: worker", true);
  if (r.l2_persist) set_l2_window(s, nullptr, 0, false);
  if (rc != ATOS_OK) return rc;
  ATOS_TRY(finish_queue(p, s, st, "bfs"));
  if (((QueueCtl*)p.host_pinned)->status.v & kStatusDeep) {
    *deep = true;
    return ATOS_OK;
  }
  if (r.map_o2n && r.map_done) {
    k_bfs_byte_output_mapped<<<148 * 8, 256, 0, s>>>(state, r.map_o2n, (uint32_t*)r.map_out, n);
    *r.map_done = true;
  } else {
    k_bfs_byte_output<<<148 * 8, 256, 0, s>>>(state, depth, n);
  }
  g_launches++;
  ATOS_CUDA(cudaGetLastError());
  return ATOS_OK;
}

int bfs_single(atos_csr* g, Part& p, int64_t src, uint32_t* depth, const Resolved& r, atos_stats* st) {
  cudaStream_t s = r.stream;
  const int64_t n = p.n_local;
  uint64_t want = r.queue_capacity ? r.queue_capacity : (uint64_t)std::max<int64_t>(2 * n, 1024);
  if (!r.dedupe && !r.queue_capacity) want = (uint64_t)std::max<int64_t>(4 * n, 4096);
  trace_mark("bfs: enter", true);
  ATOS_TRY(ensure_queue(p, pow2_at_least(want), s));
  trace_mark("bfs: ensure_queue", true);
  // byte state first (dedupe mode); a traversal deeper than 125 levels re-runs with u32 words
  // A graph on which a byte-state traversal already ran out of depth codes (a high-diameter mesh or road
  // network) starts every later BFS with the u32 words instead of paying the aborted first attempt again
  // (stats.flags bit 1).
  if (r.dedupe && r.depth_state != 2 && g->bfs_deep_seen && st) st->flags |= 2;
  if (r.dedupe && r.depth_state != 2 && !g->bfs_deep_seen) {
    bool deep = false;
    ATOS_TRY(bfs_single_bytes(p, src, depth, r, st, &deep));
    if (!deep) return ATOS_OK;
    g->bfs_deep_seen = true;
    if (st) {
      st->flags |= 1;  // re-run with the u32 state; rounds describe the final run (worker_ms keeps both)
      st->rounds = 0;
    }
    ATOS_TRY(ensure_queue(p, pow2_at_least(want), s));  // resets the ring the stopped run left behind
  }
  ATOS_CUDA(cudaMemsetAsync(depth, 0xFF, (size_t)n * 4, s));
  ATOS_TRY(p.shadow.ensure((size_t)n));
  uint8_t* shadow = p.shadow.as<uint8_t>();
  ATOS_CUDA(cudaMemsetAsync(shadow, 0xFF, (size_t)n, s));
  Ring q = ring_of(p);
  k_bfs_init<<<1, 32, 0, s>>>(depth, r.dedupe, shadow, q, (uint32_t)src, r.watchdog_ns);
  g_launches++;
  ATOS_CUDA(cudaGetLastError());
  if (r.l2_persist) set_l2_window(s, depth, (size_t)n * 4, true);
  const GhostView nogv{0u, (uint32_t)n, nullptr, nullptr, nullptr};
  p.ring_clean = false;
  int rc;
  if (r.dedupe) rc = launch_relax(BfsDedupeApp{p.row_ptr, p.col, depth, 1, shadow, 0ull, 0ull, nogv}, q, r, p, st);
  else rc = launch_relax(BfsApp{p.row_ptr, p.col, depth, 0, shadow, 0ull, 0ull, nogv}, q, r, p, st);
  if (r.l2_persist) set_l2_window(s, nullptr, 0, false);
  if (rc != ATOS_OK) return rc;
  return finish_queue(p, s, st, "bfs");
}

// ---------------------------------------------------------------- PageRank
// Alg.3 init (R-PR-init): rank = 1 - alpha, residue[w] += (1-alpha)*alpha/deg(v)
// over every edge v -> w.  Shared by the asynchronous path and the BSP baseline (bsp.cu).
int pr_init_state(Part& p, double alpha, double* rank, double* res, cudaStream_t s) {
  const int64_t n = p.n_local;
  const int gs = 148 * 8;
  k_pr_init_vertices<<<gs, 256, 0, s>>>(rank, res, n, 1.0 - alpha);
  g_launches++;
  if (p.m_local > 0) {
    k_pr_init_edges<<<gs * 2, 256, 0, s>>>(p.row_ptr, p.col, res, (uint32_t)n, (uint32_t)p.m_local,
                                            (1.0 - alpha) * alpha);
    g_launches++;
  }
  ATOS_CUDA(cudaGetLastError());
  return ATOS_OK;
}

// rank_out = x / n (R-PR-4) and the residual sum (conservation check) into *h_sum.
int pr_finalize(Part& p, double* rank, const double* res, double* h_sum, cudaStream_t s) {
  ATOS_TRY(p.scratch.ensure(64));
  double* sum = p.scratch.as<double>();
  ATOS_CUDA(cudaMemsetAsync(sum, 0, 8, s));
  k_pr_finalize_n<<<148 * 8, 256, 0, s>>>(rank, res, p.n_local, (double)p.n_local, sum);
  g_launches++;
  ATOS_CUDA(cudaGetLastError());
  ATOS_CUDA(cudaMemcpyAsync(h_sum, sum, 8, cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  return ATOS_OK;
}

int pagerank_single(atos_csr* g, Part& p, double alpha, double eps, double* rank, const Resolved& r,
                    atos_stats* st) {
  cudaStream_t s = r.stream;
  const int64_t n = p.n_local;
  const uint64_t want = r.queue_capacity ? r.queue_capacity : (uint64_t)std::max<int64_t>(2 * n, 1024);
  ATOS_TRY(ensure_queue(p, pow2_at_least(want), s));
  ATOS_TRY(p.vbuf_a.ensure((size_t)n * 8));
  ATOS_TRY(p.scratch.ensure(64));
  double* res = p.vbuf_a.as<double>();
  double* sum = p.scratch.as<double>();
  Ring q = ring_of(p);
  k_run_begin<<<1, 32, 0, s>>>(q.ctl);
  g_launches++;
  // residue slots on a degree-layout graph: T = 65536 (or the largest power of two with 16T <= n)
  uint32_t rs_log = 0;
  if (g->relabeled && g->parts.size() == 1)
    while (rs_log < 16 && (16ll << (rs_log + 1)) <= n) ++rs_log;
  if (const char* e = getenv("ATOS_PR_SLOT_LOG")) rs_log = (uint32_t)std::max(0, std::min(atoi(e), (int)rs_log));
  const int gs = 148 * 8;
  // slot-addressed rank accumulator (the caller's buffer receives rank_out in vertex order at the end)
  double* const rank_out = rank;
  if (rs_log) {
    ATOS_TRY(p.vbuf_b.ensure((size_t)n * 8));
    rank = p.vbuf_b.as<double>();
  }
  k_pr_init_vertices<<<gs, 256, 0, s>>>(rank, res, n, 1.0 - alpha);
  g_launches++;
  if (p.m_local > 0) {
    k_pr_init_edges<<<gs * 2, 256, 0, s>>>(p.row_ptr, p.col, res, (uint32_t)n, (uint32_t)p.m_local,
                                            (1.0 - alpha) * alpha, rs_log);
    g_launches++;
  }
  k_pr_seed<<<gs, 1024, 0, s>>>(res, n, eps, q, r.watchdog_ns, rs_log);
  g_launches++;
  ATOS_CUDA(cudaGetLastError());
  if (r.l2_persist) set_l2_window(s, res, (size_t)n * 8, true);
  PrApp app{p.row_ptr, p.col, 0ull, rank, res, alpha, eps, r.check_size > 0 ? 0 : 1, nullptr,
            GhostView{0u, (uint32_t)n, nullptr, nullptr, nullptr}};
  app.rs_log = rs_log;
  uint32_t* dbg_edge = nullptr;
  const bool dbg = getenv("ATOS_DEBUG_EDGES") != nullptr;
  if (dbg) {
    ATOS_CUDA(cudaMalloc(&dbg_edge, (size_t)p.m_local * 4 + 4));
    ATOS_CUDA(cudaMalloc(&app.dbg_expand, (size_t)n * 4 + 4));
    ATOS_CUDA(cudaMemset(dbg_edge, 0, (size_t)p.m_local * 4 + 4));
    ATOS_CUDA(cudaMemset(app.dbg_expand, 0, (size_t)n * 4 + 4));
    g_dbg_edge = dbg_edge;
    if (!g_dbg_claim) {
      cudaMalloc(&g_dbg_claim, 64 * 4096 * 4);
      cudaMemset(g_dbg_claim, 0, 64 * 4096 * 4);
    }
  }
  p.ring_clean = false;
  int rc = ATOS_OK;
  if (r.check_size <= 0) {
    rc = launch_relax(app, q, r, p, st);
  } else {
    // Check_Size variant: activation only by round-robin sweeps of
    // Check_Size ids.  Drain the queue, sweep all n ids, repeat until a full
    // sweep enqueues nothing (every residue <= eps).
    unsigned long long* h = (unsigned long long*)p.host_pinned;
    for (int iter = 0; iter < 100000 && rc == ATOS_OK; ++iter) {
      rc = launch_relax(app, q, r, p, st);
      if (rc != ATOS_OK) break;
      ATOS_CUDA(cudaMemcpyAsync(h, &q.ctl->tail.v, 8, cudaMemcpyDeviceToHost, s));
      ATOS_CUDA(cudaMemcpyAsync(h + 1, &q.ctl->status.v, 8, cudaMemcpyDeviceToHost, s));
      ATOS_TRY(stream_wait(s, r.timeout_s));
      if (h[1] != 0) break;  // watchdog/overflow: reported by finish_queue
      const unsigned long long t_before = h[0];
      ATOS_CUDA(cudaMemsetAsync(&q.ctl->check.v, 0, 8, s));
      k_pr_sweep<<<gs, 256, 0, s>>>(res, n, eps, q, (uint32_t)r.check_size, r.watchdog_ns, rs_log);
      g_launches++;
      ATOS_CUDA(cudaMemcpyAsync(h, &q.ctl->tail.v, 8, cudaMemcpyDeviceToHost, s));
      ATOS_TRY(stream_wait(s, r.timeout_s));
      if (h[0] == t_before) break;
    }
  }
  if (r.l2_persist) set_l2_window(s, nullptr, 0, false);
  g_dbg_edge = nullptr;
  if (dbg) {
    g_dbg_claim = g_dbg_claim;  // kept across calls (generations keep increasing)
    cudaDeviceSynchronize();
    std::vector<uint32_t> ec(p.m_local), xc(n), rp(n + 1);
    cudaMemcpy(ec.data(), dbg_edge, p.m_local * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(xc.data(), app.dbg_expand, n * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(rp.data(), p.row_ptr, (n + 1) * 4, cudaMemcpyDeviceToHost);
    long over = 0, under = 0, vbad = 0;
    for (int64_t v = 0; v < n; ++v) {
      bool b = false;
      for (uint32_t e = rp[v]; e < rp[v + 1]; ++e) {
        if (ec[e] > xc[v]) { ++over; b = true; }
        if (ec[e] < xc[v]) { ++under; b = true; }
      }
      if (b && vbad < 8) {
        fprintf(stderr, "  v=%lld deg=%u expands=%u edge counts:", (long long)v, rp[v + 1] - rp[v], xc[v]);
        for (uint32_t e = rp[v]; e < rp[v + 1] && e < rp[v] + 24; ++e) fprintf(stderr, " %u", ec[e]);
        fprintf(stderr, "\n");
      }
      vbad += b;
    }
    fprintf(stderr, "[atos debug edges] over=%ld under=%ld bad_vertices=%ld\n", over, under, vbad);
    cudaFree(dbg_edge);
    cudaFree(app.dbg_expand);
  }
  if (rc != ATOS_OK) return rc;
  ATOS_CUDA(cudaMemsetAsync(sum, 0, 8, s));
  if (rs_log) k_pr_finalize_slots<<<gs, 256, 0, s>>>(rank, rank_out, res, n, (double)n, rs_log, sum);
  else k_pr_finalize_n<<<gs, 256, 0, s>>>(rank, res, n, (double)n, sum);
  g_launches++;
  ATOS_CUDA(cudaGetLastError());
  rc = finish_queue(p, s, st, "pagerank");
  if (rc != ATOS_OK) return rc;
  if (st) {
    double h_sum = 0;
    ATOS_CUDA(cudaMemcpy(&h_sum, sum, 8, cudaMemcpyDeviceToHost));
    st->residual_sum = h_sum;
  }
  return ATOS_OK;
}

}  // namespace atos

// =========================================================================
// Partitioned BFS / PageRank (S10): rounds of
//   local persistent phase -> pack touched ghosts per owner -> exchange ->
//   apply inbox (relax + activate) -> global "anything sent?" reduction.
// Loopback (P partitions in one process) and NCCL (one partition per rank)
// share this code; only the exchange/reduction differ.
// =========================================================================
namespace atos {

// The touched list is split into gridDim.x contiguous block ranges; every block
// histograms its range per destination part in shared memory (P counters) and
// touches the global counters once per part -- no same-address global atomic
// per touched vertex.
__device__ __forceinline__ void block_range(unsigned long long nt, unsigned long long& b, unsigned long long& e) {
  const unsigned long long per = (nt + gridDim.x - 1) / gridDim.x;
  b = blockIdx.x * per;
  e = b + per < nt ? b + per : nt;
}

// Byte-state BFS ghosts: list every vertex whose ghost byte has bit 7 set
// (improved this round) -- a coalesced scan of n_global bytes, one list append
// (atomicAdd) per block.
__global__ void k_ghost_flags_to_list(const uint32_t* __restrict__ ghost_words, int64_t nwords, uint32_t* touched,
                                      unsigned long long* ntouched) {
  __shared__ uint32_t tmp[40];
  __shared__ unsigned long long s_base;
  for (int64_t w0 = (int64_t)blockIdx.x * blockDim.x; w0 < nwords; w0 += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = w0 + threadIdx.x;
    const uint32_t word = i < nwords ? ghost_words[i] : 0u;
    const uint32_t fl = word & 0x80808080u;
    const uint32_t cnt = __popc(fl);
    uint32_t tot = 0;
    const uint32_t ex = block_exclusive_scan(cnt, tmp, &tot);  // uniform trip count: every thread calls it
    if (tot == 0) continue;
    if (threadIdx.x == 0) s_base = atomicAdd(ntouched, (unsigned long long)tot);
    __syncthreads();
    uint32_t k = 0;
#pragma unroll
    for (int b = 0; b < 4; ++b)
      if (fl & (0x80u << (8 * b))) touched[s_base + ex + k++] = (uint32_t)(4 * i + b);
    __syncthreads();
  }
}

// PageRank ghosts: list every REMOTE vertex (outside [vb, vb+nl)) whose ghost
// mass is non-zero -- the relax adds remote mass with red.add (no return, so no
// first-touch test and no list append in the relax loop).
__global__ void k_ghost_mass_to_list(const double* __restrict__ ghost, int64_t n, int64_t vb, int64_t nl,
                                     uint32_t* touched, unsigned long long* ntouched) {
  __shared__ uint32_t tmp[40];
  __shared__ unsigned long long s_base;
  const int64_t nr = n - nl;  // remote ids: r < vb -> r, else r + nl
  for (int64_t r0 = (int64_t)blockIdx.x * blockDim.x; r0 < nr; r0 += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = r0 + threadIdx.x;
    const int64_t w = r < vb ? r : r + nl;
    const uint32_t f = (r < nr && ghost[w] != 0.0) ? 1u : 0u;
    uint32_t tot = 0;
    const uint32_t ex = block_exclusive_scan(f, tmp, &tot);
    if (tot == 0) continue;
    if (threadIdx.x == 0) s_base = atomicAdd(ntouched, (unsigned long long)tot);
    __syncthreads();
    if (f) touched[s_base + ex] = (uint32_t)w;
    __syncthreads();
  }
}

// count touched ghosts per destination part
__global__ void k_pack_count(const uint32_t* touched, const unsigned long long* ntouched, uint32_t chunk,
                             unsigned long long* counts, uint32_t P) {
  extern __shared__ unsigned int s_cnt[];
  for (uint32_t d = threadIdx.x; d < P; d += blockDim.x) s_cnt[d] = 0;
  __syncthreads();
  unsigned long long b, e;
  block_range(*ntouched, b, e);
  for (unsigned long long i0 = b; i0 < e; i0 += blockDim.x) {  // uniform trip count: warp-collective below
    const unsigned long long i = i0 + threadIdx.x;
    const bool valid = i < e;
    const uint32_t owner = valid ? touched[i] / chunk : 0xFFFFFFFFu;
    const unsigned same = __match_any_sync(0xffffffffu, owner);
    if (valid && (__ffs(same) - 1) == (int)lane_id()) atomicAdd(s_cnt + owner, (unsigned)__popc(same));
  }
  __syncthreads();
  for (uint32_t d = threadIdx.x; d < P; d += blockDim.x)
    if (s_cnt[d]) atomicAdd(counts + d, (unsigned long long)s_cnt[d]);
}

// exclusive scan of the P counts into cursors (P is small)
__global__ void k_pack_scan(const unsigned long long* counts, unsigned long long* cursor, uint32_t P) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    unsigned long long acc = 0;
    for (uint32_t d = 0; d < P; ++d) {
      cursor[d] = acc;
      acc += counts[d];
    }
  }
}

// write (owner-local id, combined value) grouped by owner; reset the ghost.
// Each block reserves one contiguous run per part (one global atomic per part)
// and places its entries with shared-memory cursors.
// How a packed ghost is read and reset: the combined value is shipped and the
// ghost returns to `reset` (PageRank mass, u32 BFS depth) ...
template <class G, class V>
struct TakeReset {
  G reset;
  __device__ __forceinline__ V operator()(G& g) const {
    const V v = (V)g;
    g = reset;
    return v;
  }
};
// ... or (byte-state BFS) keeps its depth as the cross-round filter and only
// drops the touched flag (bit 7).
struct TakeKeepByte {
  __device__ __forceinline__ uint32_t operator()(uint8_t& g) const {
    const uint32_t v = g & 0x7Fu;
    g = (uint8_t)v;
    return v;
  }
};

template <class G, class V, class Take>
__global__ void k_pack_write(const uint32_t* touched, unsigned long long* ntouched, G* ghost, uint32_t chunk,
                             unsigned long long* cursor, uint32_t* out_vid, V* out_val, Take take, uint32_t P) {
  extern __shared__ unsigned long long s_cur[];  // P cursors
  unsigned int* s_cnt = (unsigned int*)(s_cur + P);
  for (uint32_t d = threadIdx.x; d < P; d += blockDim.x) s_cnt[d] = 0;
  __syncthreads();
  unsigned long long b, e;
  block_range(*ntouched, b, e);
  for (unsigned long long i0 = b; i0 < e; i0 += blockDim.x) {
    const unsigned long long i = i0 + threadIdx.x;
    const bool valid = i < e;
    const uint32_t owner = valid ? touched[i] / chunk : 0xFFFFFFFFu;
    const unsigned same = __match_any_sync(0xffffffffu, owner);
    if (valid && (__ffs(same) - 1) == (int)lane_id()) atomicAdd(s_cnt + owner, (unsigned)__popc(same));
  }
  __syncthreads();
  for (uint32_t d = threadIdx.x; d < P; d += blockDim.x)
    s_cur[d] = s_cnt[d] ? atomicAdd(cursor + d, (unsigned long long)s_cnt[d]) : 0ull;
  __syncthreads();
  for (unsigned long long i0 = b; i0 < e; i0 += blockDim.x) {
    const unsigned long long i = i0 + threadIdx.x;
    const bool valid = i < e;
    const uint32_t w = valid ? touched[i] : 0u, owner = valid ? w / chunk : 0xFFFFFFFFu;
    const unsigned same = __match_any_sync(0xffffffffu, owner);
    const int leader = __ffs(same) - 1;
    unsigned long long base = 0;
    if (valid && leader == (int)lane_id()) base = atomicAdd(s_cur + owner, (unsigned long long)__popc(same));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (valid) {
      const unsigned long long pos = base + __popc(same & ((1u << lane_id()) - 1u));
      out_vid[pos] = w - owner * chunk;
      out_val[pos] = take(ghost[w]);
    }
  }
}

__global__ void k_reset_u64(unsigned long long* p) {
  if (threadIdx.x == 0 && blockIdx.x == 0) *p = 0;
}

// apply an inbox: owner-local relax + activation through the normal queue
template <class App>
__global__ void k_apply(App app, const uint32_t* vid, const typename App::Payload* val, unsigned long long total,
                        Ring q, unsigned long long wd) {
  __shared__ uint32_t bufs[32 * kPushBuf];
  WarpPusher pusher = make_pusher(bufs);
  app.prepare();
  const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
  for (unsigned long long base = (unsigned long long)blockIdx.x * blockDim.x; base < total; base += stride) {
    const unsigned long long i = base + threadIdx.x;
    bool want = false;
    uint32_t out = 0;
    if (i < total) want = app.apply(val[i], vid[i], out);
    pusher.push(q, want, out, wd);
  }
  pusher.flush(q, wd);
  if (lane_id() == 0) atomicAdd(&q.ctl->stat_pushes.v, (unsigned long long)pusher.total);
}

// PageRank residue init for a partition: local rows, GLOBAL columns
__global__ void k_pr_init_edges_part(const uint32_t* __restrict__ row_ptr, const uint32_t* __restrict__ col,
                                     double* res, uint32_t nl, uint32_t m, double c, GhostView gv) {
  __shared__ uint32_t s_r[2];
  for (uint64_t t0 = (uint64_t)blockIdx.x * blockDim.x; t0 < m; t0 += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t e0 = (uint32_t)t0;
    const uint64_t tend = t0 + blockDim.x < (uint64_t)m ? t0 + blockDim.x : (uint64_t)m;
    const uint32_t e1 = (uint32_t)(tend - 1);
    if (threadIdx.x == 0) s_r[0] = row_of(row_ptr, 0, nl - 1, e0);
    if (threadIdx.x == 32 || (blockDim.x <= 32 && threadIdx.x == 0)) s_r[1] = row_of(row_ptr, 0, nl - 1, e1);
    __syncthreads();
    const uint32_t e = e0 + threadIdx.x;
    if (e <= e1) {
      const uint32_t v = row_of(row_ptr, s_r[0], s_r[1], e);
      const uint32_t deg = __ldg(row_ptr + v + 1) - __ldg(row_ptr + v);
      const uint32_t w = __ldg(col + e);
      const double add = c / (double)deg;
      if (gv.remote_dyn(w)) {
        red_add_f64((double*)gv.ghost + w, add);  // listed by the pack's ghost scan
      } else {
        red_add_f64(res + (w - gv.vb), add);
      }
    }
    __syncthreads();
  }
}

__global__ void k_bfs_init_part(uint32_t* depth, int dedupe, uint8_t* shadow, Ring q, uint32_t lsrc, int has_src,
                                unsigned long long wd) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    run_begin(q.ctl);
    if (has_src) {
      depth[lsrc] = dedupe ? kInq : 0u;
      if (shadow) shadow[lsrc] = 0;
      const unsigned long long idx = q.ctl->tail.v;
      q.ctl->tail.v = idx + 1;
      publish_one(q, idx, lsrc, wd);
    }
  }
}

namespace {

struct PartRun {
  Part* p;
  int scan_flags = 0;  // build the touched list from the ghost first: 1 byte bit-7 flags (BFS), 2 non-zero mass (PR)
  int64_t ghost_words = 0;  // words of ghost bytes to scan (n_global bytes, rounded up)
  uint32_t* state;      // depth (u32) or rank (f64) -- local slice of the output
  GhostView gv;
  unsigned long long* counts;   // device: P counts, then P cursors
  unsigned long long* ntouched; // device
};

template <class G, class V, class Take>
int pack_part(PartRun& pr, uint32_t chunk, uint32_t P, Take take, ExchangeIO& io, cudaStream_t s) {
  Part& p = *pr.p;
  if (pr.scan_flags == 1) {
    k_ghost_flags_to_list<<<148 * 8, 256, 0, s>>>((const uint32_t*)pr.gv.ghost, pr.ghost_words,
                                                  p.touched.as<uint32_t>(), pr.ntouched);
    ++g_launches;
  } else if (pr.scan_flags == 2) {
    k_ghost_mass_to_list<<<148 * 8, 256, 0, s>>>((const double*)pr.gv.ghost, pr.ghost_words, (int64_t)pr.gv.vb,
                                                 (int64_t)pr.gv.nl, p.touched.as<uint32_t>(), pr.ntouched);
    ++g_launches;
  }
  ATOS_CUDA(cudaMemsetAsync(pr.counts, 0, sizeof(unsigned long long) * P, s));
  k_pack_count<<<592, 256, P * 4, s>>>(p.touched.as<uint32_t>(), pr.ntouched, chunk, pr.counts, P);
  k_pack_scan<<<1, 32, 0, s>>>(pr.counts, pr.counts + P, P);
  k_pack_write<G, V, Take><<<592, 256, P * 12, s>>>(p.touched.as<uint32_t>(), pr.ntouched, (G*)pr.gv.ghost, chunk,
                                                    pr.counts + P, p.outbox.as<uint32_t>(), p.out_val.as<V>(), take,
                                                    P);
  k_reset_u64<<<1, 32, 0, s>>>(pr.ntouched);
  g_launches += 4;
  ATOS_CUDA(cudaGetLastError());
  std::vector<unsigned long long> h(P);
  ATOS_CUDA(cudaMemcpyAsync(h.data(), pr.counts, sizeof(unsigned long long) * P, cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  io.out_vid = p.outbox.as<uint32_t>();
  io.out_val = p.out_val.p;
  io.counts.assign(h.begin(), h.end());
  io.in_vid = &p.inbox;
  io.in_val = &p.in_val;
  return ATOS_OK;
}

// allocate the ghost machinery of one partition (n_global-sized ghost, touched list, outbox)
int ensure_ghosts(Part& p, int64_t n_global, size_t ghost_bytes, size_t val_bytes, uint32_t P, cudaStream_t s) {
  ATOS_TRY(p.ghost_a.ensure(((size_t)n_global * ghost_bytes + 3) / 4 * 4));
  ATOS_TRY(p.touched.ensure((size_t)n_global * 4));
  ATOS_TRY(p.outbox.ensure((size_t)n_global * 4));
  ATOS_TRY(p.out_val.ensure((size_t)n_global * val_bytes));
  ATOS_TRY(p.pack.ensure(sizeof(unsigned long long) * (2 * P + 2)));
  return ATOS_OK;
}

// Between-round hook: decides termination after an exchange (default: nothing
// was sent anywhere).
struct NoHook {
  template <class App>
  int between(std::vector<App>&, std::vector<PartRun>&, uint64_t sent, bool* done, const Resolved&) {
    *done = sent == 0;
    return ATOS_OK;
  }
};

// Partitioned PageRank threshold schedule: local phases
// run to quiescence at eps_k = max(eps, eps_0 * factor^k) instead of eps, so a
// round does not drive every local residue down to eps only for the next
// round's remote mass to raise it again.  When the threshold drops, every
// vertex with eps_{k+1} < residue is queued (before the inbox is applied with
// the crossing rule at eps_{k+1}, so nothing is queued twice).  The run ends
// only after a round at the final eps sent nothing, so the result satisfies the
// same bound as the unscheduled run.
struct PrEpsHook {
  double cur, fin, factor, defer_c = 0.0;
  template <class App>
  int between(std::vector<App>& apps, std::vector<PartRun>& runs, uint64_t sent, bool* done, const Resolved& r) {
    if (cur <= fin) {
      *done = sent == 0;
      return ATOS_OK;
    }
    cur = cur * factor > fin ? cur * factor : fin;
    *done = false;
    for (size_t i = 0; i < runs.size(); ++i) {
      Part& p = *runs[i].p;
      apps[i].eps = cur;
      apps[i].defer = cur > fin ? defer_c * cur : 0.0;
      if (!p.n_local) continue;
      k_pr_seed<<<148 * 8, 1024, 0, r.stream>>>(apps[i].res, p.n_local, cur, ring_of(p), r.watchdog_ns);
      ++g_launches;
    }
    ATOS_CUDA(cudaGetLastError());
    return ATOS_OK;
  }
};

// One run of the round protocol.  G = ghost element type, V = the exchanged
// value (the app's payload).  *deep (byte-state BFS): some partition met a depth
// the byte state cannot encode -- the caller re-runs with the u32 state.
template <class App, class G, class Take, class Hook = NoHook>
int run_rounds(atos_csr* g, std::vector<PartRun>& runs, std::vector<App>& apps, const Resolved& r, Take take,
               atos_stats* st, bool* deep = nullptr, Hook hook = Hook{}) {
  using V = typename App::Payload;
  cudaStream_t s = r.stream;
  const uint32_t P = g->comm ? (uint32_t)g->nranks : (uint32_t)g->num_parts;
  const uint32_t chunk = (uint32_t)((g->n + P - 1) / P);
  Resolved rl = r;
  rl.persistent = 1;  // each local phase runs to local quiescence
  uint64_t rounds = 0, bytes = 0;
  std::vector<ExchangeIO> io(runs.size());
  // ATOS_ROUND_TRACE=1 (tools): per-round stage times on stderr
  const bool trace = getenv("ATOS_ROUND_TRACE") != nullptr;
  WorkerTimer tw[4];
  double tsum[4] = {0, 0, 0, 0};
  while (true) {
    if (trace) tw[0].start(s);
    for (size_t i = 0; i < runs.size(); ++i) {
      Part& p = *runs[i].p;
      Ring q = ring_of(p);
      ATOS_TRY(launch_relax(apps[i], q, rl, p, st));
    }
    if (trace) { tw[0].stop(s); tw[1].start(s); }
    for (size_t i = 0; i < runs.size(); ++i) ATOS_TRY((pack_part<G, V, Take>(runs[i], chunk, P, take, io[i], s)));
    if (trace) { tw[1].stop(s); tw[2].start(s); }
    if (deep) {
      // pack_part synchronised the stream: the control blocks are final for this round
      uint64_t dp = 0;
      for (auto& pr : runs) {
        uint32_t stw = 0;
        ATOS_CUDA(cudaMemcpy(&stw, &pr.p->ctl.as<QueueCtl>()->status.v, 4, cudaMemcpyDeviceToHost));
        if (stw & kStatusDeep) dp = 1;
      }
      if (g->comm) ATOS_TRY(allreduce_u64(g->comm, &dp, s));
      if (dp) {
        for (auto& pr : runs) pr.p->ring_clean = false;
        *deep = true;
        return ATOS_OK;
      }
    }
    uint64_t sent = 0;
    for (auto& x : io)
      for (uint32_t d = 0; d < P; ++d) sent += x.counts[d];
    if (g->comm) {
      uint64_t b = 0;
      ATOS_TRY(exchange_nccl(g->comm, io[0], sizeof(V), s, &b));
      bytes += b;
      ATOS_TRY(allreduce_u64(g->comm, &sent, s));
    } else {
      for (auto& x : io)
        for (uint32_t d = 0; d < P; ++d) bytes += x.counts[d] * (4 + sizeof(V));
      ATOS_TRY(exchange_loopback(io, sizeof(V), s));
    }
    if (trace) { tw[2].stop(s); tw[3].start(s); }
    ++rounds;
    bool done = false;
    ATOS_TRY(hook.between(apps, runs, sent, &done, r));
    if (done) break;
    for (size_t i = 0; i < runs.size(); ++i) {
      if (!io[i].in_total) continue;
      Part& p = *runs[i].p;
      Ring q = ring_of(p);
      k_apply<App><<<(unsigned)std::min<uint64_t>((io[i].in_total + 1023) / 1024, 1184), 1024, 0, s>>>(
          apps[i], io[i].in_vid->as<uint32_t>(), (const typename App::Payload*)io[i].in_val->p, io[i].in_total, q,
          r.watchdog_ns);
      ++g_launches;
      ATOS_CUDA(cudaGetLastError());
    }
    if (trace) {
      tw[3].stop(s);
      double t[4];
      for (int k = 0; k < 4; ++k) tsum[k] += (t[k] = tw[k].elapsed());
      fprintf(stderr, "[round %llu] local %.3f ms  pack %.3f  exchange %.3f  apply %.3f  sent %llu\n",
              (unsigned long long)rounds, t[0], t[1], t[2], t[3], (unsigned long long)sent);
    }
    if (rounds > 100000) {
      set_error("partitioned run did not converge within 100000 rounds");
      return ATOS_ERR_TIMEOUT;
    }
  }
  if (trace)
    fprintf(stderr, "[rounds %llu] local %.3f ms  pack %.3f  exchange %.3f  apply %.3f\n", (unsigned long long)rounds,
            tsum[0], tsum[1], tsum[2], tsum[3]);
  for (auto& pr : runs) ATOS_TRY(finish_queue(*pr.p, s, st, "partitioned"));
  if (st) {
    st->rounds = rounds;
    st->bytes_exchanged += bytes;
  }
  return ATOS_OK;
}

}  // namespace

__global__ void k_bfs_byte_init_part(uint8_t* state, Ring q, uint32_t lsrc, int has_src, unsigned long long wd) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    run_begin(q.ctl);
    if (has_src) {
      state[lsrc] = (uint8_t)kBInq;
      const unsigned long long idx = q.ctl->tail.v;
      q.ctl->tail.v = idx + 1;
      publish_one(q, idx, lsrc, wd);
    }
  }
}

// Byte-state partitioned BFS: per-partition state bytes (local), ghost bytes
// (n_global, kBUnreached = untouched) min-combined, u32 depths exchanged.
static int bfs_partitioned_bytes(atos_csr* g, int64_t src, uint32_t* depth_out, const Resolved& r, atos_stats* st,
                                 bool* deep) {
  cudaStream_t s = r.stream;
  const uint32_t P = g->comm ? (uint32_t)g->nranks : (uint32_t)g->num_parts;
  std::vector<PartRun> runs(g->parts.size());
  std::vector<BfsBytePartApp> apps(g->parts.size());
  for (size_t i = 0; i < g->parts.size(); ++i) {
    Part& p = g->parts[i];
    const int64_t n = p.n_local;
    ATOS_TRY(ensure_queue(p, pow2_at_least((uint64_t)std::max<int64_t>(2 * n, 1024)), s));
    ATOS_TRY(ensure_ghosts(p, g->n, 1, 4, P, s));
    const size_t nb = (size_t)(std::max<int64_t>(n, 1) + 3) / 4 * 4;
    ATOS_TRY(p.shadow.ensure(nb));
    ATOS_CUDA(cudaMemsetAsync(p.shadow.p, (int)kBUnreached, nb, s));
    ATOS_CUDA(cudaMemsetAsync(p.ghost_a.p, (int)kBUnreached, ((size_t)g->n + 3) / 4 * 4, s));
    unsigned long long* pk = p.pack.as<unsigned long long>();
    ATOS_CUDA(cudaMemsetAsync(pk, 0, sizeof(unsigned long long) * (2 * P + 2), s));
    PartRun& pr = runs[i];
    pr.p = &p;
    pr.scan_flags = 1;
    pr.ghost_words = (g->n + 3) / 4;
    pr.state = g->comm ? depth_out : depth_out + p.v_begin;
    pr.counts = pk;
    pr.ntouched = pk + 2 * P;
    pr.gv = GhostView{(uint32_t)p.v_begin, (uint32_t)n, p.ghost_a.p, p.touched.as<uint32_t>(), pr.ntouched};
    const bool has = src >= p.v_begin && src < p.v_end;
    Ring q = ring_of(p);
    k_bfs_byte_init_part<<<1, 32, 0, s>>>(p.shadow.as<uint8_t>(), q, has ? (uint32_t)(src - p.v_begin) : 0u,
                                          has ? 1 : 0, r.watchdog_ns);
    ++g_launches;
    p.ring_clean = false;
    apps[i] = BfsBytePartApp{p.row_ptr, p.col, p.shadow.as<uint8_t>(), (uint32_t*)&q.ctl->status.v, 0ull, 0ull, pr.gv};
  }
  ATOS_CUDA(cudaGetLastError());
  ATOS_TRY((run_rounds<BfsBytePartApp, uint8_t>(g, runs, apps, r, TakeKeepByte{}, st, deep)));
  if (*deep) return ATOS_OK;
  for (auto& pr : runs) {
    if (!pr.p->n_local) continue;
    k_bfs_byte_output<<<148 * 8, 256, 0, s>>>(pr.p->shadow.as<uint8_t>(), pr.state, pr.p->n_local);
    ++g_launches;
  }
  ATOS_CUDA(cudaGetLastError());
  return ATOS_OK;
}

int bfs_partitioned(atos_csr* g, int64_t src, uint32_t* depth_out, const Resolved& r, atos_stats* st) {
  cudaStream_t s = r.stream;
  const uint32_t P = g->comm ? (uint32_t)g->nranks : (uint32_t)g->num_parts;
  if (r.dedupe && r.depth_state != 2) {
    bool deep = false;
    ATOS_TRY(bfs_partitioned_bytes(g, src, depth_out, r, st, &deep));
    if (!deep) return ATOS_OK;
    if (st) {
      st->flags |= 1;  // re-run with the u32 state (rounds/bytes describe both runs)
    }
  }
  std::vector<PartRun> runs(g->parts.size());
  std::vector<BfsPartApp> apps(g->parts.size());
  for (size_t i = 0; i < g->parts.size(); ++i) {
    Part& p = g->parts[i];
    const int64_t n = p.n_local;
    ATOS_TRY(ensure_queue(p, pow2_at_least((uint64_t)std::max<int64_t>(2 * n, 1024)), s));
    ATOS_TRY(ensure_ghosts(p, g->n, 4, 4, P, s));
    ATOS_TRY(p.shadow.ensure((size_t)std::max<int64_t>(n, 1)));
    // loopback: the partition writes its slice of the full output; NCCL: the local output
    uint32_t* depth = g->comm ? depth_out : depth_out + p.v_begin;
    if (n) ATOS_CUDA(cudaMemsetAsync(depth, 0xFF, (size_t)n * 4, s));
    ATOS_CUDA(cudaMemsetAsync(p.shadow.p, 0xFF, (size_t)std::max<int64_t>(n, 1), s));
    ATOS_CUDA(cudaMemsetAsync(p.ghost_a.p, 0xFF, (size_t)g->n * 4, s));
    unsigned long long* pk = p.pack.as<unsigned long long>();
    ATOS_CUDA(cudaMemsetAsync(pk, 0, sizeof(unsigned long long) * (2 * P + 2), s));
    PartRun& pr = runs[i];
    pr.p = &p;
    pr.state = depth;
    pr.counts = pk;
    pr.ntouched = pk + 2 * P;
    pr.gv = GhostView{(uint32_t)p.v_begin, (uint32_t)n, p.ghost_a.p, p.touched.as<uint32_t>(), pr.ntouched};
    const bool has = src >= p.v_begin && src < p.v_end;
    Ring q = ring_of(p);
    k_bfs_init_part<<<1, 32, 0, s>>>(depth, r.dedupe, p.shadow.as<uint8_t>(), q,
                                     has ? (uint32_t)(src - p.v_begin) : 0u, has ? 1 : 0, r.watchdog_ns);
    ++g_launches;
    p.ring_clean = false;
    apps[i] = BfsPartApp{p.row_ptr, p.col, depth, r.dedupe, p.shadow.as<uint8_t>(), 0ull, 0ull, pr.gv};
  }
  ATOS_CUDA(cudaGetLastError());
  return run_rounds<BfsPartApp, uint32_t>(g, runs, apps, r, TakeReset<uint32_t, uint32_t>{0xFFFFFFFFu}, st);
}

int pagerank_partitioned(atos_csr* g, double alpha, double eps, double* rank_out, const Resolved& r,
                         atos_stats* st) {
  cudaStream_t s = r.stream;
  const uint32_t P = g->comm ? (uint32_t)g->nranks : (uint32_t)g->num_parts;
  if (r.check_size > 0) {
    set_error("check_size sweeps are single-partition only");
    return ATOS_ERR_UNSUPPORTED;
  }
  std::vector<PartRun> runs(g->parts.size());
  std::vector<PrPartApp> apps(g->parts.size());
  const int gs = 148 * 8;
  // threshold schedule: eps_0 = 1e-2 (unnormalised residue, per-vertex mass ~1), x0.85 per round
  // (measured on RMAT S23, 2 loopback partitions: 1130 -> 822 ms, 73 -> 18 pops/n).
  // Tools: ATOS_PR_EPS0 / ATOS_PR_EPSF override; EPS0 <= eps disables.
  PrEpsHook hook{eps, eps, 1.0};
  {
    const char* e0 = getenv("ATOS_PR_EPS0");
    const char* ef = getenv("ATOS_PR_EPSF");
    const double eps0 = e0 ? atof(e0) : 1e-2;
    if (eps0 > eps) hook = PrEpsHook{eps0, eps, ef ? atof(ef) : 0.85};
    if (!(hook.factor > 0.0 && hook.factor < 1.0)) hook = PrEpsHook{eps, eps, 1.0};
    // hub deferral while the threshold is above eps: a popped vertex with deg > 32 and residue below
    // 0.05 * eps_k * deg hands its residue back (re-seeded when the threshold drops) -- hubs are
    // expanded when their residue pays for their edge count instead of in every round.  Measured
    // (S23, P=2 / P=8 loopback): 477 -> 284 ms / 730 -> 620 ms, 213 -> 105 edge relaxations per m.
    const char* dc = getenv("ATOS_PR_DEFER");
    hook.defer_c = dc ? atof(dc) : 0.05;
  }
  for (size_t i = 0; i < g->parts.size(); ++i) {
    Part& p = g->parts[i];
    const int64_t n = p.n_local;
    ATOS_TRY(ensure_queue(p, pow2_at_least((uint64_t)std::max<int64_t>(2 * n, 1024)), s));
    ATOS_TRY(ensure_ghosts(p, g->n, 8, 8, P, s));
    ATOS_TRY(p.vbuf_a.ensure((size_t)std::max<int64_t>(n, 1) * 8));
    double* rank = g->comm ? rank_out : rank_out + p.v_begin;
    double* res = p.vbuf_a.as<double>();
    ATOS_CUDA(cudaMemsetAsync(p.ghost_a.p, 0, (size_t)g->n * 8, s));
    unsigned long long* pk = p.pack.as<unsigned long long>();
    ATOS_CUDA(cudaMemsetAsync(pk, 0, sizeof(unsigned long long) * (2 * P + 2), s));
    PartRun& pr = runs[i];
    pr.p = &p;
    pr.state = nullptr;
    pr.counts = pk;
    pr.ntouched = pk + 2 * P;
    pr.gv = GhostView{(uint32_t)p.v_begin, (uint32_t)n, p.ghost_a.p, p.touched.as<uint32_t>(), pr.ntouched};
    pr.scan_flags = 2;
    pr.ghost_words = g->n;  // elements (f64)
    Ring q = ring_of(p);
    k_run_begin<<<1, 32, 0, s>>>(q.ctl);
    if (n) {
      k_pr_init_vertices<<<gs, 256, 0, s>>>(rank, res, n, 1.0 - alpha);
      g_launches += 1;
    }
    if (p.m_local) {
      k_pr_init_edges_part<<<gs * 2, 256, 0, s>>>(p.row_ptr, p.col, res, (uint32_t)n, (uint32_t)p.m_local,
                                                  (1.0 - alpha) * alpha, pr.gv);
      ++g_launches;
    }
    if (n) {
      k_pr_seed<<<gs, 1024, 0, s>>>(res, n, hook.cur, q, r.watchdog_ns);
      ++g_launches;
    }
    g_launches += 1;
    p.ring_clean = false;
    apps[i] = PrPartApp{p.row_ptr, p.col, 0ull, rank, res, alpha, hook.cur, 1, nullptr, pr.gv};
    apps[i].defer = hook.cur > hook.fin ? hook.defer_c * hook.cur : 0.0;
  }
  ATOS_CUDA(cudaGetLastError());
  ATOS_TRY((run_rounds<PrPartApp, double>(g, runs, apps, r, TakeReset<double, double>{0.0}, st, nullptr, hook)));
  // finalize: rank / n_global, residual sum over all partitions (conservation)
  double total = 0.0;
  for (size_t i = 0; i < g->parts.size(); ++i) {
    Part& p = g->parts[i];
    ATOS_TRY(p.scratch.ensure(64));
    double* sum = p.scratch.as<double>();
    ATOS_CUDA(cudaMemsetAsync(sum, 0, 8, s));
    double* rank = g->comm ? rank_out : rank_out + p.v_begin;
    if (p.n_local) {
      // rank_out = rank / n_global
      k_pr_finalize_n<<<gs, 256, 0, s>>>(rank, p.vbuf_a.as<double>(), p.n_local, (double)g->n, sum);
      ++g_launches;
    }
    double h = 0;
    ATOS_CUDA(cudaMemcpyAsync(&h, sum, 8, cudaMemcpyDeviceToHost, s));
    ATOS_CUDA(cudaStreamSynchronize(s));
    total += h;
  }
  if (g->comm) ATOS_TRY(allreduce_f64(g->comm, &total, s));
  if (st) st->residual_sum = total;
  return ATOS_OK;
}

}  // namespace atos
