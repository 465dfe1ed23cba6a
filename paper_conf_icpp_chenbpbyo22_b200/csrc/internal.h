// internal.h -- host-side internals of libatos (C++17, not part of the ABI).
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/atos.h"
#include "engine.cuh"

namespace atos {

// ------------------------------------------------------------------ errors
void set_error(const char* fmt, ...);
extern std::atomic<uint64_t> g_launches;

#define ATOS_CUDA(call)                                                                   \
  do {                                                                                   \
    cudaError_t e_ = (call);                                                             \
    if (e_ != cudaSuccess) {                                                             \
      ::atos::set_error("%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, \
                        __LINE__);                                                       \
      return e_ == cudaErrorMemoryAllocation ? ATOS_ERR_OOM : ATOS_ERR_CUDA;             \
    }                                                                                    \
  } while (0)

#define ATOS_TRY(expr)        \
  do {                        \
    int rc_ = (expr);         \
    if (rc_ != ATOS_OK) return rc_; \
  } while (0)

// Device memory of the library: a stream-ordered pool per device (cudaMallocFromPoolAsync) whose release
// threshold keeps freed blocks reserved, so the graph arrays and workspaces of a handle created and
// destroyed per step (the e2e path) are re-used instead of being mapped and unmapped by cudaMalloc /
// cudaFree every time.  dev_free waits for the device first (the same guarantee cudaFree gives).
int dev_alloc(void** p, size_t bytes);
void dev_free(void* p);
// 4 KB pinned host pages (control-block reads), recycled through a free list: no cudaHostAlloc /
// cudaFreeHost per handle
int pinned_page(void** p);
void pinned_page_release(void* p);
template <class T>
inline int dev_alloc_t(T** p, size_t count) { return dev_alloc((void**)p, count * sizeof(T)); }

// a device allocation owned by the handle
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
  int ensure(size_t want);  // grow-only
  void release();
  template <class T> T* as() const { return (T*)p; }
};

// One partition of a graph resident on one device (a whole graph when P = 1).
struct Part {
  int64_t v_begin = 0, v_end = 0;   // owned global vertices
  int64_t n_local = 0, m_local = 0;
  uint32_t* row_ptr = nullptr;      // n_local + 1, local offsets
  uint32_t* col = nullptr;          // m_local, GLOBAL ids (single-partition: the ids)
  // cached workspaces (grow-only, reused across calls)
  DevBuf ring, ctl, big, bitmap, shadow, vbuf_a, vbuf_b, vbuf_c, scratch;
  DevBuf ghost_a, ghost_b, touched, outbox, inbox, out_val, in_val, pack;
  DevBuf bsp_fa, bsp_fb, bsp_off, bsp_tmp, bsp_ctr;  // BSP baselines (bsp.cu)
  DevBuf nb_ring, nb_ctl, nb_peers;                   // barrier-free partitioned PageRank (nobarrier.cu)
  // barrier-free across PROCESSES (nobarrier.cu run_nobarrier_mp): this rank's peer-visible block
  // (cudaMalloc, exported with a CUDA IPC handle) and the peers' blocks mapped into this process
  void* nb_ipc = nullptr;
  size_t nb_ipc_bytes = 0;
  std::vector<void*> nb_peer_base;
  uint64_t ring_cap = 0;
  uint64_t max_deg = ~0ull;         // largest row length when known (whole-graph upload), else ~0
  void* host_pinned = nullptr;      // 4 KB pinned scratch for control-block reads
  bool ring_clean = false;          // every ring slot is EMPTY
};

// Multi-process communicator (dist.cu): NCCL loaded at run time (dlopen of
// libnccl.so.2 -- the copy torch already loaded), so the library has no link
// dependency on NCCL and CPU-only processes never touch it.
struct Comm {
  int nranks = 1, rank = 0, device = 0;
  void* nccl = nullptr;  // ncclComm_t
  // host-staged transport (atos_comm_create_host): the caller's collectives move host buffers
  atos_host_alltoallv_fn h_a2a = nullptr;
  atos_host_allreduce_fn h_ar = nullptr;
  void* h_user = nullptr;
};

// One partition's side of an exchange round.
struct ExchangeIO {
  uint32_t* out_vid = nullptr;        // outbox ids (owner-local), grouped by destination part
  void* out_val = nullptr;            // outbox values (u32 depth or f64 mass)
  std::vector<uint64_t> counts;       // items for each destination part (P entries)
  DevBuf* in_vid = nullptr;           // inbox (grown as needed)
  DevBuf* in_val = nullptr;
  uint64_t in_total = 0;
};
int exchange_loopback(std::vector<ExchangeIO>& io, size_t val_bytes, cudaStream_t s);
int exchange_nccl(Comm* c, ExchangeIO& io, size_t val_bytes, cudaStream_t s, uint64_t* bytes_sent);
int allreduce_u64(Comm* c, uint64_t* v, cudaStream_t s);
// every rank's `bytes` bytes (host memory) into out[rank * bytes] on every rank
int allgather_host(Comm* c, const void* in, size_t bytes, void* out, cudaStream_t s);
int allreduce_f64(Comm* c, double* v, cudaStream_t s);

}  // namespace atos

struct atos_csr {
  int device = 0;
  int64_t n = 0, m = 0;
  int num_parts = 1;                       // > 1: loopback partitions on one device
  std::vector<atos::Part> parts;
  atos::Comm* comm = nullptr;              // distributed partition (one per process)
  int rank = 0, nranks = 1;
  int64_t max_degree = 0;
  bool symmetric_checked = false, symmetric = false;
  bool bfs_deep_seen = false;              // a byte-state BFS on this graph met depth >= 126: start with u32 words
  bool relabeled = false;                  // degree layout (layout.cu): internal id = o2n[caller id]
  atos::DevBuf o2n, n2o, perm_out;         // u32[n] maps; output staging for host outputs
  std::mutex mu;
};

namespace atos {

// RAII device guard
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

struct Resolved {
  int persistent, worker, fetch, num_blocks, block_threads, dedupe, check_size;
  int conflict_policy, permute_init, validate, out_where, l2_persist, big_threshold, big_chunk, depth_state;
  int engine_variant;
  int barrier_free;
  int recolor_spread;
  int knobs_set;  // a scheduler knob the barrier-free kernel ignores was set (persistent=0, dedupe=0, worker,
                  // fetch_size, queue_capacity, depth_state, engine_variant)
  unsigned long long* timeline;
  uint32_t timeline_cap, timeline_interval_ns;
  uint64_t queue_capacity;
  double timeout_s;
  cudaStream_t stream;
  atos_stats* stats;
  unsigned long long watchdog_ns;
  // degree layout (layout.cu): a solver that can write the CALLER's ids directly (out[j] = f(state[o2n[j]]))
  // does so into map_out and sets *map_done; otherwise run_with_output scatters its internal-order result.
  const uint32_t* map_o2n = nullptr;
  void* map_out = nullptr;
  bool* map_done = nullptr;
};
// smallest fair-share claim for an app's workers (EngineParams::min_claim): ATOS_MIN_CLAIM overrides `dflt`
inline uint32_t min_claim_for(uint32_t dflt) {
  const char* e = getenv("ATOS_MIN_CLAIM");
  const long v = e ? atol(e) : 0;
  return v > 0 ? (uint32_t)v : dflt;
}
// defaults: app = 'b' (bfs) / 'p' (pagerank) / 'c' (color)
int resolve_cfg(const atos_cfg* cfg, char app, Resolved* r);

inline int mode_of(int worker) {
  return worker == 1 ? MODE_THREAD : (worker == 32 ? MODE_WARP : MODE_CTA);
}

constexpr uint32_t kBigSlots = 64;

// Ring/control workspace of a partition (+ the big-task table): capacity >= want (power of two), all slots EMPTY.
int ensure_queue(Part& p, uint64_t want_cap, cudaStream_t s);
// persistent grid size: occupancy max x SMs
int persistent_grid(const void* fn, int block, size_t smem, int* grid);
// L2 persisting window (best effort)
void set_l2_window(cudaStream_t s, void* base, size_t bytes, bool on);

// timing helper: events on the call stream
struct CallTimer {
  cudaEvent_t a = nullptr, b = nullptr;
  cudaStream_t s;
  explicit CallTimer(cudaStream_t st) : s(st) {
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a, s);
  }
  double stop() {
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    return ms;
  }
  ~CallTimer() {
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
  }
};

// events around the worker kernel(s) of one call; elapsed() after the stream synchronised
struct WorkerTimer {
  cudaEvent_t a = nullptr, b = nullptr;
  void start(cudaStream_t s) {
    if (!a) { cudaEventCreate(&a); cudaEventCreate(&b); }
    cudaEventRecord(a, s);
  }
  void stop(cudaStream_t s) { cudaEventRecord(b, s); }
  double elapsed() {
    float ms = 0;
    if (a && cudaEventSynchronize(b) == cudaSuccess) cudaEventElapsedTime(&ms, a, b);
    return ms;
  }
  ~WorkerTimer() {
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
  }
};

// Host-side phase tracer (tools: ATOS_TRACE=1): prints the wall time since the previous mark of this
// thread; `sync` first waits for the device so the time covers the enqueued work.
void trace_mark(const char* what, bool sync = false);

// wait for the stream, honouring cfg.timeout_s (polling) -- returns ATOS_ERR_TIMEOUT on expiry
int stream_wait(cudaStream_t s, double timeout_s);

// degree layout (layout.cu)
int create_single(atos_csr* g, const int64_t* row_ptr, const int32_t* col, int where, int flags);
template <class T>
int layout_scatter(const atos_csr* g, const T* in, T* out, cudaStream_t s);
int64_t layout_vertex(const atos_csr* g, int64_t v);  // caller id -> internal id (-1 on a CUDA error)

// single-partition solvers (relax.cu / color.cu)
int bfs_single(atos_csr* g, Part& p, int64_t src, uint32_t* depth_dev, const Resolved& r,
               atos_stats* st);
int pagerank_single(atos_csr* g, Part& p, double alpha, double eps, double* rank_dev,
                    const Resolved& r, atos_stats* st);
int color_single(atos_csr* g, Part& p, uint64_t seed, int32_t* color_dev, const Resolved& r,
                 atos_stats* st);
// bulk-synchronous baselines (bsp.cu): Alg.1 / Alg.3 / Alg.5
int bfs_bsp_single(atos_csr* g, Part& p, int64_t src, uint32_t* depth_dev, const Resolved& r, atos_stats* st);
int pagerank_bsp_single(atos_csr* g, Part& p, double alpha, double eps, double* rank_dev, const Resolved& r,
                        atos_stats* st);
int color_bsp_single(atos_csr* g, Part& p, uint64_t seed, int32_t* color_dev, const Resolved& r, atos_stats* st);
// helpers shared by the asynchronous and BSP paths
int pr_init_state(Part& p, double alpha, double* rank, double* res, cudaStream_t s);
int pr_finalize(Part& p, double* rank, const double* res, double* h_sum, cudaStream_t s);
int check_symmetric_if(Part& p, const Resolved& r);
int color_count(Part& p, const int32_t* color, int64_t* used, cudaStream_t s);
// partitioned solvers (dist.cu)
int bfs_partitioned(atos_csr* g, int64_t src, uint32_t* depth_dev, const Resolved& r, atos_stats* st);
int pagerank_partitioned(atos_csr* g, double alpha, double eps, double* rank_dev, const Resolved& r,
                         atos_stats* st);
// barrier-free partitioned BFS / PageRank, loopback partitions (nobarrier.cu, NEXT-4)
int bfs_nobarrier(atos_csr* g, int64_t src, uint32_t* depth_dev, const Resolved& r, atos_stats* st);
int pagerank_nobarrier(atos_csr* g, double alpha, double eps, double* rank_dev, const Resolved& r,
                       atos_stats* st);

// read the control block after a run: status -> error code, stats
int finish_queue(Part& p, cudaStream_t s, atos_stats* st, const char* what);

}  // namespace atos
