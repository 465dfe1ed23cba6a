// api.cu -- the C ABI (include/atos.h): handles, configuration, errors, and
// the host-side plumbing shared by all solvers.
#include <cstdarg>
#include <cstdlib>
#include <cstring>
#include <chrono>
#include <thread>
#include <algorithm>
#include <functional>
#include <unordered_map>

#include "internal.h"

namespace atos {

static thread_local char g_err[1024] = "";
std::atomic<uint64_t> g_launches{0};

void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}

namespace {
struct PoolOf {
  cudaMemPool_t pool = nullptr;
  cudaStream_t s = nullptr;  // allocation stream (no kernels run on it)
};
std::mutex g_pool_mu;
PoolOf g_pools[64];

int pool_of(int dev, PoolOf** out) {
  std::lock_guard<std::mutex> lk(g_pool_mu);
  if (dev < 0 || dev >= 64) {
    set_error("device %d out of range for the memory pool", dev);
    return ATOS_ERR_CUDA;
  }
  PoolOf& P = g_pools[dev];
  if (!P.pool) {
    cudaMemPoolProps props;
    memset(&props, 0, sizeof(props));
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    ATOS_CUDA(cudaMemPoolCreate(&P.pool, &props));
    // keep up to 96 GB of freed blocks reserved (a C5 handle plus its workspaces is ~25 GB)
    uint64_t keep = 96ull << 30;
    ATOS_CUDA(cudaMemPoolSetAttribute(P.pool, cudaMemPoolAttrReleaseThreshold, &keep));
    ATOS_CUDA(cudaStreamCreateWithFlags(&P.s, cudaStreamNonBlocking));
  }
  *out = &P;
  return ATOS_OK;
}
}  // namespace

// Block cache on top of the pool: freed blocks are kept by exact size class, so a handle created and
// destroyed per step gets the same blocks back without the pool re-mapping memory (measured: the pool
// alone still cost 20-55 ms on some steps when a multi-GB request no longer fit its split blocks).
namespace {
struct CacheEnt {
  void* p;
  size_t bytes;
  int dev;
};
std::mutex g_cache_mu;
std::vector<CacheEnt> g_cache;                       // free blocks, oldest first
std::unordered_map<void*, std::pair<size_t, int>> g_live;  // every library block: size, device
size_t g_cache_bytes = 0;
constexpr size_t kCacheCap = 48ull << 30;
}  // namespace

int dev_alloc(void** p, size_t bytes) {
  *p = nullptr;
  int dev = 0;
  ATOS_CUDA(cudaGetDevice(&dev));
  if (!bytes) bytes = 16;
  {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    size_t best = (size_t)-1;
    for (size_t i = 0; i < g_cache.size(); ++i) {
      const CacheEnt& c = g_cache[i];
      if (c.dev == dev && c.bytes >= bytes && c.bytes <= bytes + bytes / 4 &&
          (best == (size_t)-1 || c.bytes < g_cache[best].bytes))
        best = i;
    }
    if (best != (size_t)-1) {
      *p = g_cache[best].p;
      g_cache_bytes -= g_cache[best].bytes;
      g_cache.erase(g_cache.begin() + best);
      return ATOS_OK;
    }
  }
  PoolOf* P = nullptr;
  ATOS_TRY(pool_of(dev, &P));
  cudaError_t e = cudaMallocFromPoolAsync(p, bytes, P->pool, P->s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(P->s);  // usable by every stream from here on
  if (e != cudaSuccess) {
    *p = nullptr;
    cudaGetLastError();
    set_error("device allocation of %zu bytes failed: %s", bytes, cudaGetErrorString(e));
    return e == cudaErrorMemoryAllocation ? ATOS_ERR_OOM : ATOS_ERR_CUDA;
  }
  std::lock_guard<std::mutex> lk(g_cache_mu);
  g_live[*p] = {bytes, dev};
  return ATOS_OK;
}

void dev_free(void* p) {
  if (!p) return;
  size_t bytes = 0;
  int dev = 0;
  {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    auto it = g_live.find(p);
    if (it == g_live.end()) return;  // not ours
    bytes = it->second.first;
    dev = it->second.second;
  }
  DeviceGuard dg(dev);
  cudaDeviceSynchronize();  // no kernel may still use the block (cudaFree's own guarantee)
  std::vector<CacheEnt> evict;
  {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    g_cache.push_back({p, bytes, dev});
    g_cache_bytes += bytes;
    while (g_cache_bytes > kCacheCap && !g_cache.empty()) {
      evict.push_back(g_cache.front());
      g_cache_bytes -= g_cache.front().bytes;
      g_live.erase(g_cache.front().p);
      g_cache.erase(g_cache.begin());
    }
  }
  for (const CacheEnt& c : evict) {
    PoolOf* P = nullptr;
    if (pool_of(c.dev, &P) != ATOS_OK) continue;
    DeviceGuard dg2(c.dev);
    cudaFreeAsync(c.p, P->s);
  }
  cudaGetLastError();
}

namespace {
std::mutex g_pin_mu;
std::vector<void*> g_pin_free;
}  // namespace

int pinned_page(void** p) {
  {
    std::lock_guard<std::mutex> lk(g_pin_mu);
    if (!g_pin_free.empty()) {
      *p = g_pin_free.back();
      g_pin_free.pop_back();
      return ATOS_OK;
    }
  }
  ATOS_CUDA(cudaHostAlloc(p, 4096, cudaHostAllocPortable));
  return ATOS_OK;
}

void pinned_page_release(void* p) {
  if (!p) return;
  std::lock_guard<std::mutex> lk(g_pin_mu);
  g_pin_free.push_back(p);
}

int DevBuf::ensure(size_t want) {
  if (want <= bytes && p) return ATOS_OK;
  release();
  if (want == 0) want = 16;
  ATOS_TRY(dev_alloc(&p, want));
  bytes = want;
  return ATOS_OK;
}

void DevBuf::release() {
  if (p) dev_free(p);
  p = nullptr;
  bytes = 0;
}

int resolve_cfg(const atos_cfg* cfg, char app, Resolved* r) {
  atos_cfg d;
  atos_cfg_default(&d);
  if (cfg) {
    if (cfg->struct_size != sizeof(atos_cfg)) {
      set_error("atos_cfg.struct_size = %u, expected %zu (call atos_cfg_default)", cfg->struct_size,
                sizeof(atos_cfg));
      return ATOS_ERR_INVALID_ARG;
    }
    d = *cfg;
  }
  r->persistent = d.persistent ? 1 : 0;
  r->worker = d.worker;
  // defaults measured on B200: CTA workers with load-balancing search
  // win for all three apps (tools/sweep.py, gpurun_out sweep: BFS C5 256/256, PageRank C3 512/512,
  // colouring C4 1024/128)
  if (r->worker == 0) r->worker = (app == 'c') ? 1024 : (app == 'p' ? 512 : 256);
  if (!(r->worker == 1 || r->worker == 32 || (r->worker >= 64 && r->worker <= 1024 && r->worker % 32 == 0))) {
    set_error("worker must be 1, 32 or a multiple of 32 in [64, 1024] (got %d)", r->worker);
    return ATOS_ERR_INVALID_ARG;
  }
  r->fetch = d.fetch_size;
  // CTA defaults: BFS fetch = worker; colouring min(worker, 48) (fewer vertices assigned concurrently, fewer
  // recolour cascades on a dense core: C4 1024:128 7.95 ms / 10.7 edge visits per m / 695 colours vs 1024:48
  // 6.3 ms / 6.0 / 713-719, profiles/r02_gc_fetch_sweep.txt); PageRank min(worker, 256) (512:256 vs
  // 512:512 measured C3 61.7 vs 63.6 ms, C5 even -- profiles/r02_pr_fetch_sweep.txt)
  if (r->fetch == 0)
    r->fetch = (r->worker >= 64) ? (app == 'c' ? std::min(r->worker, 48) : (app == 'p' ? std::min(r->worker, 256) : r->worker))
                                 : (r->worker == 32 ? 8 : 1);
  if (r->fetch < 1 || r->fetch > 4096) {
    set_error("fetch_size must be in [1, 4096] (got %d)", r->fetch);
    return ATOS_ERR_INVALID_ARG;
  }
  r->num_blocks = std::max(0, d.num_blocks);
  r->block_threads = d.block_threads ? d.block_threads : 256;
  if (r->block_threads < 32 || r->block_threads > 1024 || r->block_threads % 32) {
    set_error("block_threads must be a multiple of 32 in [32, 1024] (got %d)", r->block_threads);
    return ATOS_ERR_INVALID_ARG;
  }
  r->dedupe = d.dedupe ? 1 : 0;
  r->check_size = d.check_size;
  if (r->check_size < 0) {
    set_error("check_size must be >= 0");
    return ATOS_ERR_INVALID_ARG;
  }
  r->conflict_policy = d.conflict_policy;
  if (r->conflict_policy < 0 || r->conflict_policy > 2) {
    set_error("conflict_policy must be 0, 1 or 2 (got %d)", r->conflict_policy);
    return ATOS_ERR_INVALID_ARG;
  }
  r->permute_init = d.permute_init;
  r->validate = d.validate;
  r->out_where = d.out_where;
  if (r->out_where != ATOS_MEM_DEVICE && r->out_where != ATOS_MEM_HOST) {
    set_error("out_where must be ATOS_MEM_DEVICE or ATOS_MEM_HOST");
    return ATOS_ERR_INVALID_ARG;
  }
  r->l2_persist = d.l2_persist;
  r->timeline = (unsigned long long*)d.timeline;
  r->timeline_cap = d.timeline ? d.timeline_cap : 0;
  r->timeline_interval_ns = d.timeline_interval_ns ? d.timeline_interval_ns : 5000;
  r->big_threshold = d.big_threshold;
  r->depth_state = d.depth_state;
  if (r->depth_state != 0 && r->depth_state != 2) {
    set_error("depth_state must be 0 (auto) or 2 (u32 words) (got %d)", r->depth_state);
    return ATOS_ERR_INVALID_ARG;
  }
  r->engine_variant = d.engine_variant;
  if (r->engine_variant != 0 && r->engine_variant != 1) {
    set_error("engine_variant must be 0 (auto) or 1 (64-register build) (got %d)", r->engine_variant);
    return ATOS_ERR_INVALID_ARG;
  }
  r->barrier_free = d.barrier_free;
  r->recolor_spread = d.recolor_spread;
  if (r->recolor_spread < 0 || r->recolor_spread > 64) {
    set_error("recolor_spread must be in [0, 64] (got %d)", r->recolor_spread);
    return ATOS_ERR_INVALID_ARG;
  }
  r->knobs_set = (!d.persistent || !d.dedupe || d.worker != 0 || d.fetch_size != 0 || d.queue_capacity != 0 ||
                  d.depth_state != 0 || d.engine_variant != 0) ? 1 : 0;
  if (r->barrier_free != 0 && r->barrier_free != 1) {
    set_error("barrier_free must be 0 or 1 (got %d)", r->barrier_free);
    return ATOS_ERR_INVALID_ARG;
  }
  r->big_chunk = d.big_chunk;
  if (r->big_chunk < 0) {
    set_error("big_chunk must be >= 0");
    return ATOS_ERR_INVALID_ARG;
  }
  r->queue_capacity = d.queue_capacity;
  r->timeout_s = d.timeout_s;
  if (r->timeout_s < 0) {
    set_error("timeout_s must be >= 0");
    return ATOS_ERR_INVALID_ARG;
  }
  r->stream = (cudaStream_t)d.stream;
  r->stats = d.stats;
  // no-progress watchdog: cfg.timeout_s, else 10 s (ATOS_WATCHDOG_S overrides the default -- tools, e.g.
  // kernels slowed 100x under compute-sanitizer)
  const char* wd_env = getenv("ATOS_WATCHDOG_S");
  const double wd_default = wd_env && atof(wd_env) > 0 ? atof(wd_env) : 10.0;
  r->watchdog_ns = (unsigned long long)((r->timeout_s > 0 ? r->timeout_s : wd_default) * 1e9);
  return ATOS_OK;
}

// Fresh ring: slot i free for index i (seq = i), all counters 0.
__global__ void k_ring_init(unsigned long long* slots, unsigned long long cap, QueueCtl* ctl, BigTask* big,
                            uint32_t nbig) {
  for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < cap;
       i += (unsigned long long)gridDim.x * blockDim.x)
    slots[i] = make_slot(i, 0u);
  if (blockIdx.x == 0) {
    for (uint32_t i = threadIdx.x; i < nbig; i += blockDim.x) {
      big[i].state = 0;
      big[i].ctr = 0;
      big[i].finished = 0;
    }
    if (threadIdx.x == 0) {
      ctl->head.v = 0;
      ctl->tail.v = 0;
      ctl->done.v = 0;
      ctl->status.v = 0;
      ctl->big_count.v = 0;
      ctl->big_rr.v = 0;
    }
  }
}

int ensure_queue(Part& p, uint64_t cap, cudaStream_t s) {
  if (p.ring_cap < cap || !p.ring.p) {
    ATOS_TRY(p.ring.ensure(cap * 8));
    p.ring_cap = cap;
    p.ring_clean = false;
  }
  if (!p.ctl.p) ATOS_TRY(p.ctl.ensure(sizeof(QueueCtl)));
  if (!p.big.p) ATOS_TRY(p.big.ensure(sizeof(BigTask) * kBigSlots));
  if (!p.host_pinned) ATOS_TRY(pinned_page(&p.host_pinned));
  if (!p.ring_clean) {
    k_ring_init<<<1184, 256, 0, s>>>(p.ring.as<unsigned long long>(), p.ring_cap, p.ctl.as<QueueCtl>(),
                                     p.big.as<BigTask>(), kBigSlots);
    g_launches++;
    ATOS_CUDA(cudaGetLastError());
    p.ring_clean = true;
  }
  return ATOS_OK;
}

int persistent_grid(const void* fn, int block, size_t smem, int* grid) {
  int dev = 0, sms = 0, per = 0;
  ATOS_CUDA(cudaGetDevice(&dev));
  ATOS_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  ATOS_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, block, smem));
  if (per < 1) {
    set_error("kernel cannot be resident with block=%d smem=%zu", block, smem);
    return ATOS_ERR_INVALID_ARG;
  }
  *grid = per * sms;
  return ATOS_OK;
}

void set_l2_window(cudaStream_t s, void* base, size_t bytes, bool on) {
  cudaStreamAttrValue v;
  memset(&v, 0, sizeof(v));
  if (on && base && bytes) {
    int dev = 0, maxwin = 0, persist_max = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&maxwin, cudaDevAttrMaxAccessPolicyWindowSize, dev);
    cudaDeviceGetAttribute(&persist_max, cudaDevAttrMaxPersistingL2CacheSize, dev);
    if (maxwin <= 0 || persist_max <= 0) return;
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)persist_max);
    size_t win = std::min(bytes, (size_t)maxwin);
    v.accessPolicyWindow.base_ptr = base;
    v.accessPolicyWindow.num_bytes = win;
    v.accessPolicyWindow.hitRatio = std::min(1.0f, (float)persist_max / (float)win);
    v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
  } else {
    v.accessPolicyWindow.num_bytes = 0;
  }
  cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v);
  cudaGetLastError();  // best effort
}

void trace_mark(const char* what, bool sync) {
  static const bool on = getenv("ATOS_TRACE") != nullptr;
  if (!on) return;
  static thread_local std::chrono::steady_clock::time_point last = std::chrono::steady_clock::now();
  if (sync) cudaDeviceSynchronize();
  const auto now = std::chrono::steady_clock::now();
  fprintf(stderr, "[atos trace] %-28s %9.3f ms\n", what, std::chrono::duration<double, std::milli>(now - last).count());
  last = now;
}

int stream_wait(cudaStream_t s, double timeout_s) {
  if (timeout_s <= 0) {
    ATOS_CUDA(cudaStreamSynchronize(s));
    return ATOS_OK;
  }
  auto t0 = std::chrono::steady_clock::now();
  for (uint64_t polls = 0;; ++polls) {
    cudaError_t e = cudaStreamQuery(s);
    if (e == cudaSuccess) return ATOS_OK;
    if (e != cudaErrorNotReady) ATOS_CUDA(e);
    // busy-poll first: a discrete per-frontier launch lasts microseconds and a sleep would dominate it
    if (polls < 20000) continue;
    double el = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    if (el > timeout_s * 1.5 + 1.0) {
      set_error("stream did not finish within timeout_s=%.3f", timeout_s);
      return ATOS_ERR_TIMEOUT;
    }
    std::this_thread::sleep_for(std::chrono::microseconds(50));
  }
}

int finish_queue(Part& p, cudaStream_t s, atos_stats* st, const char* what) {
  QueueCtl* h = (QueueCtl*)p.host_pinned;  // first 1152 bytes of the pinned page
  static_assert(sizeof(QueueCtl) <= 4096, "control block fits the pinned page");
  ATOS_CUDA(cudaMemcpyAsync(h, p.ctl.p, sizeof(QueueCtl), cudaMemcpyDeviceToHost, s));
  ATOS_CUDA(cudaStreamSynchronize(s));
  ATOS_CUDA(cudaGetLastError());
  const uint32_t status = (uint32_t)h->status.v;
  if ((status || h->done.v != h->tail.v) && getenv("ATOS_DEBUG")) {
    fprintf(stderr, "[atos debug] %s: status=%u head=%llu tail=%llu done=%llu big_count=%lld pops=%llu\n", what,
            status, (unsigned long long)h->head.v, (unsigned long long)h->tail.v, (unsigned long long)h->done.v,
            (long long)h->big_count.v, (unsigned long long)h->stat_pops.v);
    if (p.big.p) {
      std::vector<BigTask> tb(kBigSlots);
      cudaMemcpy(tb.data(), p.big.p, sizeof(BigTask) * kBigSlots, cudaMemcpyDeviceToHost);
      for (uint32_t i = 0; i < kBigSlots; ++i)
        if (tb[i].state)
          fprintf(stderr, "  slot %u state=%u gen=%u nchunks=%u next=%u finished=%u deg=%u\n", i, tb[i].state,
                  big_gen(tb[i].ctr), big_nchunks(tb[i].ctr), big_next(tb[i].ctr), tb[i].finished, tb[i].deg);
    }
  }
  if (status & kStatusOverflow) {
    p.ring_clean = false;
    set_error("%s: queue overflow (ring of %llu slots lapped an unconsumed slot)", what,
              (unsigned long long)p.ring_cap);
    return ATOS_ERR_QUEUE_OVERFLOW;
  }
  if (status & kStatusTimeout) {
    p.ring_clean = false;
    set_error("%s: device watchdog expired (no progress)", what);
    return ATOS_ERR_TIMEOUT;
  }
  if (status & kStatusDeep) {
    // byte-state BFS stopped at an unencodable depth: the caller re-runs (the ring is reset then)
    p.ring_clean = false;
    return ATOS_OK;
  }
  if (h->done.v != h->tail.v) {
    p.ring_clean = false;
    set_error("%s: queue not drained (done=%llu tail=%llu)", what, (unsigned long long)h->done.v,
              (unsigned long long)h->tail.v);
    return ATOS_ERR_CUDA;
  }
  p.ring_clean = true;
  if (st) {
    st->pops += h->stat_pops.v;
    st->pushes += h->stat_pushes.v;
    st->edges += h->stat_edges.v;
    st->timeline_len = h->tl_count.v;
    if (h->stat_maxocc.v > st->max_queue_occupancy) st->max_queue_occupancy = h->stat_maxocc.v;
  }
  return ATOS_OK;
}

// ----------------------------------------------------- CSR upload / checks
__global__ void k_narrow_row_ptr(const int64_t* in, uint32_t* out, int64_t count, int64_t m, unsigned* bad) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = in[i];
    if (x < 0 || x > m || (i > 0 && in[i - 1] > x) || (i == 0 && x != 0) || (i == count - 1 && x != m))
      atomicOr(bad, 1u);
    out[i] = (uint32_t)x;
  }
}

__global__ void k_rebase_row_ptr(const int64_t* in, uint32_t* out, int64_t count, int64_t base) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = (uint32_t)(in[i] - base);
}

__global__ void k_check_col(const int32_t* col, uint32_t* out, int64_t m, int64_t n, unsigned* bad) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t c = col[i];
    if (c < 0 || (int64_t)c >= n) atomicOr(bad, 2u);
    if (out) out[i] = (uint32_t)c;
  }
}

// Upload a partition given its LOCAL arrays: row_ptr[0..nl] (any base offset,
// host or device) and the matching col[0..ml) (global ids).
int upload_part_local(Part& p, const int64_t* row_ptr, const int32_t* col, int where, int64_t nl, int64_t ml) {
  p.n_local = nl;
  p.m_local = ml;
  ATOS_TRY(dev_alloc_t(&p.row_ptr, nl + 1));
  ATOS_TRY(dev_alloc_t(&p.col, std::max<int64_t>(ml, 1)));
  if (where == ATOS_MEM_HOST) {
    const int64_t base = row_ptr[0];
    std::vector<uint32_t> rp((size_t)nl + 1);
    for (int64_t i = 0; i <= nl; ++i) rp[(size_t)i] = (uint32_t)(row_ptr[i] - base);
    ATOS_CUDA(cudaMemcpy(p.row_ptr, rp.data(), rp.size() * 4, cudaMemcpyHostToDevice));
    if (ml) ATOS_CUDA(cudaMemcpy(p.col, col, (size_t)ml * 4, cudaMemcpyHostToDevice));
    return ATOS_OK;
  }
  int64_t base = 0;
  ATOS_CUDA(cudaMemcpy(&base, row_ptr, 8, cudaMemcpyDeviceToHost));
  k_rebase_row_ptr<<<1024, 256>>>(row_ptr, p.row_ptr, nl + 1, base);
  g_launches++;
  ATOS_CUDA(cudaGetLastError());
  if (ml) ATOS_CUDA(cudaMemcpy(p.col, col, (size_t)ml * 4, cudaMemcpyDeviceToDevice));
  ATOS_CUDA(cudaDeviceSynchronize());
  return ATOS_OK;
}

// host CSR: the end points are checked here; monotonicity while the offsets are
// narrowed on the device (single partition: k_narrow_row_ptr in upload_part; loopback
// partitions: the host loop below) and col ids after the upload
// (validate_uploaded_cols) -- a host pass over n or m would cost more than the copy
static int validate_host_csr(int64_t n, int64_t m, const int64_t* row_ptr, const int32_t* col, bool full) {
  if (row_ptr[0] != 0 || row_ptr[n] != m) {
    set_error("row_ptr[0] must be 0 and row_ptr[n] must equal m");
    return ATOS_ERR_INVALID_ARG;
  }
  if (full)
    for (int64_t v = 0; v < n; ++v)
      if (row_ptr[v + 1] < row_ptr[v]) {
        set_error("row_ptr is not non-decreasing at %lld", (long long)v);
        return ATOS_ERR_INVALID_ARG;
      }
  (void)col;
  return ATOS_OK;
}

static int validate_uploaded_cols(atos_csr* g) {
  unsigned* bad = nullptr;
  ATOS_CUDA(cudaMalloc(&bad, 4));
  ATOS_CUDA(cudaMemset(bad, 0, 4));
  for (auto& p : g->parts)
    if (p.m_local) {
      k_check_col<<<1024, 256>>>((const int32_t*)p.col, nullptr, p.m_local, g->n, bad);
      g_launches++;
    }
  unsigned h = 0;
  ATOS_CUDA(cudaMemcpy(&h, bad, 4, cudaMemcpyDeviceToHost));
  cudaFree(bad);
  if (h) {
    set_error("col has ids outside [0, n)");
    return ATOS_ERR_INVALID_ARG;
  }
  return ATOS_OK;
}

static int validate_device_csr(int64_t n, int64_t m, const int64_t* row_ptr, const int32_t* col) {
  unsigned* bad = nullptr;
  uint32_t* scratch = nullptr;
  ATOS_CUDA(cudaMalloc(&bad, 4));
  ATOS_CUDA(cudaMemset(bad, 0, 4));
  ATOS_CUDA(cudaMalloc(&scratch, (size_t)(n + 1) * 4));
  k_narrow_row_ptr<<<1024, 256>>>(row_ptr, scratch, n + 1, m, bad);
  g_launches++;
  if (m) {
    k_check_col<<<1024, 256>>>(col, nullptr, m, n, bad);
    g_launches++;
  }
  unsigned h = 0;
  ATOS_CUDA(cudaMemcpy(&h, bad, 4, cudaMemcpyDeviceToHost));
  cudaFree(bad);
  cudaFree(scratch);
  if (h & 1u) {
    set_error("row_ptr invalid (must start at 0, be non-decreasing and end at m)");
    return ATOS_ERR_INVALID_ARG;
  }
  if (h & 2u) {
    set_error("col has ids outside [0, n)");
    return ATOS_ERR_INVALID_ARG;
  }
  return ATOS_OK;
}

void destroy_part(Part& p) {
  if (p.row_ptr) dev_free(p.row_ptr);
  if (p.col) dev_free(p.col);
  p.row_ptr = nullptr;
  p.col = nullptr;
  DevBuf* bufs[] = {&p.ring, &p.ctl, &p.big, &p.bitmap, &p.shadow, &p.vbuf_a, &p.vbuf_b, &p.vbuf_c, &p.scratch,
                    &p.ghost_a, &p.ghost_b, &p.touched, &p.outbox, &p.inbox, &p.out_val, &p.in_val, &p.pack,
                    &p.bsp_fa, &p.bsp_fb, &p.bsp_off, &p.bsp_tmp, &p.bsp_ctr, &p.nb_ring, &p.nb_ctl,
                    &p.nb_peers};
  for (DevBuf* b : bufs) b->release();
  pinned_page_release(p.host_pinned);
  for (void* b : p.nb_peer_base)
    if (b) cudaIpcCloseMemHandle(b);
  p.nb_peer_base.clear();
  if (p.nb_ipc) cudaFree(p.nb_ipc);
  p.nb_ipc = nullptr;
  p.nb_ipc_bytes = 0;
  p.host_pinned = nullptr;
}

int create_loopback_parts(atos_csr* g, const int64_t* row_ptr, const int32_t* col, int where);

// Output staging: device pointer given -> use it; host pointer -> internal buffer + D2H at the end.
template <class T>
int run_with_output(atos_csr* g, T* out, int64_t len, const Resolved& r, DevBuf& staging,
                           const std::function<int(T*)>& body) {
  if (g->relabeled) {
    // degree layout: the solver writes internal ids into staging and we scatter to the caller's ids,
    // unless it wrote the caller's ids itself (r.map_*: the byte-state BFS output pass gathers)
    ATOS_TRY(staging.ensure((size_t)std::max<int64_t>(len, 1) * sizeof(T)));
    T* dst = out;
    if (r.out_where != ATOS_MEM_DEVICE) {
      ATOS_TRY(g->perm_out.ensure((size_t)std::max<int64_t>(len, 1) * sizeof(T)));
      dst = g->perm_out.as<T>();
    }
    bool mapped = false;
    Resolved& rm = const_cast<Resolved&>(r);
    rm.map_o2n = g->o2n.as<uint32_t>();
    rm.map_out = dst;
    rm.map_done = &mapped;
    const int rc = body(staging.as<T>());
    rm.map_o2n = nullptr;
    rm.map_out = nullptr;
    rm.map_done = nullptr;
    ATOS_TRY(rc);
    if (!mapped) ATOS_TRY(layout_scatter<T>(g, staging.as<T>(), dst, r.stream));
    trace_mark("output: device", true);
    if (r.out_where != ATOS_MEM_DEVICE) {
      ATOS_CUDA(cudaMemcpyAsync(out, dst, (size_t)len * sizeof(T), cudaMemcpyDeviceToHost, r.stream));
      ATOS_CUDA(cudaStreamSynchronize(r.stream));
      trace_mark("output: D2H", true);
    }
    return ATOS_OK;
  }
  if (r.out_where == ATOS_MEM_DEVICE) return body(out);
  ATOS_TRY(staging.ensure((size_t)std::max<int64_t>(len, 1) * sizeof(T)));
  ATOS_TRY(body(staging.as<T>()));
  ATOS_CUDA(cudaMemcpyAsync(out, staging.p, (size_t)len * sizeof(T), cudaMemcpyDeviceToHost, r.stream));
  ATOS_CUDA(cudaStreamSynchronize(r.stream));
  return ATOS_OK;
}

}  // namespace atos

using namespace atos;

extern "C" {

void atos_cfg_default(atos_cfg* cfg) {
  if (!cfg) return;
  memset(cfg, 0, sizeof(*cfg));
  cfg->struct_size = sizeof(atos_cfg);
  cfg->persistent = 1;
  cfg->worker = 0;
  cfg->fetch_size = 0;
  cfg->dedupe = 1;
  cfg->out_where = ATOS_MEM_DEVICE;
}

const char* atos_last_error(void) { return g_err; }
int atos_version(void) { return ATOS_VERSION; }
uint64_t atos_kernel_launches(void) { return g_launches.load(); }

int atos_csr_create(atos_csr** out, int64_t n, int64_t m, const int64_t* row_ptr, const int32_t* col, int where,
                    int device, int num_parts) {
  return atos_csr_create_ex(out, n, m, row_ptr, col, where, device, num_parts, ATOS_LAYOUT_AUTO);
}

int atos_csr_create_ex(atos_csr** out, int64_t n, int64_t m, const int64_t* row_ptr, const int32_t* col, int where,
                       int device, int num_parts, int flags) {
  if (!out || n < 0 || m < 0 || (n > 0 && !row_ptr) || (m > 0 && !col) || num_parts < 1 ||
      (where != ATOS_MEM_HOST && where != ATOS_MEM_DEVICE) ||
      (flags != ATOS_LAYOUT_AUTO && flags != ATOS_LAYOUT_INPUT && flags != ATOS_LAYOUT_DEGREE)) {
    set_error("atos_csr_create: invalid argument");
    return ATOS_ERR_INVALID_ARG;
  }
  *out = nullptr;
  if (m >= (int64_t)0xFFFFFFFFll || n >= (int64_t)0x7FFFFFFFll) {
    set_error("atos_csr_create: n < 2^31 and m < 2^32 required (n=%lld m=%lld)", (long long)n, (long long)m);
    return ATOS_ERR_UNSUPPORTED;
  }
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    set_error("atos_csr_create: no CUDA device (%s)", cudaGetErrorString(e));
    return ATOS_ERR_CUDA;
  }
  if (device < 0 || device >= ndev) {
    set_error("atos_csr_create: device %d out of range (have %d)", device, ndev);
    return ATOS_ERR_INVALID_ARG;
  }
  DeviceGuard dg(device);
  if (n > 0 && where == ATOS_MEM_HOST) {
    int rc = validate_host_csr(n, m, row_ptr, col, num_parts > 1);  // end points (+ monotone for partitions)
    if (rc != ATOS_OK) return rc;
  }
  if (n > 0 && where == ATOS_MEM_DEVICE && num_parts > 1) {
    int rc = validate_device_csr(n, m, row_ptr, col);
    if (rc != ATOS_OK) return rc;
  }
  atos_csr* g = new atos_csr();
  g->device = device;
  g->n = n;
  g->m = m;
  g->num_parts = num_parts;
  // single partition: pipelined upload, validation and layout in one pass (layout.cu); partitions keep the ids
  int rc = num_parts == 1 ? create_single(g, row_ptr, col, where, flags) : create_loopback_parts(g, row_ptr, col, where);
  if (rc == ATOS_OK && num_parts > 1 && where == ATOS_MEM_HOST) rc = validate_uploaded_cols(g);
  if (rc != ATOS_OK) {
    atos_csr_destroy(g);
    return rc;
  }
  *out = g;
  return ATOS_OK;
}

void atos_csr_destroy(atos_csr* g) {
  if (!g) return;
  {
    DeviceGuard dg(g->device);
    for (auto& p : g->parts) destroy_part(p);
    g->o2n.release();
    g->n2o.release();
    g->perm_out.release();
  }
  delete g;
}

int atos_csr_info(const atos_csr* g, int64_t* n, int64_t* m, int* num_parts) {
  if (!g) {
    set_error("atos_csr_info: null handle");
    return ATOS_ERR_INVALID_ARG;
  }
  if (n) *n = g->n;
  if (m) *m = g->m;
  if (num_parts) *num_parts = g->comm ? g->nranks : g->num_parts;
  return ATOS_OK;
}

int atos_csr_layout(const atos_csr* g, int* layout) {
  if (!g || !layout) {
    set_error("atos_csr_layout: null argument");
    return ATOS_ERR_INVALID_ARG;
  }
  *layout = g->relabeled ? ATOS_LAYOUT_DEGREE : ATOS_LAYOUT_INPUT;
  return ATOS_OK;
}

int atos_bfs(const atos_csr* gc, int64_t src, uint32_t* depth_out, const atos_cfg* cfg) {
  atos_csr* g = const_cast<atos_csr*>(gc);
  if (!g || !depth_out) {
    set_error("atos_bfs: null argument");
    return ATOS_ERR_INVALID_ARG;
  }
  if (src < 0 || src >= g->n) {
    set_error("atos_bfs: src %lld out of range [0, %lld)", (long long)src, (long long)g->n);
    return ATOS_ERR_INVALID_ARG;
  }
  Resolved r;
  ATOS_TRY(resolve_cfg(cfg, 'b', &r));
  std::lock_guard<std::mutex> lk(g->mu);
  DeviceGuard dg(g->device);
  atos_stats local{};
  atos_stats* st = r.stats ? &local : nullptr;
  CallTimer tm(r.stream);
  int rc;
  if (r.barrier_free) {
    if (!g->comm && g->num_parts < 2) {
      set_error("atos_bfs: barrier_free needs a partitioned graph (loopback num_parts > 1, or one partition per "
                "process)");
      return ATOS_ERR_UNSUPPORTED;
    }
    const int64_t len = g->comm ? g->parts[0].n_local : g->n;
    rc = run_with_output<uint32_t>(g, depth_out, len, r, g->parts[0].vbuf_c,
                                   [&](uint32_t* d) { return bfs_nobarrier(g, src, d, r, st); });
  } else if (g->comm || g->num_parts > 1) {
    const int64_t len = g->comm ? g->parts[0].n_local : g->n;
    rc = run_with_output<uint32_t>(g, depth_out, len, r, g->parts[0].vbuf_c,
                                   [&](uint32_t* d) { return bfs_partitioned(g, src, d, r, st); });
  } else {
    rc = run_with_output<uint32_t>(g, depth_out, g->n, r, g->parts[0].vbuf_c,
                                   [&](uint32_t* d) {
                                     const int64_t isrc = layout_vertex(g, src);  // degree layout: internal id
                                     if (isrc < 0) return (int)ATOS_ERR_CUDA;
                                     return bfs_single(g, g->parts[0], isrc, d, r, st);
                                   });
    if (st) st->pushes += 1;
  }
  const double ms = tm.stop();
  if (rc == ATOS_OK && r.stats) {
    local.kernel_ms = ms;
    *r.stats = local;
  }
  return rc;
}

int atos_pagerank(const atos_csr* gc, double alpha, double eps, double* rank_out, const atos_cfg* cfg) {
  atos_csr* g = const_cast<atos_csr*>(gc);
  if (!g || !rank_out) {
    set_error("atos_pagerank: null argument");
    return ATOS_ERR_INVALID_ARG;
  }
  if (!(alpha > 0.0 && alpha < 1.0) || !(eps > 0.0)) {
    set_error("atos_pagerank: alpha must be in (0,1) and eps > 0 (alpha=%g eps=%g)", alpha, eps);
    return ATOS_ERR_INVALID_ARG;
  }
  Resolved r;
  ATOS_TRY(resolve_cfg(cfg, 'p', &r));
  std::lock_guard<std::mutex> lk(g->mu);
  DeviceGuard dg(g->device);
  atos_stats local{};
  atos_stats* st = r.stats ? &local : nullptr;
  CallTimer tm(r.stream);
  int rc;
  if (g->n == 0) return ATOS_OK;
  if (r.barrier_free) {
    if (!g->comm && g->num_parts < 2) {
      set_error("atos_pagerank: barrier_free needs a partitioned graph (loopback num_parts > 1, or one partition "
                "per process)");
      return ATOS_ERR_UNSUPPORTED;
    }
    const int64_t len = g->comm ? g->parts[0].n_local : g->n;
    rc = run_with_output<double>(g, rank_out, len, r, g->parts[0].vbuf_c,
                                 [&](double* d) { return pagerank_nobarrier(g, alpha, eps, d, r, st); });
  } else if (g->comm || g->num_parts > 1) {
    const int64_t len = g->comm ? g->parts[0].n_local : g->n;
    rc = run_with_output<double>(g, rank_out, len, r, g->parts[0].vbuf_c,
                                 [&](double* d) { return pagerank_partitioned(g, alpha, eps, d, r, st); });
  } else {
    rc = run_with_output<double>(g, rank_out, g->n, r, g->parts[0].vbuf_c,
                                 [&](double* d) { return pagerank_single(g, g->parts[0], alpha, eps, d, r, st); });
  }
  const double ms = tm.stop();
  if (rc == ATOS_OK && r.stats) {
    local.kernel_ms = ms;
    *r.stats = local;
  }
  return rc;
}

int atos_color(const atos_csr* gc, uint64_t seed, int32_t* color_out, const atos_cfg* cfg) {
  atos_csr* g = const_cast<atos_csr*>(gc);
  if (!g || !color_out) {
    set_error("atos_color: null argument");
    return ATOS_ERR_INVALID_ARG;
  }
  if (g->comm || g->num_parts > 1) {
    set_error("atos_color: colouring runs on a single partition only (replicas only, DESIGN.md)");
    return ATOS_ERR_UNSUPPORTED;
  }
  Resolved r;
  ATOS_TRY(resolve_cfg(cfg, 'c', &r));
  std::lock_guard<std::mutex> lk(g->mu);
  DeviceGuard dg(g->device);
  atos_stats local{};
  atos_stats* st = r.stats ? &local : nullptr;
  CallTimer tm(r.stream);
  if (g->n == 0) return ATOS_OK;
  int rc = run_with_output<int32_t>(g, color_out, g->n, r, g->parts[0].vbuf_c,
                                    [&](int32_t* d) { return color_single(g, g->parts[0], seed, d, r, st); });
  const double ms = tm.stop();
  if (rc == ATOS_OK && r.stats) {
    local.kernel_ms = ms;
    *r.stats = local;
  }
  return rc;
}

// ---- bulk-synchronous baselines (bsp.cu) ----------------
int atos_bfs_bsp(const atos_csr* gc, int64_t src, uint32_t* depth_out, const atos_cfg* cfg) {
  atos_csr* g = const_cast<atos_csr*>(gc);
  if (!g || !depth_out) {
    set_error("atos_bfs_bsp: null argument");
    return ATOS_ERR_INVALID_ARG;
  }
  if (src < 0 || src >= g->n) {
    set_error("atos_bfs_bsp: src %lld out of range [0, %lld)", (long long)src, (long long)g->n);
    return ATOS_ERR_INVALID_ARG;
  }
  if (g->comm || g->num_parts > 1) {
    set_error("atos_bfs_bsp: the BSP baseline runs on a single partition only");
    return ATOS_ERR_UNSUPPORTED;
  }
  Resolved r;
  ATOS_TRY(resolve_cfg(cfg, 'b', &r));
  std::lock_guard<std::mutex> lk(g->mu);
  DeviceGuard dg(g->device);
  atos_stats local{};
  atos_stats* st = r.stats ? &local : nullptr;
  CallTimer tm(r.stream);
  if (g->n == 0) return ATOS_OK;
  int rc = run_with_output<uint32_t>(g, depth_out, g->n, r, g->parts[0].vbuf_c,
                              [&](uint32_t* d) {
                                const int64_t isrc = layout_vertex(g, src);
                                if (isrc < 0) return (int)ATOS_ERR_CUDA;
                                return bfs_bsp_single(g, g->parts[0], isrc, d, r, st);
                              });
  const double ms = tm.stop();
  if (rc == ATOS_OK && r.stats) {
    local.kernel_ms = ms;
    *r.stats = local;
  }
  return rc;
}

int atos_pagerank_bsp(const atos_csr* gc, double alpha, double eps, double* rank_out, const atos_cfg* cfg) {
  atos_csr* g = const_cast<atos_csr*>(gc);
  if (!g || !rank_out) {
    set_error("atos_pagerank_bsp: null argument");
    return ATOS_ERR_INVALID_ARG;
  }
  if (!(alpha > 0.0 && alpha < 1.0) || !(eps > 0.0)) {
    set_error("atos_pagerank_bsp: alpha must be in (0,1) and eps > 0 (alpha=%g eps=%g)", alpha, eps);
    return ATOS_ERR_INVALID_ARG;
  }
  if (g->comm || g->num_parts > 1) {
    set_error("atos_pagerank_bsp: the BSP baseline runs on a single partition only");
    return ATOS_ERR_UNSUPPORTED;
  }
  Resolved r;
  ATOS_TRY(resolve_cfg(cfg, 'p', &r));
  std::lock_guard<std::mutex> lk(g->mu);
  DeviceGuard dg(g->device);
  atos_stats local{};
  atos_stats* st = r.stats ? &local : nullptr;
  CallTimer tm(r.stream);
  if (g->n == 0) return ATOS_OK;
  int rc = run_with_output<double>(g, rank_out, g->n, r, g->parts[0].vbuf_c,
                              [&](double* d) { return pagerank_bsp_single(g, g->parts[0], alpha, eps, d, r, st); });
  const double ms = tm.stop();
  if (rc == ATOS_OK && r.stats) {
    local.kernel_ms = ms;
    *r.stats = local;
  }
  return rc;
}

int atos_color_bsp(const atos_csr* gc, uint64_t seed, int32_t* color_out, const atos_cfg* cfg) {
  atos_csr* g = const_cast<atos_csr*>(gc);
  if (!g || !color_out) {
    set_error("atos_color_bsp: null argument");
    return ATOS_ERR_INVALID_ARG;
  }
  if (g->comm || g->num_parts > 1) {
    set_error("atos_color_bsp: the BSP baseline runs on a single partition only");
    return ATOS_ERR_UNSUPPORTED;
  }
  Resolved r;
  ATOS_TRY(resolve_cfg(cfg, 'c', &r));
  std::lock_guard<std::mutex> lk(g->mu);
  DeviceGuard dg(g->device);
  atos_stats local{};
  atos_stats* st = r.stats ? &local : nullptr;
  CallTimer tm(r.stream);
  if (g->n == 0) return ATOS_OK;
  int rc = run_with_output<int32_t>(g, color_out, g->n, r, g->parts[0].vbuf_c,
                              [&](int32_t* d) { return color_bsp_single(g, g->parts[0], seed, d, r, st); });
  const double ms = tm.stop();
  if (rc == ATOS_OK && r.stats) {
    local.kernel_ms = ms;
    *r.stats = local;
  }
  return rc;
}

int atos_partition_range(int64_t n, int nparts, int part, int64_t* v_begin, int64_t* v_end) {
  if (n < 0 || nparts < 1 || part < 0 || part >= nparts || !v_begin || !v_end) {
    set_error("atos_partition_range: invalid argument");
    return ATOS_ERR_INVALID_ARG;
  }
  const int64_t chunk = (n + nparts - 1) / nparts;
  *v_begin = std::min<int64_t>(n, (int64_t)part * chunk);
  *v_end = std::min<int64_t>(n, (int64_t)(part + 1) * chunk);
  return ATOS_OK;
}

}  // extern "C"
