// layout.cu -- S0 residency of a single-partition graph: the pipelined upload and validation, and the
// degree layout ("Degree layout").
//
// The generators (and real inputs) hand us vertex ids in random order, so the
// per-vertex state of the hubs -- which receive most relaxations -- is spread
// over the whole state array.  When that array is larger than L2 (C5: the
// PageRank residue is 537 MB, L2 126 MB) most of the per-edge f64 atomics miss
// L2.  At creation the CSR is relabelled once:
//   rank r = position of v in descending-degree order (stable, by old id);
//   new id = r (T = 1 since round 2: the interleave below moved into PageRank's residue addressing,
//            apps.cuh res_slot); with T > 1 (ATOS_LAYOUT_T) the first 16*T ranks are interleaved as
//            (r mod T) * 16 + r / T,
// which packs the hot set into a prefix of the state arrays (L2-resident) but
// gives each of the T hottest vertices its own 128-byte line of an f64 array,
// so the hubs' atomics do not serialise on shared lines/slices (without the
// interleave C3 PageRank, whose state already fits L2, ran 2x slower).
// Measured (tools/relabel_probe.py): C5 PageRank 2652 -> 1243 ms, C5 BFS
// 14.7 -> 13.2 ms, C3 within 3 %.  The interleave width T trades the two C5 workloads (tools/layout_probe.py,
// profiles/r02_layout_interleave.txt): the BFS byte state wants the hubs packed (32 per sector), the PageRank
// f64 residues want them apart -- T = 65536 / 4096 / 1 (none): BFS 13.15 / 12.77 / 12.59 ms, PageRank 1173 /
// 1192 / 1775 ms.  Since round 2 the ids use T = 1 and PageRank interleaves its own residue / rank arrays
// (apps.cuh res_slot): BFS 12.6 ms and PageRank 1.19 s at once.
//
// The method is unchanged: every call maps the source into the internal ids
// and scatters its output back (out[old] = result[new]); colouring seeds its
// queue in the caller's vertex-id order.  Loopback / NCCL partitions keep the
// input ids (a degree-sorted block partition would put every hub on part 0).
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <algorithm>
#include <vector>

#include "internal.h"

namespace atos {

__global__ void k_layout_degrees(const uint32_t* __restrict__ rp, int64_t n, uint32_t* deg, uint32_t* ids) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    deg[v] = rp[v + 1] - rp[v];
    ids[v] = (uint32_t)v;
  }
}

__global__ void k_layout_place(const uint32_t* __restrict__ deg_sorted, const uint32_t* __restrict__ order, int64_t n,
                               uint32_t T, uint32_t* n2o, uint32_t* o2n, uint32_t* ndeg) {
  const int64_t spread = 16 * (int64_t)T;
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t pos = r < spread ? (r % T) * 16 + r / T : r;
    const uint32_t old = order[r];
    n2o[pos] = old;
    o2n[old] = (uint32_t)pos;
    ndeg[pos] = deg_sorted[r];
  }
}

__global__ void k_layout_set_last(uint32_t* rp_new, int64_t n, uint32_t m) {
  if (threadIdx.x == 0 && blockIdx.x == 0) rp_new[n] = m;
}

// Per old row v: the offset that moves its edges to their new row, base[v] = rp_new[o2n[v]] - rp_old[v]
// (an edge e of old row v lands at e + base[v]).
__global__ void k_layout_row_base(const uint32_t* __restrict__ rp_old, const uint32_t* __restrict__ rp_new,
                                  const uint32_t* __restrict__ o2n, int64_t n, uint32_t* base) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    base[v] = rp_new[o2n[v]] - rp_old[v];
}

// Edge-parallel relabel of one chunk [e0, e0 + cnt) of the OLD col array (a staging buffer of the H2D
// pipeline, or the caller's device array): col_new[e + base[row(e)]] = o2n[col[e]], with the ids
// checked (< n) on the way.  A block takes tiles of kTile consecutive edges; two global searches bound
// the tile's old rows, whose starts and bases are staged in shared memory, and every thread finds its
// edges' rows by binary search there (rows of consecutive edges are consecutive, so the new positions
// -- and the writes -- stay contiguous within a row).  Replaces a warp-per-row gather (64 ms at C5,
// 34 M isolated rows).
constexpr int kRemapThreads = 256, kRemapPer = 8, kRemapTile = kRemapThreads * kRemapPer, kRemapRows = 2048;
__global__ void __launch_bounds__(kRemapThreads) k_layout_remap(const uint32_t* __restrict__ rp_old, int64_t n,
                                                               const uint32_t* __restrict__ base,
                                                               const int32_t* __restrict__ col_chunk, uint32_t e0,
                                                               uint32_t cnt, const uint32_t* __restrict__ o2n,
                                                               uint32_t* __restrict__ col_new, unsigned* bad) {
  __shared__ uint32_t s_start[kRemapRows + 1], s_base[kRemapRows];
  __shared__ uint32_t s_r[2];
  for (uint64_t t = (uint64_t)blockIdx.x * kRemapTile; t < cnt; t += (uint64_t)gridDim.x * kRemapTile) {
    const uint32_t a = e0 + (uint32_t)t;
    const uint64_t tend = t + kRemapTile < (uint64_t)cnt ? t + kRemapTile : (uint64_t)cnt;
    const uint32_t b = e0 + (uint32_t)tend - 1;  // last edge of the tile
    if (threadIdx.x == 0 || threadIdx.x == 32) {
      const uint32_t e = threadIdx.x == 0 ? a : b;
      uint32_t lo = 0, hi = (uint32_t)n - 1;  // largest r with rp_old[r] <= e (skips empty rows)
      while (lo < hi) {
        const uint32_t mid = lo + ((hi - lo + 1) >> 1);
        if (__ldg(rp_old + mid) <= e) lo = mid; else hi = mid - 1;
      }
      s_r[threadIdx.x == 0 ? 0 : 1] = lo;
    }
    __syncthreads();
    const uint32_t r0 = s_r[0], nr = s_r[1] - s_r[0] + 1;
    const bool staged = nr <= kRemapRows;
    if (staged)
      for (uint32_t i = threadIdx.x; i < nr; i += kRemapThreads) {
        s_start[i] = __ldg(rp_old + r0 + i);
        s_base[i] = __ldg(base + r0 + i);
      }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kRemapPer; ++k) {
      const uint32_t e = a + k * kRemapThreads + threadIdx.x;
      if (e > b) continue;
      uint32_t lo = 0, hi = nr - 1, off;
      if (staged) {
        while (lo < hi) {
          const uint32_t mid = lo + ((hi - lo + 1) >> 1);
          if (s_start[mid] <= e) lo = mid; else hi = mid - 1;
        }
        off = s_base[lo];
      } else {
        while (lo < hi) {
          const uint32_t mid = lo + ((hi - lo + 1) >> 1);
          if (__ldg(rp_old + r0 + mid) <= e) lo = mid; else hi = mid - 1;
        }
        off = __ldg(base + r0 + lo);
      }
      const int32_t w = __ldcs(col_chunk + (e - e0));
      if (w < 0 || (int64_t)w >= n) {
        atomicOr(bad, 2u);
        continue;
      }
      col_new[e + off] = __ldg(o2n + w);
    }
    __syncthreads();
  }
}

// o2n / n2o and the new offsets rp_new[n+1] from the (narrowed) old offsets; `base` = per-old-row shift.
int layout_prepare(atos_csr* g, const uint32_t* rp_old, int64_t n, int64_t m, cudaStream_t s, DevBuf& rp_new,
                   DevBuf& base) {
  // T = 1: no interleave of the ids (the BFS byte state wants the hubs packed); single-partition PageRank
  // spreads its residues itself (res_slot in apps.cuh)
  uint32_t T = 1;
  if (const char* e = getenv("ATOS_LAYOUT_T")) T = (uint32_t)std::max<int64_t>(1, std::min<int64_t>(atol(e), n / 16));
  struct Scratch {  // released on every return path
    DevBuf deg, ids, deg_s, order, ndeg, tmp;
    ~Scratch() {
      for (DevBuf* b : {&deg, &ids, &deg_s, &order, &ndeg, &tmp}) b->release();
    }
  } w;
  ATOS_TRY(w.deg.ensure(n * 4));
  ATOS_TRY(w.ids.ensure(n * 4));
  ATOS_TRY(w.deg_s.ensure(n * 4));
  ATOS_TRY(w.order.ensure(n * 4));
  ATOS_TRY(w.ndeg.ensure(n * 4));
  ATOS_TRY(rp_new.ensure((n + 1) * 4));
  ATOS_TRY(base.ensure(n * 4));
  ATOS_TRY(g->o2n.ensure(n * 4));
  ATOS_TRY(g->n2o.ensure(n * 4));
  const int gs = 148 * 8;
  k_layout_degrees<<<gs, 256, 0, s>>>(rp_old, n, w.deg.as<uint32_t>(), w.ids.as<uint32_t>());
  size_t tb = 0, tb2 = 0;
  ATOS_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, w.deg.as<uint32_t>(), w.deg_s.as<uint32_t>(),
                                                      w.ids.as<uint32_t>(), w.order.as<uint32_t>(), (int)n, 0, 32, s));
  ATOS_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb2, w.ndeg.as<uint32_t>(), rp_new.as<uint32_t>(), (int)n, s));
  ATOS_TRY(w.tmp.ensure(std::max(tb, tb2)));
  ATOS_CUDA(cub::DeviceRadixSort::SortPairsDescending(w.tmp.p, tb, w.deg.as<uint32_t>(), w.deg_s.as<uint32_t>(),
                                                      w.ids.as<uint32_t>(), w.order.as<uint32_t>(), (int)n, 0, 32, s));
  k_layout_place<<<gs, 256, 0, s>>>(w.deg_s.as<uint32_t>(), w.order.as<uint32_t>(), n, T, g->n2o.as<uint32_t>(),
                                    g->o2n.as<uint32_t>(), w.ndeg.as<uint32_t>());
  ATOS_CUDA(cub::DeviceScan::ExclusiveSum(w.tmp.p, tb2, w.ndeg.as<uint32_t>(), rp_new.as<uint32_t>(), (int)n, s));
  k_layout_set_last<<<1, 32, 0, s>>>(rp_new.as<uint32_t>(), n, (uint32_t)m);
  k_layout_row_base<<<gs, 256, 0, s>>>(rp_old, rp_new.as<uint32_t>(), g->o2n.as<uint32_t>(), n, base.as<uint32_t>());
  g_launches += 7;
  ATOS_CUDA(cudaGetLastError());
  ATOS_CUDA(cudaStreamSynchronize(s));  // the scratch buffers are released at return
  return ATOS_OK;
}

// ------------------------------------------------------------------ S0 residency
__global__ void k_narrow_offsets(const int64_t* in, uint32_t* out, int64_t count, int64_t m, unsigned* bad) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = in[i];
    if (x < 0 || x > m || (i > 0 && in[i - 1] > x) || (i == 0 && x != 0) || (i == count - 1 && x != m))
      atomicOr(bad, 1u);
    out[i] = (uint32_t)x;
  }
}

__global__ void k_copy_check_col(const int32_t* __restrict__ col, uint32_t* __restrict__ out, int64_t cnt, int64_t n,
                                 unsigned* bad) {
  // 16-byte vectors when both pointers allow it (pool blocks and chunk starts do; a caller's array may not)
  const int64_t nv = (((uintptr_t)col | (uintptr_t)out) & 15u) ? 0 : cnt / 4;
  const int4* in4 = (const int4*)col;
  uint4* out4 = (uint4*)out;
  unsigned b = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nv; i += (int64_t)gridDim.x * blockDim.x) {
    const int4 v = __ldcs(in4 + i);
    b |= (v.x < 0 || v.x >= n || v.y < 0 || v.y >= n || v.z < 0 || v.z >= n || v.w < 0 || v.w >= n) ? 2u : 0u;
    if (out) out4[i] = make_uint4((uint32_t)v.x, (uint32_t)v.y, (uint32_t)v.z, (uint32_t)v.w);
  }
  for (int64_t i = 4 * nv + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = col[i];
    b |= (v < 0 || v >= n) ? 2u : 0u;
    if (out) out[i] = (uint32_t)v;
  }
  if (__any_sync(0xffffffffu, b != 0) && b) atomicOr(bad, b);
}

__global__ void k_max_deg(const uint32_t* row_ptr, int64_t n, unsigned long long* mx) {
  unsigned long long best = 0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    best = max(best, (unsigned long long)(row_ptr[v + 1] - row_ptr[v]));
  for (int o = 16; o; o >>= 1) best = max(best, __shfl_xor_sync(0xffffffffu, best, o));
  if (lane_id() == 0) atomicMax(mx, best);
}

namespace {
// streams / events of one creation (released on every return path)
struct UploadCtx {
  cudaStream_t cs = nullptr, ks = nullptr;  // copy stream, kernel stream
  std::vector<cudaEvent_t> ev;
  ~UploadCtx() {
    if (cs) cudaStreamSynchronize(cs);
    if (ks) cudaStreamSynchronize(ks);
    for (cudaEvent_t e : ev) cudaEventDestroy(e);
    if (cs) cudaStreamDestroy(cs);
    if (ks) cudaStreamDestroy(ks);
  }
};
constexpr int64_t kChunkEdges = 32ll << 20;  // 128 MB of col per pipeline stage
constexpr int kStages = 4;
}  // namespace

// Single-partition residency (S0): narrow + validate the offsets, decide the layout, and bring col in
// -- from HOST memory as a pipeline of chunked H2D copies on one stream with the per-chunk kernel
// (check ids; with the degree layout, relabel straight into the final array) on another, so the
// transfer overlaps all device work and the old col never exists on the device in full; from DEVICE
// memory in one pass (check + copy, or check + relabel) over the caller's array.
int create_single(atos_csr* g, const int64_t* row_ptr, const int32_t* col, int where, int flags) {
  g->parts.resize(1);
  Part& p = g->parts[0];
  const int64_t n = g->n, m = g->m;
  p.v_begin = 0;
  p.v_end = n;
  p.n_local = n;
  p.m_local = m;
  // device input may still be in flight on the caller's stream (e.g. just produced by torch): the
  // creation streams below are non-blocking, so wait for the device first
  if (where == ATOS_MEM_DEVICE) ATOS_CUDA(cudaDeviceSynchronize());
  UploadCtx cx;
  ATOS_CUDA(cudaStreamCreateWithFlags(&cx.cs, cudaStreamNonBlocking));
  ATOS_CUDA(cudaStreamCreateWithFlags(&cx.ks, cudaStreamNonBlocking));
  DevBuf rp64, flags_buf, rp_new, base, stage;
  struct Rel {
    DevBuf* b[5];
    ~Rel() { for (DevBuf* x : b) x->release(); }
  } rel{{&rp64, &flags_buf, &base, &stage, &rp_new}};
  ATOS_TRY(flags_buf.ensure(64));
  unsigned* bad = flags_buf.as<unsigned>();
  unsigned long long* mxd = (unsigned long long*)(flags_buf.as<char>() + 16);
  ATOS_CUDA(cudaMemsetAsync(flags_buf.p, 0, 64, cx.ks));
  ATOS_TRY(dev_alloc_t(&p.row_ptr, n + 1));
  const int gs = 148 * 8;
  // 1. offsets: narrow to u32 and validate (monotone, 0 .. m) on the device
  const int64_t* rp_src = row_ptr;
  if (where == ATOS_MEM_HOST) {
    ATOS_TRY(rp64.ensure((size_t)(n + 1) * 8));
    ATOS_CUDA(cudaMemcpyAsync(rp64.p, row_ptr, (size_t)(n + 1) * 8, cudaMemcpyHostToDevice, cx.ks));
    rp_src = rp64.as<int64_t>();
  }
  k_narrow_offsets<<<gs, 256, 0, cx.ks>>>(rp_src, p.row_ptr, n + 1, m, bad);
  k_max_deg<<<gs, 256, 0, cx.ks>>>(p.row_ptr, n, mxd);
  g_launches += 2;
  unsigned long long hmx = 0;
  unsigned hbad = 0;
  ATOS_CUDA(cudaMemcpyAsync(&hmx, mxd, 8, cudaMemcpyDeviceToHost, cx.ks));
  ATOS_CUDA(cudaMemcpyAsync(&hbad, bad, 4, cudaMemcpyDeviceToHost, cx.ks));
  ATOS_CUDA(cudaStreamSynchronize(cx.ks));
  rp64.release();
  if (hbad) {
    set_error("row_ptr invalid (must start at 0, be non-decreasing and end at m)");
    return ATOS_ERR_INVALID_ARG;
  }
  g->max_degree = (int64_t)hmx;
  p.max_deg = hmx;
  // 2. layout decision (ATOS_LAYOUT_AUTO: an f64 per-vertex array would not fit half of L2, and the
  //    degrees are skewed)
  bool want = flags == ATOS_LAYOUT_DEGREE;
  if (flags == ATOS_LAYOUT_AUTO) {
    int l2 = 0;
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, g->device);
    const int64_t avg = std::max<int64_t>(1, n > 0 ? m / n : 1);
    want = n * 8 > (int64_t)l2 / 2 && g->max_degree >= 32 * avg;
  }
  if (n < 2) want = false;
  if (want) ATOS_TRY(layout_prepare(g, p.row_ptr, n, m, cx.ks, rp_new, base));
  // 3. col
  ATOS_TRY(dev_alloc_t(&p.col, std::max<int64_t>(m, 1)));
  if (m > 0) {
    if (where == ATOS_MEM_DEVICE) {
      if (want) {
        k_layout_remap<<<gs * 2, kRemapThreads, 0, cx.ks>>>(p.row_ptr, n, base.as<uint32_t>(), col, 0, (uint32_t)m,
                                                           g->o2n.as<uint32_t>(), p.col, bad);
      } else {
        k_copy_check_col<<<gs * 2, 256, 0, cx.ks>>>(col, p.col, m, n, bad);
      }
      g_launches++;
    } else {
      // pipelined H2D: chunk c is copied on cs into its final place (input layout) or into staging slot
      // c % kStages (degree layout), then checked / relabelled on ks; a staging slot is re-filled only
      // after the kernel that read it finished.
      const int64_t nchunks = (m + kChunkEdges - 1) / kChunkEdges;
      if (want) ATOS_TRY(stage.ensure((size_t)kStages * kChunkEdges * 4));
      cx.ev.resize(2 * nchunks);
      for (auto& e : cx.ev) ATOS_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
      for (int64_t c = 0; c < nchunks; ++c) {
        const int64_t e0 = c * kChunkEdges, cnt = std::min(kChunkEdges, m - e0);
        int32_t* dst = want ? stage.as<int32_t>() + (c % kStages) * kChunkEdges : (int32_t*)(p.col + e0);
        if (want && c >= kStages) ATOS_CUDA(cudaStreamWaitEvent(cx.cs, cx.ev[2 * (c - kStages) + 1], 0));
        ATOS_CUDA(cudaMemcpyAsync(dst, col + e0, (size_t)cnt * 4, cudaMemcpyHostToDevice, cx.cs));
        ATOS_CUDA(cudaEventRecord(cx.ev[2 * c], cx.cs));
        ATOS_CUDA(cudaStreamWaitEvent(cx.ks, cx.ev[2 * c], 0));
        if (want) {
          k_layout_remap<<<gs, kRemapThreads, 0, cx.ks>>>(p.row_ptr, n, base.as<uint32_t>(), dst, (uint32_t)e0,
                                                         (uint32_t)cnt, g->o2n.as<uint32_t>(), p.col, bad);
        } else {
          k_copy_check_col<<<gs, 256, 0, cx.ks>>>(dst, nullptr, cnt, n, bad);
        }
        g_launches++;
        ATOS_CUDA(cudaEventRecord(cx.ev[2 * c + 1], cx.ks));
      }
    }
  }
  ATOS_CUDA(cudaGetLastError());
  ATOS_CUDA(cudaMemcpyAsync(&hbad, bad, 4, cudaMemcpyDeviceToHost, cx.ks));
  ATOS_CUDA(cudaStreamSynchronize(cx.cs));
  ATOS_CUDA(cudaStreamSynchronize(cx.ks));
  if (hbad & 2u) {
    set_error("col has ids outside [0, n)");
    return ATOS_ERR_INVALID_ARG;
  }
  if (want) {
    dev_free(p.row_ptr);
    p.row_ptr = rp_new.as<uint32_t>();
    rp_new.p = nullptr;
    rp_new.bytes = 0;
    g->relabeled = true;
  }
  return ATOS_OK;
}

template <class T>
__global__ void k_layout_scatter(const T* __restrict__ in, const uint32_t* __restrict__ n2o, int64_t n, T* out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    out[n2o[i]] = in[i];
}

template <class T>
int layout_scatter(const atos_csr* g, const T* in, T* out, cudaStream_t s) {
  k_layout_scatter<T><<<148 * 8, 256, 0, s>>>(in, g->n2o.as<uint32_t>(), g->n, out);
  g_launches++;
  ATOS_CUDA(cudaGetLastError());
  return ATOS_OK;
}
template int layout_scatter<uint32_t>(const atos_csr*, const uint32_t*, uint32_t*, cudaStream_t);
template int layout_scatter<int32_t>(const atos_csr*, const int32_t*, int32_t*, cudaStream_t);
template int layout_scatter<double>(const atos_csr*, const double*, double*, cudaStream_t);

int64_t layout_vertex(const atos_csr* g, int64_t v) {
  if (!g->relabeled) return v;
  uint32_t x = 0;
  if (cudaMemcpy(&x, g->o2n.as<uint32_t>() + v, 4, cudaMemcpyDeviceToHost) != cudaSuccess) return -1;
  return (int64_t)x;
}

}  // namespace atos
