// layout.cu -- S0 residency: the degree layout of a single-partition graph
// ("Degree layout").
//
// The generators (and real inputs) hand us vertex ids in random order, so the
// per-vertex state of the hubs -- which receive most relaxations -- is spread
// over the whole state array.  When that array is larger than L2 (C5: the
// PageRank residue is 537 MB, L2 126 MB) most of the per-edge f64 atomics miss
// L2.  At creation the CSR is relabelled once:
//   rank r = position of v in descending-degree order (stable, by old id);
//   new id = r, except that the first 16*T ranks are interleaved as
//            (r mod T) * 16 + r / T  (T = min(65536, n / 16)),
// which packs the hot set into a prefix of the state arrays (L2-resident) but
// gives each of the T hottest vertices its own 128-byte line of an f64 array,
// so the hubs' atomics do not serialise on shared lines/slices (without the
// interleave C3 PageRank, whose state already fits L2, ran 2x slower).
// Measured (tools/relabel_probe.py): C5 PageRank 2652 -> 1243 ms, C5 BFS
// 14.7 -> 13.2 ms, C3 within 3 %.
//
// The method is unchanged: every call maps the source into the internal ids
// and scatters its output back (out[old] = result[new]); colouring seeds its
// queue in the caller's vertex-id order.  Loopback / NCCL partitions keep the
// input ids (a degree-sorted block partition would put every hub on part 0).
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <algorithm>

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

// one warp per new row: copy the old row with every neighbour id mapped
__global__ void k_layout_rows(const uint32_t* __restrict__ rp_old, const uint32_t* __restrict__ col_old,
                              const uint32_t* __restrict__ rp_new, const uint32_t* __restrict__ n2o,
                              const uint32_t* __restrict__ o2n, int64_t n, uint32_t* col_new) {
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t i = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); i < n; i += warps) {
    const uint32_t old = n2o[i];
    const uint32_t b = rp_old[old], d = rp_old[old + 1] - b, nb = rp_new[i];
    for (uint32_t j = threadIdx.x & 31u; j < d; j += 32) col_new[nb + j] = o2n[col_old[b + j]];
  }
}

__global__ void k_layout_set_last(uint32_t* rp_new, int64_t n, uint32_t m) {
  if (threadIdx.x == 0 && blockIdx.x == 0) rp_new[n] = m;
}

int layout_by_degree(atos_csr* g) {
  Part& p = g->parts[0];
  const int64_t n = p.n_local, m = p.m_local;
  if (n < 2) return ATOS_OK;
  cudaStream_t s = 0;
  const uint32_t T = (uint32_t)std::min<int64_t>(65536, n / 16);
  struct Scratch {  // released on every return path
    DevBuf deg, ids, deg_s, order, ndeg, rp_new, col_new, tmp;
    ~Scratch() {
      for (DevBuf* b : {&deg, &ids, &deg_s, &order, &ndeg, &rp_new, &col_new, &tmp}) b->release();
    }
  } w;
  DevBuf &deg = w.deg, &ids = w.ids, &deg_s = w.deg_s, &order = w.order, &ndeg = w.ndeg, &rp_new = w.rp_new,
         &col_new = w.col_new, &tmp = w.tmp;
  ATOS_TRY(deg.ensure(n * 4));
  ATOS_TRY(ids.ensure(n * 4));
  ATOS_TRY(deg_s.ensure(n * 4));
  ATOS_TRY(order.ensure(n * 4));
  ATOS_TRY(ndeg.ensure(n * 4));
  ATOS_TRY(rp_new.ensure((n + 1) * 4));
  ATOS_TRY(g->o2n.ensure(n * 4));
  ATOS_TRY(g->n2o.ensure(n * 4));
  const int gs = 148 * 8;
  k_layout_degrees<<<gs, 256, 0, s>>>(p.row_ptr, n, deg.as<uint32_t>(), ids.as<uint32_t>());
  size_t tb = 0;
  ATOS_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, deg.as<uint32_t>(), deg_s.as<uint32_t>(),
                                                      ids.as<uint32_t>(), order.as<uint32_t>(), (int)n, 0, 32, s));
  ATOS_TRY(tmp.ensure(tb));
  ATOS_CUDA(cub::DeviceRadixSort::SortPairsDescending(tmp.p, tb, deg.as<uint32_t>(), deg_s.as<uint32_t>(),
                                                      ids.as<uint32_t>(), order.as<uint32_t>(), (int)n, 0, 32, s));
  k_layout_place<<<gs, 256, 0, s>>>(deg_s.as<uint32_t>(), order.as<uint32_t>(), n, T, g->n2o.as<uint32_t>(),
                                    g->o2n.as<uint32_t>(), ndeg.as<uint32_t>());
  size_t tb2 = 0;
  ATOS_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb2, ndeg.as<uint32_t>(), rp_new.as<uint32_t>(), (int)n, s));
  ATOS_TRY(tmp.ensure(tb2));
  ATOS_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, tb2, ndeg.as<uint32_t>(), rp_new.as<uint32_t>(), (int)n, s));
  k_layout_set_last<<<1, 32, 0, s>>>(rp_new.as<uint32_t>(), n, (uint32_t)m);
  deg.release();
  ids.release();
  deg_s.release();
  order.release();
  ndeg.release();
  tmp.release();
  if (m > 0) {
    ATOS_TRY(col_new.ensure(m * 4));
    k_layout_rows<<<148 * 16, 256, 0, s>>>(p.row_ptr, p.col, rp_new.as<uint32_t>(), g->n2o.as<uint32_t>(),
                                          g->o2n.as<uint32_t>(), n, col_new.as<uint32_t>());
  }
  g_launches += 4;
  ATOS_CUDA(cudaGetLastError());
  ATOS_CUDA(cudaStreamSynchronize(s));
  // swap in the relabelled arrays (the Part owns row_ptr / col as raw allocations)
  cudaFree(p.row_ptr);
  p.row_ptr = rp_new.as<uint32_t>();
  rp_new.p = nullptr;
  if (m > 0) {
    cudaFree(p.col);
    p.col = col_new.as<uint32_t>();
    col_new.p = nullptr;
  }
  g->relabeled = true;
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
