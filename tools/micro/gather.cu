// Microbenchmark (tools only): the BFS per-edge access pattern without the queue --
// stream col[] and gather shadow[col[e]] (u8), counting hits <= thr.  Measures the
// B200 ceiling of the pattern the BFS worker is made of.
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long pol_first() {
  unsigned long long p;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ unsigned long long pol_last() {
  unsigned long long p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}

template <int U>
__global__ void k_gather(const uint32_t* __restrict__ col, const uint8_t* __restrict__ sh, uint64_t m, uint32_t thr,
                         unsigned long long* out) {
  const unsigned long long pf = pol_first(), pl = pol_last();
  unsigned long long cnt = 0;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x * U;
  for (uint64_t base = (uint64_t)blockIdx.x * blockDim.x * U + threadIdx.x; base < m; base += stride) {
    uint32_t w[U];
#pragma unroll
    for (int k = 0; k < U; ++k) {
      const uint64_t e = base + (uint64_t)k * blockDim.x;
      if (e < m) asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(w[k]) : "l"(col + e), "l"(pf));
    }
#pragma unroll
    for (int k = 0; k < U; ++k) {
      const uint64_t e = base + (uint64_t)k * blockDim.x;
      if (e < m) {
        uint16_t v;
        asm volatile("ld.global.L2::cache_hint.u8 %0, [%1], %2;" : "=h"(v) : "l"(sh + w[k]), "l"(pl));
        cnt += (v <= thr);
      }
    }
  }
  for (int o = 16; o; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
  if ((threadIdx.x & 31) == 0) atomicAdd(out, cnt);
}

extern "C" float gather_bench(const uint32_t* col, const uint8_t* sh, uint64_t m, int U, int grid, int block,
                              unsigned long long* out) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  if (U == 1) k_gather<1><<<grid, block>>>(col, sh, m, 3, out);
  else if (U == 2) k_gather<2><<<grid, block>>>(col, sh, m, 3, out);
  else if (U == 4) k_gather<4><<<grid, block>>>(col, sh, m, 3, out);
  else k_gather<8><<<grid, block>>>(col, sh, m, 3, out);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  return ms;
}
