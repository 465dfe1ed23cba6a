// Microbenchmark (tools only): throughput of the PageRank per-edge atomic on B200 --
// random-target 64-bit adds over the C3-sized residue array (4M doubles, L2-resident),
// f64 vs u64, with return (atom, needed for the crossing test) vs without (red).
#include <cstdint>
#include <cuda_runtime.h>

template <int KIND>
__global__ void k_atom(const uint32_t* __restrict__ col, uint64_t m, double* res, unsigned long long* out) {
  unsigned long long acc = 0;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x * 4;
  for (uint64_t base = (uint64_t)blockIdx.x * blockDim.x * 4 + threadIdx.x; base < m; base += stride) {
    uint32_t w[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const uint64_t e = base + (uint64_t)k * blockDim.x;
      w[k] = e < m ? __ldg(col + e) : 0u;
    }
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const uint64_t e = base + (uint64_t)k * blockDim.x;
      if (e >= m) continue;
      if (KIND == 0) acc += atomicAdd(res + w[k], 1e-7) > 1e-6;                                  // atom.add.f64
      if (KIND == 1) atomicAdd(res + w[k], 1e-7);                                                 // red.add.f64
      if (KIND == 2) acc += atomicAdd((unsigned long long*)res + w[k], 12345ull) > 1000000ull;   // atom.add.u64
      if (KIND == 3) atomicAdd((unsigned long long*)res + w[k], 12345ull);                        // red.add.u64
      if (KIND == 4) acc += atomicAdd((float*)res + w[k], 1e-7f) > 1e-6f;                         // atom.add.f32
    }
  }
  if (acc) atomicAdd(out, acc);
}

extern "C" float atom_bench(const uint32_t* col, uint64_t m, double* res, int kind, int grid, int block,
                            unsigned long long* out) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  switch (kind) {
    case 0: k_atom<0><<<grid, block>>>(col, m, res, out); break;
    case 1: k_atom<1><<<grid, block>>>(col, m, res, out); break;
    case 2: k_atom<2><<<grid, block>>>(col, m, res, out); break;
    case 3: k_atom<3><<<grid, block>>>(col, m, res, out); break;
    default: k_atom<4><<<grid, block>>>(col, m, res, out); break;
  }
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  return ms;
}
