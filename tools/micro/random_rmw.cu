// Ceiling probe for the Hugewiki-shaped Hogwild kernel's P traffic (profiles/r02_hugewiki_mlp.md):
// random read-modify-write of 256-B rows (k = 128 fp16) spread over a 12.8-GB array, with D rows in
// flight per 16-lane group, against a streaming copy.  Reports DRAM-level GB/s (bytes read + written).
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/rrmw tools/micro/random_rmw.cu && /tmp/rrmw
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t z) {
  z = (z ^ (z >> 33)) * 0xff51afd7ed558ccdULL;
  z = (z ^ (z >> 33)) * 0xc4ceb9fe1a85ec53ULL;
  return z ^ (z >> 33);
}

// each group of 16 lanes owns a stream of random rows; lane l moves bytes [16 l, 16 l + 16) of a row
template <int D>
__global__ void __launch_bounds__(256) k_rmw(uint4* P, uint64_t rows, uint64_t iters, int write) {
  const int lane = threadIdx.x & 15;
  const uint64_t grp = (blockIdx.x * 256ull + threadIdx.x) >> 4;
  uint4 v[D];
  uint64_t r[D];
  for (uint64_t it = 0; it < iters; it += D) {
#pragma unroll
    for (int d = 0; d < D; ++d) {
      r[d] = mix(grp * 0x9E3779B97F4A7C15ULL + it + d) % rows;
      v[d] = P[r[d] * 16 + lane];
    }
#pragma unroll
    for (int d = 0; d < D; ++d) {
      v[d].x += 1;
      if (write) P[r[d] * 16 + lane] = v[d];
    }
  }
}

__global__ void k_copy(const uint4* a, uint4* b, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    b[i] = a[i];
}

int main() {
  const uint64_t rows = 50082604ull, bytes = rows * 256;
  uint4* P;
  if (cudaMalloc(&P, bytes) != cudaSuccess) { printf("alloc failed\n"); return 1; }
  cudaMemset(P, 0, bytes);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  float ms;
  // streaming copy of 4 GB -> 4 GB
  {
    uint64_t n = (4ull << 30) / 16;
    for (int w = 0; w < 2; ++w) k_copy<<<148 * 8, 512>>>(P, P + n, n);
    cudaEventRecord(e0);
    for (int w = 0; w < 5; ++w) k_copy<<<148 * 8, 512>>>(P, P + n, n);
    cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
    printf("stream copy: %.0f GB/s\n", 5 * 2.0 * n * 16 / (ms * 1e6));
  }
  const int grids[] = {740, 888, 1184};
  for (int write = 0; write < 2; ++write)
    for (int gi = 0; gi < 3; ++gi) {
      int grid = grids[gi];
      uint64_t groups = grid * 16ull, iters = 2048;
      auto go = [&](int D) {
        auto launch = [&]() {
          if (D == 1) k_rmw<1><<<grid, 256>>>(P, rows, iters, write);
          if (D == 2) k_rmw<2><<<grid, 256>>>(P, rows, iters, write);
          if (D == 4) k_rmw<4><<<grid, 256>>>(P, rows, iters, write);
        };
        launch();
        cudaEventRecord(e0);
        launch(); launch();
        cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        double b = 2.0 * groups * iters * 256.0 * (write ? 2 : 1);
        printf("%s grid %d D %d: %.0f GB/s  (%.2f G rows/s)\n", write ? "rmw " : "read", grid, D, b / (ms * 1e6),
               2.0 * groups * iters / (ms * 1e6));
      };
      go(1); go(2); go(4);
    }
  cudaError_t err = cudaGetLastError();
  printf("status %s\n", cudaGetErrorString(err));
  return 0;
}
