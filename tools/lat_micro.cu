// Dependent-chain latencies on one warp (cycles per link), to size the deterministic kernel's
// per-update critical path: SHFL.BFLY+FADD (one butterfly level), FADD, FFMA, LDS pointer chase,
// a whole 32-lane butterfly all-reduce and an smem all-reduce (STS, __syncwarp, 8x LDS.128,
// 31 FADD in a fixed tree: same result on every lane).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/bin/lat_micro tools/lat_micro.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int IT = 4096;

__global__ void k_chain(float* out, long long* cyc, float seed) {
  __shared__ __align__(16) float sm[32 * 4 + 64];
  __shared__ int chase[64];
  const int l = threadIdx.x;
  float x = seed + l;
  long long t0, t1;
  // 1. butterfly level: x = x + shfl_xor(x, 1)
  t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) x = x * 0.5f + __shfl_xor_sync(~0u, x, 1);
  t1 = clock64();
  if (l == 0) cyc[0] = t1 - t0;
  // 2. FFMA chain
  t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) x = fmaf(x, 0.999f, 0.001f);
  t1 = clock64();
  if (l == 0) cyc[1] = t1 - t0;
  // 3. LDS chase
  chase[l] = (l + 1) & 31;
  chase[l + 32] = 0;
  __syncwarp();
  int p = l;
  t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) p = chase[p];
  t1 = clock64();
  if (l == 0) cyc[2] = t1 - t0;
  x += p;
  // 4. full 5-level butterfly all-reduce, chained
  t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < IT / 8; ++i) {
    float s = x;
#pragma unroll
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(~0u, s, o);
    x = x * 0.5f + s * 1e-3f;
  }
  t1 = clock64();
  if (l == 0) cyc[3] = t1 - t0;
  // 5. smem all-reduce, chained
  t0 = clock64();
#pragma unroll 2
  for (int i = 0; i < IT / 8; ++i) {
    sm[l] = x;
    __syncwarp();
    float v[32];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const float4 t = reinterpret_cast<const float4*>(sm)[q];
      v[4 * q] = t.x; v[4 * q + 1] = t.y; v[4 * q + 2] = t.z; v[4 * q + 3] = t.w;
    }
#pragma unroll
    for (int w = 16; w; w >>= 1)
#pragma unroll
      for (int q = 0; q < w; ++q) v[q] += v[q + w];
    __syncwarp();
    x = x * 0.5f + v[0] * 1e-3f;
  }
  t1 = clock64();
  if (l == 0) cyc[4] = t1 - t0;
  // 6. 2x16-lane butterfly on packed halves: reduce 2 values at once, 4 levels + 1
  t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < IT / 8; ++i) {
    float s = x;
#pragma unroll
    for (int o = 8; o; o >>= 1) s += __shfl_xor_sync(~0u, s, o);
    x = x * 0.5f + s * 1e-3f;
  }
  t1 = clock64();
  if (l == 0) cyc[5] = t1 - t0;
  // 7. integer warp reduction (REDUX.SUM) chained
  int xi = (int)x;
  t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) xi = __reduce_add_sync(~0u, xi) >> 5;
  t1 = clock64();
  if (l == 0) cyc[6] = t1 - t0;
  x += xi;
  // 8. fixed-point all-reduce: F2I (scale 2^24) + REDUX.SUM + I2F, chained
  t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < IT / 8; ++i) {
    const int q = __float2int_rn(x * 16777216.f);
    const float s = (float)__reduce_add_sync(~0u, q) * (1.f / 16777216.f);
    x = x * 0.5f + s * 1e-3f;
  }
  t1 = clock64();
  if (l == 0) cyc[7] = t1 - t0;
  out[l] = x;
}

int main() {
  float* out;
  long long* cyc;
  cudaMalloc(&out, 32 * 4);
  cudaMallocManaged(&cyc, 16 * 8);
  for (int rep = 0; rep < 2; ++rep) {
    k_chain<<<1, 32>>>(out, cyc, 1.0f);
    cudaDeviceSynchronize();
  }
  printf("shfl+fma level   %.1f cyc\n", (double)cyc[0] / IT);
  printf("ffma             %.1f cyc\n", (double)cyc[1] / IT);
  printf("lds chase        %.1f cyc\n", (double)cyc[2] / IT);
  printf("bfly32 allreduce %.1f cyc (+2 fp)\n", (double)cyc[3] / (IT / 8));
  printf("smem allreduce   %.1f cyc (+2 fp)\n", (double)cyc[4] / (IT / 8));
  printf("bfly16 allreduce %.1f cyc (+2 fp)\n", (double)cyc[5] / (IT / 8));
  printf("redux.add.s32    %.1f cyc (+1 shift)\n", (double)cyc[6] / IT);
  printf("fixed-pt redux   %.1f cyc (+2 fp)\n", (double)cyc[7] / (IT / 8));
  return 0;
}
