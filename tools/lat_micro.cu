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
  // 9. the kernel's split fixed-point group sum (hi 2^-12 + lo 2^-36, two F2I, two REDUX)
  t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < IT / 8; ++i) {
    const int hi = __float2int_rn(x * 4096.f);
    const float rem = fmaf((float)hi, -1.f / 4096.f, x);
    const int lo = __float2int_rn(rem * 68719476736.f);
    const int shi = __reduce_add_sync(~0u, hi), slo = __reduce_add_sync(~0u, lo);
    const float s = fmaf((float)shi, 1.f / 4096.f, (float)slo * (1.f / 68719476736.f));
    x = x * 0.5f + s * 1e-3f;
  }
  t1 = clock64();
  if (l == 0) cyc[8] = t1 - t0;
  // 10. the same sum with magic-number rounding (FADD to 1.5*2^k) instead of F2I / I2F
  t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < IT / 8; ++i) {
    const float M1 = 12582912.f * (1.f / 4096.f);          // 1.5*2^23 * 2^-12: ulp 2^-12
    const float t = x + M1;                                 // RNE to a multiple of 2^-12
    const int hi = __float_as_int(t) - __float_as_int(M1);  // that multiple, in units of 2^-12
    const float rem = x - (t - M1);                         // exact
    const float M2 = 12582912.f;                            // ulp 1
    const float t2 = fmaf(rem, 68719476736.f, M2);          // rem*2^36 rounded to an integer
    const int lo = __float_as_int(t2) - __float_as_int(M2);
    const int shi = __reduce_add_sync(~0u, hi), slo = __reduce_add_sync(~0u, lo);
    const float s = fmaf((float)shi, 1.f / 4096.f, (float)slo * (1.f / 68719476736.f));
    x = x * 0.5f + s * 1e-3f;
  }
  t1 = clock64();
  if (l == 0) cyc[9] = t1 - t0;
  // 11. F2I.rn chain, 12. I2F chain
  t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) xi = __float2int_rn((float)xi * 0.5f);
  t1 = clock64();
  if (l == 0) cyc[10] = t1 - t0;
  x += xi;
  t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) xi = (int)__int2float_rn(xi + 1) ;
  t1 = clock64();
  if (l == 0) cyc[11] = t1 - t0;
  out[l] = x + xi;
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
  printf("split redux (kernel) %.1f cyc (+2 fp)\n", (double)cyc[8] / (IT / 8));
  printf("split redux magic    %.1f cyc (+2 fp)\n", (double)cyc[9] / (IT / 8));
  printf("f2i.rn+fmul chain    %.1f cyc\n", (double)cyc[10] / IT);
  printf("i2f+f2i(trunc)+iadd  %.1f cyc\n", (double)cyc[11] / IT);
  return 0;
}
