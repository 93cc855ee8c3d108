// rmw_ceiling.cu -- what does the B200 memory system deliver for the hot path's access
// pattern WITHOUT the SGD dependency chain?  Each "update" reads row P[u] and row Q[v]
// (k*S bytes each), writes both back (+1 so the write depends on the read), and streams a 12-B
// rating.  u uniform over m, v power-law over n (Netflix shape).  Independent samples, U per
// group in flight.  Prints algorithmic GB/s (12 + 4kS per update) per variant.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o rmw_ceiling tools/rmw_ceiling.cu
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <random>
#include <vector>

struct Rating { int u, v; float r; };

template <int L, int U, bool WRITE, bool WP = true, bool WQ = true, int ST = 0>
__global__ void rmw(const Rating* __restrict__ s, long long N, uint4* __restrict__ P,
                    uint4* __restrict__ Q, int row16) {  // row16 = row bytes / 16 = L
  const int lane = threadIdx.x & 31, gl = lane % L;
  const long long groups = (long long)gridDim.x * blockDim.x / L;
  const long long gid = ((long long)blockIdx.x * blockDim.x + threadIdx.x) / L;
  for (long long base = gid * U; base < N; base += groups * U) {
    uint4 a[U], b[U];
    int uu[U], vv[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {
      long long i = base + j;
      if (i < N) {
        uu[j] = __ldcs(&s[i].u);
        vv[j] = __ldcs(&s[i].v);
      } else {
        uu[j] = -1;
      }
    }
#pragma unroll
    for (int j = 0; j < U; ++j)
      if (uu[j] >= 0) {
        a[j] = __ldcg(P + (long long)uu[j] * row16 + gl);
        b[j] = __ldcg(Q + (long long)vv[j] * row16 + gl);
      }
    if (WRITE) {
#pragma unroll
      for (int j = 0; j < U; ++j)
        if (uu[j] >= 0) {
          a[j].x += 1; b[j].x += 1;
          if (ST == 0) {
            if (WP) __stcg(P + (long long)uu[j] * row16 + gl, a[j]);
            if (WQ) __stcg(Q + (long long)vv[j] * row16 + gl, b[j]);
          } else {
            if (WP) P[(long long)uu[j] * row16 + gl] = a[j];
            if (WQ) Q[(long long)vv[j] * row16 + gl] = b[j];
          }
          if (!WP) { if (a[j].y == 0x12345u) P[0] = a[j]; }
          if (!WQ) { if (b[j].y == 0x12345u) Q[0] = b[j]; }
        }
    } else {
      unsigned acc = 0;
#pragma unroll
      for (int j = 0; j < U; ++j) if (uu[j] >= 0) acc ^= a[j].x ^ b[j].y;
      if (acc == 0x12345678u) P[0].x = acc;
    }
  }
}

template <int L, int U, bool W, bool WP = true, bool WQ = true, int ST = 0>
float run(const Rating* s, long long N, uint4* P, uint4* Q, int blocks_per_sm, int sms) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  int grid = blocks_per_sm * sms;
  rmw<L, U, W, WP, WQ, ST><<<grid, 256>>>(s, N, P, Q, L);
  cudaEventRecord(e0);
  for (int it = 0; it < 3; ++it) rmw<L, U, W, WP, WQ, ST><<<grid, 256>>>(s, N, P, Q, L);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  return ms / 3;
}

int main(int argc, char** argv) {
  const long long m = 480190, n = 17771, N = 99072112;
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  std::vector<Rating> h(N);
  std::mt19937_64 rng(1);
  std::vector<double> cdf(n);
  double acc = 0;
  for (long long x = 0; x < n; ++x) { acc += std::pow(x + 1.0, -0.45); cdf[x] = acc; }
  std::vector<int> perm(n);
  for (int i = 0; i < n; ++i) perm[i] = i;
  std::shuffle(perm.begin(), perm.end(), rng);
  std::uniform_real_distribution<double> U01(0, 1);
  for (long long i = 0; i < N; ++i) {
    h[i].u = (int)(rng() % m);
    long long r = std::lower_bound(cdf.begin(), cdf.end(), U01(rng) * acc) - cdf.begin();
    h[i].v = perm[std::min(r, n - 1)];
    h[i].r = 1.f;
  }
  Rating* s;
  cudaMalloc(&s, N * sizeof(Rating));
  cudaMemcpy(s, h.data(), N * sizeof(Rating), cudaMemcpyHostToDevice);
  // uniform-v copy of the stream (no hot columns)
  std::vector<Rating> hu(h);
  for (long long i = 0; i < N; ++i) hu[i].v = (int)(rng() % n);
  Rating* su;
  cudaMalloc(&su, N * sizeof(Rating));
  cudaMemcpy(su, hu.data(), N * sizeof(Rating), cudaMemcpyHostToDevice);
  const int rowbytes = 256;
  uint4 *P, *Q;
  cudaMalloc(&P, m * rowbytes);
  cudaMalloc(&Q, n * rowbytes);
  cudaMemset(P, 0, m * rowbytes);
  cudaMemset(Q, 0, n * rowbytes);
  const double alg = (double)N * (12 + 4 * 256);
  const int bps = 4;
  float t;
#define R(label, expr) t = expr; printf("%-40s %.3f ms  %.2f Gupd/s  %.0f GB/s(alg fp16)\n", label, t, N / t / 1e6, alg / t / 1e6);
  R("rmw P+Q  .cg store  powerlaw v", (run<16, 4, true, true, true, 0>(s, N, P, Q, bps, sms)));
  R("rmw P+Q  wb  store  powerlaw v", (run<16, 4, true, true, true, 1>(s, N, P, Q, bps, sms)));
  R("rmw P+Q  .cg store  uniform v", (run<16, 4, true, true, true, 0>(su, N, P, Q, bps, sms)));
  R("rmw P only .cg      powerlaw v", (run<16, 4, true, true, false, 0>(s, N, P, Q, bps, sms)));
  R("rmw Q only .cg      powerlaw v", (run<16, 4, true, false, true, 0>(s, N, P, Q, bps, sms)));
  R("rmw Q only .cg      uniform v", (run<16, 4, true, false, true, 0>(su, N, P, Q, bps, sms)));
  R("read P+Q            powerlaw v", (run<16, 4, false>(s, N, P, Q, bps, sms)));
  R("rmw P+Q  .cg U=8    powerlaw v", (run<16, 8, true, true, true, 0>(s, N, P, Q, bps, sms)));
  R("rmw P+Q  .cg L=8(32B)  powerlaw", (run<16, 4, true, true, true, 0>(s, N, P, Q, 8, sms)));
  cudaFree(P);
  cudaFree(Q);
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
