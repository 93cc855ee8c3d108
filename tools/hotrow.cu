// hotrow.cu -- update rate of ONE hot feature row under Hogwild concurrency (B200).
//
// tools/ncols_probe.py shows that with power-law columns the Hogwild kernel's throughput is set
// by the hottest column: ~13-18 M updates/s land on the top q_v row whatever the worker count.
// This microbenchmark isolates that: G groups of 16 lanes (one 256-B fp16 row = 16 x 16 B, k=128)
// repeatedly read-modify-write one of H hot rows (row = (group + iteration) mod H), with
//   V0  ld.global.cg  + st.global.cg   (the SGD kernel's path)
//   V1  ld.global.cg  + st.global (wb)
//   V2  ld.global.cg  + red.global.add.noftz.v4.f16x2  (write the DELTA as an L2 reduction)
//   V3  store only (st.cg, no load)
//   V4  load only (ld.cg)
//   V5  red only
// Prints updates/s per hot row and in total.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o hotrow tools/hotrow.cu
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <cstdio>

template <int V>
__global__ void hot(uint4* __restrict__ rows, int H, int iters, unsigned* sink) {
  const int lane = threadIdx.x & 31, gl = lane & 15;
  const int gid = (int)((blockIdx.x * blockDim.x + threadIdx.x) >> 4);
  unsigned acc = 0;
  for (int it = 0; it < iters; ++it) {
    uint4* p = rows + (size_t)((gid + it) % H) * 16 + gl;
    if constexpr (V == 0 || V == 1 || V == 2 || V == 4) {
      uint4 x = __ldcg(p);
      acc += x.x;
      if constexpr (V == 0) { x.x += 1; __stcg(p, x); }
      if constexpr (V == 1) { x.x += 1; *p = x; }
      if constexpr (V == 2) {
        const unsigned d = 0x00010001u ^ (x.y & 0x80008000u);   // tiny delta, depends on the load
        asm volatile("red.global.add.noftz.v4.f16x2 [%0], {%1,%1,%1,%1};" ::"l"(p), "r"(d) : "memory");
      }
    } else if constexpr (V == 3) {
      __stcg(p, make_uint4(it, gid, 0, 0));
    } else {
      asm volatile("red.global.add.noftz.v4.f16x2 [%0], {%1,%1,%1,%1};" ::"l"(p), "r"(0x00010001u) : "memory");
    }
  }
  if (acc == 0x7fffffffu) *sink = acc;
}

template <int V>
float run(uint4* rows, int H, int groups, int iters, unsigned* sink) {
  const int threads = 256, blocks = groups * 16 / threads;
  hot<V><<<blocks, threads>>>(rows, H, iters, sink);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  hot<V><<<blocks, threads>>>(rows, H, iters, sink);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  return ms;
}

int main() {
  uint4* rows;
  unsigned* sink;
  cudaMalloc(&rows, 1 << 26);
  cudaMemset(rows, 0, 1 << 26);
  cudaMalloc(&sink, 4);
  const char* names[] = {"ld.cg+st.cg", "ld.cg+st.wb", "ld.cg+red.v4.f16x2", "st.cg only",
                         "ld.cg only", "red only"};
  for (int H : {1, 4, 16, 256}) {
    for (int groups : {148, 1184, 4736, 9472}) {
      const int iters = 2000;
      float ms[6] = {run<0>(rows, H, groups, iters, sink), run<1>(rows, H, groups, iters, sink),
                     run<2>(rows, H, groups, iters, sink), run<3>(rows, H, groups, iters, sink),
                     run<4>(rows, H, groups, iters, sink), run<5>(rows, H, groups, iters, sink)};
      for (int v = 0; v < 6; ++v) {
        const double upd = (double)groups * iters;
        printf("H=%4d groups=%5d %-20s %8.3f ms  total %7.3f G/s  per-row %8.2f M/s\n", H, groups,
               names[v], ms[v], upd / ms[v] / 1e6, upd / ms[v] / 1e3 / H);
      }
    }
  }
  cudaError_t e = cudaGetLastError();
  printf("%s\n", cudaGetErrorString(e));
  return 0;
}
