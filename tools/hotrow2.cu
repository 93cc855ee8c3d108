// hotrow2.cu -- what limits the read-modify-write rate of hot feature rows (B200)?
//
// die_probe.cu showed the per-row rate does not depend on dies (one die of SMs gets the same
// per-row rate as both; die-affine rows do not help).  This probe varies the access instead,
// H hot 256-B rows (fp16 k=128 q_v), 9,472 groups, each group RMWs row (gid + it) mod H:
//   V0 ld.cg.v4 + st.cg.v4, 16 lanes x 16 B     (the Hogwild kernel)
//   V1 ld.v8 + st.v8, 8 lanes x 32 B            (256-bit accesses, half the requests)
//   V2 ld.cg + st.cs (evict-first store)
//   V3 ld.cg + st.wt (write-through)
//   V4 ld.cg row (gid+it), st.cg row (gid+it+H/2): loads and stores to the same set of lines,
//      never the same line within one group's iteration (is it the same-thread RAW order?)
//   V5 ld.relaxed.gpu + st.relaxed.gpu (explicit memory-model ops)
//   V6 ld.cg + st.cg of a 512-B fp32 row (32 lanes x 16 B)
//   V7 half the groups only load, half only store (no per-group dependency)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o hotrow2 tools/hotrow2.cu
#include <cuda_runtime.h>

#include <cstdio>

template <int V>
__global__ void hot(uint4* __restrict__ rows, int H, int iters, unsigned* sink) {
  constexpr int GL = (V == 1) ? 8 : (V == 6 ? 32 : 16);      // lanes per group
  constexpr int ROW16 = (V == 6) ? 32 : 16;                   // row size in 16-B units
  const int lane = threadIdx.x & 31, gl = lane % GL;
  const int gid = (int)((blockIdx.x * blockDim.x + threadIdx.x) / GL);
  unsigned acc = 0;
  for (int it = 0; it < iters; ++it) {
    const int row = (gid + it) % H;
    if constexpr (V == 1) {
      uint4* p = rows + (size_t)row * ROW16 + gl * 2;
      unsigned a0, a1, a2, a3, a4, a5, a6, a7;
      asm volatile("ld.global.cg.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                   : "=r"(a0), "=r"(a1), "=r"(a2), "=r"(a3), "=r"(a4), "=r"(a5), "=r"(a6), "=r"(a7)
                   : "l"(p)
                   : "memory");
      acc += a0;
      a0 += 1;
      asm volatile("st.global.cg.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(a0), "r"(a1),
                   "r"(a2), "r"(a3), "r"(a4), "r"(a5), "r"(a6), "r"(a7)
                   : "memory");
    } else if constexpr (V == 4) {
      uint4 x = __ldcg(rows + (size_t)row * ROW16 + gl);
      acc += x.x;
      x.x += 1;
      __stcg(rows + (size_t)((row + H / 2) % H) * ROW16 + gl, x);
    } else if constexpr (V == 5) {
      uint4* p = rows + (size_t)row * ROW16 + gl;
      unsigned a, b, c, d;
      asm volatile("ld.relaxed.gpu.global.v4.b32 {%0,%1,%2,%3}, [%4];"
                   : "=r"(a), "=r"(b), "=r"(c), "=r"(d)
                   : "l"(p)
                   : "memory");
      acc += a;
      a += 1;
      asm volatile("st.relaxed.gpu.global.v4.b32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(a), "r"(b), "r"(c),
                   "r"(d)
                   : "memory");
    } else if constexpr (V == 7) {
      uint4* p = rows + (size_t)row * ROW16 + gl;
      if (gid & 1) {
        uint4 x = __ldcg(p);
        acc += x.x;
      } else {
        __stcg(p, make_uint4(it, gid, 0, 0));
      }
    } else {
      uint4* p = rows + (size_t)row * ROW16 + gl;
      uint4 x = __ldcg(p);
      acc += x.x;
      x.x += 1;
      if constexpr (V == 2) __stcs(p, x);
      else if constexpr (V == 3) __stwt(p, x);
      else __stcg(p, x);
    }
  }
  if (acc == 0x7fffffffu) *sink = acc;
}

template <int V>
float run(uint4* rows, int H, int groups, int iters, unsigned* sink) {
  constexpr int GL = (V == 1) ? 8 : (V == 6 ? 32 : 16);
  const int threads = 256, blocks = groups * GL / threads;
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
  const char* names[] = {"ld.cg+st.cg 16x16B", "ld+st v8 8x32B",   "ld.cg+st.cs",       "ld.cg+st.wt",
                         "ld row, st row+H/2", "ld/st.relaxed.gpu", "fp32 row 32x16B",   "half ld / half st"};
  for (int H : {1, 16, 256, 4096}) {
    const int groups = 9472, iters = H >= 256 ? 2000 : 500;
    float ms[8] = {run<0>(rows, H, groups, iters, sink), run<1>(rows, H, groups, iters, sink),
                   run<2>(rows, H, groups, iters, sink), run<3>(rows, H, groups, iters, sink),
                   run<4>(rows, H, groups, iters, sink), run<5>(rows, H, groups, iters, sink),
                   run<6>(rows, H, groups, iters, sink), run<7>(rows, H, groups, iters, sink)};
    for (int v = 0; v < 8; ++v) {
      const double upd = (double)groups * iters;
      printf("H=%5d %-22s %8.3f ms  total %7.3f G/s  per-row %8.2f M/s\n", H, names[v], ms[v],
             upd / ms[v] / 1e6, upd / ms[v] / 1e3 / H);
    }
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
