// die_probe.cu -- does the hot-row limit of Hogwild come from the two-die L2 (B200)?
//
// profiles/r01_scaling_hot_rows.md section 4: interleaved ld.cg + st.cg of the same 256-B rows
// from every SM serialise at ~10-30 M updates/s per row, while loads alone and stores alone run
// at L2 speed.  B200 is two dies with the L2 split between them (each 2-KB granule of the
// address space is homed on one die).  This probe
//   1. finds each SM's die: one CTA per SM times dependent ld.cg loads of 64 granules; SMs on
//      the same die see the same near/far pattern (234 vs 262 cycles on B300),
//   2. finds each test row's home die (the die whose SMs see it near),
//   3. times the hot-row RMW (ld.cg + st.cg of a 256-B fp16 k=128 row per group of 16 lanes)
//      with H hot rows under:
//        all      every SM, rows of both homes               (what the SGD kernel sees)
//        one-die  only die-0 SMs work (same groups per SM)
//        near     only die-0 SMs, rows homed on die 0
//        far      only die-0 SMs, rows homed on die 1
//        split    every SM, but die d's SMs touch only rows homed on die d (die-affine columns)
//        split-x  every SM, die d's SMs touch only rows homed on the OTHER die
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o die_probe tools/die_probe.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

constexpr int NPROBE = 64;      // probed granules
constexpr int GRAN = 2048;      // address->die granule

__device__ __forceinline__ unsigned smid() {
  unsigned s;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  return s;
}

// Latency of one ld.cg from this SM to *p: a chain of 32 dependent loads (the loaded value,
// always 0, is added to the next address), closed by a shared-memory store of the result
// before the clock read so the clock waits for the last load.
__device__ __forceinline__ long long chain_lat(const unsigned* p, volatile unsigned* sink_smem) {
  unsigned x = 0;
  long long best = 1LL << 40;
  for (int rep = 0; rep < 4; ++rep) {
    const long long t0 = clock64();
#pragma unroll
    for (int i = 0; i < 32; ++i)
      asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(x) : "l"(p + x) : "memory");
    *sink_smem = x;
    const long long t1 = clock64();
    if (rep > 0 && t1 - t0 < best) best = t1 - t0;
  }
  return best / 32;
}

// One CTA per SM (forced by dynamic smem); thread 0 times dependent loads.
__global__ void k_latency(const unsigned* __restrict__ base, int* out_smid, float* lat) {
  extern __shared__ char smem[];
  if (threadIdx.x != 0) return;
  smem[0] = 0;
  const unsigned s = smid();
  out_smid[blockIdx.x] = (int)s;
  for (int g = 0; g < NPROBE; ++g) {
    const unsigned* p = base + (size_t)g * (GRAN / 4) * 3;   // granules 3 apart
    lat[blockIdx.x * NPROBE + g] = (float)chain_lat(p, (volatile unsigned*)smem);
  }
}

// Per-row latency from one SM: probes rows, returns best latency per row.
__global__ void k_row_latency(const uint4* __restrict__ rows, const int* __restrict__ row_ids, int nrows,
                              int want_sm, float* lat, int* hit) {
  extern __shared__ char smem[];
  if (threadIdx.x != 0) return;
  smem[0] = 0;
  if ((int)smid() != want_sm) return;
  *hit = 1;
  for (int r = 0; r < nrows; ++r)
    lat[r] = (float)chain_lat((const unsigned*)(rows + (size_t)row_ids[r] * 16), (volatile unsigned*)smem);
}

// mode: 0 all, 1 only die-0 SMs (rows set A), 2 split (die d uses set d), 3 split-x
__global__ void k_hot(uint4* __restrict__ rows, const int* __restrict__ setA, int nA,
                      const int* __restrict__ setB, int nB, const signed char* __restrict__ die_of,
                      int mode, int iters, unsigned* sink) {
  const int lane = threadIdx.x & 31, gl = lane & 15;
  const int gid = (int)((blockIdx.x * blockDim.x + threadIdx.x) >> 4);
  const int d = die_of[smid()];
  const int* set = setA;
  int n = nA;
  if (mode == 1 && d != 0) return;
  if (mode == 2 && d == 1) { set = setB; n = nB; }
  if (mode == 3 && d == 0) { set = setB; n = nB; }
  unsigned acc = 0;
  for (int it = 0; it < iters; ++it) {
    uint4* p = rows + (size_t)set[(gid + it) % n] * 16 + gl;
    uint4 x = __ldcg(p);
    acc += x.x;
    x.x += 1;
    __stcg(p, x);
  }
  if (acc == 0x7fffffffu) *sink = acc;
}

static float time_hot(uint4* rows, const int* A, int nA, const int* B, int nB, const signed char* die,
                      int mode, int groups, int iters, unsigned* sink, long long* done_groups,
                      const std::vector<int>& die_h, const std::vector<int>& sm_of_block) {
  const int threads = 256, blocks = groups * 16 / threads;
  k_hot<<<blocks, threads>>>(rows, A, nA, B, nB, die, mode, iters, sink);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  k_hot<<<blocks, threads>>>(rows, A, nA, B, nB, die, mode, iters, sink);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  (void)die_h; (void)sm_of_block;
  *done_groups = groups;
  return ms;
}

int main() {
  int dev = 0, nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  unsigned* probe;
  cudaMalloc(&probe, (size_t)NPROBE * GRAN * 4);
  cudaMemset(probe, 0, (size_t)NPROBE * GRAN * 4);
  int* d_smid;
  float* d_lat;
  cudaMalloc(&d_smid, nsm * 4);
  cudaMalloc(&d_lat, (size_t)nsm * NPROBE * 4);
  const int big = 160 * 1024;
  cudaFuncSetAttribute(k_latency, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k_row_latency, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  k_latency<<<nsm, 32, big>>>(probe, d_smid, d_lat);
  k_latency<<<nsm, 32, big>>>(probe, d_smid, d_lat);
  std::vector<int> smid(nsm);
  std::vector<float> lat((size_t)nsm * NPROBE);
  cudaMemcpy(smid.data(), d_smid, nsm * 4, cudaMemcpyDeviceToHost);
  cudaMemcpy(lat.data(), d_lat, lat.size() * 4, cudaMemcpyDeviceToHost);
  // Cluster: each granule's latency relative to that granule's median across SMs -> sign pattern.
  std::vector<int> die(256, -1);
  std::vector<float> med(NPROBE);
  for (int g = 0; g < NPROBE; ++g) {
    std::vector<float> col(nsm);
    for (int b = 0; b < nsm; ++b) col[b] = lat[(size_t)b * NPROBE + g];
    std::nth_element(col.begin(), col.begin() + nsm / 2, col.end());
    med[g] = col[nsm / 2];
  }
  // reference = block 0's sign pattern
  std::vector<int> ref(NPROBE);
  for (int g = 0; g < NPROBE; ++g) ref[g] = lat[g] < med[g] ? 1 : -1;
  int n0 = 0, n1 = 0, ambiguous = 0;
  for (int b = 0; b < nsm; ++b) {
    int agree = 0;
    for (int g = 0; g < NPROBE; ++g) agree += ((lat[(size_t)b * NPROBE + g] < med[g] ? 1 : -1) == ref[g]) ? 1 : -1;
    if (std::abs(agree) < NPROBE / 2) ++ambiguous;
    die[smid[b]] = agree > 0 ? 0 : 1;
    (agree > 0 ? n0 : n1)++;
  }
  printf("SMs %d: die0 %d die1 %d ambiguous %d\n", nsm, n0, n1, ambiguous);
  printf("latency granule 0..7 from block0 / a die-1 block:");
  int b1 = -1;
  for (int b = 0; b < nsm; ++b) if (die[smid[b]] == 1) { b1 = b; break; }
  for (int g = 0; g < 8; ++g) printf(" %.0f/%.0f", lat[g], b1 >= 0 ? lat[(size_t)b1 * NPROBE + g] : -1.f);
  printf("\nsmid die map:");
  for (int s = 0; s < nsm; ++s) printf("%d", die[s]);
  printf("\n");
  if (b1 < 0) return 0;
  const int sm0 = smid[0], sm1 = smid[b1];

  // Test rows: 4096 rows of 256 B; classify each by near/far from sm0 vs sm1.
  const int R = 4096;
  uint4* rows;
  cudaMalloc(&rows, (size_t)R * 256);
  cudaMemset(rows, 0, (size_t)R * 256);
  std::vector<int> ids(R);
  for (int r = 0; r < R; ++r) ids[r] = r;
  int* d_ids;
  float* d_rl;
  int* d_hit;
  cudaMalloc(&d_ids, R * 4);
  cudaMalloc(&d_rl, R * 4);
  cudaMalloc(&d_hit, 4);
  cudaMemcpy(d_ids, ids.data(), R * 4, cudaMemcpyHostToDevice);
  std::vector<float> l0(R), l1(R);
  k_row_latency<<<nsm, 32, big>>>(rows, d_ids, R, sm0, d_rl, d_hit);
  k_row_latency<<<nsm, 32, big>>>(rows, d_ids, R, sm0, d_rl, d_hit);
  cudaMemcpy(l0.data(), d_rl, R * 4, cudaMemcpyDeviceToHost);
  k_row_latency<<<nsm, 32, big>>>(rows, d_ids, R, sm1, d_rl, d_hit);
  cudaMemcpy(l1.data(), d_rl, R * 4, cudaMemcpyDeviceToHost);
  std::vector<int> home0, home1;
  for (int r = 0; r < R; ++r) (l0[r] < l1[r] ? home0 : home1).push_back(r);
  printf("rows homed near die0 %zu, die1 %zu (row0 lat %.0f/%.0f)\n", home0.size(), home1.size(), l0[0], l1[0]);

  signed char* d_die;
  cudaMalloc(&d_die, 256);
  std::vector<signed char> die8(256);
  for (int s = 0; s < 256; ++s) die8[s] = (signed char)(die[s] < 0 ? 0 : die[s]);
  cudaMemcpy(d_die, die8.data(), 256, cudaMemcpyHostToDevice);
  unsigned* sink;
  cudaMalloc(&sink, 4);
  int *dA, *dB, *dMix;
  cudaMalloc(&dA, R * 4);
  cudaMalloc(&dB, R * 4);
  cudaMalloc(&dMix, R * 4);
  for (int H : {1, 16, 256}) {
    if ((int)home0.size() < H || (int)home1.size() < H) continue;
    // mixed set: H rows alternating homes; A = H rows homed die0; B = H rows homed die1
    std::vector<int> mix, A(home0.begin(), home0.begin() + H), B(home1.begin(), home1.begin() + H);
    for (int i = 0; i < H; ++i) mix.push_back(i % 2 ? home1[i / 2] : home0[i / 2]);
    if (H == 1) mix = {home0[0]};
    cudaMemcpy(dMix, mix.data(), H * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dA, A.data(), H * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, B.data(), H * 4, cudaMemcpyHostToDevice);
    const int groups = 9472, iters = 1000;
    long long g;
    std::vector<int> dummy;
    struct Case { const char* name; const int* a; const int* b; int mode; double frac; };
    // split with H rows total: H/2 per die (H>=2)
    const int Hh = std::max(1, H / 2);
    const double f0 = (double)n0 / nsm;
    Case cs[] = {{"all (mixed homes)", dMix, dMix, 0, 1.0},
                 {"one-die SMs, mixed rows", dMix, dMix, 1, f0},
                 {"one-die SMs, near rows", dA, dA, 1, f0},
                 {"one-die SMs, far rows", dB, dB, 1, f0},
                 {"split: die d -> rows homed d", dA, dB, 2, 1.0},
                 {"split-x: die d -> rows homed 1-d", dA, dB, 3, 1.0}};
    for (auto& c : cs) {
      const int n = (c.mode >= 2) ? Hh : H;
      const float ms = time_hot(rows, c.a, n, c.b, n, d_die, c.mode, groups, iters, sink, &g, dummy, dummy);
      const double upd = (double)groups * iters * c.frac;   // one-die: the die-0 share of the CTAs
      const int rows_touched = (c.mode >= 2) ? 2 * n : n;
      printf("H=%4d %-34s %8.3f ms  total %7.3f G/s  per-row %8.2f M/s\n", H, c.name, ms,
             upd / ms / 1e6, upd / ms / 1e3 / rows_touched);
    }
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
