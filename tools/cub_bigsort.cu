// Check cub::DeviceRadixSort::SortPairs with int64 num_items > 2^31 (the shuffle sort at
// Hugewiki scale, N = 3.07e9): keys sorted, values a permutation (sum + xor checks).
#include <cub/cub.cuh>
#include <cstdio>
#include <cstdint>
__global__ void fill(uint64_t* k, uint32_t* v, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t z = (uint64_t)i * 0x9E3779B97F4A7C15ull + 12345;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
    k[i] = z; v[i] = (uint32_t)i;
  }
}
__global__ void check(const uint64_t* k, const uint32_t* v, int64_t n, unsigned long long* bad,
                      unsigned long long* vsum, unsigned long long* vx) {
  unsigned long long s = 0, x = 0, b = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    if (i + 1 < n && k[i] > k[i + 1]) b++;
    s += v[i]; x ^= v[i];
  }
  atomicAdd(bad, b); atomicAdd(vsum, s); atomicXor(vx, x);
}
int main() {
  const int64_t n = 2400000000LL;
  uint64_t *k0, *k1; uint32_t *v0, *v1;
  cudaMalloc(&k0, n * 8); cudaMalloc(&k1, n * 8); cudaMalloc(&v0, n * 4); cudaMalloc(&v1, n * 4);
  fill<<<4096, 256>>>(k0, v0, n);
  size_t tb = 0; void* tmp = nullptr;
  cub::DeviceRadixSort::SortPairs(tmp, tb, k0, k1, v0, v1, n, 0, 64);
  cudaMalloc(&tmp, tb);
  cudaError_t e = cub::DeviceRadixSort::SortPairs(tmp, tb, k0, k1, v0, v1, n, 0, 64);
  cudaDeviceSynchronize();
  unsigned long long *d; cudaMalloc(&d, 24); cudaMemset(d, 0, 24);
  check<<<4096, 256>>>(k1, v1, n, d, d + 1, d + 2);
  unsigned long long h[3]; cudaMemcpy(h, d, 24, cudaMemcpyDeviceToHost);
  unsigned long long want_sum = 0, want_x = 0;
  for (int64_t i = 0; i < n; ++i) { want_sum += (uint32_t)i; want_x ^= (uint32_t)i; }
  printf("sort err=%s  unsorted pairs=%llu  vsum ok=%d  vxor ok=%d  temp=%zu MB\n", cudaGetErrorString(e), h[0],
         h[1] == want_sum, h[2] == want_x, tb >> 20);
  return 0;
}
