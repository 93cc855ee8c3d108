// mf_common.cuh -- shared definitions of the product path (libmf_b200.so).
// Independent of oracle/: the keyed hash below is this library's own rendering of the
// SURVEY.md Appendix A specification (the two implementations agree by specification only).
#pragma once

#include <cstdint>
#include <cuda_bf16.h>
#include <cuda_fp16.h>

namespace mfb {

constexpr uint64_t kPhi = 0x9E3779B97F4A7C15ull;  // A: golden-ratio increment

// A: SplitMix64 finaliser (bijective), stream derivation and per-index key.
__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__host__ __device__ __forceinline__ uint64_t make_stream(uint64_t seed, uint64_t tag, uint64_t a,
                                                         uint64_t b) {
  return mix64(mix64(mix64(seed + tag * kPhi) + a * kPhi) + b * kPhi);
}
__host__ __device__ __forceinline__ uint64_t hkey(uint64_t S, uint64_t i) {
  return mix64(S + i * kPhi);
}

// Stream tags (A: table "Streams").
enum : uint64_t {
  kTagShuf = 1, kTagRow = 2, kTagCol = 3, kTagP = 4, kTagQ = 5, kTagHW = 6, kTagWF = 7,
  kTagStrata = 8, kTagCycTau = 9, kTagCycSigma = 10
};

// One COO rating as the paper stores it: two ints and one float, 12 bytes.
// In device memory u, v are the RELABELLED indices (rho_R(u), rho_C(v)) and r = r/rating_scale.
struct Rating {
  int32_t u, v;
  float r;
};
static_assert(sizeof(Rating) == 12, "12-byte COO sample");

constexpr int32_t kSentinel = -1;  // padding slot (u = v = -1), skipped by every kernel

__host__ __device__ __forceinline__ int64_t cdiv64(int64_t x, int64_t y) { return (x + y - 1) / y; }

}  // namespace mfb
