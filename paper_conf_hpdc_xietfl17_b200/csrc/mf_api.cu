// mf_api.cu -- host runtime of libmf_b200.so: the C ABI of include/mf.h, the one-time GPU
// preprocessing (validate, shuffle, relabel, bucket, init), the per-epoch schedule build
// (chunk order, column sequences, tickets) and the epoch driver.  All device work runs in
// this library's kernels (plus CUB radix sort as the sort primitive); nothing falls back to
// the CPU.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <map>
#include <cub/cub.cuh>
#include <nvtx3/nvToolsExt.h>
#include <string>
#include <vector>

#include "mf.h"
#include "mf_comm.h"
#include "mf_internal.h"

using namespace mfb;

// NVTX ranges (SURVEY 5 tracing): per load phase, epoch, schedule build, sub-epoch, Q rotation
// and evaluation -- visible in nsys / ncu --nvtx timelines; header-only, no cost unattached.
struct Nvtx {
  explicit Nvtx(const char* fmt, ...) {
    char buf[96];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    nvtxRangePushA(buf);
  }
  ~Nvtx() { nvtxRangePop(); }
  Nvtx(const Nvtx&) = delete;
  Nvtx& operator=(const Nvtx&) = delete;
};

// =============================================================================================
// preprocessing / schedule kernels
// =============================================================================================
namespace {

__global__ void k_validate(const int32_t* __restrict__ u, const int32_t* __restrict__ v,
                           const float* __restrict__ r, int64_t N, int64_t m, int64_t n,
                           int* __restrict__ bad) {
  int local = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t a = u[i], b = v[i];
    const float x = r[i];
    if (a < 0 || a >= m || b < 0 || b >= n || !isfinite(x)) local = 1;
  }
  if (__syncthreads_or(local) && threadIdx.x == 0) atomicOr(bad, 1);
}

// keys[i] = key(S, i), vals[i] = i  (A: "perm(S, n) = [0..n) sorted ascending by key(S,.)")
__global__ void k_iota_keys(uint64_t S, int64_t n, uint64_t* __restrict__ keys,
                            uint32_t* __restrict__ vals) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    keys[i] = hkey(S, (uint64_t)i);
    vals[i] = (uint32_t)i;
  }
}

// keys[j] = key(S, idx[j]) (idx == nullptr: idx[j] = j), vals[j] = idx[j]
__global__ void k_keys_of(uint64_t S, const uint32_t* __restrict__ idx, int64_t n,
                          uint64_t* __restrict__ keys, uint32_t* __restrict__ vals) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n;
       j += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t i = idx ? idx[j] : (uint32_t)j;
    keys[j] = hkey(S, (uint64_t)i);
    vals[j] = i;
  }
}

// world > 1: flag the caller's ratings whose row segment this rank owns
__global__ void k_own_caller(const int32_t* __restrict__ u, int64_t N, const int32_t* __restrict__ rho_r,
                             int64_t m, int64_t a, int64_t lo_seg, int64_t hi_seg,
                             char* __restrict__ flag) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = (int64_t)rho_r[u[i]] * a / m;
    flag[i] = (r >= lo_seg && r < hi_seg) ? 1 : 0;
  }
}

// rho[perm[j]] = j
__global__ void k_rank_of(const uint32_t* __restrict__ perm, int64_t n, int32_t* __restrict__ rho) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n;
       j += (int64_t)gridDim.x * blockDim.x)
    rho[perm[j]] = (int32_t)j;
}

struct Grid {
  int64_t m, n, a, s, c;  // s, c only for wavefront
  bool wf;
  int64_t ac;             // column segments: a (a x a strata grid) or 1 (a x 1 row blocks, R27)
};

__device__ __forceinline__ int64_t seg_lo(int64_t r, int64_t a, int64_t n) {
  return cdiv64(r * n, a);
}

// Bucket of a (relabelled) sample: strata block b = r*ac + J (ac = a, or 1 for the a x 1 row
// blocks), and for the wavefront the sub-block (b*s + i)*c + j inside it (A: "Segments and
// blocks").
__device__ __forceinline__ uint32_t bucket_of(const Grid& G, int64_t ru, int64_t rc) {
  const int64_t r = ru * G.a / G.m, J = rc * G.ac / G.n;
  const int64_t b = r * G.ac + J;
  if (!G.wf) return (uint32_t)b;
  const int64_t rlo = seg_lo(r, G.a, G.m), rhi = seg_lo(r + 1, G.a, G.m);
  const int64_t clo = seg_lo(J, G.ac, G.n), chi = seg_lo(J + 1, G.ac, G.n);
  const int64_t i = (ru - rlo) * G.s / (rhi - rlo);
  const int64_t j = (rc - clo) * G.c / (chi - clo);
  return (uint32_t)((b * G.s + i) * G.c + j);
}

// storage order j (Alg. 1 l.2): sample perm[j], relabelled and scaled; plus its bucket.
__global__ void k_build_storage(const uint32_t* __restrict__ perm, int64_t N,
                                const int32_t* __restrict__ u, const int32_t* __restrict__ v,
                                const float* __restrict__ r, const int32_t* __restrict__ rho_r,
                                const int32_t* __restrict__ rho_c, double rs, Grid G,
                                Rating* __restrict__ stor, uint32_t* __restrict__ bucket,
                                uint32_t* __restrict__ pos) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < N;
       j += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t i = perm[j];
    Rating x;
    x.u = rho_r[u[i]];
    x.v = rho_c[v[i]];
    x.r = (float)((double)r[i] / rs);     // R5: r' = r / rating_scale, rounded once
    stor[j] = x;
    if (bucket) bucket[j] = bucket_of(G, x.u, x.v);
    if (pos) pos[j] = (uint32_t)j;
  }
}

__global__ void k_build_test(const int32_t* __restrict__ u, const int32_t* __restrict__ v,
                             const float* __restrict__ r, int64_t N,
                             const int32_t* __restrict__ rho_r, const int32_t* __restrict__ rho_c,
                             double rs, Rating* __restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N;
       i += (int64_t)gridDim.x * blockDim.x) {
    Rating x;
    x.u = rho_r[u[i]];
    x.v = rho_c[v[i]];
    x.r = (float)((double)r[i] / rs);
    out[i] = x;
  }
}

// world > 1: a test rating is evaluated by the rank owning its row segment
__global__ void k_own_rows(const Rating* __restrict__ t, int64_t N, int64_t m, int64_t a,
                           int64_t lo_seg, int64_t hi_seg, char* __restrict__ flag) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = (int64_t)t[i].u * a / m;
    flag[i] = (r >= lo_seg && r < hi_seg) ? 1 : 0;
  }
}

__global__ void k_histogram(const uint32_t* __restrict__ bucket, int64_t N,
                            unsigned int* __restrict__ cnt) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < N;
       j += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(cnt + bucket[j], 1u);
}

// Few buckets (strata blocks, a*a <= 4096): per-CTA shared-memory counts, one global atomic
// per bucket per CTA (a single global counter would serialise N atomics).
constexpr int kSmemBuckets = 4096;
__global__ void k_histogram_smem(const uint32_t* __restrict__ bucket, int64_t N, int nb,
                                 unsigned int* __restrict__ cnt) {
  __shared__ unsigned int h[kSmemBuckets];
  for (int i = threadIdx.x; i < nb; i += blockDim.x) h[i] = 0u;
  __syncthreads();
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < N;
       j += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(h + bucket[j], 1u);
  __syncthreads();
  for (int i = threadIdx.x; i < nb; i += blockDim.x)
    if (h[i]) atomicAdd(cnt + i, h[i]);
}

// Place sorted sample x (bucket b = key[x]) at slot dst_off[b] + (x - src_off[b]).
__global__ void k_place(const uint32_t* __restrict__ keys_sorted,
                        const uint32_t* __restrict__ pos_sorted, int64_t N,
                        const int64_t* __restrict__ src_off, const int64_t* __restrict__ dst_off,
                        const Rating* __restrict__ stor, Rating* __restrict__ slots,
                        uint32_t* __restrict__ slot_pos) {
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < N;
       x += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t b = keys_sorted ? keys_sorted[x] : 0u;
    const uint32_t j = pos_sorted[x];
    const int64_t slot = dst_off[b] + (x - src_off[b]);
    slots[slot] = stor[j];
    if (slot_pos) slot_pos[slot] = j;
  }
}

// Ring-staged wavefront metadata: for slot x, the distance to the previous slot of the same
// sub-block with the same u (low byte) / same v (high byte) when it is <= W, else 0.
__global__ void k_dupdist(const Rating* __restrict__ slots, int64_t N, Grid G, int W,
                          uint16_t* __restrict__ dup) {
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < N;
       x += (int64_t)gridDim.x * blockDim.x) {
    const Rating a = slots[x];
    const uint32_t b = bucket_of(G, a.u, a.v);
    int pd = 0, qd = 0;
    for (int d = 1; d <= W && x - d >= 0; ++d) {
      const Rating y = slots[x - d];
      if (bucket_of(G, y.u, y.v) != b) break;
      if (!pd && y.u == a.u) pd = d;
      if (!qd && y.v == a.v) qd = d;
    }
    dup[x] = (uint16_t)(pd | (qd << 8));
  }
}

// Packed staging records (the out-of-core H2D stream, section 6.2): (u, v) as ONE integer
// uv = u << bv | v of bu + bv bits (bu = bits(m), bv = bits(n - 1)) stored in 4 + hib bytes --
// a u32 low word and hib (1 or 2) high bytes -- plus r as fp32: 9 B per rating when
// bu + bv <= 40 (Netflix, Yahoo shapes), 10 B up to 48 (Hugewiki), instead of the 12-B slot.
// The sentinel pad slot (u = v = -1) is the all-ones uv: its u field 2^bu - 1 >= m is never a
// real row.
struct PackFmt {
  int bu, bv, hib;
};
__global__ void k_split_slots(const Rating* __restrict__ s, int64_t N, PackFmt F,
                              uint32_t* __restrict__ lo, uint8_t* __restrict__ hi,
                              float* __restrict__ r) {
  const uint64_t ones = (1ull << (F.bu + F.bv)) - 1ull;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < N;
       x += (int64_t)gridDim.x * blockDim.x) {
    const Rating a = s[x];
    const uint64_t uv = a.u < 0 ? ones : (((uint64_t)(uint32_t)a.u << F.bv) | (uint32_t)a.v);
    lo[x] = (uint32_t)uv;
    if (F.hib == 1) {
      hi[x] = (uint8_t)(uv >> 32);
    } else {
      reinterpret_cast<uint16_t*>(hi)[x] = (uint16_t)(uv >> 32);
    }
    r[x] = a.r;
  }
}
__global__ void k_expand_slots(const uint32_t* __restrict__ lo, const uint8_t* __restrict__ hi,
                               const float* __restrict__ r, int64_t N, PackFmt F,
                               Rating* __restrict__ s) {
  const uint32_t usent = (1u << F.bu) - 1u, vmask = (1u << F.bv) - 1u;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < N;
       x += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t h = F.hib == 1 ? (uint64_t)__ldcs(hi + x)
                                  : (uint64_t)__ldcs(reinterpret_cast<const unsigned short*>(hi) + x);
    const uint64_t uv = (uint64_t)__ldcs(lo + x) | (h << 32);
    const uint32_t u = (uint32_t)(uv >> F.bv);
    Rating a;
    a.u = u == usent ? -1 : (int32_t)u;
    a.v = u == usent ? -1 : (int32_t)((uint32_t)uv & vmask);
    a.r = __ldcs(r + x);
    s[x] = a;
  }
}

// Alg. 1 l.3 (R5): X[rho[id]][d] = round_S((float)U24(S, id*k+d) * 2^-24 * amp),
// keyed by the ORIGINAL id (A: S_P / S_Q).
template <typename T>
__global__ void k_init(T* __restrict__ X, const int32_t* __restrict__ rho, int64_t rows, int k,
                       uint64_t S, float amp) {
  const int64_t total = rows * k;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t id = x / k, d = x % k;
    const float u01 = (float)(hkey(S, (uint64_t)x) >> 40) * 0x1p-24f;
    const float val = u01 * amp;
    X[(int64_t)rho[id] * k + d] = static_cast<T>(val);
  }
}

template <typename T> __device__ __forceinline__ float to_f32(T x) { return static_cast<float>(x); }
template <> __device__ __forceinline__ float to_f32<__half>(__half x) { return __half2float(x); }
template <> __device__ __forceinline__ float to_f32<__nv_bfloat16>(__nv_bfloat16 x) {
  return __bfloat162float(x);
}
template <typename T> __device__ __forceinline__ T from_f32(float x);
template <> __device__ __forceinline__ float from_f32<float>(float x) { return x; }
template <> __device__ __forceinline__ __half from_f32<__half>(float x) { return __float2half_rn(x); }
template <> __device__ __forceinline__ __nv_bfloat16 from_f32<__nv_bfloat16>(float x) {
  return __float2bfloat16_rn(x);
}

// inv[rho[i]] = i (relabelled row -> original id)
__global__ void k_invert(const int32_t* __restrict__ rho, int64_t n, int32_t* __restrict__ inv) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    inv[rho[i]] = (int32_t)i;
}

// Alg. 1 l.3 for relabelled rows [lo, lo + rows) into a segment buffer (staged == 2): the same
// value as k_init for every (id, d), id = inv[row].
template <typename T>
__global__ void k_init_rows(T* __restrict__ X, const int32_t* __restrict__ inv, int64_t lo,
                            int64_t rows, int k, uint64_t S, float amp) {
  const int64_t total = rows * k;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t id = inv[lo + x / k], d = x % k;
    const float u01 = (float)(hkey(S, (uint64_t)(id * k + d)) >> 40) * 0x1p-24f;
    X[x] = static_cast<T>(u01 * amp);
  }
}

// model_shuffle (Alg. 1 l.15): out[id][d] = fp32(X[rho[id]][d])
template <typename T>
__global__ void k_unrelabel(const T* __restrict__ X, const int32_t* __restrict__ rho, int64_t rows,
                            int k, float* __restrict__ out) {
  const int64_t total = rows * k;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t id = x / k, d = x % k;
    out[x] = to_f32<T>(X[(int64_t)rho[id] * k + d]);
  }
}
template <typename T>
__global__ void k_relabel_store(T* __restrict__ X, const int32_t* __restrict__ rho, int64_t rows,
                                int k, const float* __restrict__ in) {
  const int64_t total = rows * k;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t id = x / k, d = x % k;
    X[(int64_t)rho[id] * k + d] = from_f32<T>(in[x]);
  }
}

// Hogwild chunk keys of epoch t: global chunk gc of block b (local q = gc - choff[b]) gets
// key(S_HW(t,b), q) (A).  nb <= 64 blocks -> linear search is fine.
__global__ void k_chunk_keys(const int64_t* __restrict__ choff, int nb, uint64_t seed, int32_t t,
                             uint64_t* __restrict__ keys, uint32_t* __restrict__ vals) {
  const int64_t total = choff[nb];
  for (int64_t gc = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; gc < total;
       gc += (int64_t)gridDim.x * blockDim.x) {
    int b = 0;
    while (gc >= choff[b + 1]) ++b;
    const uint64_t S = make_stream(seed, kTagHW, (uint64_t)t, (uint64_t)b);
    keys[gc] = hkey(S, (uint64_t)(gc - choff[b]));
    vals[gc] = (uint32_t)gc;
  }
}

// block id of each (sorted) chunk, for the stable second pass
__global__ void k_chunk_block(const uint32_t* __restrict__ vals, const int64_t* __restrict__ choff,
                              int nb, int64_t total, uint32_t* __restrict__ blk) {
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t gc = vals[x];
    int b = 0;
    while (gc >= choff[b + 1]) ++b;
    blk[x] = (uint32_t)b;
  }
}

// wavefront column-sequence keys: item (b*s + i)*c + j gets key(S_WF(t,b,i), j) (A).
__global__ void k_wf_keys(int64_t nseg, int s, int c, uint64_t seed, int32_t t,
                          uint64_t* __restrict__ keys, uint32_t* __restrict__ vals) {
  const int64_t total = nseg * c;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t sg = x / c, j = x % c;
    const int64_t b = sg / s, i = sg % s;
    const uint64_t S = make_stream(seed, kTagWF, (uint64_t)t, ((uint64_t)b << 32) + (uint64_t)i);
    keys[x] = hkey(S, (uint64_t)j);
    vals[x] = (uint32_t)x;
  }
}

// generic: keys for nseg independent permutations of length c with per-segment stream
// make_stream(seed, tag, t, seg) (cyclic variant's tau / sigma per block)
__global__ void k_perm_keys(int64_t nseg, int c, uint64_t seed, uint64_t tag, int32_t t,
                            uint64_t* __restrict__ keys, uint32_t* __restrict__ vals) {
  const int64_t total = nseg * c;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t sg = x / c, j = x % c;
    keys[x] = hkey(make_stream(seed, tag, (uint64_t)t, (uint64_t)sg), (uint64_t)j);
    vals[x] = (uint32_t)x;
  }
}

__global__ void k_seg_of(const uint32_t* __restrict__ vals, int64_t total, int c,
                         uint32_t* __restrict__ seg) {
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x)
    seg[x] = (uint32_t)(vals[x] / (uint32_t)c);
}

// sorted (segment-major) vals -> position-in-segment j values
__global__ void k_mod_c(const uint32_t* __restrict__ vals, int64_t total, int c,
                        int32_t* __restrict__ out) {
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x)
    out[x] = (int32_t)(vals[x] % (uint32_t)c);
}

// cyclic variant (A): seq_i[w] = sigma[(tau[i] + w) mod c] per block b
__global__ void k_cyclic_seq(const int32_t* __restrict__ tau, const int32_t* __restrict__ sigma,
                             int64_t nb, int s, int c, int32_t* __restrict__ seq) {
  const int64_t total = nb * s * (int64_t)c;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t w = x % c, bi = x / c, i = bi % s, b = bi / s;
    seq[x] = sigma[b * c + (tau[b * c + i] + w) % c];
  }
}

// Cyclic variant, ticket ranks in closed form (no sort).  Worker i visits column
// sigma[(tau[i] + w) mod c] in wave w, so the s visits of one column fall in distinct waves,
// and the rank of visit (w, i) -- the number of earlier (w', i') visits of that column -- is
// the number of workers i' whose offset lies in the cyclic window (tau[i], tau[i] + w].  With
// P_b(y) = #{i' < s : tau_b[i'] < y} that is P(a+w+1) - P(a+1), or across the wrap
// (P(c) - P(a+1)) + P(a+w-c+1), a = tau_b[i].
// k_tau_prefix: one CTA per block b builds P_b(0..c) (occupancy of the first s offsets, then
// an inclusive scan in place).
__global__ void __launch_bounds__(1024) k_tau_prefix(const int32_t* __restrict__ tau, int s, int c,
                                                     int32_t* __restrict__ P) {
  __shared__ int32_t part[1024];
  const int64_t b = blockIdx.x;
  int32_t* Pb = P + b * (int64_t)(c + 1);
  for (int y = threadIdx.x; y <= c; y += blockDim.x) Pb[y] = 0;
  __syncthreads();
  for (int i = threadIdx.x; i < s; i += blockDim.x) Pb[1 + tau[b * (int64_t)c + i]] = 1;
  __syncthreads();
  const int ch = (c + (int)blockDim.x - 1) / (int)blockDim.x;
  const int lo = 1 + (int)threadIdx.x * ch, hi = min(c + 1, lo + ch);
  int32_t sum = 0;
  for (int y = lo; y < hi; ++y) sum += Pb[y];
  part[threadIdx.x] = sum;
  __syncthreads();
  for (int o = 1; o < (int)blockDim.x; o <<= 1) {     // Hillis-Steele inclusive scan
    const int32_t add = (int)threadIdx.x >= o ? part[threadIdx.x - o] : 0;
    __syncthreads();
    part[threadIdx.x] += add;
    __syncthreads();
  }
  int32_t run = part[threadIdx.x] - sum;               // exclusive prefix of this chunk
  for (int y = lo; y < hi; ++y) {
    run += Pb[y];
    Pb[y] = run;
  }
}

__global__ void k_cyclic_rank(const int32_t* __restrict__ tau, const int32_t* __restrict__ P,
                              int64_t nb, int s, int c, int32_t* __restrict__ rank) {
  const int64_t total = nb * s * (int64_t)c;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t w = x % c, bi = x / c, i = bi % s, b = bi / s;
    const int32_t* Pb = P + b * (int64_t)(c + 1);
    const int64_t a = tau[b * c + i], e = a + w;
    rank[x] = e < c ? Pb[e + 1] - Pb[a + 1] : (Pb[c] - Pb[a + 1]) + Pb[e - c + 1];
  }
}

// ticket keys: visit (b,i,w) to column col = seq[(b*s+i)*c+w] gets key ((b*c+col)*c + w)*s + i
__global__ void k_ticket_keys(const int32_t* __restrict__ seq, int64_t nb, int s, int c,
                              uint64_t* __restrict__ keys, uint32_t* __restrict__ vals) {
  const int64_t total = nb * s * (int64_t)c;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t w = x % c, bi = x / c, i = bi % s, b = bi / s;
    const int64_t col = seq[x];
    keys[x] = (uint64_t)(((b * c + col) * c + w) * s + i);
    vals[x] = (uint32_t)x;
  }
}

// rank of visit = sorted position - first position of its (b, col) group (each column is
// visited exactly s times per block and epoch).
__global__ void k_ticket_rank(const uint32_t* __restrict__ vals, int64_t total, int s,
                              int32_t* __restrict__ rank) {
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
       x += (int64_t)gridDim.x * blockDim.x)
    rank[vals[x]] = (int32_t)(x % s);
}

int bits_for(uint64_t maxval) {
  int b = 1;
  while (b < 64 && (maxval >> b) != 0) ++b;
  return b;
}

inline int grid_for(int64_t n, int num_sms) {
  int64_t b = (n + 255) / 256;
  int64_t cap = (int64_t)num_sms * 16;
  if (b > cap) b = cap;
  if (b < 1) b = 1;
  return (int)b;
}

// Eq. 9, t 0-based (R4): evaluated in double with t^1.5 = t*sqrt(t), rounded once.
float gamma_of(float alpha, float beta, int32_t t) {
  const double td = (double)t;
  return (float)((double)alpha / (1.0 + (double)beta * td * std::sqrt(td)));
}

// ---- out-of-core (chunked) preprocessing (section 6): the caller's COO streams
// through the device in chunks; pass 1 partitions each chunk by strata block, pass 2 orders one
// block at a time.  Same slots as the resident path, bit for bit.
// Pass 1: record i0 + j of the caller's set -> (block, shuffle key, relabelled rating).  Samples
// of row segments this rank does not own get block = nb (sorted last, dropped).
__global__ void k_chunk_records(const int32_t* __restrict__ u, const int32_t* __restrict__ v,
                                const float* __restrict__ r, int64_t C, int64_t i0, uint64_t S,
                                const int32_t* __restrict__ rho_r, const int32_t* __restrict__ rho_c,
                                double rs, int64_t m, int64_t n, int64_t a, int64_t ac,
                                int64_t lo_seg, int64_t hi_seg, uint32_t* __restrict__ blk,
                                uint32_t* __restrict__ idx, uint64_t* __restrict__ keys,
                                Rating* __restrict__ recs) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < C;
       j += (int64_t)gridDim.x * blockDim.x) {
    Rating x;
    x.u = rho_r[u[j]];
    x.v = rho_c[v[j]];
    x.r = (float)((double)r[j] / rs);                  // R5, rounded once (as k_build_storage)
    const int64_t seg = (int64_t)x.u * a / m;
    const bool own = seg >= lo_seg && seg < hi_seg;
    blk[j] = own ? (uint32_t)(seg * ac + (int64_t)x.v * ac / n) : (uint32_t)(a * ac);
    idx[j] = (uint32_t)j;
    keys[j] = hkey(S, (uint64_t)(i0 + j));              // A: key(S_SHUF, caller index)
    recs[j] = x;
  }
}

// Column-grouped batches (group_cols, reading R24): key of slot x of a chunk-aligned piece =
// (chunk within the piece, relabelled column); a stable sort by it orders every batch of f
// consecutive samples by column, ties in storage order (sentinel pads, v = -1, stay last).
__global__ void k_group_keys(const Rating* __restrict__ slots, int64_t n, int f,
                             uint64_t* __restrict__ keys, uint32_t* __restrict__ vals) {
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < n;
       x += (int64_t)gridDim.x * blockDim.x) {
    keys[x] = ((uint64_t)(x / f) << 32) | (uint32_t)slots[x].v;
    vals[x] = (uint32_t)x;
  }
}
__global__ void k_permute_slots(const uint32_t* __restrict__ order, int64_t n,
                                const Rating* __restrict__ in, Rating* __restrict__ out,
                                const uint32_t* __restrict__ pin, uint32_t* __restrict__ pout) {
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < n;
       x += (int64_t)gridDim.x * blockDim.x) {
    out[x] = in[order[x]];
    if (pout) pout[x] = pin[order[x]];
  }
}

__global__ void k_test_seg(const Rating* __restrict__ t, int64_t N, int64_t m, int64_t a,
                           uint32_t* __restrict__ seg, uint32_t* __restrict__ idx) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N;
       i += (int64_t)gridDim.x * blockDim.x) {
    seg[i] = (uint32_t)((int64_t)t[i].u * a / m);
    idx[i] = (uint32_t)i;
  }
}

__global__ void k_iota_u32(uint32_t* __restrict__ x, int64_t n) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n;
       j += (int64_t)gridDim.x * blockDim.x)
    x[j] = (uint32_t)j;
}

__global__ void k_gather_records(const uint32_t* __restrict__ order, int64_t n,
                                 const uint64_t* __restrict__ kin, const Rating* __restrict__ rin,
                                 uint64_t* __restrict__ kout, Rating* __restrict__ rout) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n;
       j += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t o = order[j];
    if (kout) kout[j] = kin[o];
    rout[j] = rin[o];
  }
}

// Pass 2 (wavefront): sub-block of each (key-ordered) sample of block b, local to the block.
__global__ void k_local_sub(const Rating* __restrict__ recs, int64_t n, Grid G, int64_t b,
                            uint32_t* __restrict__ sub, uint32_t* __restrict__ idx) {
  const int64_t per = G.s * G.c;
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n;
       j += (int64_t)gridDim.x * blockDim.x) {
    sub[j] = (uint32_t)((int64_t)bucket_of(G, recs[j].u, recs[j].v) - b * per);
    idx[j] = (uint32_t)j;
  }
}

// A: host perm of a small set (strata order pi_t).
std::vector<int64_t> host_perm(uint64_t S, int64_t n) {
  std::vector<std::pair<uint64_t, int64_t>> t((size_t)n);
  for (int64_t i = 0; i < n; ++i) t[(size_t)i] = {hkey(S, (uint64_t)i), i};
  std::sort(t.begin(), t.end());
  std::vector<int64_t> out((size_t)n);
  for (int64_t i = 0; i < n; ++i) out[(size_t)i] = t[(size_t)i].second;
  return out;
}

}  // namespace

// =============================================================================================
// context
// =============================================================================================
struct mf_ctx {
  mf_params p{};
  uint8_t nccl_id[128]{};
  int dev = 0, num_sms = 0;
  cudaStream_t st = nullptr;
  bool own_stream = false;
  mf_status sticky = MF_OK;
  std::string err;
  bool train_loaded = false, test_loaded = false;

  int64_t m = 0, n = 0, N = 0, Ntest = 0;
  int k = 0, a = 1, s = 1, c = 1, f = 256, G = 1, rank = 0;
  int ac = 1;                        // column segments of the grid: a, or 1 (a x 1, R27)
  int32_t t = 0;
  bool wf = false;

  // device state
  Rating* slots = nullptr;         int64_t nslots = 0;
  uint32_t* slot_pos = nullptr;    // storage position of each slot (0xFFFFFFFF = pad)
  uint32_t* perm = nullptr;        // caller index of storage position j
  int32_t* rho_r = nullptr;
  int32_t* rho_c = nullptr;
  void* P = nullptr;
  void* Q = nullptr;
  Rating* test = nullptr;
  uint16_t* dup = nullptr;         // wavefront ring kernel: per-slot duplicate distances
  int64_t* sub_off = nullptr;      // wavefront: a*a*s*c + 1
  std::vector<int64_t> blk_off;    // a*a + 1 slot offsets (Hogwild: padded to f)
  std::vector<int64_t> blk_len;    // a*a sample counts
  std::vector<int64_t> ch_off;     // a*a + 1 chunk offsets (Hogwild)
  int64_t* d_choff = nullptr;
  // schedule scratch
  uint64_t *sk0 = nullptr, *sk1 = nullptr;
  uint32_t *sv0 = nullptr, *sv1 = nullptr, *sb = nullptr;
  int64_t sched_cap = 0;
  uint32_t* chunk_order = nullptr;  // Hogwild: sorted global chunk ids, blocks ascending
  // Hogwild: the next epoch's chunk order is built on a side stream (ss) into chunk_order_alt
  // while this epoch's SGD kernel runs (its sorts fill the SMs its retiring blocks free).
  uint32_t* chunk_order_alt = nullptr;
  uint32_t* chunk_seq = nullptr;     // a x 1 resident: the epoch's chunk ids, blocks in pi_t order
  cudaStream_t ss = nullptr;
  cudaEvent_t ev_ss_go = nullptr, ev_ss_done = nullptr;
  int32_t prebuilt_t = -1;           // epoch whose order chunk_order_alt holds (-1: none)
  bool ss_pending = false;           // a side build may still use the sort scratch
  int32_t *seq = nullptr, *rank_arr = nullptr, *tickets = nullptr;
  int32_t *tau = nullptr, *sigma = nullptr;
  unsigned long long* counter = nullptr;
  // Exactly-once evidence (Eq. 7): per work unit (Hogwild chunk / wavefront sub-block /
  // LIBMF block) the number of claims since load, and the device count of the samples the SGD
  // kernels updated in the current epoch.  mf_check_visits compares the former with epochs_run.
  unsigned* visits = nullptr;
  int64_t n_units = 0;
  unsigned long long* upd_dev = nullptr;
  unsigned long long* chk_dev = nullptr;
  int32_t epochs_run = 0;
  int* owners = nullptr;             // params.check_owners: wavefront column tags (c)
  unsigned* own_viol = nullptr;      // violations found by the ownership checker
  double* rm_partial = nullptr;
  double* rm_out = nullptr;
  void* tmp = nullptr;
  size_t tmp_bytes = 0;
  int sched_built_for = -1;

  // stats
  std::vector<cudaEvent_t> ev;     // pairs for SGD launches
  cudaEvent_t ev_e0 = nullptr, ev_e1 = nullptr, ev_s0 = nullptr, ev_s1 = nullptr;
  cudaEvent_t ev_c0 = nullptr, ev_c1 = nullptr;
  int n_sgd = 0, n_launch = 0;
  int last_workers = 0, last_lanes = 0, last_grid = 0, last_block = 0, last_q_l1 = 0;
  bool have_stats = false;
  std::vector<double> comm_ms_acc;

  mf::Comm* comm = nullptr;

  // out-of-core staging (params.staged; section 6.2): the bucketed ratings live in
  // pinned host memory; each stratum's blocks are copied into one of two device buffers on a
  // copy stream while the previous stratum computes.
  float* GP = nullptr;             // ADAGRAD accumulators (lr_rule 1), fp32, relabelled rows
  float* GQ = nullptr;
  bool libmf = false;              // LIBMF-GPU table-scheduler baseline (MF_LIBMF)
  int64_t *d_blk_off = nullptr, *d_blk_len = nullptr;
  int *lm_lock = nullptr, *lm_row = nullptr, *lm_col = nullptr, *lm_done = nullptr, *lm_rem = nullptr;

  bool staged = false;
  // Packed staging (n <= 65535): the pinned host copy and the H2D stream carry 10 B per rating
  // (u int32, v uint16, r fp32, structure of arrays) instead of the 12-B slot; the compute
  // stream expands each staged stratum back into 12-B slots before its SGD launch.
  bool stg_packed = false;
  PackFmt pk{0, 0, 0};               // packed record format (bits of u, v; high bytes)
  uint32_t* h_u = nullptr;           // packed: low words of uv
  uint8_t* h_v16 = nullptr;          // packed: pk.hib high bytes of uv per rating
  float* h_r = nullptr;
  uint32_t* stg_u[2] = {nullptr, nullptr};
  uint8_t* stg_v16[2] = {nullptr, nullptr};
  float* stg_r[2] = {nullptr, nullptr};
  int64_t stg_len[2] = {0, 0};
  Rating* h_slots = nullptr;
  uint16_t* h_dup = nullptr;
  Rating* stg[2] = {nullptr, nullptr};
  uint16_t* stg_dup[2] = {nullptr, nullptr};
  int64_t stg_cap = 0;
  cudaStream_t cs = nullptr;
  cudaEvent_t ev_h2d[2] = {nullptr, nullptr}, ev_free[2] = {nullptr, nullptr};
  std::vector<std::pair<int64_t, int64_t>> stg_shift[2];   // (block, slot shift) per buffer
  int64_t staged_t = -1, staged_j = -1;
  int cur_buf = 0;
  int64_t h2d_bytes = 0;
  // staged == 2 (section 6.1 step 3): P is out of core too.  Its row segments live
  // in pinned host memory and one strata block at a time is trained with its segment staged
  // into one of two device slots: copy-in stream cs, compute stream st, write-back stream ds
  // (the three streams of section 6.3).  Q stays resident.
  bool pq = false;
  char* h_P = nullptr;
  char* Pslot[2] = {nullptr, nullptr};
  int64_t pseg_max = 0;
  cudaStream_t ds = nullptr;
  cudaEvent_t ev_pin[2] = {nullptr, nullptr}, ev_pcomp[2] = {nullptr, nullptr};
  cudaEvent_t ev_pout[2] = {nullptr, nullptr};
  std::vector<int64_t> test_seg_off;   // pq: test ratings grouped by row segment (a + 1)

  mf_status fail(mf_status s, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    err = buf;
    if (s == MF_E_CUDA || s == MF_E_NCCL) sticky = s;
    return s;
  }
  mf_status cuda_fail(cudaError_t e, const char* what, int line) {
    cudaGetLastError();
    if (e == cudaErrorMemoryAllocation) return fail(MF_E_NOMEM, "%s: out of device memory (line %d)", what, line);
    return fail(MF_E_CUDA, "%s: %s (line %d)", what, cudaGetErrorString(e), line);
  }
  mf_status enter() {
    if (sticky != MF_OK) return fail(MF_E_STATE, "ctx is in an error state after: %s", err.c_str());
    cudaError_t e = cudaSetDevice(dev);
    if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice", __LINE__);
    return MF_OK;
  }

  template <typename X>
  mf_status alloc(X** out, size_t count) {
    *out = nullptr;
    size_t bytes = count * sizeof(X);
    if (bytes == 0) bytes = 16;
    void* ptr = nullptr;
    if (p.alloc && p.alloc->alloc) {
      ptr = p.alloc->alloc(bytes, (void*)st, p.alloc->user);
      if (!ptr) return fail(MF_E_NOMEM, "allocator returned NULL for %zu bytes", bytes);
    } else {
      cudaError_t e = cudaMallocAsync(&ptr, bytes, st);
      if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(MF_E_NOMEM, "cudaMallocAsync(%zu): %s", bytes, cudaGetErrorString(e));
      }
    }
    sizes.push_back({ptr, bytes});
    *out = static_cast<X*>(ptr);
    return MF_OK;
  }
  template <typename X>
  void release(X*& ptr) {
    if (!ptr) return;
    size_t bytes = 0;
    for (size_t i = 0; i < sizes.size(); ++i)
      if (sizes[i].first == (void*)ptr) {
        bytes = sizes[i].second;
        sizes.erase(sizes.begin() + (long)i);
        break;
      }
    if (p.alloc && p.alloc->free) p.alloc->free((void*)ptr, bytes, (void*)st, p.alloc->user);
    else cudaFreeAsync((void*)ptr, st);
    ptr = nullptr;
  }
  std::vector<std::pair<void*, size_t>> sizes;

  mf_status need_tmp(size_t bytes) {
    if (bytes <= tmp_bytes) return MF_OK;
    release(tmp);
    tmp_bytes = 0;
    mf_status s2 = alloc((char**)&tmp, bytes);
    if (s2) return s2;
    tmp_bytes = bytes;
    return MF_OK;
  }
  template <typename K, typename V>
  mf_status sort_pairs(const K* kin, K* kout, const V* vin, V* vout, int64_t n_items, int end_bit) {
    size_t bytes = 0;
    cudaError_t e = cub::DeviceRadixSort::SortPairs(nullptr, bytes, kin, kout, vin, vout, n_items, 0,
                                                    end_bit, st);
    if (e != cudaSuccess) return cuda_fail(e, "cub sort (size)", __LINE__);
    mf_status s2 = need_tmp(bytes);
    if (s2) return s2;
    e = cub::DeviceRadixSort::SortPairs(tmp, bytes, kin, kout, vin, vout, n_items, 0, end_bit, st);
    if (e != cudaSuccess) return cuda_fail(e, "cub sort", __LINE__);
    return MF_OK;
  }
  // Error path of mf_load_coo: release every device allocation made since `before` (a snapshot
  // of `sizes` taken on entry) and null the members that pointed at them, so the ctx stays
  // usable and a retried load does not accumulate the failed attempt's buffers.
  void drop_allocations_since(const std::vector<std::pair<void*, size_t>>& before) {
    std::vector<void*> fresh;
    for (auto& x : sizes) {
      bool old = false;
      for (auto& y : before) old = old || y.first == x.first;
      if (!old) fresh.push_back(x.first);
    }
    void** members[] = {
        (void**)&slots, (void**)&slot_pos, (void**)&perm, (void**)&rho_r, (void**)&rho_c, &P, &Q,
        (void**)&test, (void**)&dup, (void**)&sub_off, (void**)&d_choff, (void**)&sk0,
        (void**)&sk1, (void**)&sv0, (void**)&sv1, (void**)&sb, (void**)&chunk_order,
        (void**)&chunk_order_alt, (void**)&chunk_seq, (void**)&seq, (void**)&rank_arr, (void**)&tickets,
        (void**)&tau, (void**)&sigma, &tmp, (void**)&GP, (void**)&GQ, (void**)&d_blk_off,
        (void**)&d_blk_len, (void**)&lm_lock, (void**)&lm_row, (void**)&lm_col, (void**)&lm_done,
        (void**)&lm_rem, (void**)&stg[0], (void**)&stg[1], (void**)&stg_dup[0],
        (void**)&stg_dup[1], (void**)&stg_u[0], (void**)&stg_u[1], (void**)&stg_v16[0],
        (void**)&stg_v16[1], (void**)&stg_r[0], (void**)&stg_r[1], (void**)&visits,
        (void**)&owners, (void**)&own_viol, (void**)&Pslot[0], (void**)&Pslot[1]};
    for (void* ptr : fresh) {
      for (void** m : members)
        if (*m == ptr) *m = nullptr;
      void* q = ptr;
      release(q);
      if (ptr == tmp) tmp = nullptr;
    }
    if (!tmp) tmp_bytes = 0;
    for (void** h : {(void**)&h_slots, (void**)&h_u, (void**)&h_v16, (void**)&h_r, (void**)&h_dup,
                     (void**)&h_P})
      if (*h) { cudaFreeHost(*h); *h = nullptr; }
    cudaGetLastError();
  }
  int ssize() const { return p.storage == MF_FP32 ? 4 : 2; }
  int lo_row_seg() const { return rank * (a / G); }
  int hi_row_seg() const { return (rank + 1) * (a / G); }
};

#define TRY(expr)                         \
  do {                                    \
    mf_status _s = (expr);                \
    if (_s != MF_OK) return _s;           \
  } while (0)
#define CUDA_TRY(ctx, expr)                                                  \
  do {                                                                       \
    cudaError_t _e = (expr);                                                 \
    if (_e != cudaSuccess) return (ctx)->cuda_fail(_e, #expr, __LINE__);     \
  } while (0)
#define KERNEL_TRY(ctx) CUDA_TRY(ctx, cudaGetLastError())

// =============================================================================================
// C ABI
// =============================================================================================
// Definitions take C linkage from the extern "C" declarations in mf.h.
int32_t mf_abi_version(void) { return MF_ABI_VERSION; }

const char* mf_status_string(mf_status s) {
  switch (s) {
    case MF_OK: return "MF_OK";
    case MF_E_INVAL: return "MF_E_INVAL";
    case MF_E_NOMEM: return "MF_E_NOMEM";
    case MF_E_CUDA: return "MF_E_CUDA";
    case MF_E_NCCL: return "MF_E_NCCL";
    case MF_E_STATE: return "MF_E_STATE";
    case MF_E_RANGE: return "MF_E_RANGE";
    case MF_E_UNSUPPORTED: return "MF_E_UNSUPPORTED";
  }
  return "MF_E_?";
}

const char* mf_last_error(const mf_ctx* ctx) { return ctx ? ctx->err.c_str() : "null ctx"; }

mf_status mf_params_default(mf_params* p) {
  if (!p) return MF_E_INVAL;
  std::memset(p, 0, sizeof *p);
  p->struct_size = (uint32_t)sizeof(mf_params);
  p->k = 128;
  p->lambda_p = p->lambda_q = 0.05f;  // Table 3 Netflix
  p->alpha = 0.08f;
  p->beta = 0.3f;
  p->init_scale = 1.0f;
  p->rating_scale = 1.0f;
  p->seed = 42;
  p->schedule = MF_HOGWILD;
  p->storage = MF_FP32;
  p->batch_f = 256;
  p->world = 1;
  return MF_OK;
}

mf_status mf_strata_holders(uint64_t seed, int32_t a, int32_t world, int32_t t, int32_t j,
                            int32_t* holder) {
  if (a < 1 || world < 1 || a % world != 0 || j < 0 || j >= a || t < 0 || !holder)
    return MF_E_INVAL;
  std::vector<int64_t> pi = host_perm(make_stream(seed, kTagStrata, (uint64_t)t, 0), a);
  const int per = a / world;
  // segment J is trained in sub-epoch j by the owner of row segment (J - pi_t[j]) mod a
  for (int J = 0; J < a; ++J) {
    const int r = (int)(((J - pi[(size_t)j]) % a + a) % a);
    holder[J] = r / per;
  }
  return MF_OK;
}

mf_status mf_strata_plan(uint64_t seed, int32_t a, int32_t world, int32_t rank, int64_t n,
                         int32_t t, int32_t j, int32_t* holders, int64_t* blocks,
                         int32_t* nblocks, int64_t* xfers, int32_t* nxfers) {
  if (!holders || !blocks || !nblocks || !xfers || !nxfers || rank < 0 || rank >= world || n < a)
    return MF_E_INVAL;
  std::vector<int32_t> next((size_t)std::max(a, 1));
  mf_status s = mf_strata_holders(seed, a, world, t, j, next.data());
  if (s != MF_OK) return s;
  const std::vector<int64_t> pi = host_perm(make_stream(seed, kTagStrata, (uint64_t)t, 0), a);
  // A: rank g owns row segments [g a/G, (g+1) a/G); in sub-epoch j row segment r trains
  // block (r, (r + pi_t[j]) mod a)
  const int per = a / world;
  *nblocks = 0;
  for (int r = rank * per; r < (rank + 1) * per; ++r)
    blocks[(*nblocks)++] = (int64_t)r * a + (r + pi[(size_t)j]) % a;
  // a segment moves iff its valid copy is on one rank (>= 0) that is not the next holder;
  // segment J = relabelled Q rows [ceil(J n / a), ceil((J+1) n / a))
  *nxfers = 0;
  for (int J = 0; J < a; ++J) {
    if (holders[J] >= 0 && holders[J] != next[(size_t)J]) {
      int64_t* x = xfers + 5 * (*nxfers)++;
      x[0] = J;
      x[1] = holders[J];
      x[2] = next[(size_t)J];
      x[3] = cdiv64((int64_t)J * n, a);
      x[4] = cdiv64((int64_t)(J + 1) * n, a);
    }
    holders[J] = next[(size_t)J];
  }
  return MF_OK;
}

mf_status mf_comm_selftest(const void* comm_id, int32_t world, int32_t rank, int32_t device,
                           int32_t transport, char* msg, int32_t msg_len) {
  std::string text;
  auto done = [&](mf_status s, const std::string& t) {
    if (msg && msg_len > 0) std::snprintf(msg, (size_t)msg_len, "%s", t.c_str());
    return s;
  };
  if (!comm_id || world < 1 || rank < 0 || rank >= world || transport < 0 || transport > 1)
    return done(MF_E_INVAL, "bad arguments");
  if (cudaSetDevice(device) != cudaSuccess) return done(MF_E_CUDA, "cudaSetDevice failed");
  cudaStream_t st = nullptr;
  if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess)
    return done(MF_E_CUDA, "cudaStreamCreate failed");
  uint8_t id[128];
  std::memcpy(id, comm_id, 128);
  std::string why;
  mf::Comm* cm = transport == 1 ? mf::Comm::create_loopback(id, world, rank, st, &why)
                                : mf::Comm::create(id, world, rank, st, &why);
  if (!cm) {
    cudaStreamDestroy(st);
    return done(MF_E_NCCL, "communicator: " + why);
  }
  const size_t seg = 4096, rowb = 16;
  const int64_t rows = 3 * (int64_t)world + 1;
  auto pat = [](int r) { return (unsigned char)(r * 13 + 1); };
  double* d = nullptr;
  unsigned char *buf = nullptr, *bc = nullptr, *rw = nullptr;
  mf_status s = MF_OK;
  bool ok = cudaMalloc(&d, 4 * sizeof(double)) == cudaSuccess &&
            cudaMalloc(&buf, seg * (size_t)world) == cudaSuccess &&
            cudaMalloc(&bc, seg) == cudaSuccess &&
            cudaMalloc(&rw, rowb * (size_t)rows) == cudaSuccess;
  std::vector<double> hd(4);
  for (int i = 0; i < 4; ++i) hd[(size_t)i] = (double)(rank + 1) * (i + 1);
  ok = ok && cudaMemcpyAsync(d, hd.data(), 4 * sizeof(double), cudaMemcpyHostToDevice, st) == cudaSuccess;
  ok = ok && cudaMemsetAsync(bc, pat(rank), seg, st) == cudaSuccess;
  ok = ok && cudaMemsetAsync(buf, 0xEE, seg * (size_t)world, st) == cudaSuccess;
  ok = ok && cudaMemsetAsync(buf + seg * (size_t)rank, pat(rank), seg, st) == cudaSuccess;
  ok = ok && cudaMemsetAsync(rw, 0, rowb * (size_t)rows, st) == cudaSuccess;
  const int64_t lo = cdiv64((int64_t)rank * rows, world), hi = cdiv64((int64_t)(rank + 1) * rows, world);
  if (hi > lo) ok = ok && cudaMemsetAsync(rw + lo * rowb, pat(rank), (size_t)(hi - lo) * rowb, st) == cudaSuccess;
  if (!ok) s = MF_E_CUDA, text = "device buffers";
  std::vector<mf::Xfer> xs;
  for (int r = 0; r < world; ++r) xs.push_back(mf::Xfer{buf + seg * (size_t)r, seg, r, (r + 1) % world});
  if (s == MF_OK && !cm->allreduce_sum(d, 4, &why)) s = MF_E_NCCL, text = "all-reduce: " + why;
  if (s == MF_OK && !cm->broadcast(bc, seg, world - 1, &why)) s = MF_E_NCCL, text = "broadcast: " + why;
  if (s == MF_OK && !cm->exchange(xs, rank, &why)) s = MF_E_NCCL, text = "send/recv: " + why;
  if (s == MF_OK && !cm->gather_rows(rw, rows, world, world, rowb, &why)) s = MF_E_NCCL, text = "gather: " + why;
  std::vector<unsigned char> hb(seg * (size_t)world), hc(seg), hr(rowb * (size_t)rows);
  if (s == MF_OK) {
    ok = cudaMemcpyAsync(hd.data(), d, 4 * sizeof(double), cudaMemcpyDeviceToHost, st) == cudaSuccess &&
         cudaMemcpyAsync(hb.data(), buf, hb.size(), cudaMemcpyDeviceToHost, st) == cudaSuccess &&
         cudaMemcpyAsync(hc.data(), bc, seg, cudaMemcpyDeviceToHost, st) == cudaSuccess &&
         cudaMemcpyAsync(hr.data(), rw, hr.size(), cudaMemcpyDeviceToHost, st) == cudaSuccess &&
         cudaStreamSynchronize(st) == cudaSuccess;
    if (!ok) s = MF_E_CUDA, text = "read-back";
  }
  if (s == MF_OK) {
    const double tri = (double)world * (world + 1) / 2.0;
    for (int i = 0; i < 4 && s == MF_OK; ++i)
      if (hd[(size_t)i] != tri * (i + 1)) s = MF_E_RANGE, text = "all-reduce value";
    for (size_t x = 0; x < seg && s == MF_OK; ++x)
      if (hc[x] != pat(world - 1)) s = MF_E_RANGE, text = "broadcast value";
    const int from = (rank + world - 1) % world;
    for (int r = 0; r < world && s == MF_OK; ++r) {
      const unsigned char want = (r == rank || r == from) ? pat(r) : 0xEE;
      for (size_t x = 0; x < seg; ++x)
        if (hb[seg * (size_t)r + x] != want) {
          s = MF_E_RANGE, text = "send/recv value";
          break;
        }
    }
    for (int r = 0; r < world && s == MF_OK; ++r) {
      const int64_t a0 = cdiv64((int64_t)r * rows, world), a1 = cdiv64((int64_t)(r + 1) * rows, world);
      for (int64_t x = a0 * (int64_t)rowb; x < a1 * (int64_t)rowb; ++x)
        if (hr[(size_t)x] != pat(r)) {
          s = MF_E_RANGE, text = "gather value";
          break;
        }
    }
  }
  if (s == MF_OK) {
    char line[160];
    std::snprintf(line, sizeof(line), "ok: %s, rank %d of %d: all-reduce, broadcast, %d-segment send/recv, "
                  "%lld-row gather checked", transport ? "loopback" : "NCCL", rank, world, world,
                  (long long)rows);
    text = line;
  }
  mf::Comm::destroy(cm);
  for (void* x : {(void*)d, (void*)buf, (void*)bc, (void*)rw})
    if (x) cudaFree(x);
  cudaStreamDestroy(st);
  cudaGetLastError();
  return done(s, text);
}

mf_status mf_create(const mf_params* p, mf_ctx** out) {
  if (!out) return MF_E_INVAL;
  *out = nullptr;
  if (!p || p->struct_size != sizeof(mf_params)) return MF_E_INVAL;
  if (p->m <= 0 || p->n <= 0 || p->m >= INT32_MAX || p->n >= INT32_MAX) return MF_E_INVAL;
  if (!(p->k == 16 || p->k == 32 || p->k == 64 || p->k == 128 || p->k == 256))
    return MF_E_UNSUPPORTED;
  if (p->storage < 0 || p->storage > 2 || p->schedule < 0 || p->schedule > 2) return MF_E_INVAL;
  const bool libmf = p->schedule == MF_LIBMF;
  if (libmf && (p->world > 1 || p->staged)) return MF_E_UNSUPPORTED;
  if (!(p->alpha >= 0.f) || !(p->beta >= 0.f) || !(p->lambda_p >= 0.f) || !(p->lambda_q >= 0.f))
    return MF_E_INVAL;
  if (!(p->rating_scale > 0.f) || !(p->init_scale > 0.f)) return MF_E_INVAL;
  if (p->lane_bytes != 0 && p->lane_bytes != 8 && p->lane_bytes != 16 && p->lane_bytes != 32 &&
      p->lane_bytes != 64)
    return MF_E_INVAL;
  if (p->prefetch < 0 || p->prefetch > 2) return MF_E_INVAL;
  if (p->wf_kernel < 0 || p->wf_kernel > 2 || p->launch_blocks < 0) return MF_E_INVAL;
  if (p->transport < 0 || p->transport > 1) return MF_E_INVAL;
  if (p->staged < 0 || p->staged > 2) return MF_E_INVAL;
  if (p->staged == 2 && (p->world > 1 || p->lr_rule != 0 || p->schedule == MF_LIBMF))
    return MF_E_UNSUPPORTED;                     // P out of core: one GPU, Eq. 9 step
  if (p->lr_rule < 0 || p->lr_rule > 1 || !(p->ada_eps >= 0.f)) return MF_E_INVAL;
  if (p->exact_order < 0 || p->exact_order > 1) return MF_E_INVAL;
  if (p->group_cols < 0 || p->group_cols > 1) return MF_E_INVAL;
  if (p->check_owners < 0 || p->check_owners > 1) return MF_E_INVAL;
  if (p->group_cols && (p->schedule != MF_HOGWILD || p->rating_stage || p->prefetch > 1))
    return MF_E_UNSUPPORTED;
  if (p->rating_stage < 0 || p->rating_stage > 2) return MF_E_INVAL;
  // the staged rating streams are instantiated for plain Eq. 9 updates in the fast form only;
  // the row ring (2) needs 16-B lane slices: k S <= 512 at the default 16-B lanes
  if (p->rating_stage && (p->exact_order || p->lr_rule == 1 || p->schedule != MF_HOGWILD))
    return MF_E_UNSUPPORTED;
  if (p->rating_stage == 2 && ((p->lane_bytes && p->lane_bytes != 16) || p->prefetch > 1 ||
                               (int64_t)p->k * (p->storage == MF_FP32 ? 4 : 2) > 512))
    return MF_E_UNSUPPORTED;
  if (p->rating_stage == 1 && ((p->batch_f > 0 ? p->batch_f : 256) % 64 != 0 ||
                               p->prefetch > 1 || (p->lane_bytes && p->lane_bytes != 16)))
    return MF_E_UNSUPPORTED;                      // TMA stream: f % 64 == 0, default geometry
  if (p->lr_rule == 1 && p->schedule == MF_LIBMF) return MF_E_UNSUPPORTED;
  const int world = p->world > 0 ? p->world : 1;
  if (p->rank < 0 || p->rank >= world) return MF_E_INVAL;
  if (p->grid_cols < 0 || p->grid_cols > 1) return MF_E_INVAL;
  if (p->q_cache < 0 || p->q_cache > 1) return MF_E_INVAL;
  const bool rows_only = p->grid_cols == 1;      // a x 1 row blocks (R27)
  // a x 1 with grid_a = 0: blocks whose P row segment is ~32 MiB, a fraction of the 126-MB L2
  // (profiles/r02_row_blocks.md)
  const int64_t seg_target = (int64_t)32 << 20;
  const int64_t p_bytes = p->m * (int64_t)p->k * (p->storage == MF_FP32 ? 4 : 2);
  const int a = p->grid_a > 0 ? p->grid_a
                : rows_only ? (int)std::max<int64_t>(1, std::min<int64_t>(std::min<int64_t>(256, p->m),
                                                                         cdiv64(p_bytes, seg_target)))
                : (libmf ? 64 : (world == 1 ? 1 : 8));
  if (rows_only && (world > 1 || p->schedule != MF_HOGWILD || p->lr_rule != 0))
    return MF_E_UNSUPPORTED;                     // one GPU, batch-Hogwild, Eq. 9
  if (a % world != 0 || a > p->m || (!rows_only && a > p->n)) return MF_E_INVAL;
  if (rows_only && a > 256) return MF_E_INVAL;
  if (!libmf && !rows_only && (a > 64 || a / world > kMaxSegs)) return MF_E_INVAL;
  if (libmf && a > 1024) return MF_E_INVAL;
  if (p->batch_f < 0 || p->workers < 0 || p->wf_cols < 0) return MF_E_INVAL;

  mf_ctx* c = new (std::nothrow) mf_ctx();
  if (!c) return MF_E_NOMEM;
  c->p = *p;
  c->dev = p->device;
  c->m = p->m;
  c->n = p->n;
  c->k = p->k;
  c->a = a;
  c->ac = rows_only ? 1 : a;
  c->G = world;
  c->rank = p->rank;
  c->f = p->batch_f > 0 ? p->batch_f : 256;
  c->wf = p->schedule == MF_WAVEFRONT;
  c->libmf = p->schedule == MF_LIBMF;
  c->staged = p->staged >= 1;
  c->pq = p->staged == 2;
  if (c->wf) {
    const int64_t rows_per_seg = p->m / a;
    // default s: 768 workers per launch (all co-resident in every ring geometry), shared by the
    // a / G blocks of a stratum that one launch runs together
    const int64_t cap = std::max<int64_t>(1, 768 / std::max(1, a / world));
    int64_t s = p->workers > 0 ? p->workers
                               : std::min<int64_t>(cap, std::max<int64_t>(1, rows_per_seg / 4));
    c->s = (int)s;
    c->c = p->wf_cols > 0 ? p->wf_cols : 2 * c->s;
    if (p->cyclic && c->c < c->s) { delete c; return MF_E_INVAL; }
    if ((int64_t)a * a * c->s * c->c >= ((int64_t)1 << 31)) { delete c; return MF_E_UNSUPPORTED; }
  }
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    delete c;
    return MF_E_UNSUPPORTED;
  }
  if (c->dev < 0 || c->dev >= ndev) { delete c; return MF_E_INVAL; }
  if (cudaSetDevice(c->dev) != cudaSuccess ||
      cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, c->dev) != cudaSuccess) {
    cudaGetLastError();
    delete c;
    return MF_E_CUDA;
  }
  if (p->stream) {
    c->st = (cudaStream_t)p->stream;
  } else {
    if (cudaStreamCreateWithFlags(&c->st, cudaStreamDefault) != cudaSuccess) {
      delete c;
      return MF_E_CUDA;
    }
    c->own_stream = true;
  }
  cudaEventCreate(&c->ev_e0);
  cudaEventCreate(&c->ev_e1);
  cudaEventCreate(&c->ev_s0);
  cudaEventCreate(&c->ev_s1);
  cudaEventCreate(&c->ev_c0);
  cudaEventCreate(&c->ev_c1);
  if (world > 1) {
    if (!p->nccl_id) { mf_destroy(c); return MF_E_INVAL; }
    std::memcpy(c->nccl_id, p->nccl_id, 128);
    std::string why;
    c->comm = p->transport == 1 ? mf::Comm::create_loopback(c->nccl_id, world, p->rank, c->st, &why)
                                : mf::Comm::create(c->nccl_id, world, p->rank, c->st, &why);
    if (!c->comm) {
      c->fail(MF_E_NCCL, "NCCL init failed: %s", why.c_str());
      mf_destroy(c);
      return MF_E_NCCL;
    }
  }
  if (c->alloc(&c->counter, 1) || c->alloc(&c->rm_partial, (size_t)c->num_sms * 4) ||
      c->alloc(&c->rm_out, 2) || c->alloc(&c->upd_dev, 1) || c->alloc(&c->chk_dev, 1)) {
    mf_destroy(c);
    return MF_E_NOMEM;
  }
  *out = c;
  return MF_OK;
}

// The out-of-core state a train load creates outside the allocator: pinned host copies of the
// ratings and P, the copy / write-back streams and their events.  Streams must be idle.
static void release_host_staging(mf_ctx* c) {
  for (void** h : {(void**)&c->h_slots, (void**)&c->h_u, (void**)&c->h_v16, (void**)&c->h_r,
                   (void**)&c->h_dup, (void**)&c->h_P}) {
    if (*h) cudaFreeHost(*h);
    *h = nullptr;
  }
  for (int i = 0; i < 2; ++i)
    for (cudaEvent_t* e : {&c->ev_pin[i], &c->ev_pcomp[i], &c->ev_pout[i], &c->ev_h2d[i], &c->ev_free[i]}) {
      if (*e) cudaEventDestroy(*e);
      *e = nullptr;
    }
  for (cudaStream_t* q : {&c->ds, &c->cs}) {
    if (*q) cudaStreamDestroy(*q);
    *q = nullptr;
  }
}

void mf_destroy(mf_ctx* c) {
  if (!c) return;
  cudaSetDevice(c->dev);
  // every stream that may still touch ctx memory drains before the stream-ordered frees: the
  // side schedule stream, the staging copy stream (an epoch ends by queueing the next
  // stratum's H2D into a staging buffer on cs, which nothing on st waits for) and st itself
  if (c->ss) cudaStreamSynchronize(c->ss);
  if (c->cs) cudaStreamSynchronize(c->cs);
  if (c->ds) cudaStreamSynchronize(c->ds);
  if (c->st) cudaStreamSynchronize(c->st);
  std::vector<std::pair<void*, size_t>> all = c->sizes;
  for (auto& x : all) {
    void* ptr = x.first;
    c->release(ptr);
  }
  if (c->st) cudaStreamSynchronize(c->st);
  for (auto e : c->ev) cudaEventDestroy(e);
  for (cudaEvent_t e : {c->ev_e0, c->ev_e1, c->ev_s0, c->ev_s1, c->ev_c0, c->ev_c1})
    if (e) cudaEventDestroy(e);
  if (c->comm) mf::Comm::destroy(c->comm);
  release_host_staging(c);
  for (cudaEvent_t e : {c->ev_ss_go, c->ev_ss_done})
    if (e) cudaEventDestroy(e);
  if (c->ss) cudaStreamDestroy(c->ss);
  if (c->own_stream && c->st) cudaStreamDestroy(c->st);
  cudaGetLastError();
  delete c;
}

// ---------------------------------------------------------------------------------------------
// load
// ---------------------------------------------------------------------------------------------
static mf_status stage_input(mf_ctx* c, int64_t nnz, const int32_t* u, const int32_t* v,
                             const float* r, int on_device, const int32_t** du,
                             const int32_t** dv, const float** dr, int32_t** own_u,
                             int32_t** own_v, float** own_r) {
  *own_u = nullptr; *own_v = nullptr; *own_r = nullptr;
  if (on_device) {
    *du = u; *dv = v; *dr = r;
    return MF_OK;
  }
  TRY(c->alloc(own_u, (size_t)nnz));
  TRY(c->alloc(own_v, (size_t)nnz));
  TRY(c->alloc(own_r, (size_t)nnz));
  CUDA_TRY(c, cudaMemcpyAsync(*own_u, u, nnz * 4, cudaMemcpyHostToDevice, c->st));
  CUDA_TRY(c, cudaMemcpyAsync(*own_v, v, nnz * 4, cudaMemcpyHostToDevice, c->st));
  CUDA_TRY(c, cudaMemcpyAsync(*own_r, r, nnz * 4, cudaMemcpyHostToDevice, c->st));
  *du = *own_u; *dv = *own_v; *dr = *own_r;
  return MF_OK;
}

static mf_status validate(mf_ctx* c, int64_t nnz, const int32_t* du, const int32_t* dv,
                          const float* dr) {
  int* flag = nullptr;
  TRY(c->alloc(&flag, 1));
  CUDA_TRY(c, cudaMemsetAsync(flag, 0, 4, c->st));
  if (nnz > 0) {
    k_validate<<<grid_for(nnz, c->num_sms), 256, 0, c->st>>>(du, dv, dr, nnz, c->m, c->n, flag);
    KERNEL_TRY(c);
  }
  int h = 0;
  CUDA_TRY(c, cudaMemcpyAsync(&h, flag, 4, cudaMemcpyDeviceToHost, c->st));
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  c->release(flag);
  if (h) return c->fail(MF_E_RANGE, "rating index out of range or non-finite rating");
  return MF_OK;
}

static mf_status relabel(mf_ctx* c, uint64_t tag, int64_t count, int32_t** rho) {
  uint64_t *k0 = nullptr, *k1 = nullptr;
  uint32_t *v0 = nullptr, *v1 = nullptr;
  TRY(c->alloc(&k0, (size_t)count));
  TRY(c->alloc(&k1, (size_t)count));
  TRY(c->alloc(&v0, (size_t)count));
  TRY(c->alloc(&v1, (size_t)count));
  TRY(c->alloc(rho, (size_t)count));
  k_iota_keys<<<grid_for(count, c->num_sms), 256, 0, c->st>>>(make_stream(c->p.seed, tag, 0, 0),
                                                              count, k0, v0);
  KERNEL_TRY(c);
  TRY(c->sort_pairs(k0, k1, v0, v1, count, 64));
  k_rank_of<<<grid_for(count, c->num_sms), 256, 0, c->st>>>(v1, count, *rho);
  KERNEL_TRY(c);
  c->release(k0); c->release(k1); c->release(v0); c->release(v1);
  return MF_OK;
}

template <typename T>
static void launch_init(mf_ctx* c, void* X, const int32_t* rho, int64_t rows, uint64_t S, float amp) {
  k_init<T><<<grid_for(rows * c->k, c->num_sms), 256, 0, c->st>>>((T*)X, rho, rows, c->k, S, amp);
}

template <typename T>
static void launch_init_rows(mf_ctx* c, void* X, const int32_t* inv, int64_t lo, int64_t rows,
                             uint64_t S, float amp) {
  k_init_rows<T><<<grid_for(rows * c->k, c->num_sms), 256, 0, c->st>>>((T*)X, inv, lo, rows, c->k,
                                                                         S, amp);
}

// staged == 2: P initialised segment by segment in a device slot and written to pinned host
// memory; the two device slots of one row segment each are all the HBM P ever takes.
static mf_status init_p_out_of_core(mf_ctx* c, float amp, uint64_t SP) {
  const size_t rowb = (size_t)c->k * c->ssize();
  c->pseg_max = 0;
  for (int r = 0; r < c->a; ++r)
    c->pseg_max = std::max(c->pseg_max, cdiv64((int64_t)(r + 1) * c->m, c->a) - cdiv64((int64_t)r * c->m, c->a));
  CUDA_TRY(c, cudaMallocHost(&c->h_P, (size_t)c->m * rowb));
  TRY(c->alloc(&c->Pslot[0], (size_t)c->pseg_max * rowb));
  TRY(c->alloc(&c->Pslot[1], (size_t)c->pseg_max * rowb));
  int32_t* inv = nullptr;
  TRY(c->alloc(&inv, (size_t)c->m));
  k_invert<<<grid_for(c->m, c->num_sms), 256, 0, c->st>>>(c->rho_r, c->m, inv);
  KERNEL_TRY(c);
  for (int r = 0; r < c->a; ++r) {
    const int64_t lo = cdiv64((int64_t)r * c->m, c->a), hi = cdiv64((int64_t)(r + 1) * c->m, c->a);
    switch (c->p.storage) {
      case MF_FP32: launch_init_rows<float>(c, c->Pslot[0], inv, lo, hi - lo, SP, amp); break;
      case MF_FP16: launch_init_rows<__half>(c, c->Pslot[0], inv, lo, hi - lo, SP, amp); break;
      default: launch_init_rows<__nv_bfloat16>(c, c->Pslot[0], inv, lo, hi - lo, SP, amp); break;
    }
    KERNEL_TRY(c);
    CUDA_TRY(c, cudaMemcpyAsync(c->h_P + (size_t)lo * rowb, c->Pslot[0], (size_t)(hi - lo) * rowb,
                                cudaMemcpyDeviceToHost, c->st));
    CUDA_TRY(c, cudaStreamSynchronize(c->st));
  }
  c->release(inv);
  return MF_OK;
}

static mf_status init_factors(mf_ctx* c) {
  const size_t es = (size_t)c->ssize();
  const float amp = (float)std::sqrt(1.0 / ((double)c->k * (double)c->p.init_scale));
  const uint64_t SP = make_stream(c->p.seed, kTagP, 0, 0), SQ = make_stream(c->p.seed, kTagQ, 0, 0);
  if (c->pq) {
    TRY(c->alloc((char**)&c->Q, (size_t)c->n * c->k * es));
    switch (c->p.storage) {
      case MF_FP32: launch_init<float>(c, c->Q, c->rho_c, c->n, SQ, amp); break;
      case MF_FP16: launch_init<__half>(c, c->Q, c->rho_c, c->n, SQ, amp); break;
      default: launch_init<__nv_bfloat16>(c, c->Q, c->rho_c, c->n, SQ, amp); break;
    }
    KERNEL_TRY(c);
    return init_p_out_of_core(c, amp, SP);
  }
  TRY(c->alloc((char**)&c->P, (size_t)c->m * c->k * es));
  TRY(c->alloc((char**)&c->Q, (size_t)c->n * c->k * es));
  switch (c->p.storage) {
    case MF_FP32: launch_init<float>(c, c->P, c->rho_r, c->m, SP, amp);
                  launch_init<float>(c, c->Q, c->rho_c, c->n, SQ, amp); break;
    case MF_FP16: launch_init<__half>(c, c->P, c->rho_r, c->m, SP, amp);
                  launch_init<__half>(c, c->Q, c->rho_c, c->n, SQ, amp); break;
    default: launch_init<__nv_bfloat16>(c, c->P, c->rho_r, c->m, SP, amp);
             launch_init<__nv_bfloat16>(c, c->Q, c->rho_c, c->n, SQ, amp); break;
  }
  KERNEL_TRY(c);
  return MF_OK;
}

// a x 1 row blocks (R27) with a > 1, Hogwild, resident: the epoch is one launch over the blocks'
// concatenated chunk orders (train_epoch_rows).  The 1 x 1 grid (ac == 1 as well) and the
// wavefront keep the per-stratum path.
static bool rows_one_launch(const mf_ctx* c) {
  return !c->wf && c->ac == 1 && c->a > 1 && !c->staged;
}

static mf_status alloc_schedule(mf_ctx* c) {
  const int64_t nb = (int64_t)c->a * c->ac;
  int64_t cap = 1;
  if (c->wf) cap = nb * c->s * (int64_t)c->c;
  else cap = c->ch_off.back();
  if (c->wf && c->p.cyclic) cap = std::max<int64_t>(cap, 2 * nb * c->c);
  cap = std::max<int64_t>(cap, 1);
  TRY(c->alloc(&c->sk0, (size_t)cap));
  TRY(c->alloc(&c->sk1, (size_t)cap));
  TRY(c->alloc(&c->sv0, (size_t)cap));
  TRY(c->alloc(&c->sv1, (size_t)cap));
  TRY(c->alloc(&c->sb, (size_t)cap));
  c->sched_cap = cap;
  if (c->wf) {
    TRY(c->alloc(&c->seq, (size_t)cap));
    TRY(c->alloc(&c->rank_arr, (size_t)cap));
    const size_t per_launch = (size_t)(c->a / c->G) * c->c;   // c per block of a stratum
    TRY(c->alloc(&c->tickets, per_launch));
    if (c->p.check_owners) {
      TRY(c->alloc(&c->owners, per_launch));
      TRY(c->alloc(&c->own_viol, 1));
      CUDA_TRY(c, cudaMemsetAsync(c->owners, 0xFF, per_launch * 4, c->st));   // all free (-1)
      CUDA_TRY(c, cudaMemsetAsync(c->own_viol, 0, 4, c->st));
    }
    if (c->p.cyclic) {
      TRY(c->alloc(&c->tau, (size_t)(nb * c->c)));
      TRY(c->alloc(&c->sigma, (size_t)(nb * c->c)));
    }
  } else {
    TRY(c->alloc(&c->chunk_order, (size_t)cap));
    TRY(c->alloc(&c->chunk_order_alt, (size_t)cap));
    if (rows_one_launch(c)) TRY(c->alloc(&c->chunk_seq, (size_t)cap));
  }
  return MF_OK;
}

// The packed staging format of this ctx (k_split_slots): bu = bits(m), bv = bits(n - 1).
static void set_pack_format(mf_ctx* c) {
  const int bu = bits_for((uint64_t)c->m), bv = bits_for((uint64_t)std::max<int64_t>(c->n - 1, 1));
  c->pk = PackFmt{bu, bv, bu + bv <= 40 ? 1 : 2};
  c->stg_packed = bu + bv <= 48;
}
static int64_t staged_bytes_per_rating(const mf_ctx* c) {
  return (c->stg_packed ? 8 + c->pk.hib : (int64_t)sizeof(Rating)) + (c->h_dup ? 2 : 0);
}

// Move the bucketed ratings (and the wavefront dup metadata) from HBM to pinned host memory
// (the resident preprocessing path; the chunked path writes them there directly).
static mf_status setup_staging(mf_ctx* c) {
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  const size_t ns = (size_t)std::max<int64_t>(c->nslots, 1);
  set_pack_format(c);
  if (c->stg_packed) {
    uint32_t* du = nullptr;
    uint8_t* dv = nullptr;
    float* dr = nullptr;
    const size_t hb = (size_t)c->pk.hib;
    TRY(c->alloc(&du, ns));
    TRY(c->alloc(&dv, ns * hb));
    TRY(c->alloc(&dr, ns));
    if (c->nslots > 0) {
      k_split_slots<<<grid_for(c->nslots, c->num_sms), 256, 0, c->st>>>(c->slots, c->nslots, c->pk, du, dv, dr);
      KERNEL_TRY(c);
    }
    CUDA_TRY(c, cudaMallocHost(&c->h_u, ns * 4));
    CUDA_TRY(c, cudaMallocHost(&c->h_v16, ns * hb));
    CUDA_TRY(c, cudaMallocHost(&c->h_r, ns * 4));
    CUDA_TRY(c, cudaMemcpyAsync(c->h_u, du, ns * 4, cudaMemcpyDeviceToHost, c->st));
    CUDA_TRY(c, cudaMemcpyAsync(c->h_v16, dv, ns * hb, cudaMemcpyDeviceToHost, c->st));
    CUDA_TRY(c, cudaMemcpyAsync(c->h_r, dr, ns * 4, cudaMemcpyDeviceToHost, c->st));
    CUDA_TRY(c, cudaStreamSynchronize(c->st));
    c->release(du);
    c->release(dv);
    c->release(dr);
  } else {
    CUDA_TRY(c, cudaMallocHost(&c->h_slots, ns * sizeof(Rating)));
    CUDA_TRY(c, cudaMemcpyAsync(c->h_slots, c->slots, ns * sizeof(Rating), cudaMemcpyDeviceToHost, c->st));
  }
  if (c->dup) {
    CUDA_TRY(c, cudaMallocHost(&c->h_dup, ns * sizeof(uint16_t)));
    CUDA_TRY(c, cudaMemcpyAsync(c->h_dup, c->dup, ns * sizeof(uint16_t), cudaMemcpyDeviceToHost, c->st));
  }
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  c->release(c->slots);
  c->release(c->dup);
  c->release(c->slot_pos);
  c->release(c->perm);
  return MF_OK;
}

// The two device staging buffers, sized for the largest stratum this rank can meet:
// sum over owned row segments r of max_J |block (r, J)|; the copy stream and its events.
static mf_status setup_staging_buffers(mf_ctx* c) {
  int64_t cap = 1;
  int64_t sum = 0;
  for (int r = c->lo_row_seg(); r < c->hi_row_seg(); ++r) {
    int64_t mx = 0;
    for (int J = 0; J < c->ac; ++J) {
      const int64_t b = (int64_t)r * c->ac + J;
      mx = std::max(mx, c->blk_off[(size_t)b + 1] - c->blk_off[(size_t)b]);
    }
    sum = c->ac == 1 ? std::max(sum, mx) : sum + mx;   // a x 1: a stratum is one block
  }
  cap = std::max<int64_t>(cap, sum);
  if (c->pq) {                         // one strata block at a time
    cap = 1;
    for (size_t b = 0; b + 1 < c->blk_off.size(); ++b) cap = std::max(cap, c->blk_off[b + 1] - c->blk_off[b]);
    CUDA_TRY(c, cudaStreamCreateWithFlags(&c->ds, cudaStreamNonBlocking));
    for (int i = 0; i < 2; ++i) {
      CUDA_TRY(c, cudaEventCreateWithFlags(&c->ev_pin[i], cudaEventDisableTiming));
      CUDA_TRY(c, cudaEventCreateWithFlags(&c->ev_pcomp[i], cudaEventDisableTiming));
      CUDA_TRY(c, cudaEventCreateWithFlags(&c->ev_pout[i], cudaEventDisableTiming));
      CUDA_TRY(c, cudaEventRecord(c->ev_pout[i], c->ds));
    }
  }
  c->stg_cap = cap;
  for (int i = 0; i < 2; ++i) {
    TRY(c->alloc(&c->stg[i], (size_t)cap));
    if (c->h_dup) TRY(c->alloc(&c->stg_dup[i], (size_t)cap));
    if (c->stg_packed) {
      TRY(c->alloc(&c->stg_u[i], (size_t)cap));
      TRY(c->alloc(&c->stg_v16[i], (size_t)cap * c->pk.hib));
      TRY(c->alloc(&c->stg_r[i], (size_t)cap));
    }
    CUDA_TRY(c, cudaEventCreateWithFlags(&c->ev_h2d[i], cudaEventDisableTiming));
    CUDA_TRY(c, cudaEventCreateWithFlags(&c->ev_free[i], cudaEventDisableTiming));
    CUDA_TRY(c, cudaEventRecord(c->ev_free[i], c->st));
  }
  CUDA_TRY(c, cudaStreamCreateWithFlags(&c->cs, cudaStreamNonBlocking));
  return MF_OK;
}

// The blocks this rank trains in sub-epoch j of epoch t (A: strata order; a x 1 row blocks,
// R27: block pi_t[j] alone).
static std::vector<int64_t> stratum_blocks(const mf_ctx* c, int32_t t, int32_t j) {
  const std::vector<int64_t> pi = host_perm(make_stream(c->p.seed, kTagStrata, (uint64_t)t, 0), c->a);
  if (c->ac == 1) return std::vector<int64_t>(1, pi[(size_t)j]);
  std::vector<int64_t> out;
  for (int r = c->lo_row_seg(); r < c->hi_row_seg(); ++r)
    out.push_back((int64_t)r * c->a + (r + pi[(size_t)j]) % c->a);
  return out;
}

// Copy the blocks of (t, j) from pinned host memory into staging buffer `buf`, packed, on the
// copy stream, after the compute stream released the buffer.
static mf_status stage(mf_ctx* c, int32_t t, int32_t j, int buf) {
  CUDA_TRY(c, cudaStreamWaitEvent(c->cs, c->ev_free[buf], 0));
  c->stg_shift[buf].clear();
  int64_t off = 0;
  for (int64_t b : stratum_blocks(c, t, j)) {
    const int64_t lo = c->blk_off[(size_t)b], len = c->blk_off[(size_t)b + 1] - lo;
    c->stg_shift[buf].push_back({b, off - lo});
    if (len == 0) continue;
    if (c->stg_packed) {
      CUDA_TRY(c, cudaMemcpyAsync(c->stg_u[buf] + off, c->h_u + lo, (size_t)len * 4,
                                  cudaMemcpyHostToDevice, c->cs));
      CUDA_TRY(c, cudaMemcpyAsync(c->stg_v16[buf] + off * c->pk.hib, c->h_v16 + lo * c->pk.hib,
                                  (size_t)len * c->pk.hib, cudaMemcpyHostToDevice, c->cs));
      CUDA_TRY(c, cudaMemcpyAsync(c->stg_r[buf] + off, c->h_r + lo, (size_t)len * 4,
                                  cudaMemcpyHostToDevice, c->cs));
    } else {
      CUDA_TRY(c, cudaMemcpyAsync(c->stg[buf] + off, c->h_slots + lo, (size_t)len * sizeof(Rating),
                                  cudaMemcpyHostToDevice, c->cs));
    }
    if (c->h_dup)
      CUDA_TRY(c, cudaMemcpyAsync(c->stg_dup[buf] + off, c->h_dup + lo, (size_t)len * 2,
                                  cudaMemcpyHostToDevice, c->cs));
    c->h2d_bytes += len * staged_bytes_per_rating(c);
    off += len;
  }
  c->stg_len[buf] = off;
  CUDA_TRY(c, cudaEventRecord(c->ev_h2d[buf], c->cs));
  c->staged_t = t;
  c->staged_j = j;
  return MF_OK;
}

// group_cols (R24): order every Hogwild batch of f slots in [lo, lo + len) (a padded strata
// block, chunk aligned) by column, in pieces of at most ~2^26 slots (whole chunks).
static mf_status group_batches(mf_ctx* c, Rating* slots, uint32_t* slot_pos, int64_t len) {
  if (!c->p.group_cols || len == 0) return MF_OK;
  const int64_t piece = std::max<int64_t>(c->f, (((int64_t)1 << 26) / c->f) * c->f);
  const int64_t cap = std::min(piece, len);
  uint64_t *k0 = nullptr, *k1 = nullptr;
  uint32_t *v0 = nullptr, *v1 = nullptr, *p1 = nullptr;
  Rating* tmp = nullptr;
  TRY(c->alloc(&k0, (size_t)cap)); TRY(c->alloc(&k1, (size_t)cap));
  TRY(c->alloc(&v0, (size_t)cap)); TRY(c->alloc(&v1, (size_t)cap));
  TRY(c->alloc(&tmp, (size_t)cap));
  if (slot_pos) TRY(c->alloc(&p1, (size_t)cap));
  for (int64_t lo = 0; lo < len; lo += piece) {
    const int64_t n = std::min(piece, len - lo);
    const int g = grid_for(n, c->num_sms);
    k_group_keys<<<g, 256, 0, c->st>>>(slots + lo, n, c->f, k0, v0);
    KERNEL_TRY(c);
    TRY(c->sort_pairs(k0, k1, v0, v1, n, 32 + bits_for((uint64_t)cdiv64(n, c->f))));
    k_permute_slots<<<g, 256, 0, c->st>>>(v1, n, slots + lo, tmp, slot_pos ? slot_pos + lo : nullptr, p1);
    KERNEL_TRY(c);
    CUDA_TRY(c, cudaMemcpyAsync(slots + lo, tmp, (size_t)n * sizeof(Rating), cudaMemcpyDeviceToDevice, c->st));
    if (slot_pos)
      CUDA_TRY(c, cudaMemcpyAsync(slot_pos + lo, p1, (size_t)n * 4, cudaMemcpyDeviceToDevice, c->st));
  }
  c->release(k0); c->release(k1); c->release(v0); c->release(v1); c->release(tmp); c->release(p1);
  return MF_OK;
}

// staged == 2: one strata block's ratings (and duplicate distances) into staging buffer buf,
// on the copy stream (the caller orders it after the buffer's previous use).
static mf_status stage_block(mf_ctx* c, int64_t b, int buf) {
  const int64_t lo = c->blk_off[(size_t)b], len = c->blk_off[(size_t)b + 1] - lo;
  c->stg_shift[buf].assign(1, {b, -lo});
  c->stg_len[buf] = len;
  if (len == 0) return MF_OK;
  if (c->stg_packed) {
    CUDA_TRY(c, cudaMemcpyAsync(c->stg_u[buf], c->h_u + lo, (size_t)len * 4, cudaMemcpyHostToDevice, c->cs));
    CUDA_TRY(c, cudaMemcpyAsync(c->stg_v16[buf], c->h_v16 + lo * c->pk.hib, (size_t)len * c->pk.hib,
                                cudaMemcpyHostToDevice, c->cs));
    CUDA_TRY(c, cudaMemcpyAsync(c->stg_r[buf], c->h_r + lo, (size_t)len * 4, cudaMemcpyHostToDevice, c->cs));
  } else {
    CUDA_TRY(c, cudaMemcpyAsync(c->stg[buf], c->h_slots + lo, (size_t)len * sizeof(Rating),
                                cudaMemcpyHostToDevice, c->cs));
  }
  if (c->h_dup)
    CUDA_TRY(c, cudaMemcpyAsync(c->stg_dup[buf], c->h_dup + lo, (size_t)len * 2, cudaMemcpyHostToDevice, c->cs));
  c->h2d_bytes += len * staged_bytes_per_rating(c);
  return MF_OK;
}

static mf_status load_train(mf_ctx* c, int64_t N, const int32_t* u, const int32_t* v,
                            const float* r, int on_device) {
  if (N >= (int64_t)UINT32_MAX) return c->fail(MF_E_UNSUPPORTED, "N >= 2^32 not supported");
  const int32_t *du, *dv;
  const float* dr;
  int32_t *ou, *ov;
  float* orr;
  TRY(stage_input(c, N, u, v, r, on_device, &du, &dv, &dr, &ou, &ov, &orr));
  {
    Nvtx rv("validate");
    TRY(validate(c, N, du, dv, dr));
  }

  // relabel (A: S_ROW, S_COL) first: a rank only needs the ratings of the row segments it owns
  TRY(relabel(c, kTagRow, c->m, &c->rho_r));
  TRY(relabel(c, kTagCol, c->n, &c->rho_c));
  uint32_t* own = nullptr;                  // caller indices of this rank's ratings (world > 1)
  if (c->G > 1 && N > 0) {
    char* flag = nullptr;
    int64_t* nsel = nullptr;
    TRY(c->alloc(&flag, (size_t)N));
    TRY(c->alloc(&own, (size_t)N));
    TRY(c->alloc(&nsel, 1));
    k_own_caller<<<grid_for(N, c->num_sms), 256, 0, c->st>>>(du, N, c->rho_r, c->m, c->a,
                                                             c->lo_row_seg(), c->hi_row_seg(), flag);
    KERNEL_TRY(c);
    cub::CountingInputIterator<uint32_t> iota(0);
    size_t bytes = 0;
    CUDA_TRY(c, cub::DeviceSelect::Flagged(nullptr, bytes, iota, flag, own, nsel, N, c->st));
    TRY(c->need_tmp(bytes));
    CUDA_TRY(c, cub::DeviceSelect::Flagged(c->tmp, bytes, iota, flag, own, nsel, N, c->st));
    int64_t h = 0;
    CUDA_TRY(c, cudaMemcpyAsync(&h, nsel, 8, cudaMemcpyDeviceToHost, c->st));
    CUDA_TRY(c, cudaStreamSynchronize(c->st));
    c->release(flag);
    c->release(nsel);
    N = h;
  }
  c->N = N;

  // Alg. 1 l.2 random_shuffle: storage order = perm(S_SHUF, N) over caller indices.
  // A rank sorts only its own ratings by the same keys: their relative order is the global one.
  {
    Nvtx rs("shuffle (Alg. 1 l.2)");
    uint64_t *k0 = nullptr, *k1 = nullptr;
    uint32_t* v0 = nullptr;
    TRY(c->alloc(&k0, (size_t)N));
    TRY(c->alloc(&k1, (size_t)N));
    TRY(c->alloc(&v0, (size_t)N));
    TRY(c->alloc(&c->perm, (size_t)N));
    if (N > 0) {
      k_keys_of<<<grid_for(N, c->num_sms), 256, 0, c->st>>>(make_stream(c->p.seed, kTagShuf, 0, 0),
                                                           own, N, k0, v0);
      KERNEL_TRY(c);
      TRY(c->sort_pairs(k0, k1, v0, c->perm, N, 64));
    }
    c->release(k0); c->release(k1); c->release(v0);
    c->release(own);
  }

  // storage-order samples (relabelled, scaled) and their buckets
  Grid Gd{c->m, c->n, c->a, c->s, c->c, c->wf, c->ac};
  const int64_t nb = (int64_t)c->a * c->ac;
  const int64_t nbuckets = c->wf ? nb * c->s * (int64_t)c->c : nb;
  Rating* stor = nullptr;
  uint32_t *bk0 = nullptr, *bk1 = nullptr, *pos0 = nullptr, *pos1 = nullptr;
  TRY(c->alloc(&stor, (size_t)N));
  TRY(c->alloc(&bk0, (size_t)N));
  TRY(c->alloc(&bk1, (size_t)N));
  TRY(c->alloc(&pos0, (size_t)N));
  TRY(c->alloc(&pos1, (size_t)N));
  if (N > 0) {
    k_build_storage<<<grid_for(N, c->num_sms), 256, 0, c->st>>>(
        c->perm, N, du, dv, dr, c->rho_r, c->rho_c, (double)c->p.rating_scale, Gd, stor, bk0, pos0);
    KERNEL_TRY(c);
  }
  c->release(ou); c->release(ov); c->release(orr);
  const bool keep_maps = N <= ((int64_t)1 << 30);   // per-sample index maps only feed exports
  if (!keep_maps) c->release(c->perm);

  // bucket counts -> offsets
  unsigned int* cnt = nullptr;
  TRY(c->alloc(&cnt, (size_t)nbuckets));
  CUDA_TRY(c, cudaMemsetAsync(cnt, 0, nbuckets * 4, c->st));
  if (N > 0) {
    if (nbuckets <= kSmemBuckets)
      k_histogram_smem<<<grid_for(N, c->num_sms), 256, 0, c->st>>>(bk0, N, (int)nbuckets, cnt);
    else
      k_histogram<<<grid_for(N, c->num_sms), 256, 0, c->st>>>(bk0, N, cnt);
    KERNEL_TRY(c);
  }
  // stable sort of storage positions by bucket (radix sort is stable; storage order kept, R12)
  const uint32_t* keys_sorted = nullptr;
  const uint32_t* pos_sorted = pos0;
  if (nbuckets > 1 && N > 0) {
    TRY(c->sort_pairs(bk0, bk1, pos0, pos1, N, bits_for((uint64_t)(nbuckets - 1))));
    keys_sorted = bk1;
    pos_sorted = pos1;
  }
  int64_t *src_off = nullptr, *dst_off = nullptr;
  TRY(c->alloc(&src_off, (size_t)nbuckets + 1));
  if (c->wf) {
    // sub-block offsets: exclusive scan of the counts (int64)
    std::vector<unsigned int> hc((size_t)nbuckets);
    CUDA_TRY(c, cudaMemcpyAsync(hc.data(), cnt, nbuckets * 4, cudaMemcpyDeviceToHost, c->st));
    CUDA_TRY(c, cudaStreamSynchronize(c->st));
    std::vector<int64_t> off((size_t)nbuckets + 1, 0);
    for (int64_t x = 0; x < nbuckets; ++x) off[(size_t)x + 1] = off[(size_t)x] + hc[(size_t)x];
    CUDA_TRY(c, cudaMemcpyAsync(src_off, off.data(), (nbuckets + 1) * 8, cudaMemcpyHostToDevice, c->st));
    c->blk_off.assign((size_t)nb + 1, 0);
    c->blk_len.assign((size_t)nb, 0);
    for (int64_t b = 0; b < nb; ++b) {
      c->blk_off[(size_t)b + 1] = off[(size_t)((b + 1) * c->s * c->c)];
      c->blk_len[(size_t)b] = c->blk_off[(size_t)b + 1] - c->blk_off[(size_t)b];
    }
    c->nslots = N;
    c->sub_off = src_off;
    dst_off = src_off;
    src_off = nullptr;
    CUDA_TRY(c, cudaStreamSynchronize(c->st));  // host vector `off` goes out of scope
  } else {
    // Hogwild: pad every block to a multiple of f (sentinel slots) so chunk q of block b is
    // slots [blk_off[b] + q f, + f) (A: "Padding").
    std::vector<unsigned int> hc((size_t)nb);
    CUDA_TRY(c, cudaMemcpyAsync(hc.data(), cnt, nb * 4, cudaMemcpyDeviceToHost, c->st));
    CUDA_TRY(c, cudaStreamSynchronize(c->st));
    std::vector<int64_t> so((size_t)nb + 1, 0);
    c->blk_off.assign((size_t)nb + 1, 0);
    c->blk_len.assign((size_t)nb, 0);
    c->ch_off.assign((size_t)nb + 1, 0);
    for (int64_t b = 0; b < nb; ++b) {
      c->blk_len[(size_t)b] = hc[(size_t)b];
      so[(size_t)b + 1] = so[(size_t)b] + hc[(size_t)b];
      const int64_t nch = cdiv64(hc[(size_t)b], c->f);
      c->ch_off[(size_t)b + 1] = c->ch_off[(size_t)b] + nch;
      c->blk_off[(size_t)b + 1] = c->blk_off[(size_t)b] + nch * c->f;
    }
    c->nslots = c->blk_off.back();
    TRY(c->alloc(&dst_off, (size_t)nb + 1));
    CUDA_TRY(c, cudaMemcpyAsync(src_off, so.data(), (nb + 1) * 8, cudaMemcpyHostToDevice, c->st));
    CUDA_TRY(c, cudaMemcpyAsync(dst_off, c->blk_off.data(), (nb + 1) * 8, cudaMemcpyHostToDevice, c->st));
    TRY(c->alloc(&c->d_choff, (size_t)nb + 1));
    CUDA_TRY(c, cudaMemcpyAsync(c->d_choff, c->ch_off.data(), (nb + 1) * 8, cudaMemcpyHostToDevice, c->st));
    if (c->libmf) {
      TRY(c->alloc(&c->d_blk_off, (size_t)nb + 1));
      TRY(c->alloc(&c->d_blk_len, (size_t)nb));
      TRY(c->alloc(&c->lm_lock, 1));
      TRY(c->alloc(&c->lm_rem, 1));
      TRY(c->alloc(&c->lm_row, (size_t)c->a));
      TRY(c->alloc(&c->lm_col, (size_t)c->a));
      TRY(c->alloc(&c->lm_done, (size_t)nb));
      CUDA_TRY(c, cudaMemcpyAsync(c->d_blk_off, c->blk_off.data(), (nb + 1) * 8, cudaMemcpyHostToDevice, c->st));
      CUDA_TRY(c, cudaMemcpyAsync(c->d_blk_len, c->blk_len.data(), nb * 8, cudaMemcpyHostToDevice, c->st));
    }
    CUDA_TRY(c, cudaStreamSynchronize(c->st));  // host vectors used by async copies
  }
  // free the bucket sort's inputs before the slot array (peak HBM at Hugewiki scale)
  if (keys_sorted) {
    c->release(bk0);
    c->release(pos0);
  } else {
    c->release(bk0);
    c->release(bk1);
    c->release(pos1);
  }
  TRY(c->alloc(&c->slots, (size_t)std::max<int64_t>(c->nslots, 1)));
  if (keep_maps) TRY(c->alloc(&c->slot_pos, (size_t)std::max<int64_t>(c->nslots, 1)));
  if (c->nslots > N) {
    CUDA_TRY(c, cudaMemsetAsync(c->slots, 0xFF, c->nslots * sizeof(Rating), c->st));  // u=v=-1
    if (c->slot_pos) CUDA_TRY(c, cudaMemsetAsync(c->slot_pos, 0xFF, c->nslots * 4, c->st));
  }
  if (N > 0) {
    k_place<<<grid_for(N, c->num_sms), 256, 0, c->st>>>(
        keys_sorted, pos_sorted, N, c->wf ? c->sub_off : src_off, c->wf ? c->sub_off : dst_off,
        stor, c->slots, c->slot_pos);
    KERNEL_TRY(c);
  }
  if (!c->wf) { c->release(src_off); c->release(dst_off); }
  c->release(cnt); c->release(stor); c->release(bk0); c->release(bk1);
  c->release(pos0); c->release(pos1);
  if (!c->wf && !c->libmf)
    for (int64_t b = 0; b < nb; ++b)
      TRY(group_batches(c, c->slots + c->blk_off[(size_t)b],
                        c->slot_pos ? c->slot_pos + c->blk_off[(size_t)b] : nullptr,
                        c->blk_off[(size_t)b + 1] - c->blk_off[(size_t)b]));

  if (c->wf && c->p.wf_kernel != 2) {
    TRY(c->alloc(&c->dup, (size_t)std::max<int64_t>(c->nslots, 1)));
    if (N > 0) {
      k_dupdist<<<grid_for(N, c->num_sms), 256, 0, c->st>>>(c->slots, N, Gd,
                                                          ring_window(c->k, c->p.storage, c->p.lane_bytes), c->dup);
      KERNEL_TRY(c);
    }
  }
  {
    Nvtx ri("init P, Q (Alg. 1 l.3)");
    TRY(init_factors(c));
  }
  if (c->p.lr_rule == 1) {
    TRY(c->alloc(&c->GP, (size_t)(c->m * c->k)));
    TRY(c->alloc(&c->GQ, (size_t)(c->n * c->k)));
    CUDA_TRY(c, cudaMemsetAsync(c->GP, 0, (size_t)(c->m * c->k) * 4, c->st));
    CUDA_TRY(c, cudaMemsetAsync(c->GQ, 0, (size_t)(c->n * c->k) * 4, c->st));
  }
  TRY(alloc_schedule(c));
  c->n_units = c->libmf ? nb : (c->wf ? nbuckets : c->ch_off.back());
  TRY(c->alloc(&c->visits, (size_t)std::max<int64_t>(c->n_units, 1)));
  CUDA_TRY(c, cudaMemsetAsync(c->visits, 0, (size_t)std::max<int64_t>(c->n_units, 1) * 4, c->st));
  c->epochs_run = 0;
  if (c->staged) {
    TRY(setup_staging(c));
    TRY(setup_staging_buffers(c));
  }
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  c->train_loaded = true;
  return MF_OK;
}


// ---------------------------------------------------------------------------------------------
// Out-of-core load (params.staged with a HOST rating set; section 6, "partition the
// data sets and stage the partitions to GPUs in batches"): the caller's COO never resides in
// HBM as a whole.  Device memory holds one chunk of stage_chunk samples (pass 1) or one strata
// block (pass 2) at a time, so a set larger than the device budget loads.
//   pass 1, per chunk: H2D, validate, relabel, strata block + shuffle key key(S_SHUF, i) of
//     every sample (i = caller index, 64-bit), stable sort by block, D2H appended to per-block
//     host runs (rank-foreign samples dropped);
//   pass 2, per block: H2D its runs, sort by key (= the storage order of Alg. 1 l.2 restricted
//     to the block, R12), wavefront: stable sort by sub-block, sub-block offsets and duplicate
//     distances; padded (Hogwild) and written to the pinned host slots the epochs stream from.
// The slots are those of the resident path, bit for bit (tests/test_gpu_parity.py), and
// N >= 2^32 is allowed (keys and block runs are 64-bit indexed; a block must stay < 2^32).
// ---------------------------------------------------------------------------------------------
static mf_status load_train_chunked(mf_ctx* c, int64_t N, const int32_t* u, const int32_t* v,
                                    const float* r) {
  const int64_t nb = (int64_t)c->a * c->ac;
  const int64_t C = std::max<int64_t>(
      1, std::min<int64_t>(std::max<int64_t>(N, 1),
                           c->p.stage_chunk > 0 ? c->p.stage_chunk : ((int64_t)1 << 26)));
  TRY(relabel(c, kTagRow, c->m, &c->rho_r));
  TRY(relabel(c, kTagCol, c->n, &c->rho_c));
  const uint64_t S = make_stream(c->p.seed, kTagShuf, 0, 0);
  std::vector<std::vector<uint64_t>> hk((size_t)nb);
  std::vector<std::vector<Rating>> hr((size_t)nb);
  std::vector<int64_t> bcount((size_t)nb, 0);
  {  // ---- pass 1
    Nvtx rp1("out-of-core pass 1 (chunks of %lld)", (long long)C);
    int32_t *cu = nullptr, *cv = nullptr;
    float* cr = nullptr;
    uint32_t *b0 = nullptr, *b1 = nullptr, *i0 = nullptr, *i1 = nullptr;
    uint64_t *k0 = nullptr, *k1 = nullptr;
    Rating *r0 = nullptr, *r1 = nullptr;
    int* bad = nullptr;
    unsigned* cnt = nullptr;
    TRY(c->alloc(&cu, (size_t)C)); TRY(c->alloc(&cv, (size_t)C)); TRY(c->alloc(&cr, (size_t)C));
    TRY(c->alloc(&b0, (size_t)C)); TRY(c->alloc(&b1, (size_t)C));
    TRY(c->alloc(&i0, (size_t)C)); TRY(c->alloc(&i1, (size_t)C));
    TRY(c->alloc(&k0, (size_t)C)); TRY(c->alloc(&k1, (size_t)C));
    TRY(c->alloc(&r0, (size_t)C)); TRY(c->alloc(&r1, (size_t)C));
    TRY(c->alloc(&bad, 1)); TRY(c->alloc(&cnt, (size_t)nb + 1));
    uint64_t* hkb = nullptr;
    Rating* hrb = nullptr;
    CUDA_TRY(c, cudaMallocHost(&hkb, (size_t)C * 8));
    CUDA_TRY(c, cudaMallocHost(&hrb, (size_t)C * sizeof(Rating)));
    std::vector<unsigned> hc((size_t)nb + 1);
    mf_status st = MF_OK;
    for (int64_t s0 = 0; s0 < N && st == MF_OK; s0 += C) {
      const int64_t n = std::min(C, N - s0);
      const int g = grid_for(n, c->num_sms);
      cudaError_t e = cudaMemcpyAsync(cu, u + s0, (size_t)n * 4, cudaMemcpyHostToDevice, c->st);
      if (e == cudaSuccess) e = cudaMemcpyAsync(cv, v + s0, (size_t)n * 4, cudaMemcpyHostToDevice, c->st);
      if (e == cudaSuccess) e = cudaMemcpyAsync(cr, r + s0, (size_t)n * 4, cudaMemcpyHostToDevice, c->st);
      if (e == cudaSuccess) e = cudaMemsetAsync(bad, 0, 4, c->st);
      if (e != cudaSuccess) { st = c->cuda_fail(e, "chunk H2D", __LINE__); break; }
      k_validate<<<g, 256, 0, c->st>>>(cu, cv, cr, n, c->m, c->n, bad);
      int hbad = 0;
      e = cudaMemcpyAsync(&hbad, bad, 4, cudaMemcpyDeviceToHost, c->st);
      if (e == cudaSuccess) e = cudaStreamSynchronize(c->st);
      if (e != cudaSuccess) { st = c->cuda_fail(e, "chunk validate", __LINE__); break; }
      if (hbad) { st = c->fail(MF_E_RANGE, "rating index out of range or non-finite rating"); break; }
      k_chunk_records<<<g, 256, 0, c->st>>>(cu, cv, cr, n, s0, S, c->rho_r, c->rho_c,
                                            (double)c->p.rating_scale, c->m, c->n, c->a, c->ac,
                                            c->lo_row_seg(), c->hi_row_seg(), b0, i0, k0, r0);
      if ((e = cudaGetLastError()) != cudaSuccess) { st = c->cuda_fail(e, "k_chunk_records", __LINE__); break; }
      if ((st = c->sort_pairs(b0, b1, i0, i1, n, bits_for((uint64_t)nb))) != MF_OK) break;
      k_gather_records<<<g, 256, 0, c->st>>>(i1, n, k0, r0, k1, r1);
      e = cudaMemsetAsync(cnt, 0, (nb + 1) * 4, c->st);
      if (nb + 1 <= kSmemBuckets)
        k_histogram_smem<<<g, 256, 0, c->st>>>(b1, n, (int)nb + 1, cnt);
      else
        k_histogram<<<g, 256, 0, c->st>>>(b1, n, cnt);
      if (e == cudaSuccess) e = cudaMemcpyAsync(hc.data(), cnt, (nb + 1) * 4, cudaMemcpyDeviceToHost, c->st);
      if (e == cudaSuccess) e = cudaMemcpyAsync(hkb, k1, (size_t)n * 8, cudaMemcpyDeviceToHost, c->st);
      if (e == cudaSuccess) e = cudaMemcpyAsync(hrb, r1, (size_t)n * sizeof(Rating), cudaMemcpyDeviceToHost, c->st);
      if (e == cudaSuccess) e = cudaStreamSynchronize(c->st);
      if (e != cudaSuccess) { st = c->cuda_fail(e, "chunk partition", __LINE__); break; }
      int64_t off = 0;                       // the chunk's block runs, in block order
      for (int64_t b = 0; b < nb; ++b) {
        const int64_t len = hc[(size_t)b];
        if (len) {
          hk[(size_t)b].insert(hk[(size_t)b].end(), hkb + off, hkb + off + len);
          hr[(size_t)b].insert(hr[(size_t)b].end(), hrb + off, hrb + off + len);
        }
        bcount[(size_t)b] += len;
        off += len;
      }
    }
    cudaFreeHost(hkb);
    cudaFreeHost(hrb);
    for (void* x : {(void*)cu, (void*)cv, (void*)cr, (void*)b0, (void*)b1, (void*)i0, (void*)i1,
                    (void*)k0, (void*)k1, (void*)r0, (void*)r1, (void*)bad, (void*)cnt}) {
      void* y = x;
      c->release(y);
    }
    if (st != MF_OK) return st;
  }
  // ---- block layout (A: padding of Hogwild blocks to a multiple of f)
  int64_t Nown = 0, maxlen = 1;
  c->blk_off.assign((size_t)nb + 1, 0);
  c->blk_len.assign((size_t)nb, 0);
  c->ch_off.assign((size_t)nb + 1, 0);
  for (int64_t b = 0; b < nb; ++b) {
    const int64_t len = bcount[(size_t)b];
    if (len >= ((int64_t)1 << 32)) return c->fail(MF_E_UNSUPPORTED, "a strata block holds >= 2^32 ratings");
    Nown += len;
    c->blk_len[(size_t)b] = len;
    const int64_t padded = c->wf ? len : cdiv64(len, c->f) * c->f;
    c->ch_off[(size_t)b + 1] = c->ch_off[(size_t)b] + (c->wf ? 0 : cdiv64(len, c->f));
    c->blk_off[(size_t)b + 1] = c->blk_off[(size_t)b] + padded;
    maxlen = std::max(maxlen, padded);
  }
  c->N = Nown;
  c->nslots = c->blk_off.back();
  const size_t ns = (size_t)std::max<int64_t>(c->nslots, 1);
  set_pack_format(c);
  if (c->stg_packed) {
    CUDA_TRY(c, cudaMallocHost(&c->h_u, ns * 4));
    CUDA_TRY(c, cudaMallocHost(&c->h_v16, ns * (size_t)c->pk.hib));
    CUDA_TRY(c, cudaMallocHost(&c->h_r, ns * 4));
  } else {
    CUDA_TRY(c, cudaMallocHost(&c->h_slots, ns * sizeof(Rating)));
  }
  const bool want_dup = c->wf && c->p.wf_kernel != 2;
  if (want_dup) CUDA_TRY(c, cudaMallocHost(&c->h_dup, ns * sizeof(uint16_t)));
  // ---- pass 2
  {
    Nvtx rp2("out-of-core pass 2 (per block)");
    Grid Gd{c->m, c->n, c->a, c->s, c->c, c->wf, c->ac};
    const int64_t per = (int64_t)c->s * c->c;
    uint64_t *k0 = nullptr, *k1 = nullptr;
    uint32_t *i0 = nullptr, *i1 = nullptr, *s0 = nullptr, *s1 = nullptr;
    Rating *r0 = nullptr, *r1 = nullptr;
    unsigned* cnt = nullptr;
    uint16_t* dd = nullptr;
    uint32_t* du = nullptr;
    uint8_t* dv = nullptr;
    float* dr = nullptr;
    TRY(c->alloc(&k0, (size_t)maxlen)); TRY(c->alloc(&k1, (size_t)maxlen));
    TRY(c->alloc(&i0, (size_t)maxlen)); TRY(c->alloc(&i1, (size_t)maxlen));
    TRY(c->alloc(&r0, (size_t)maxlen)); TRY(c->alloc(&r1, (size_t)maxlen));
    if (c->wf) {
      TRY(c->alloc(&s0, (size_t)maxlen)); TRY(c->alloc(&s1, (size_t)maxlen));
      TRY(c->alloc(&cnt, (size_t)per));
    }
    if (want_dup) TRY(c->alloc(&dd, (size_t)maxlen));
    if (c->stg_packed) {
      TRY(c->alloc(&du, (size_t)maxlen)); TRY(c->alloc(&dv, (size_t)maxlen * c->pk.hib));
      TRY(c->alloc(&dr, (size_t)maxlen));
    }
    std::vector<int64_t> subo;
    std::vector<unsigned> hcnt;
    if (c->wf) {
      subo.assign((size_t)(nb * per + 1), 0);
      hcnt.resize((size_t)per);
    }
    const int W = want_dup ? ring_window(c->k, c->p.storage, c->p.lane_bytes) : 0;
    for (int64_t b = 0; b < nb; ++b) {
      const int64_t len = c->blk_len[(size_t)b], lo = c->blk_off[(size_t)b];
      const int64_t padded = c->blk_off[(size_t)b + 1] - lo;
      if (c->wf)
        for (int64_t q = 0; q <= per; ++q) subo[(size_t)(b * per + q)] = lo;   // empty default
      if (len == 0) continue;
      const int g = grid_for(len, c->num_sms);
      CUDA_TRY(c, cudaMemcpyAsync(k0, hk[(size_t)b].data(), (size_t)len * 8, cudaMemcpyHostToDevice, c->st));
      CUDA_TRY(c, cudaMemcpyAsync(r0, hr[(size_t)b].data(), (size_t)len * sizeof(Rating),
                                  cudaMemcpyHostToDevice, c->st));
      k_iota_u32<<<g, 256, 0, c->st>>>(i0, len);
      KERNEL_TRY(c);
      TRY(c->sort_pairs(k0, k1, i0, i1, len, 64));                 // storage order in the block
      k_gather_records<<<g, 256, 0, c->st>>>(i1, len, nullptr, r0, nullptr, r1);
      KERNEL_TRY(c);
      Rating* fin = r1;
      if (c->wf) {
        k_local_sub<<<g, 256, 0, c->st>>>(r1, len, Gd, b, s0, i0);
        KERNEL_TRY(c);
        TRY(c->sort_pairs(s0, s1, i0, i1, len, bits_for((uint64_t)std::max<int64_t>(per - 1, 1))));
        k_gather_records<<<g, 256, 0, c->st>>>(i1, len, nullptr, r1, nullptr, r0);
        CUDA_TRY(c, cudaMemsetAsync(cnt, 0, (size_t)per * 4, c->st));
        k_histogram<<<g, 256, 0, c->st>>>(s1, len, cnt);
        KERNEL_TRY(c);
        CUDA_TRY(c, cudaMemcpyAsync(hcnt.data(), cnt, (size_t)per * 4, cudaMemcpyDeviceToHost, c->st));
        fin = r0;
        if (want_dup) {
          k_dupdist<<<g, 256, 0, c->st>>>(fin, len, Gd, W, dd);
          KERNEL_TRY(c);
          CUDA_TRY(c, cudaMemcpyAsync(c->h_dup + lo, dd, (size_t)len * 2, cudaMemcpyDeviceToHost, c->st));
        }
      } else {
        if (padded > len)
          CUDA_TRY(c, cudaMemsetAsync(fin + len, 0xFF, (size_t)(padded - len) * sizeof(Rating), c->st));
        TRY(group_batches(c, fin, nullptr, padded));
      }
      if (c->stg_packed) {
        k_split_slots<<<grid_for(padded, c->num_sms), 256, 0, c->st>>>(fin, padded, c->pk, du, dv, dr);
        KERNEL_TRY(c);
        CUDA_TRY(c, cudaMemcpyAsync(c->h_u + lo, du, (size_t)padded * 4, cudaMemcpyDeviceToHost, c->st));
        CUDA_TRY(c, cudaMemcpyAsync(c->h_v16 + lo * c->pk.hib, dv, (size_t)padded * c->pk.hib,
                                    cudaMemcpyDeviceToHost, c->st));
        CUDA_TRY(c, cudaMemcpyAsync(c->h_r + lo, dr, (size_t)padded * 4, cudaMemcpyDeviceToHost, c->st));
      } else {
        CUDA_TRY(c, cudaMemcpyAsync(c->h_slots + lo, fin, (size_t)padded * sizeof(Rating),
                                    cudaMemcpyDeviceToHost, c->st));
      }
      CUDA_TRY(c, cudaStreamSynchronize(c->st));
      if (c->wf) {
        int64_t run = lo;
        for (int64_t q = 0; q < per; ++q) {
          subo[(size_t)(b * per + q)] = run;
          run += hcnt[(size_t)q];
        }
        subo[(size_t)(b * per + per)] = run;
      }
      std::vector<uint64_t>().swap(hk[(size_t)b]);               // host runs of b done
      std::vector<Rating>().swap(hr[(size_t)b]);
    }
    for (void* x : {(void*)k0, (void*)k1, (void*)i0, (void*)i1, (void*)r0, (void*)r1, (void*)s0,
                    (void*)s1, (void*)cnt, (void*)dd, (void*)du, (void*)dv, (void*)dr}) {
      void* y = x;
      c->release(y);
    }
    if (c->wf) {
      TRY(c->alloc(&c->sub_off, subo.size()));
      CUDA_TRY(c, cudaMemcpyAsync(c->sub_off, subo.data(), subo.size() * 8, cudaMemcpyHostToDevice, c->st));
      CUDA_TRY(c, cudaStreamSynchronize(c->st));
    } else {
      TRY(c->alloc(&c->d_choff, (size_t)nb + 1));
      CUDA_TRY(c, cudaMemcpyAsync(c->d_choff, c->ch_off.data(), (nb + 1) * 8, cudaMemcpyHostToDevice, c->st));
      CUDA_TRY(c, cudaStreamSynchronize(c->st));
    }
  }
  TRY(init_factors(c));
  if (c->p.lr_rule == 1) {
    TRY(c->alloc(&c->GP, (size_t)(c->m * c->k)));
    TRY(c->alloc(&c->GQ, (size_t)(c->n * c->k)));
    CUDA_TRY(c, cudaMemsetAsync(c->GP, 0, (size_t)(c->m * c->k) * 4, c->st));
    CUDA_TRY(c, cudaMemsetAsync(c->GQ, 0, (size_t)(c->n * c->k) * 4, c->st));
  }
  TRY(alloc_schedule(c));
  c->n_units = c->wf ? nb * (int64_t)c->s * c->c : c->ch_off.back();
  TRY(c->alloc(&c->visits, (size_t)std::max<int64_t>(c->n_units, 1)));
  CUDA_TRY(c, cudaMemsetAsync(c->visits, 0, (size_t)std::max<int64_t>(c->n_units, 1) * 4, c->st));
  c->epochs_run = 0;
  TRY(setup_staging_buffers(c));
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  c->train_loaded = true;
  return MF_OK;
}

static mf_status join_side(mf_ctx* c);

static mf_status load_test(mf_ctx* c, int64_t N, const int32_t* u, const int32_t* v, const float* r,
                           int on_device) {
  // the side stream may still be building the next epoch's chunk order in the shared sort
  // scratch (tmp), which the world > 1 test-set selection below reuses
  TRY(join_side(c));
  const int32_t *du, *dv;
  const float* dr;
  int32_t *ou, *ov;
  float* orr;
  TRY(stage_input(c, N, u, v, r, on_device, &du, &dv, &dr, &ou, &ov, &orr));
  TRY(validate(c, N, du, dv, dr));
  TRY(c->alloc(&c->test, (size_t)std::max<int64_t>(N, 1)));
  if (N > 0) {
    k_build_test<<<grid_for(N, c->num_sms), 256, 0, c->st>>>(du, dv, dr, N, c->rho_r, c->rho_c,
                                                             (double)c->p.rating_scale, c->test);
    KERNEL_TRY(c);
  }
  c->release(ou); c->release(ov); c->release(orr);
  if (c->G > 1 && N > 0) {
    // keep only the test ratings of this rank's row segments (SSE and count are all-reduced)
    char* flag = nullptr;
    Rating* kept = nullptr;
    int64_t* nsel = nullptr;
    TRY(c->alloc(&flag, (size_t)N));
    TRY(c->alloc(&kept, (size_t)N));
    TRY(c->alloc(&nsel, 1));
    k_own_rows<<<grid_for(N, c->num_sms), 256, 0, c->st>>>(c->test, N, c->m, c->a, c->lo_row_seg(),
                                                          c->hi_row_seg(), flag);
    KERNEL_TRY(c);
    size_t bytes = 0;
    CUDA_TRY(c, cub::DeviceSelect::Flagged(nullptr, bytes, c->test, flag, kept, nsel, N, c->st));
    TRY(c->need_tmp(bytes));
    CUDA_TRY(c, cub::DeviceSelect::Flagged(c->tmp, bytes, c->test, flag, kept, nsel, N, c->st));
    int64_t h = 0;
    CUDA_TRY(c, cudaMemcpyAsync(&h, nsel, 8, cudaMemcpyDeviceToHost, c->st));
    CUDA_TRY(c, cudaStreamSynchronize(c->st));
    c->release(c->test);
    c->release(flag);
    c->release(nsel);
    c->test = kept;
    N = h;
  }
  if (c->pq && N > 0) {
    // P out of core: the test ratings grouped by row segment (stable), evaluated one staged
    // segment at a time
    Nvtx rg("group test ratings by row segment");
    uint32_t *k0 = nullptr, *k1 = nullptr, *i0 = nullptr, *i1 = nullptr;
    unsigned* cnt = nullptr;
    Rating* sorted = nullptr;
    TRY(c->alloc(&k0, (size_t)N)); TRY(c->alloc(&k1, (size_t)N));
    TRY(c->alloc(&i0, (size_t)N)); TRY(c->alloc(&i1, (size_t)N));
    TRY(c->alloc(&cnt, (size_t)c->a)); TRY(c->alloc(&sorted, (size_t)N));
    const int g = grid_for(N, c->num_sms);
    k_test_seg<<<g, 256, 0, c->st>>>(c->test, N, c->m, c->a, k0, i0);
    KERNEL_TRY(c);
    TRY(c->sort_pairs(k0, k1, i0, i1, N, bits_for((uint64_t)c->a)));
    k_gather_records<<<g, 256, 0, c->st>>>(i1, N, nullptr, c->test, nullptr, sorted);
    CUDA_TRY(c, cudaMemsetAsync(cnt, 0, (size_t)c->a * 4, c->st));
    k_histogram<<<g, 256, 0, c->st>>>(k1, N, cnt);
    KERNEL_TRY(c);
    std::vector<unsigned> hc((size_t)c->a);
    CUDA_TRY(c, cudaMemcpyAsync(hc.data(), cnt, (size_t)c->a * 4, cudaMemcpyDeviceToHost, c->st));
    CUDA_TRY(c, cudaStreamSynchronize(c->st));
    c->test_seg_off.assign((size_t)c->a + 1, 0);
    for (int r = 0; r < c->a; ++r) c->test_seg_off[(size_t)r + 1] = c->test_seg_off[(size_t)r] + hc[(size_t)r];
    c->release(c->test);
    c->test = sorted;
    c->release(k0); c->release(k1); c->release(i0); c->release(i1); c->release(cnt);
  }
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  c->Ntest = N;
  c->test_loaded = true;
  return MF_OK;
}

mf_status mf_load_coo(mf_ctx* c, int32_t set, int64_t nnz, const int32_t* u, const int32_t* v,
                      const float* r, int32_t on_device) {
  if (!c) return MF_E_INVAL;
  TRY(c->enter());
  if (nnz < 0 || (nnz > 0 && (!u || !v || !r))) return c->fail(MF_E_INVAL, "bad COO arguments");
  const std::vector<std::pair<void*, size_t>> before = c->sizes;
  Nvtx range("mf_load_coo(%s, N=%lld)", set == MF_TRAIN ? "train" : "test", (long long)nnz);
  mf_status s = MF_OK;
  if (set == MF_TRAIN) {
    if (c->train_loaded) return c->fail(MF_E_STATE, "train set already loaded");
    // out-of-core mode with a host rating set: chunked preprocessing (never all in HBM)
    s = (c->staged && !on_device) ? load_train_chunked(c, nnz, u, v, r)
                                  : load_train(c, nnz, u, v, r, on_device);
  } else if (set == MF_TEST) {
    if (!c->train_loaded) return c->fail(MF_E_STATE, "load the train set first");
    if (c->test_loaded) return c->fail(MF_E_STATE, "test set already loaded");
    s = load_test(c, nnz, u, v, r, on_device);
  } else {
    return c->fail(MF_E_INVAL, "set must be MF_TRAIN or MF_TEST");
  }
  if (s != MF_OK && c->sticky == MF_OK) {
    // recoverable failure (MF_E_RANGE, MF_E_NOMEM, ...): the ctx stays usable
    cudaStreamSynchronize(c->st);
    if (c->cs) cudaStreamSynchronize(c->cs);
    if (c->ds) cudaStreamSynchronize(c->ds);
    c->drop_allocations_since(before);
    if (set == MF_TRAIN) release_host_staging(c);   // a retried load allocates them again
  }
  return s;
}

// ---------------------------------------------------------------------------------------------
// per-epoch schedule (A: "Orders")
// ---------------------------------------------------------------------------------------------
// The main stream waits for an in-flight side-stream schedule build (they share the scratch).
static mf_status join_side(mf_ctx* c) {
  if (c->ss_pending) {
    CUDA_TRY(c, cudaStreamWaitEvent(c->st, c->ev_ss_done, 0));
    c->ss_pending = false;
  }
  return MF_OK;
}

static mf_status build_schedule(mf_ctx* c, int32_t t) {
  TRY(join_side(c));
  const int64_t nb = (int64_t)c->a * c->ac;
  if (c->libmf) return MF_OK;             // blocks are picked at run time from the table
  if (!c->wf) {
    const int64_t total = c->ch_off.back();
    if (total == 0) return MF_OK;
    k_chunk_keys<<<grid_for(total, c->num_sms), 256, 0, c->st>>>(c->d_choff, (int)nb, c->p.seed, t,
                                                                 c->sk0, c->sv0);
    KERNEL_TRY(c);
    ++c->n_launch;
    if (nb == 1) {
      TRY(c->sort_pairs(c->sk0, c->sk1, c->sv0, c->chunk_order, total, 64));
    } else {
      TRY(c->sort_pairs(c->sk0, c->sk1, c->sv0, c->sv1, total, 64));
      k_chunk_block<<<grid_for(total, c->num_sms), 256, 0, c->st>>>(c->sv1, c->d_choff, (int)nb,
                                                                    total, c->sb);
      KERNEL_TRY(c);
      ++c->n_launch;
      // stable by block: keeps each block's key order
      uint32_t* bk_out = reinterpret_cast<uint32_t*>(c->sk0);
      TRY(c->sort_pairs(c->sb, bk_out, c->sv1, c->chunk_order, total, bits_for((uint64_t)(nb - 1))));
    }
    c->sched_built_for = t;
    return MF_OK;
  }
  // wavefront: seq (per block b, worker i: perm of c columns) then ticket ranks
  const int s = c->s, cc = c->c;
  const int64_t total = nb * s * (int64_t)cc;
  if (c->p.cyclic) {
    const int64_t tt = nb * cc;
    for (int which = 0; which < 2; ++which) {
      k_perm_keys<<<grid_for(tt, c->num_sms), 256, 0, c->st>>>(
          nb, cc, c->p.seed, which == 0 ? kTagCycTau : kTagCycSigma, t, c->sk0, c->sv0);
      KERNEL_TRY(c);
      TRY(c->sort_pairs(c->sk0, c->sk1, c->sv0, c->sv1, tt, 64));
      if (nb > 1) {
        k_seg_of<<<grid_for(tt, c->num_sms), 256, 0, c->st>>>(c->sv1, tt, cc, c->sb);
        KERNEL_TRY(c);
        TRY(c->sort_pairs(c->sb, reinterpret_cast<uint32_t*>(c->sk0), c->sv1, c->sv0, tt,
                          bits_for((uint64_t)(nb - 1))));
        std::swap(c->sv0, c->sv1);
      }
      k_mod_c<<<grid_for(tt, c->num_sms), 256, 0, c->st>>>(c->sv1, tt, cc,
                                                           which == 0 ? c->tau : c->sigma);
      KERNEL_TRY(c);
    }
    k_cyclic_seq<<<grid_for(total, c->num_sms), 256, 0, c->st>>>(c->tau, c->sigma, nb, s, cc, c->seq);
    KERNEL_TRY(c);
    int32_t* P = reinterpret_cast<int32_t*>(c->sb);       // nb (c+1) <= 2 nb c = cap: free here
    k_tau_prefix<<<(unsigned)nb, 1024, 0, c->st>>>(c->tau, s, cc, P);
    KERNEL_TRY(c);
    k_cyclic_rank<<<grid_for(total, c->num_sms), 256, 0, c->st>>>(c->tau, P, nb, s, cc, c->rank_arr);
    KERNEL_TRY(c);
    c->n_launch += 3;
    c->sched_built_for = t;
    return MF_OK;
  } else {
    k_wf_keys<<<grid_for(total, c->num_sms), 256, 0, c->st>>>(nb * s, s, cc, c->p.seed, t, c->sk0,
                                                              c->sv0);
    KERNEL_TRY(c);
    TRY(c->sort_pairs(c->sk0, c->sk1, c->sv0, c->sv1, total, 64));
    if (nb * s > 1) {
      k_seg_of<<<grid_for(total, c->num_sms), 256, 0, c->st>>>(c->sv1, total, cc, c->sb);
      KERNEL_TRY(c);
      TRY(c->sort_pairs(c->sb, reinterpret_cast<uint32_t*>(c->sk0), c->sv1, c->sv0, total,
                        bits_for((uint64_t)(nb * s - 1))));
      std::swap(c->sv0, c->sv1);
    }
    k_mod_c<<<grid_for(total, c->num_sms), 256, 0, c->st>>>(c->sv1, total, cc, c->seq);
    KERNEL_TRY(c);
  }
  k_ticket_keys<<<grid_for(total, c->num_sms), 256, 0, c->st>>>(c->seq, nb, s, cc, c->sk0, c->sv0);
  KERNEL_TRY(c);
  const uint64_t maxkey = (uint64_t)(((nb - 1) * cc + (cc - 1)) * (int64_t)cc + (cc - 1)) * s + (s - 1);
  TRY(c->sort_pairs(c->sk0, c->sk1, c->sv0, c->sv1, total, bits_for(maxkey)));
  k_ticket_rank<<<grid_for(total, c->num_sms), 256, 0, c->st>>>(c->sv1, total, s, c->rank_arr);
  KERNEL_TRY(c);
  c->n_launch += 6;
  c->sched_built_for = t;
  return MF_OK;
}

static cudaEvent_t ev_at(mf_ctx* c, int i) {
  while ((int)c->ev.size() <= i) {
    cudaEvent_t e;
    cudaEventCreate(&e);
    c->ev.push_back(e);
  }
  return c->ev[(size_t)i];
}

// One strata block set (the blocks rank g trains in sub-epoch j) of epoch t.
static AdaArgs ada_args(const mf_ctx* c) {
  AdaArgs A{};
  if (c->p.lr_rule == 1) {
    A.GP = c->GP;
    A.GQ = c->GQ;
    A.lp = c->p.lambda_p;
    A.lq = c->p.lambda_q;
    A.eps = c->p.ada_eps > 0.f ? c->p.ada_eps : 1e-8f;
  }
  return A;
}

// shift of block b in the current staging buffer (0 when the ratings are resident)
static int64_t slot_shift(const mf_ctx* c, int buf, int64_t b) {
  if (!c->staged) return 0;
  for (const auto& x : c->stg_shift[buf])
    if (x.first == b) return x.second;
  return 0;
}

// Level table of the interleaved claim order (ChunkSegs): level l runs, round-robin over the
// segments whose length exceeds the previous level's, the chunk indices up to the next
// distinct segment length.
static void finalize_segs(ChunkSegs& s) {
  std::vector<int64_t> lens;
  for (int i = 0; i < s.n; ++i) lens.push_back(s.prefix[i + 1] - s.prefix[i]);
  std::vector<int64_t> cuts(lens);
  std::sort(cuts.begin(), cuts.end());
  cuts.erase(std::unique(cuts.begin(), cuts.end()), cuts.end());
  s.nlev = 0;
  int64_t lo = 0, base = 0;
  for (int64_t cut : cuts) {
    const int l = s.nlev;
    int cnt = 0;
    for (int i = 0; i < s.n; ++i)
      if (lens[(size_t)i] >= cut) s.lev_seg[l][cnt++] = (int8_t)i;
    s.lev_base[l] = base;
    s.lev_lo[l] = lo;
    s.lev_cnt[l] = cnt;
    base += (cut - lo) * cnt;
    lo = cut;
    ++s.nlev;
  }
  s.lev_base[s.nlev] = base;                 // == prefix[n]
  for (int l = s.nlev + 1; l <= kMaxSegs; ++l) s.lev_base[l] = base;
}

// One Hogwild launch over the claim order `segs` of the chunk-id list `chunks`.
static mf_status launch_chunks(mf_ctx* c, ChunkSegs& segs, const uint32_t* chunks, const Rating* slots,
                               float g) {
  finalize_segs(segs);
  CUDA_TRY(c, cudaMemsetAsync(c->counter, 0, sizeof(unsigned long long), c->st));
  {
    HogwildLaunch L{};
    L.storage = c->p.storage; L.k = c->k; L.lane_bytes = c->p.lane_bytes ? c->p.lane_bytes : 16;
    L.prefetch = c->p.prefetch ? c->p.prefetch : 1;
    L.rating_stage = c->p.rating_stage;
    L.group = c->p.group_cols;
    L.slots = slots; L.chunks = chunks; L.segs = segs; L.counter = c->counter;
    L.workers = c->p.workers; L.num_sms = c->num_sms; L.f = c->f;
    L.P = c->P; L.Q = c->Q; L.g = g; L.lp = c->p.lambda_p; L.lq = c->p.lambda_q; L.stream = c->st;
    L.ada = ada_args(c);
    L.exact = c->p.exact_order;
    if (L.ada.GP) L.g = c->p.alpha;        // ADAGRAD: constant alpha, no Eq. 9 decay
    L.out_workers = &c->last_workers; L.out_lanes = &c->last_lanes; L.out_grid = &c->last_grid;
    L.q_l1 = c->p.q_cache == 0; L.out_q_l1 = &c->last_q_l1;
    L.visits = c->visits; L.upd = c->upd_dev;
    CUDA_TRY(c, cudaEventRecord(ev_at(c, 2 * c->n_sgd), c->st));
    CUDA_TRY(c, launch_hogwild(L));
    CUDA_TRY(c, cudaEventRecord(ev_at(c, 2 * c->n_sgd + 1), c->st));
    c->last_block = 256;
    ++c->n_sgd;
    ++c->n_launch;
  }
  return MF_OK;
}

static mf_status run_stratum(mf_ctx* c, const std::vector<int64_t>& blocks, float g, int buf) {
  const Rating* slots = c->staged ? c->stg[buf] : c->slots;
  const uint16_t* dup = c->staged ? c->stg_dup[buf] : c->dup;
  if (!c->wf) {
    ChunkSegs segs{};
    segs.n = 0;
    segs.prefix[0] = 0;
    for (int64_t b : blocks) {
      const int64_t nch = c->ch_off[(size_t)b + 1] - c->ch_off[(size_t)b];
      if (nch == 0) continue;
      segs.begin[segs.n] = c->ch_off[(size_t)b];
      segs.prefix[segs.n + 1] = segs.prefix[segs.n] + nch;
      segs.shift[segs.n] = slot_shift(c, buf, b);
      ++segs.n;
    }
    if (segs.n == 0) return MF_OK;
    return launch_chunks(c, segs, c->chunk_order, slots, g);
  }
  // The non-empty blocks run together in one cooperative launch (they touch disjoint rows and
  // columns, so any concurrency gives the result of running them one after another): worker w
  // of the launch is worker w % s of block w / s, with c tickets per block.  When s x blocks
  // workers cannot all be co-resident, the blocks go in smaller groups (down to one per launch).
  std::vector<int64_t> todo;
  for (int64_t b : blocks)
    if (c->blk_len[(size_t)b] > 0) todo.push_back(b);
  size_t group = std::max<size_t>(todo.size(), 1);
  static const bool kProfWaves = std::getenv("MF_PROFILE_WAVES") != nullptr;
  for (size_t g0 = 0; g0 < todo.size();) {
    const size_t gn = std::min(group, todo.size() - g0);
    WavefrontLaunch L{};
    L.blocks.n = (int)gn;
    for (size_t i = 0; i < gn; ++i) {
      const int64_t b = todo[g0 + i];
      L.blocks.base[i] = b * (int64_t)c->s * c->c;
      L.blocks.shift[i] = slot_shift(c, buf, b);
    }
    CUDA_TRY(c, cudaMemsetAsync(c->tickets, 0, gn * (size_t)c->c * 4, c->st));
    L.storage = c->p.storage; L.k = c->k; L.slots = slots; L.sub_off = c->sub_off;
    L.variant = c->p.wf_kernel == 2 ? 0 : 1;
    L.lane_bytes = c->p.lane_bytes;
    L.dup = dup;
    L.seq = c->seq; L.rank = c->rank_arr; L.tickets = c->tickets;
    L.s = c->s; L.c = c->c; L.num_sms = c->num_sms; L.P = c->P; L.Q = c->Q; L.g = g;
    L.lp = c->p.lambda_p; L.lq = c->p.lambda_q; L.stream = c->st;
    L.ada = ada_args(c);
    L.exact = c->p.exact_order;
    if (L.ada.GP) L.g = c->p.alpha;
    L.out_lanes = &c->last_lanes; L.out_grid = &c->last_grid;
    L.visits = c->visits; L.upd = c->upd_dev;
    L.owners = c->owners; L.viol = c->own_viol;
    // Diagnostics only (MF_PROFILE_WAVES=1): per-worker clock64 totals of ticket waits and
    // sub-block runs, summarised on stderr after the launch (synchronises).
    const int nw = c->s * (int)gn;
    long long* prof = nullptr;
    if (kProfWaves && L.variant == 1) {
      CUDA_TRY(c, cudaMallocAsync(reinterpret_cast<void**>(&prof), (size_t)nw * 6 * 8, c->st));
      CUDA_TRY(c, cudaMemsetAsync(prof, 0, (size_t)nw * 6 * 8, c->st));
    }
    L.prof = prof;
    CUDA_TRY(c, cudaEventRecord(ev_at(c, 2 * c->n_sgd), c->st));
    cudaError_t e = launch_wavefront(L);
    if (e == cudaErrorCooperativeLaunchTooLarge) {
      cudaGetLastError();
      if (prof) CUDA_TRY(c, cudaFreeAsync(prof, c->st));
      if (gn == 1)
        return c->fail(MF_E_UNSUPPORTED, "wavefront: %d workers cannot all be co-resident", c->s);
      group = std::max<size_t>(1, gn / 2);                  // retry with smaller groups
      continue;
    }
    if (prof && e == cudaSuccess) {
      std::vector<long long> h((size_t)nw * 6);
      CUDA_TRY(c, cudaMemcpyAsync(h.data(), prof, h.size() * 8, cudaMemcpyDeviceToHost, c->st));
      CUDA_TRY(c, cudaStreamSynchronize(c->st));
      CUDA_TRY(c, cudaFreeAsync(prof, c->st));
      std::map<long long, int> per_smsp;
      for (int i = 0; i < nw; ++i) ++per_smsp[h[6 * i + 3] * 4 + (h[6 * i + 4] & 3)];
      double sw = 0, sr = 0, mxw = 0, mxr = 0, mxt = 0, sn = 0, shared_r = 0, solo_r = 0;
      double shared_n = 0, solo_n = 0, srel = 0;
      for (int i = 0; i < nw; ++i) {
        const double w = (double)h[6 * i], r = (double)h[6 * i + 1], n = (double)h[6 * i + 2];
        srel += (double)h[6 * i + 5];
        sw += w; sr += r; sn += n;
        mxw = std::max(mxw, w); mxr = std::max(mxr, r); mxt = std::max(mxt, w + r);
        const bool shared = per_smsp[h[6 * i + 3] * 4 + (h[6 * i + 4] & 3)] > 1;
        (shared ? shared_r : solo_r) += r;
        (shared ? shared_n : solo_n) += n;
      }
      int shared_w = 0;
      for (auto& kv : per_smsp) if (kv.second > 1) shared_w += kv.second;
      std::fprintf(stderr,
                   "[MF_PROFILE_WAVES] s=%d c=%d blocks=%d  cycles/worker: wait mean %.3g max %.3g, run mean "
                   "%.3g max %.3g, wait+run max %.3g; run cycles/sample %.1f (solo-SMSP workers %.1f, "
                   "SMSP-sharing %.1f; %d of %d workers share an SMSP); release fence mean %.3g cycles/worker\n",
                   c->s, c->c, (int)gn, sw / nw, mxw, sr / nw, mxr, mxt, sr / std::max(sn, 1.0),
                   solo_r / std::max(solo_n, 1.0), shared_r / std::max(shared_n, 1.0), shared_w, nw,
                   srel / nw);
    }
    CUDA_TRY(c, e);
    CUDA_TRY(c, cudaEventRecord(ev_at(c, 2 * c->n_sgd + 1), c->st));
    c->last_workers = nw;
    c->last_q_l1 = 0;
    c->last_block = 128;
    ++c->n_sgd;
    ++c->n_launch;
    g0 += gn;
  }
  return MF_OK;
}

// Q segment J occupies relabelled rows [ceil(J n / a), ceil((J+1) n / a)) (A: segments).
static void q_segment(const mf_ctx* c, int J, char** ptr, size_t* bytes) {
  const size_t row_bytes = (size_t)c->k * c->ssize();
  const int64_t lo = cdiv64((int64_t)J * c->n, c->a), hi = cdiv64((int64_t)(J + 1) * c->n, c->a);
  *ptr = (char*)c->Q + (size_t)lo * row_bytes;
  *bytes = (size_t)(hi - lo) * row_bytes;
}

// Move the Q segments of a sub-epoch plan (north_star (5): NCCL send/recv of Q column
// segments between sub-epochs); xf = {J, src, dst, lo, hi} per transfer (mf_strata_plan).
static mf_status rotate_q(mf_ctx* c, const int64_t* xf, int nx) {
  if (c->G == 1 || nx == 0) return MF_OK;
  std::vector<mf::Xfer> xs;
  const size_t row_bytes = (size_t)c->k * c->ssize();
  for (int i = 0; i < nx; ++i) {
    const int64_t* x = xf + 5 * i;
    mf::Xfer e;
    e.ptr = (char*)c->Q + (size_t)x[3] * row_bytes;
    e.bytes = (size_t)(x[4] - x[3]) * row_bytes;
    e.src = (int)x[1];
    e.dst = (int)x[2];
    xs.push_back(e);
  }
  std::string why;
  if (!c->comm->exchange(xs, c->rank, &why)) return c->fail(MF_E_NCCL, "Q rotation: %s", why.c_str());
  return MF_OK;
}

// Make every rank's Q complete (evaluation / get_factors): broadcast each segment from its
// current holder; afterwards every rank holds an identical valid copy (holders = -1).
static mf_status gather_q(mf_ctx* c) {
  if (c->G == 1) return MF_OK;
  const int32_t* h = c->comm->holders(c->a);
  std::vector<int32_t> hold(h, h + c->a);
  for (int J = 0; J < c->a; ++J) {
    if (hold[(size_t)J] < 0) continue;
    char* ptr;
    size_t bytes;
    q_segment(c, J, &ptr, &bytes);
    std::string why;
    if (!c->comm->broadcast(ptr, bytes, hold[(size_t)J], &why))
      return c->fail(MF_E_NCCL, "Q gather: %s", why.c_str());
  }
  c->comm->reset_holders(c->a);
  return MF_OK;
}

// Enqueue epoch tn's Hogwild chunk order on the side stream, into chunk_order_alt.  ev_ss_go
// was recorded on the main stream after this epoch's schedule and before its SGD launches, so
// the previous epoch's SGD (the last reader of chunk_order_alt) is complete when it fires.
static mf_status prebuild_schedule(mf_ctx* c, int32_t tn) {
  if (!c->ss) {
    CUDA_TRY(c, cudaStreamCreateWithFlags(&c->ss, cudaStreamNonBlocking));
    CUDA_TRY(c, cudaEventCreateWithFlags(&c->ev_ss_done, cudaEventDisableTiming));
  }
  CUDA_TRY(c, cudaStreamWaitEvent(c->ss, c->ev_ss_go, 0));
  const int32_t built = c->sched_built_for;
  std::swap(c->chunk_order, c->chunk_order_alt);
  std::swap(c->st, c->ss);
  const mf_status s = build_schedule(c, tn);
  std::swap(c->st, c->ss);
  std::swap(c->chunk_order, c->chunk_order_alt);
  c->sched_built_for = built;
  if (s != MF_OK) return s;
  CUDA_TRY(c, cudaEventRecord(c->ev_ss_done, c->ss));
  c->ss_pending = true;
  c->prebuilt_t = tn;
  return MF_OK;
}

// The a sub-epochs of epoch t (A: strata order): Q rotation between them (world > 1), the
// stratum's ratings staged from host (staged == 1), one interleaved Hogwild launch or one
// wavefront launch per block.
static mf_status train_epoch_strata(mf_ctx* c, int32_t t, float g) {
  // holders of every Q segment's valid copy persist across sub-epochs and epochs (comm);
  // world == 1 keeps a local vector (every segment is always on rank 0: no transfers)
  std::vector<int32_t> local_hold((size_t)c->a, -1);
  int32_t* hold = local_hold.data();
  std::vector<int32_t> hcopy;
  if (c->G > 1) {
    const int32_t* h = c->comm->holders(c->a);
    hcopy.assign(h, h + c->a);
    hold = hcopy.data();
  }
  std::vector<int64_t> blocks((size_t)c->a), xf((size_t)(5 * c->a));
  CUDA_TRY(c, cudaEventRecord(c->ev_c0, c->st));
  CUDA_TRY(c, cudaEventRecord(c->ev_c1, c->st));
  for (int j = 0; j < c->a; ++j) {
    Nvtx rj("sub-epoch %d", j);
    int32_t nb = 0, nx = 0;
    if (c->ac == 1) {                  // a x 1 row blocks (R27, one GPU): block pi_t[j]
      blocks[0] = stratum_blocks(c, t, j)[0];
      nb = 1;
    } else if (mf_strata_plan(c->p.seed, c->a, c->G, c->rank, c->n, t, j, hold, blocks.data(), &nb,
                              xf.data(), &nx) != MF_OK) {
      return c->fail(MF_E_INVAL, "strata plan failed");
    }
    if (nx) {
      Nvtx rq("Q rotation (%d segments)", nx);
      TRY(rotate_q(c, xf.data(), nx));
    }
    if (c->G > 1) c->comm->set_holders(hold, c->a);
    int buf = 0;
    if (c->staged) {
      // stratum (t, j) is normally pre-staged by the previous step (also across epochs)
      if (c->staged_t != t || c->staged_j != j) TRY(stage(c, t, j, c->cur_buf));
      buf = c->cur_buf;
      const bool last = j + 1 == c->a;
      TRY(stage(c, last ? t + 1 : t, last ? 0 : j + 1, 1 - buf));   // overlap the next copy
      CUDA_TRY(c, cudaStreamWaitEvent(c->st, c->ev_h2d[buf], 0));
      if (c->stg_packed) {
        if (c->stg_len[buf] > 0) {
          k_expand_slots<<<grid_for(c->stg_len[buf], c->num_sms), 256, 0, c->st>>>(
              c->stg_u[buf], c->stg_v16[buf], c->stg_r[buf], c->stg_len[buf], c->pk, c->stg[buf]);
          KERNEL_TRY(c);
          ++c->n_launch;
        }
        // the packed buffers are free again once expanded (the slots are stream-ordered);
        // not so the wavefront's duplicate distances, which the SGD launch reads in place
        if (!c->h_dup) CUDA_TRY(c, cudaEventRecord(c->ev_free[buf], c->st));
      }
    }
    const int per_launch = (!c->wf && c->p.launch_blocks > 0) ? c->p.launch_blocks : std::max(nb, 1);
    for (int b0 = 0; b0 < nb; b0 += per_launch)
      TRY(run_stratum(c, std::vector<int64_t>(blocks.begin() + b0,
                                              blocks.begin() + std::min(nb, b0 + per_launch)),
                      g, buf));
    if (c->staged) {
      if (!c->stg_packed || c->h_dup) CUDA_TRY(c, cudaEventRecord(c->ev_free[buf], c->st));
      c->cur_buf = 1 - buf;
    }
  }
  return MF_OK;
}

// a x 1 row blocks, resident (R27): the blocks' chunk orders concatenated in pi_t order and run
// by ONE Hogwild launch -- the claim order is block pi_t[0]'s chunks, then pi_t[1]'s, ..., so a
// single worker runs exactly the oracle's block-after-block order, and many workers overlap
// consecutive blocks only at their boundary instead of idling in a per-block tail.
static mf_status train_epoch_rows(mf_ctx* c, int32_t t, float g) {
  const std::vector<int64_t> pi = host_perm(make_stream(c->p.seed, kTagStrata, (uint64_t)t, 0), c->a);
  int64_t off = 0;
  for (int j = 0; j < c->a; ++j) {
    const int64_t b = pi[(size_t)j];
    const int64_t lo = c->ch_off[(size_t)b], nch = c->ch_off[(size_t)b + 1] - lo;
    if (nch == 0) continue;
    CUDA_TRY(c, cudaMemcpyAsync(c->chunk_seq + off, c->chunk_order + lo, (size_t)nch * 4,
                                cudaMemcpyDeviceToDevice, c->st));
    off += nch;
  }
  CUDA_TRY(c, cudaEventRecord(c->ev_c0, c->st));
  CUDA_TRY(c, cudaEventRecord(c->ev_c1, c->st));
  if (off == 0) return MF_OK;
  ChunkSegs segs{};
  segs.n = 1;
  segs.begin[0] = 0;
  segs.prefix[0] = 0;
  segs.prefix[1] = off;
  segs.shift[0] = 0;
  return launch_chunks(c, segs, c->chunk_seq, c->slots, g);
}

// staged == 2 (section 6.1 step 3 + 6.3): blocks one at a time in the strata order, each with
// its P row segment staged in on the copy stream, trained on the compute stream, written back on
// the write-back stream; the next block's copy-in overlaps this block's compute, and its
// write-back the next block's compute.  Two slots: block x uses slot x % 2, which is free once
// block x-2's write-back is done.  Consecutive blocks of the strata order never share a row
// segment (a >= 2); every read of a segment is ordered after its last write-back (ds is in
// order).  Same blocks, same order, same kernels: bit-identical to resident P.
static mf_status train_epoch_pq(mf_ctx* c, int32_t t, float g) {
  const size_t rowb = (size_t)c->k * c->ssize();
  const std::vector<int64_t> pi = host_perm(make_stream(c->p.seed, kTagStrata, (uint64_t)t, 0), c->a);
  CUDA_TRY(c, cudaEventRecord(c->ev_c0, c->st));
  CUDA_TRY(c, cudaEventRecord(c->ev_c1, c->st));
  for (int s = 0; s < 2; ++s) CUDA_TRY(c, cudaStreamWaitEvent(c->cs, c->ev_pout[s], 0));
  int64_t x = 0;
  for (int j = 0; j < c->a; ++j) {
    Nvtx rj("sub-epoch %d", j);
    for (int rr = 0; rr < (c->ac == 1 ? 1 : c->a); ++rr, ++x) {
      // a x a: block (r, (r + pi_t[j]) mod a) for every r; a x 1 (R27): block pi_t[j]
      const int r = c->ac == 1 ? (int)pi[(size_t)j] : rr;
      const int64_t b = c->ac == 1 ? (int64_t)r : (int64_t)r * c->a + (r + pi[(size_t)j]) % c->a;
      const int s = (int)(x & 1);
      const int64_t lo = cdiv64((int64_t)r * c->m, c->a), hi = cdiv64((int64_t)(r + 1) * c->m, c->a);
      const size_t bytes = (size_t)(hi - lo) * rowb;
      // copy-in
      CUDA_TRY(c, cudaStreamWaitEvent(c->cs, c->ev_pout[s], 0));
      TRY(stage_block(c, b, s));
      CUDA_TRY(c, cudaMemcpyAsync(c->Pslot[s], c->h_P + (size_t)lo * rowb, bytes, cudaMemcpyHostToDevice, c->cs));
      c->h2d_bytes += (int64_t)bytes;
      CUDA_TRY(c, cudaEventRecord(c->ev_pin[s], c->cs));
      // compute
      CUDA_TRY(c, cudaStreamWaitEvent(c->st, c->ev_pin[s], 0));
      if (c->stg_packed && c->stg_len[s] > 0) {
        k_expand_slots<<<grid_for(c->stg_len[s], c->num_sms), 256, 0, c->st>>>(
            c->stg_u[s], c->stg_v16[s], c->stg_r[s], c->stg_len[s], c->pk, c->stg[s]);
        KERNEL_TRY(c);
        ++c->n_launch;
      }
      c->P = c->Pslot[s] - (size_t)lo * rowb;      // P[u] for u in [lo, hi) lands in the slot
      const mf_status ms = run_stratum(c, std::vector<int64_t>(1, b), g, s);
      c->P = nullptr;
      TRY(ms);
      CUDA_TRY(c, cudaEventRecord(c->ev_pcomp[s], c->st));
      // write-back
      CUDA_TRY(c, cudaStreamWaitEvent(c->ds, c->ev_pcomp[s], 0));
      CUDA_TRY(c, cudaMemcpyAsync(c->h_P + (size_t)lo * rowb, c->Pslot[s], bytes, cudaMemcpyDeviceToHost, c->ds));
      CUDA_TRY(c, cudaEventRecord(c->ev_pout[s], c->ds));
    }
  }
  // the epoch is complete when its last write-back is
  CUDA_TRY(c, cudaStreamWaitEvent(c->st, c->ev_pout[(x - 1) & 1], 0));
  return MF_OK;
}

mf_status mf_train_epoch(mf_ctx* c, int32_t* epoch_done) {
  if (!c) return MF_E_INVAL;
  TRY(c->enter());
  if (!c->train_loaded) return c->fail(MF_E_STATE, "no train set loaded");
  const int32_t t = c->t;
  Nvtx range("epoch %d", t);
  const float g = gamma_of(c->p.alpha, c->p.beta, t);   // Eq. 9
  c->n_sgd = 0;
  c->n_launch = 0;
  c->h2d_bytes = 0;
  c->comm_ms_acc.clear();
  CUDA_TRY(c, cudaMemsetAsync(c->upd_dev, 0, sizeof(unsigned long long), c->st));
  CUDA_TRY(c, cudaEventRecord(c->ev_e0, c->st));
  CUDA_TRY(c, cudaEventRecord(c->ev_s0, c->st));
  const bool hog = !c->wf && !c->libmf && c->ch_off.back() > 0;
  {
    Nvtx rsched("schedule build");
    if (hog && c->prebuilt_t == t) {        // built on the side stream during the last epoch
      TRY(join_side(c));
      std::swap(c->chunk_order, c->chunk_order_alt);
      c->sched_built_for = t;
    } else {
      TRY(build_schedule(c, t));
    }
    c->prebuilt_t = -1;
  }
  if (hog) {
    if (!c->ev_ss_go) CUDA_TRY(c, cudaEventCreateWithFlags(&c->ev_ss_go, cudaEventDisableTiming));
    CUDA_TRY(c, cudaEventRecord(c->ev_ss_go, c->st));
  }
  CUDA_TRY(c, cudaEventRecord(c->ev_s1, c->st));
  if (c->libmf) {
    const int64_t nb = (int64_t)c->a * c->ac;
    const int rem = (int)nb;
    CUDA_TRY(c, cudaMemsetAsync(c->lm_lock, 0, 4, c->st));
    CUDA_TRY(c, cudaMemsetAsync(c->lm_row, 0, (size_t)c->a * 4, c->st));
    CUDA_TRY(c, cudaMemsetAsync(c->lm_col, 0, (size_t)c->a * 4, c->st));
    CUDA_TRY(c, cudaMemsetAsync(c->lm_done, 0, (size_t)nb * 4, c->st));
    CUDA_TRY(c, cudaMemcpyAsync(c->lm_rem, &rem, 4, cudaMemcpyHostToDevice, c->st));
    LibmfLaunch L{};
    L.storage = c->p.storage; L.k = c->k; L.slots = c->slots; L.blk_off = c->d_blk_off;
    L.blk_len = c->d_blk_len; L.a = c->a; L.lock = c->lm_lock; L.row_busy = c->lm_row;
    L.col_busy = c->lm_col; L.done = c->lm_done; L.remaining = c->lm_rem;
    L.workers = c->p.workers > 0 ? c->p.workers : std::max(1, c->a / 2);
    L.P = c->P; L.Q = c->Q; L.g = g; L.lp = c->p.lambda_p; L.lq = c->p.lambda_q;
    L.exact = c->p.exact_order;
    L.seed = make_stream(c->p.seed, 11, (uint64_t)t, 0); L.stream = c->st; L.out_lanes = &c->last_lanes;
    L.visits = c->visits; L.upd = c->upd_dev;
    CUDA_TRY(c, cudaEventRecord(ev_at(c, 0), c->st));
    CUDA_TRY(c, launch_libmf(L));
    CUDA_TRY(c, cudaEventRecord(ev_at(c, 1), c->st));
    CUDA_TRY(c, cudaStreamSynchronize(c->st));   // the host-side copy of `rem` must outlive it
    c->n_sgd = 1;
    c->n_launch += 1;
    c->last_workers = L.workers;
    c->last_q_l1 = 0;
    c->last_grid = L.workers;
    c->last_block = 32;
    CUDA_TRY(c, cudaEventRecord(c->ev_e1, c->st));
    c->t = t + 1;
    ++c->epochs_run;
    c->have_stats = true;
    if (epoch_done) *epoch_done = c->t;
    return MF_OK;
  }
  TRY(c->pq ? train_epoch_pq(c, t, g)
             : rows_one_launch(c) ? train_epoch_rows(c, t, g) : train_epoch_strata(c, t, g));
  CUDA_TRY(c, cudaEventRecord(c->ev_e1, c->st));
  if (hog) TRY(prebuild_schedule(c, t + 1));   // enqueued after this epoch's SGD launches
  c->t = t + 1;
  ++c->epochs_run;
  c->have_stats = true;
  if (epoch_done) *epoch_done = c->t;
  return MF_OK;
}

mf_status mf_get_launch_ms(mf_ctx* c, double* ms, int64_t* n) {
  if (!c || !n) return MF_E_INVAL;
  TRY(c->enter());
  const int64_t cnt = c->have_stats ? c->n_sgd : 0;
  if (!ms) {
    *n = cnt;
    return MF_OK;
  }
  if (*n < cnt) return MF_E_INVAL;
  *n = cnt;
  if (cnt == 0) return MF_OK;
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  for (int64_t i = 0; i < cnt; ++i) {
    float x = 0.f;
    CUDA_TRY(c, cudaEventElapsedTime(&x, c->ev[(size_t)(2 * i)], c->ev[(size_t)(2 * i + 1)]));
    ms[i] = x;
  }
  return MF_OK;
}

mf_status mf_get_stats(mf_ctx* c, mf_stats* out) {
  if (!c || !out) return MF_E_INVAL;
  TRY(c->enter());
  std::memset(out, 0, sizeof *out);
  if (!c->have_stats) return MF_OK;
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  float ms = 0.f;
  CUDA_TRY(c, cudaEventElapsedTime(&ms, c->ev_e0, c->ev_e1));
  out->epoch_ms = ms;
  CUDA_TRY(c, cudaEventElapsedTime(&ms, c->ev_s0, c->ev_s1));
  out->sched_ms = ms;
  double sgd = 0.0;
  for (int i = 0; i < c->n_sgd; ++i) {
    CUDA_TRY(c, cudaEventElapsedTime(&ms, c->ev[(size_t)(2 * i)], c->ev[(size_t)(2 * i + 1)]));
    sgd += ms;
  }
  out->sgd_ms = sgd;
  out->comm_ms = std::max(0.0, out->epoch_ms - out->sched_ms - sgd);
  out->sgd_launches = c->n_sgd;
  out->launches = c->n_launch;
  unsigned long long upd = 0;     // counted by the SGD kernels themselves (non-sentinel samples)
  CUDA_TRY(c, cudaMemcpyAsync(&upd, c->upd_dev, 8, cudaMemcpyDeviceToHost, c->st));
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  out->updates = (int64_t)upd;
  out->bytes_per_update = 12 + 4 * (int64_t)c->k * c->ssize() + (c->GP ? 16 * (int64_t)c->k : 0);
  out->h2d_bytes = c->h2d_bytes;
  out->workers = c->last_workers;
  out->lanes = c->last_lanes;
  out->q_l1 = c->last_q_l1;
  out->grid = c->last_grid;
  out->block = c->last_block;
  return MF_OK;
}

mf_status mf_check_visits(mf_ctx* c, int64_t* bad_units, int64_t* units, int32_t* epochs) {
  if (!c || !bad_units) return MF_E_INVAL;
  TRY(c->enter());
  if (!c->train_loaded) return c->fail(MF_E_STATE, "no train set loaded");
  CUDA_TRY(c, cudaMemsetAsync(c->chk_dev, 0, 8, c->st));
  const unsigned e = (unsigned)c->epochs_run;
  if (c->wf) {
    // a strata block's s*c sub-blocks are visited once per epoch when the rank trains the block
    // (it owns the row segment and the block holds ratings); the others never
    const int64_t per = (int64_t)c->s * c->c, nb = (int64_t)c->a * c->ac;
    for (int64_t b = 0; b < nb; ++b)
      CUDA_TRY(c, launch_visit_check(c->visits + b * per, per, c->blk_len[(size_t)b] > 0 ? e : 0u,
                                     c->chk_dev, c->num_sms, c->st));
  } else {
    CUDA_TRY(c, launch_visit_check(c->visits, c->n_units, e, c->chk_dev, c->num_sms, c->st));
  }
  unsigned long long h = 0;
  CUDA_TRY(c, cudaMemcpyAsync(&h, c->chk_dev, 8, cudaMemcpyDeviceToHost, c->st));
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  *bad_units = (int64_t)h;
  if (units) *units = c->n_units;
  if (epochs) *epochs = c->epochs_run;
  return MF_OK;
}

// ---------------------------------------------------------------------------------------------
// rmse / factors
// ---------------------------------------------------------------------------------------------
mf_status mf_rmse(mf_ctx* c, int32_t set, double* out) {
  if (!c || !out) return MF_E_INVAL;
  TRY(c->enter());
  if (!c->train_loaded) return c->fail(MF_E_STATE, "no train set loaded");
  const Rating* data;
  int64_t N;
  if (set == MF_TEST) {
    if (!c->test_loaded) return c->fail(MF_E_STATE, "no test set loaded");
    data = c->test;
    N = c->Ntest;
  } else if (set == MF_TRAIN) {
    data = c->slots;  // sentinel pad slots (u < 0) are skipped by the kernel
    N = c->nslots;
  } else {
    return c->fail(MF_E_INVAL, "bad set");
  }
  if (set == MF_TRAIN && (c->G > 1 || c->staged))
    return c->fail(MF_E_UNSUPPORTED, "train-set RMSE needs resident single-GPU ratings");
  Nvtx range("mf_rmse(%s)", set == MF_TRAIN ? "train" : "test");
  if (c->pq) {
    // P out of core: one staged row segment at a time (after the epoch's last write-back)
    CUDA_TRY(c, cudaStreamSynchronize(c->ds));
    const size_t rowb = (size_t)c->k * c->ssize();
    double sse = 0.0;
    for (int r = 0; r < c->a; ++r) {
      const int64_t t0 = c->test_seg_off.empty() ? 0 : c->test_seg_off[(size_t)r];
      const int64_t tn = c->test_seg_off.empty() ? 0 : c->test_seg_off[(size_t)r + 1] - t0;
      if (tn == 0) continue;
      const int64_t lo = cdiv64((int64_t)r * c->m, c->a), hi = cdiv64((int64_t)(r + 1) * c->m, c->a);
      CUDA_TRY(c, cudaMemcpyAsync(c->Pslot[0], c->h_P + (size_t)lo * rowb, (size_t)(hi - lo) * rowb,
                                  cudaMemcpyHostToDevice, c->st));
      RmseLaunch L{};
      L.storage = c->p.storage; L.k = c->k; L.test = data + t0; L.N = tn;
      L.P = c->Pslot[0] - (size_t)lo * rowb; L.Q = c->Q;
      L.partial = c->rm_partial; L.out = c->rm_out; L.num_sms = c->num_sms; L.stream = c->st;
      CUDA_TRY(c, launch_rmse(L));
      double h = 0.0;
      CUDA_TRY(c, cudaMemcpyAsync(&h, c->rm_out, 8, cudaMemcpyDeviceToHost, c->st));
      CUDA_TRY(c, cudaStreamSynchronize(c->st));
      sse += h;
    }
    const double rmse = (double)c->p.rating_scale * std::sqrt(sse / std::max((double)N, 1.0));
    *out = N > 0 ? rmse : 0.0;
    if (std::isnan(*out)) return c->fail(MF_E_RANGE, "RMSE is NaN (divergence)");
    return MF_OK;
  }
  // world > 1: every rank evaluates the test samples of the row segments it owns (filtered at
  // load) against a complete Q, then the SSE and count are summed over ranks.
  if (c->G > 1) TRY(gather_q(c));
  RmseLaunch L{};
  L.storage = c->p.storage; L.k = c->k; L.test = data; L.N = N; L.P = c->P; L.Q = c->Q;
  L.partial = c->rm_partial; L.out = c->rm_out; L.num_sms = c->num_sms; L.stream = c->st;
  CUDA_TRY(c, launch_rmse(L));
  double cnt = (double)(set == MF_TRAIN ? c->N : N);
  if (c->G > 1) {
    CUDA_TRY(c, cudaMemcpyAsync(c->rm_out + 1, &cnt, 8, cudaMemcpyHostToDevice, c->st));
    std::string why;
    if (!c->comm->allreduce_sum(c->rm_out, 2, &why)) return c->fail(MF_E_NCCL, "rmse: %s", why.c_str());
  }
  double h2[2] = {0.0, 0.0};
  CUDA_TRY(c, cudaMemcpyAsync(h2, c->rm_out, 16, cudaMemcpyDeviceToHost, c->st));
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  const double sse = h2[0];
  if (c->G > 1) cnt = h2[1];
  const double rmse = (double)c->p.rating_scale * std::sqrt(sse / std::max(cnt, 1.0));
  *out = cnt > 0 ? rmse : 0.0;     // global count when world > 1 (all-reduced above)
  if (std::isnan(*out)) return c->fail(MF_E_RANGE, "RMSE is NaN (divergence)");
  return MF_OK;
}

mf_status mf_owner_violations(mf_ctx* c, int64_t* out) {
  if (!c || !out) return MF_E_INVAL;
  TRY(c->enter());
  if (!c->train_loaded) return c->fail(MF_E_STATE, "no train set loaded");
  if (!c->own_viol) return c->fail(MF_E_STATE, "create the ctx with check_owners = 1 (wavefront)");
  unsigned h = 0;
  CUDA_TRY(c, cudaMemcpyAsync(&h, c->own_viol, 4, cudaMemcpyDeviceToHost, c->st));
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  *out = h;
  return MF_OK;
}

mf_status mf_loss(mf_ctx* c, double* out) {
  if (!c || !out) return MF_E_INVAL;
  TRY(c->enter());
  if (!c->train_loaded) return c->fail(MF_E_STATE, "no train set loaded");
  if (c->staged) return c->fail(MF_E_UNSUPPORTED, "the loss needs resident ratings");
  Nvtx range("mf_loss");
  if (c->G > 1) TRY(gather_q(c));
  RmseLaunch L{};
  L.storage = c->p.storage; L.k = c->k; L.test = c->slots; L.N = c->nslots; L.P = c->P; L.Q = c->Q;
  L.partial = c->rm_partial; L.out = c->rm_out; L.num_sms = c->num_sms; L.stream = c->st;
  L.loss = 1; L.lp = c->p.lambda_p; L.lq = c->p.lambda_q;
  CUDA_TRY(c, launch_rmse(L));
  if (c->G > 1) {                        // every rank holds the ratings of its own row segments
    std::string why;
    if (!c->comm->allreduce_sum(c->rm_out, 1, &why)) return c->fail(MF_E_NCCL, "loss: %s", why.c_str());
  }
  double h = 0.0;
  CUDA_TRY(c, cudaMemcpyAsync(&h, c->rm_out, 8, cudaMemcpyDeviceToHost, c->st));
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  *out = h;
  if (std::isnan(h)) return c->fail(MF_E_RANGE, "loss is NaN (divergence)");
  return MF_OK;
}

template <typename T>
static void unrelabel_t(mf_ctx* c, const void* X, const int32_t* rho, int64_t rows, float* out) {
  k_unrelabel<T><<<grid_for(rows * c->k, c->num_sms), 256, 0, c->st>>>((const T*)X, rho, rows, c->k, out);
}
template <typename T>
static void relabel_store_t(mf_ctx* c, void* X, const int32_t* rho, int64_t rows, const float* in) {
  k_relabel_store<T><<<grid_for(rows * c->k, c->num_sms), 256, 0, c->st>>>((T*)X, rho, rows, c->k, in);
}

static mf_status get_one(mf_ctx* c, const void* X, const int32_t* rho, int64_t rows, float* dst,
                         int on_device) {
  float* d = dst;
  if (!on_device) TRY(c->alloc(&d, (size_t)(rows * c->k)));
  switch (c->p.storage) {
    case MF_FP32: unrelabel_t<float>(c, X, rho, rows, d); break;
    case MF_FP16: unrelabel_t<__half>(c, X, rho, rows, d); break;
    default: unrelabel_t<__nv_bfloat16>(c, X, rho, rows, d); break;
  }
  KERNEL_TRY(c);
  if (!on_device) {
    CUDA_TRY(c, cudaMemcpyAsync(dst, d, (size_t)(rows * c->k) * 4, cudaMemcpyDeviceToHost, c->st));
    CUDA_TRY(c, cudaStreamSynchronize(c->st));
    c->release(d);
  }
  return MF_OK;
}

template <typename X>
static mf_status d2h(mf_ctx* c, std::vector<X>& h, const X* d, int64_t n) {
  h.resize((size_t)std::max<int64_t>(n, 1));
  if (n > 0) CUDA_TRY(c, cudaMemcpyAsync(h.data(), d, (size_t)n * sizeof(X), cudaMemcpyDeviceToHost, c->st));
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  return MF_OK;
}

// staged == 2: P is a host array in relabelled row order and storage type; convert on the host
// (model_shuffle, Alg. 1 l.15) -- the same values get_one produces on the device.
template <typename T> static float host_f32(T x);
template <> float host_f32<float>(float x) { return x; }
template <> float host_f32<__half>(__half x) { return __half2float(x); }
template <> float host_f32<__nv_bfloat16>(__nv_bfloat16 x) { return __bfloat162float(x); }
template <typename T> static T host_from_f32(float x);
template <> float host_from_f32<float>(float x) { return x; }
template <> __half host_from_f32<__half>(float x) { return __float2half_rn(x); }
template <> __nv_bfloat16 host_from_f32<__nv_bfloat16>(float x) { return __float2bfloat16_rn(x); }

template <typename T>
static void host_p_copy(mf_ctx* c, const std::vector<int32_t>& rho, float* out, const float* in) {
  const T* X = reinterpret_cast<const T*>(c->h_P);
  T* Y = reinterpret_cast<T*>(c->h_P);
  const int64_t k = c->k;
  for (int64_t id = 0; id < c->m; ++id) {
    const int64_t row = (int64_t)rho[(size_t)id] * k;
    for (int64_t d = 0; d < k; ++d) {
      if (out) out[id * k + d] = host_f32<T>(X[row + d]);
      else Y[row + d] = host_from_f32<T>(in[id * k + d]);
    }
  }
}

static mf_status pq_p_io(mf_ctx* c, float* out, const float* in, int on_device) {
  CUDA_TRY(c, cudaStreamSynchronize(c->ds));
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  std::vector<int32_t> rho;
  TRY(d2h(c, rho, c->rho_r, c->m));
  const size_t bytes = (size_t)(c->m * c->k) * 4;
  std::vector<float> stage;
  float* hout = out;
  const float* hin = in;
  if (on_device) {
    stage.resize((size_t)(c->m * c->k));
    if (in) {
      CUDA_TRY(c, cudaMemcpy(stage.data(), in, bytes, cudaMemcpyDeviceToHost));
      hin = stage.data();
    } else {
      hout = stage.data();
    }
  }
  switch (c->p.storage) {
    case MF_FP32: host_p_copy<float>(c, rho, hout, hin); break;
    case MF_FP16: host_p_copy<__half>(c, rho, hout, hin); break;
    default: host_p_copy<__nv_bfloat16>(c, rho, hout, hin); break;
  }
  if (on_device && out) CUDA_TRY(c, cudaMemcpy(out, stage.data(), bytes, cudaMemcpyHostToDevice));
  return MF_OK;
}

mf_status mf_get_factors(mf_ctx* c, float* P, float* Q, int32_t on_device) {
  if (!c) return MF_E_INVAL;
  TRY(c->enter());
  if (!c->train_loaded) return c->fail(MF_E_STATE, "no train set loaded");
  if (c->pq) {
    if (P) TRY(pq_p_io(c, P, nullptr, on_device));
    if (Q) TRY(get_one(c, c->Q, c->rho_c, c->n, Q, on_device));
    CUDA_TRY(c, cudaStreamSynchronize(c->st));
    return MF_OK;
  }
  if (c->G > 1) {
    TRY(gather_q(c));
    std::string why;
    const size_t row_bytes = (size_t)c->k * c->ssize();
    if (!c->comm->gather_rows(c->P, c->m, c->a, c->G, row_bytes, &why))
      return c->fail(MF_E_NCCL, "P gather: %s", why.c_str());
  }
  if (P) TRY(get_one(c, c->P, c->rho_r, c->m, P, on_device));
  if (Q) TRY(get_one(c, c->Q, c->rho_c, c->n, Q, on_device));
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  return MF_OK;
}

static mf_status set_one(mf_ctx* c, void* X, const int32_t* rho, int64_t rows, const float* src,
                         int on_device) {
  const float* d = src;
  float* own = nullptr;
  if (!on_device) {
    TRY(c->alloc(&own, (size_t)(rows * c->k)));
    CUDA_TRY(c, cudaMemcpyAsync(own, src, (size_t)(rows * c->k) * 4, cudaMemcpyHostToDevice, c->st));
    d = own;
  }
  switch (c->p.storage) {
    case MF_FP32: relabel_store_t<float>(c, X, rho, rows, d); break;
    case MF_FP16: relabel_store_t<__half>(c, X, rho, rows, d); break;
    default: relabel_store_t<__nv_bfloat16>(c, X, rho, rows, d); break;
  }
  KERNEL_TRY(c);
  if (own) {
    CUDA_TRY(c, cudaStreamSynchronize(c->st));
    c->release(own);
  }
  return MF_OK;
}

mf_status mf_set_factors(mf_ctx* c, const float* P, const float* Q, int32_t on_device) {
  if (!c) return MF_E_INVAL;
  TRY(c->enter());
  if (!c->train_loaded) return c->fail(MF_E_STATE, "no train set loaded");
  if (c->pq && P) {
    TRY(pq_p_io(c, nullptr, P, on_device));
    P = nullptr;
  }
  if (P) TRY(set_one(c, c->P, c->rho_r, c->m, P, on_device));
  if (Q) TRY(set_one(c, c->Q, c->rho_c, c->n, Q, on_device));
  if (c->G > 1 && Q) c->comm->reset_holders(c->a);  // every rank holds a valid copy again
  CUDA_TRY(c, cudaStreamSynchronize(c->st));
  return MF_OK;
}

mf_status mf_set_epoch(mf_ctx* c, int32_t t) {
  if (!c || t < 0) return MF_E_INVAL;
  c->t = t;
  return MF_OK;
}
mf_status mf_get_epoch(const mf_ctx* c, int32_t* t) {
  if (!c || !t) return MF_E_INVAL;
  *t = c->t;
  return MF_OK;
}

// ---------------------------------------------------------------------------------------------
// exports
// ---------------------------------------------------------------------------------------------

mf_status mf_export_schedule(mf_ctx* c, int32_t what, int32_t epoch, int64_t* buf, int64_t* len) {
  if (!c || !len) return MF_E_INVAL;
  TRY(c->enter());
  if (!c->train_loaded) return c->fail(MF_E_STATE, "no train set loaded");
  const int64_t nb = (int64_t)c->a * c->ac;
  int64_t need = 0;
  if ((what == MF_EX_PERM && !c->perm) || (what == MF_EX_BLOCKID && !c->slot_pos))
    return c->fail(MF_E_UNSUPPORTED, "per-sample index maps are not kept (staged mode or N > 2^30)");
  switch (what) {
    case MF_EX_PERM: case MF_EX_BLOCKID: need = c->N; break;
    case MF_EX_RHO_R: need = c->m; break;
    case MF_EX_RHO_C: need = c->n; break;
    case MF_EX_CHUNKORDER:
      if (c->wf) return c->fail(MF_E_INVAL, "no chunk order in wavefront mode");
      need = c->ch_off.back();
      break;
    case MF_EX_WFSEQ: case MF_EX_TICKETS:
      if (!c->wf) return c->fail(MF_E_INVAL, "no wavefront schedule in Hogwild mode");
      need = nb * c->s * (int64_t)c->c;
      break;
    case MF_EX_STRATA: need = c->a; break;
    default: return c->fail(MF_E_INVAL, "unknown export %d", what);
  }
  if (!buf) { *len = need; return MF_OK; }
  if (*len < need) return c->fail(MF_E_INVAL, "buffer too small (%lld < %lld)", (long long)*len, (long long)need);
  *len = need;
  switch (what) {
    case MF_EX_PERM: {
      std::vector<uint32_t> h;
      TRY(d2h(c, h, c->perm, c->N));
      for (int64_t j = 0; j < c->N; ++j) buf[j] = h[(size_t)j];
      return MF_OK;
    }
    case MF_EX_RHO_R: case MF_EX_RHO_C: {
      std::vector<int32_t> h;
      const int64_t n = what == MF_EX_RHO_R ? c->m : c->n;
      TRY(d2h(c, h, what == MF_EX_RHO_R ? c->rho_r : c->rho_c, n));
      for (int64_t j = 0; j < n; ++j) buf[j] = h[(size_t)j];
      return MF_OK;
    }
    case MF_EX_BLOCKID: {
      std::vector<uint32_t> pos;
      TRY(d2h(c, pos, c->slot_pos, c->nslots));
      if (!c->wf) {
        for (int64_t b = 0; b < nb; ++b)
          for (int64_t x = c->blk_off[(size_t)b]; x < c->blk_off[(size_t)b] + c->blk_len[(size_t)b]; ++x)
            buf[pos[(size_t)x]] = b;
      } else {
        std::vector<int64_t> off;
        TRY(d2h(c, off, c->sub_off, nb * c->s * (int64_t)c->c + 1));
        for (int64_t q = 0; q < nb * c->s * (int64_t)c->c; ++q)
          for (int64_t x = off[(size_t)q]; x < off[(size_t)q + 1]; ++x) buf[pos[(size_t)x]] = q;
      }
      return MF_OK;
    }
    case MF_EX_CHUNKORDER: {
      TRY(build_schedule(c, epoch));
      std::vector<uint32_t> h;
      TRY(d2h(c, h, c->chunk_order, need));
      for (int64_t b = 0; b < nb; ++b)
        for (int64_t x = c->ch_off[(size_t)b]; x < c->ch_off[(size_t)b + 1]; ++x)
          buf[x] = (int64_t)h[(size_t)x] - c->ch_off[(size_t)b];
      return MF_OK;
    }
    case MF_EX_WFSEQ: case MF_EX_TICKETS: {
      TRY(build_schedule(c, epoch));
      std::vector<int32_t> h;
      TRY(d2h(c, h, what == MF_EX_WFSEQ ? c->seq : c->rank_arr, need));
      for (int64_t x = 0; x < need; ++x) buf[x] = h[(size_t)x];
      return MF_OK;
    }
    case MF_EX_STRATA: {
      std::vector<int64_t> pi = host_perm(make_stream(c->p.seed, kTagStrata, (uint64_t)epoch, 0), c->a);
      for (int64_t x = 0; x < c->a; ++x) buf[x] = pi[(size_t)x];
      return MF_OK;
    }
  }
  return MF_E_INVAL;
}

