// mf_internal.h -- internal launch descriptors shared by mf_api.cu, mf_prep.cu, mf_kernels.cu.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "mf_common.cuh"
#include "mf_sgd.cuh"

namespace mfb {

constexpr int kMaxSegs = 16;  // blocks per Hogwild launch: a/G <= 16 (checked by mf_create)

// Chunk list of one Hogwild launch: segment s is chunks[begin[s] .. begin[s] + prefix[s+1]-prefix[s]).
struct ChunkSegs {
  int64_t begin[kMaxSegs];
  int64_t prefix[kMaxSegs + 1];
  int64_t shift[kMaxSegs];  // slot of chunk q = q*f + shift (0 resident; staged: buffer offset)
  int n;
  // Claim order interleaves the segments (a stratum's blocks touch disjoint P and Q rows, so
  // any interleaving gives the same result as running them one after another): level l covers
  // claim positions [lev_base[l], lev_base[l+1]) and chunk indices [lev_lo[l], ...) of the
  // lev_cnt[l] segments lev_seg[l][0..cnt) that are still that long, round-robin.  Built by
  // finalize_segs() (mf_api.cu).
  int nlev;
  int64_t lev_base[kMaxSegs + 1];
  int64_t lev_lo[kMaxSegs];
  int32_t lev_cnt[kMaxSegs];
  int8_t lev_seg[kMaxSegs][kMaxSegs];
};

struct HogwildLaunch {
  int storage, k, lane_bytes, prefetch;
  int rating_stage;         // 0 = per-lane streaming loads + shuffles, 1 = TMA bulk copies
  int group;                // params.group_cols: column-grouped batches (R24)
  int q_l1;                 // params.q_cache == 0: q_v loads through L1 where the kernel has it (R28)
  const Rating* slots;
  const uint32_t* chunks;
  ChunkSegs segs;
  unsigned long long* counter;
  int workers, num_sms, f;
  void *P, *Q;
  float g, lp, lq;
  int exact;                // params.exact_order (Step)
  AdaArgs ada;              // ada.GP != nullptr: ADAGRAD (g = alpha)
  unsigned* visits;         // per global chunk id: claims (one atomic per claimed chunk)
  unsigned long long* upd;  // non-sentinel samples updated (device count, Eq. 7)
  cudaStream_t stream;
  int *out_workers, *out_lanes, *out_grid;
  int* out_q_l1;            // 1 if the launched kernel read q_v through L1
};

// The strata blocks one wavefront launch runs concurrently (a stratum's blocks touch disjoint
// rows and columns): worker w of the launch is worker w % s of block w / s.
struct WfBlocks {
  int n;
  int64_t base[kMaxSegs];   // b * s * c: offset of the block's sub_off / seq / rank / visits
  int64_t shift[kMaxSegs];  // slot shift of the block (0 resident; staged: buffer offset - start)
};

struct WavefrontLaunch {
  int storage, k, variant;  // variant 1 = ring-staged k_wavefront2 (needs dup), 0 = k_wavefront
  int lane_bytes;           // ring kernel: 16 (default) or 32 bytes per lane
  const Rating* slots;
  WfBlocks blocks;          // the blocks of this launch (tickets / owners: c per block, in order)
  const uint16_t* dup;     // per slot: distance to previous same-u (low byte) / same-v (high
                           // byte) sample of the sub-block if <= ring_window(), else 0
  const int64_t* sub_off;  // s*c + 1 slot offsets of this strata block's sub-blocks
  const int32_t* seq;      // s*c
  const int32_t* rank;     // s*c
  int* tickets;            // c
  int s, c, num_sms;
  void *P, *Q;
  float g, lp, lq;
  int exact;                // params.exact_order (Step)
  AdaArgs ada;              // ada.GP != nullptr: ADAGRAD (register kernel; g = alpha)
  long long* prof;          // diagnostics (MF_PROFILE_WAVES): per worker {wait, run, samples, smid, warpid, release
                            // fence} clock64 totals, or nullptr
  unsigned* visits;         // s*c per strata block: visits of sub-block (i, j) (one atomic per wave)
  unsigned long long* upd;  // samples updated (device count)
  int* owners;              // params.check_owners: c column tags (-1 = free), else nullptr
  unsigned* viol;           // mutual-exclusion violations found by the checker
  cudaStream_t stream;
  int *out_lanes, *out_grid;
};

struct RmseLaunch {
  int storage, k;
  const Rating* test;
  int64_t N;
  const void *P, *Q;
  double* partial;  // num_sms*4
  double* out;      // 1
  int loss;         // 1: Eq. 2 (squared error + lp ||p||^2 + lq ||q||^2) instead of squared error
  float lp, lq;
  int num_sms;
  cudaStream_t stream;
};

struct LibmfLaunch {
  int storage, k;
  const Rating* slots;
  const int64_t *blk_off, *blk_len;  // a*a padded block starts / sample counts
  int a;
  int *lock, *row_busy, *col_busy, *done, *remaining;
  int workers;
  void *P, *Q;
  float g, lp, lq;
  int exact;                // params.exact_order (Step)
  uint64_t seed;
  unsigned* visits;         // a*a: claims of each block
  unsigned long long* upd;  // samples updated (device count)
  cudaStream_t stream;
  int* out_lanes;
};

cudaError_t launch_hogwild(const HogwildLaunch& a);
cudaError_t launch_libmf(const LibmfLaunch& a);
cudaError_t launch_wavefront(const WavefrontLaunch& a);
cudaError_t launch_rmse(const RmseLaunch& a);
// number of entries of visits[0, n) that differ from `expect`, into *out (device)
cudaError_t launch_visit_check(const unsigned* visits, int64_t n, unsigned expect,
                               unsigned long long* out, int num_sms, cudaStream_t st);
int ring_window(int k, int storage, int lane_bytes);  // history window W of k_wavefront2

}  // namespace mfb
