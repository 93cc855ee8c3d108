// mf_kernels.cu -- SGD kernels (batch-Hogwild!, wavefront) and the RMSE kernel, with the
// runtime dispatch over (k, storage, lanes) template instantiations.
#include <cuda_runtime.h>

#include "mf_internal.h"
#include "mf_sgd.cuh"

namespace mfb {

// wavefront ring geometry per (k, storage): rows of K*S bytes, 16 B per lane.  Prefetch F
// samples ahead in a ring of RS slots (history window W = RS - F - 1); deep (32/15) when a
// worker's ring fits in 32 KB, else 16/7.  The ring kernel needs F < L (lanes per worker).
constexpr int ring_lanes(int K, int S) { return (K * S / 16) >= 32 ? 32 : (K * S / 16); }
constexpr int ring_slots(int K, int S) {
  return (32 * 2 * K * S <= 32768 && ring_lanes(K, S) > 15) ? 32 : 16;
}
constexpr int ring_ahead(int K, int S) { return ring_slots(K, S) == 32 ? 15 : 7; }
// Narrow-slice full-warp ring (default for k*S = 128 or 256 bytes): 32 lanes of 4 or 8 B
// (cp.async.ca row copies), RS = 32, F = 15 -- the full-batch RS == L path and the
// integer-reduction group sum of the 32-lane geometry.
constexpr bool narrow_ring(int K, int S) { return K * S == 128 || K * S == 256; }
// 64-byte rows (fp16 k = 32, fp32 k = 16): 16 lanes of 4 B, RS = 16, F = 7 (RS == L again).
constexpr bool narrow16_ring(int K, int S) { return K * S == 64; }

// ---------------------------------------------------------------------------------------------
// batch-Hogwild! (section 5.1).  A worker is a group of L lanes; a warp holds
// 32/L workers which claim consecutive entries of the epoch's chunk list with ONE atomicAdd per
// warp (the only scheduling synchronisation, "lock-free"), then each worker updates the
// f consecutive slots of its chunk serially.  Persistent grid: workers loop until the list is
// exhausted.  The chunk list of a launch is the concatenation of up to kMaxSegs block segments.
// ---------------------------------------------------------------------------------------------
// 5 resident blocks (40 warps) per SM: 48 registers, a few bytes of stack.  Yahoo-shaped
// (DRAM-bound) 34.9 -> 33.8 ms/epoch against 4 blocks at 64 registers, Netflix unchanged (hot
// rows); the ADAGRAD, depth-2 and 32-B-per-lane variants keep the compiler's choice.
// LC: cache policy of the Hogwild row accesses (bit 0: q_v loads via L1, bit 1: p_u loads via
// L1, bit 2: q_v stores .wb, bit 3: p_u stores .wb).  0 = L2 only (.cg); kLcQ = q_v through L1
// (params.q_cache = 0, reading R28).  Measured on B200 (profiles/r02_q_l1.md): q_v via L1 is
// Netflix fp16 13.99 -> 11.63 ms, k = 32 9.09 -> 7.16 ms, Yahoo unchanged; p_u via L1 as well
// is slower (12.04 ms: p_u rows have no reuse and evict the hot q_v lines).
constexpr int kLcQ = 5;
#ifndef MF_HOG_MINB
#define MF_HOG_MINB 5
#endif
#ifndef MF_HOG_MINB_D2
#define MF_HOG_MINB_D2 1
#endif
// The column-grouped instantiation runs the batch-unrolled loop (mf_sgd.cuh, MF_BATCH_UNROLL) and
// is fastest at 4 blocks (64 registers): Netflix grouped f = 1024 10.62 -> 10.12 ms, on the 4 x 1
// row blocks 9.69 -> 9.29 ms, k = 32 7.09 -> 5.93 ms (profiles/r02_grouped_batches.md); the
// plain rolled kernel gains nothing from 64 registers and Yahoo loses (33.3 -> 35.3 ms).
#ifndef MF_HOG_MINB_GRP
#define MF_HOG_MINB_GRP 4
#endif
template <typename T, int K, int L, int D, bool ADA, bool EX, int SRC, bool GRP, int LC>
__global__ void __launch_bounds__(256, (ADA || K * (int)sizeof(T) / L > 16) ? 1
                                       : D > 1 ? MF_HOG_MINB_D2
                                       : GRP   ? MF_HOG_MINB_GRP : MF_HOG_MINB)
    k_hogwild(const Rating* __restrict__ slots,
                                                 const uint32_t* __restrict__ chunks, ChunkSegs segs,
                                                 unsigned long long* __restrict__ counter,
                                                 int workers, T* __restrict__ P, T* __restrict__ Q,
                                                 int f, Step st, AdaArgs ada,
                                                 unsigned* __restrict__ visits,
                                                 unsigned long long* __restrict__ upd) {
  constexpr int GPW = 32 / L;
  const int lane = threadIdx.x & 31;
  const int grp = lane / L, gl = lane % L, gbase = grp * L;
  const int warp = (int)((blockIdx.x * (unsigned)blockDim.x + threadIdx.x) >> 5);
  const int first = warp * GPW;
  if (first >= workers) return;                      // warp-uniform
  const int nact = min(GPW, workers - first);
  const int64_t total = segs.prefix[segs.n];
  int done = 0;                                      // this group's non-sentinel updates
  // SRC = 1: this group's rating ring in dynamic shared memory (2 mbarriers + 2 x 768 B)
  extern __shared__ __align__(16) char hsm[];
  RatingRing ring{};
  unsigned phase = 0;
  char* rowring = nullptr;                           // SRC = 2: this group's row ring (2F slots)
  if constexpr (SRC == 2) {
    const int gid = (int)(threadIdx.x >> 5) * GPW + grp;
    rowring = hsm + (size_t)gid * 4 * 2 * K * sizeof(T);
  }
  if constexpr (SRC == 1) {
    const int gid = (int)(threadIdx.x >> 5) * GPW + grp;   // group within the CTA
    const int ngroups = (int)(blockDim.x >> 5) * GPW;
    ring.bar = reinterpret_cast<uint64_t*>(hsm) + 2 * gid;
    ring.buf = hsm + 16 * ngroups + 2 * kSubBytes * gid;
    if (gl == 0) {
      mbar_init(ring.bar, 1);
      mbar_init(ring.bar + 1, 1);
      mbar_init_fence();
    }
    __syncwarp();
  }
  for (;;) {
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(counter, (unsigned long long)nact);
    base = __shfl_sync(0xffffffffu, base, 0);
    if ((int64_t)base >= total) break;
    const int64_t ci = (int64_t)base + grp;
    const bool act = grp < nact && ci < total;
    int64_t lo = 0;
    if (act) {                                       // claim position -> (block, chunk)
      int lv = 0;
      while (ci >= segs.lev_base[lv + 1]) ++lv;
      const int64_t pos = ci - segs.lev_base[lv];
      const int cnt = segs.lev_cnt[lv];
      const int sgi = segs.lev_seg[lv][(int)(pos % cnt)];
      const uint32_t chunk = __ldg(chunks + segs.begin[sgi] + segs.lev_lo[lv] + pos / cnt);
      lo = (int64_t)chunk * f + segs.shift[sgi];
      if (gl == 0) atomicAdd(visits + chunk, 1u);    // exactly-once evidence (mf_check_visits)
    }
    // every group of the warp runs f iterations in lockstep (inactive ones on sentinels)
    if constexpr (SRC == 2)
      done += run_chunk_ring<T, K, L, 2, EX>(slots, lo, f, act, P, Q, st, gl, gbase, rowring);
    else
      done += run_serial<T, K, L, D, true, ADA, EX, SRC, GRP, LC>(slots, lo, f, act, P, Q, st, gl, gbase,
                                                         0xffffffffu, ada, ring, &phase);
  }
  if (gl == 0 && done) atomicAdd(upd, (unsigned long long)done);
}

// ---------------------------------------------------------------------------------------------
// Wavefront (section 5.2, Fig. 6).  Worker i (a group of L lanes) owns row
// sub-block i and walks its column sequence seq_i[0..c).  Before wave w it waits on the 1-D
// column array ("column lock array") until the column's ticket equals the precomputed
// rank of visit (w,i) (R10: deterministic (w,i)-lexicographic tie-break), runs the sub-block
// serially, and releases the column with ticket+1.  Every wait is on a lexicographically
// smaller visit, so with all workers co-resident (cooperative launch) there is no deadlock.
// ---------------------------------------------------------------------------------------------
__device__ __forceinline__ int ld_relaxed(const int* p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed(int* p, int v) {
  asm volatile("st.relaxed.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ int ld_acquire(const int* p) {
  int v;
  asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void fence_acq_rel() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
// Release-only fence (PTX 8.6+): MEMBAR.GPU without the L1 invalidate (CCTL.IVALL) of acq_rel;
// a release needs only this thread's prior stores ordered before the ticket store.
__device__ __forceinline__ void fence_release() { asm volatile("fence.release.gpu;" ::: "memory"); }

// Acquire the column: spin with RELAXED loads (an ld.acquire per poll would emit an L1
// invalidate each time and flood L2 with strong loads on the few ticket lines) and exponential
// back-off, then one acquire fence (ld.relaxed + fence.acq_rel = acquire pattern).
__device__ __forceinline__ void ticket_acquire(const int* t, int tgt) {
  unsigned ns = 32;
  while (ld_relaxed(t) != tgt) {
    __nanosleep(ns);
    if (ns < 1024) ns <<= 1;
  }
  fence_acq_rel();
}
// Release: every lane fences its own row stores, the group re-converges (memory ordering among
// the participating lanes), and one lane publishes ticket+1 (fence + relaxed store = release).
__device__ __forceinline__ void ticket_release(int* t, int next, unsigned gmask, int gl) {
  fence_release();
  __syncwarp(gmask);
  if (gl == 0) st_relaxed(t, next);
}

// Debug ownership checker (params.check_owners; SURVEY 5 race detection): a worker tags the
// column block it acquires (atomicCAS from -1) and clears the tag on release (atomicExch back);
// any tag it finds set by another worker, or not its own on release, is a mutual-exclusion
// violation of the ticket protocol on the global P/Q rows (which compute-sanitizer's racecheck,
// shared memory only, cannot see).  Row blocks are private to their worker by construction.
__device__ __forceinline__ void own_acquire(int* owners, unsigned* viol, int col, int worker) {
  if (owners && atomicCAS(owners + col, -1, worker) != -1) atomicAdd(viol, 1u);
}
__device__ __forceinline__ void own_release(int* owners, unsigned* viol, int col, int worker) {
  if (owners && atomicExch(owners + col, -1) != worker) atomicAdd(viol, 1u);
}

template <typename T, int K, int L, bool ADA, bool EX>
__global__ void __launch_bounds__(128) k_wavefront(const Rating* __restrict__ slots,
                                                   const int64_t* __restrict__ sub_off,
                                                   const int32_t* __restrict__ seq,
                                                   const int32_t* __restrict__ rank,
                                                   int* __restrict__ tickets, int s, int c,
                                                   T* __restrict__ P, T* __restrict__ Q, Step st,
                                                   WfBlocks bl, AdaArgs ada,
                                                   unsigned* __restrict__ visits,
                                                   unsigned long long* __restrict__ upd,
                                                   int* __restrict__ owners,
                                                   unsigned* __restrict__ viol) {
  const int lane = threadIdx.x & 31;
  const int grp = lane / L, gl = lane % L, gbase = grp * L;
  const unsigned gmask = (L == 32) ? 0xffffffffu : (((1u << L) - 1u) << gbase);
  const int gw = (int)((blockIdx.x * (unsigned)blockDim.x + threadIdx.x) / L);
  if (gw >= s * bl.n) return;
  const int bi = gw / s, worker = gw - bi * s;      // block of the launch, worker in the block
  const int64_t shift = bl.shift[bi];
  sub_off += bl.base[bi];
  seq += bl.base[bi];
  rank += bl.base[bi];
  visits += bl.base[bi];
  tickets += (int64_t)bi * c;
  if (owners) owners += (int64_t)bi * c;
  const int32_t* my_seq = seq + (int64_t)worker * c;
  const int32_t* my_rank = rank + (int64_t)worker * c;
  int done = 0;
  for (int w = 0; w < c; ++w) {
    const int col = __ldg(my_seq + w);
    const int tgt = __ldg(my_rank + w);
    ticket_acquire(tickets + col, tgt);
    if (gl == 0) own_acquire(owners, viol, col, worker);
    const int64_t sb = (int64_t)worker * c + col;
    const int64_t lo = __ldg(sub_off + sb) + shift;
    done += run_serial<T, K, L, 2, false, ADA, EX>(slots, lo, (int)(__ldg(sub_off + sb + 1) + shift - lo),
                                               true, P, Q, st, gl, gbase, gmask, ada);
    if (gl == 0) atomicAdd(visits + sb, 1u);
    if (gl == 0) own_release(owners, viol, col, worker);
    ticket_release(tickets + col, tgt + 1, gmask, gl);
  }
  if (gl == 0 && done) atomicAdd(upd, (unsigned long long)done);
}


// Ring-staged wavefront (see run_subblock_ring): same schedule, tickets and result as
// k_wavefront; the rows of each sub-block stream through a per-worker shared-memory ring.
template <typename T, int K, int L, int RS, int F, bool EX>
// Register cap of the ring wavefront.  Under __launch_bounds__(128) ptxas picked 96 registers for
// the fp16/bf16 kernels and spilled 24 B in the per-wave epilogue; the reload then followed the
// acquire fence's L1 invalidate (CCTL.IVALL) and went to L2 on every ticket hand-off.  With a
// cap of 168 (126 used, no stack) on B200: fp16 39.7 -> 34.8 ms, bf16 40.7 -> 36.5 ms, fp16 k = 64
// 31.2 -> 28.8 ms, fp32 unchanged (34.3 -> 34.2 ms) (tools/gpu/run_r02az.sh).  One warp per
// block, 6 blocks per SM: registers do not limit the co-resident worker count.
#ifndef MF_WF_MAXNREG
#define MF_WF_MAXNREG 168
#endif
#if MF_WF_MAXNREG
__global__ void __maxnreg__(MF_WF_MAXNREG) k_wavefront2(
#else
__global__ void __launch_bounds__(128) k_wavefront2(
#endif
                                                    const Rating* __restrict__ slots,
                                                    const uint16_t* __restrict__ dup,
                                                    const int64_t* __restrict__ sub_off,
                                                    const int32_t* __restrict__ seq,
                                                    const int32_t* __restrict__ rank,
                                                    int* __restrict__ tickets, int s, int c,
                                                    T* __restrict__ P, T* __restrict__ Q, Step st,
                                                    WfBlocks bl,
                                                    long long* __restrict__ prof,
                                                    unsigned* __restrict__ visits,
                                                    unsigned long long* __restrict__ upd,
                                                    int* __restrict__ owners,
                                                    unsigned* __restrict__ viol) {
  extern __shared__ __align__(16) char smem[];
  constexpr int ROWB = K * (int)sizeof(T);
  const int lane = threadIdx.x & 31;
  const int grp = lane / L, gl = lane % L, gbase = grp * L;
  const unsigned gmask = (L == 32) ? 0xffffffffu : (((1u << L) - 1u) << gbase);
  // one worker per warp (lanes >= L idle): two workers sharing a warp would diverge (each
  // spins on its own ticket) and serialise each other's instruction streams
  if (lane >= L) return;
  const int local = threadIdx.x >> 5;
  const int gw = blockIdx.x * (blockDim.x >> 5) + local;
  if (gw >= s * bl.n) return;
  const int bi = gw / s, worker = gw - bi * s;      // block of the launch, worker in the block
  const int64_t shift = bl.shift[bi];
  sub_off += bl.base[bi];
  seq += bl.base[bi];
  rank += bl.base[bi];
  visits += bl.base[bi];
  tickets += (int64_t)bi * c;
  if (owners) owners += (int64_t)bi * c;
  char* ring = smem + (size_t)local * RS * 2 * ROWB;
  const int32_t* my_seq = seq + (int64_t)worker * c;
  const int32_t* my_rank = rank + (int64_t)worker * c;
  const int64_t* my_off = sub_off + (int64_t)worker * c;
  // Cross-wave pipeline: a wave's own work is ~20 samples, so its start-up chain (column id ->
  // sub-block offsets -> ratings -> rows, plus the ticket poll) would otherwise cost several
  // dependent memory round trips per wave.  While wave w runs, the next waves' inputs are in
  // flight: column ids and ticket ranks 3 ahead, sub-block offsets 2 ahead, the first rating
  // batches and an ld.acquire of the column ticket 1 ahead.  The rows (which the ticket guards)
  // are read only after an acquire: when the early ld.acquire already shows the ticket, the
  // next sub-block's first F+1 rows are prefetched before this wave's release fence, so the
  // fence's wait and their memory latency overlap (MF_PROFILE_WAVES: the release fence is
  // ~2,800 cycles per wave, a quarter of the epoch).
  auto col_at = [&](int w) { return w < c ? __ldg(my_seq + w) : 0; };
  auto tgt_at = [&](int w) { return w < c ? __ldg(my_rank + w) : 0; };
  int col0 = col_at(0), tgt0 = tgt_at(0);
  int col1 = col_at(1), tgt1 = tgt_at(1);
  int col2 = col_at(2), tgt2 = tgt_at(2);
  int64_t lo0 = __ldg(my_off + col0) + shift;
  int n0 = (int)(__ldg(my_off + col0 + 1) + shift - lo0);
  int64_t lo1 = 0;
  int n1 = 0;
  if (c > 1) {
    lo1 = __ldg(my_off + col1) + shift;
    n1 = (int)(__ldg(my_off + col1 + 1) + shift - lo1);
  }
  RingHead h0 = load_head<L>(slots, dup, lo0, n0, gl);
  bool ready = false;            // column col0 acquired and its ring prologue issued already
  long long t_wait = 0, t_run = 0, t_rel = 0, n_done = 0;
  unsigned long long n_upd = 0;                      // samples updated (no sentinels here)
  for (int w = 0; w < c; ++w) {
    const long long tw0 = prof ? clock64() : 0;
    if (!ready) {
      ticket_acquire(tickets + col0, tgt0);   // relaxed spin + fence.acq_rel
      if (gl == 0) own_acquire(owners, viol, col0, worker);
      if (n0 > 0)
        run_subblock_ring<T, K, L, RS, F, EX>(slots, dup, lo0, n0, h0, P, Q, st, gl, gbase,
                                          gmask, ring, true, false);
    }
    // next waves' inputs
    RingHead h1{};
    if (w + 1 < c) h1 = load_head<L>(slots, dup, lo1, n1, gl);
    int64_t lo2 = 0;
    int n2 = 0;
    if (w + 2 < c) {
      lo2 = __ldg(my_off + col2) + shift;
      n2 = (int)(__ldg(my_off + col2 + 1) + shift - lo2);
    }
    const int col3 = col_at(w + 3), tgt3 = tgt_at(w + 3);
    // early acquire attempt for the next column: an ld.acquire, so if it already shows the
    // ticket the next sub-block's rows may be read from here on (program order)
    const int poll1 = w + 1 < c ? ld_acquire(tickets + col1) : -1;
    const long long tw1 = prof ? clock64() : 0;
    if (n0 > 0)
      run_subblock_ring<T, K, L, RS, F, EX>(slots, dup, lo0, n0, h0, P, Q, st, gl, gbase, gmask,
                                        ring, false, true);
    // next column already released: issue its row prefetch BEFORE this wave's release fence.
    // (Its p rows may have been stored by this sub-block: same thread, issued after them.)
    ready = w + 1 < c && poll1 == tgt1;
    if (ready && gl == 0) own_acquire(owners, viol, col1, worker);
    if (ready && n1 > 0)
      run_subblock_ring<T, K, L, RS, F, EX>(slots, dup, lo1, n1, h1, P, Q, st, gl, gbase, gmask,
                                        ring, true, false);
    const long long tw2 = prof ? clock64() : 0;
    // the claim record before the release: its fence waits for it together with the rows'
    // stores (issued after the release, the next wave's acquire fence would wait for it alone:
    // measured 34.2 -> 36.4 ms on the deterministic Netflix line; without the record 33.8 ms)
    if (gl == 0) atomicAdd(visits + (int64_t)worker * c + col0, 1u);   // sub-block (worker, col0)
    n_upd += n0;
    if (gl == 0) own_release(owners, viol, col0, worker);
    ticket_release(tickets + col0, tgt0 + 1, gmask, gl);   // fence; syncwarp; relaxed store
    if (prof) {
      t_wait += tw1 - tw0;
      t_run += tw2 - tw1;
      t_rel += clock64() - tw2;
      n_done += n0;
    }
    col0 = col1; tgt0 = tgt1; lo0 = lo1; n0 = n1; h0 = h1;
    col1 = col2; tgt1 = tgt2; lo1 = lo2; n1 = n2;
    col2 = col3; tgt2 = tgt3;
  }
  if (gl == 0 && n_upd) atomicAdd(upd, n_upd);
  if (prof && gl == 0) {
    unsigned smid, wid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    asm volatile("mov.u32 %0, %%warpid;" : "=r"(wid));
    long long* o = prof + 6 * (int64_t)gw;
    o[0] = t_wait; o[1] = t_run; o[2] = n_done; o[3] = smid; o[4] = wid; o[5] = t_rel;
  }
}


// ---------------------------------------------------------------------------------------------
// LIBMF-GPU table scheduler (paper section 5, Fig. 5a): the in-tree BASELINE the
// paper's schedulers replace.  R is cut into a x a blocks; a worker (one warp, L active lanes)
// takes the single global lock, scans the table for a block whose row and column are free and
// which has not been updated this epoch (random start, then O(a^2) worst case), marks its row
// and column busy, releases the lock, updates the block serially, and frees its row/column.
// Conflict-free (serialisable) but nondeterministic order; every block once per epoch.
// ---------------------------------------------------------------------------------------------
template <typename T, int K, int L>
__global__ void __launch_bounds__(32) k_libmf(const Rating* __restrict__ slots,
                                              const int64_t* __restrict__ blk_off,
                                              const int64_t* __restrict__ blk_len, int a,
                                              int* lock, int* row_busy, int* col_busy, int* done,
                                              int* remaining, int workers, T* __restrict__ P,
                                              T* __restrict__ Q, Step st,
                                              uint64_t seed, unsigned* __restrict__ visits,
                                              unsigned long long* __restrict__ upd) {
  const int lane = threadIdx.x & 31;
  if (lane >= L) return;
  const int worker = blockIdx.x;
  if (worker >= workers) return;
  const unsigned gmask = (L == 32) ? 0xffffffffu : ((1u << L) - 1u);
  uint64_t draw = mix64(seed + (uint64_t)worker * kPhi);
  unsigned ns = 64;
  int n_upd = 0;
  for (;;) {
    int b = -1;
    if (lane == 0) {
      while (atomicCAS(lock, 0, 1) != 0) __nanosleep(64);
      __threadfence();
      if (*(volatile int*)remaining == 0) {
        b = -2;
      } else {
        draw = mix64(draw + kPhi);
        const int r0 = (int)(draw % (uint64_t)a), c0 = (int)((draw >> 32) % (uint64_t)a);
        for (int dr = 0; dr < a && b < 0; ++dr) {
          const int r = (r0 + dr) % a;
          if (((volatile int*)row_busy)[r]) continue;
          for (int dc = 0; dc < a; ++dc) {
            const int cc = (c0 + dc) % a;
            if (!((volatile int*)col_busy)[cc] && !((volatile int*)done)[r * a + cc]) {
              b = r * a + cc;
              break;
            }
          }
        }
        if (b >= 0) {
          row_busy[b / a] = 1;
          col_busy[b % a] = 1;
          done[b] = 1;
          *remaining -= 1;
        }
      }
      __threadfence();
      atomicExch(lock, 0);
    }
    b = __shfl_sync(gmask, b, 0);
    if (b == -2) break;
    if (b == -1) {                        // nothing independent is free: back off and retry
      __nanosleep(ns);
      if (ns < 4096) ns <<= 1;
      continue;
    }
    ns = 64;
    const int64_t lo = __ldg(blk_off + b);
    if (lane == 0) atomicAdd(visits + b, 1u);
    n_upd += run_serial<T, K, L, 1, false>(slots, lo, (int)__ldg(blk_len + b), true, P, Q, st,
                                           lane, 0, gmask);
    __threadfence();
    __syncwarp(gmask);
    if (lane == 0) {
      atomicExch(row_busy + b / a, 0);
      atomicExch(col_busy + b % a, 0);
    }
  }
  if (lane == 0 && n_upd) atomicAdd(upd, (unsigned long long)n_upd);
}

// ---------------------------------------------------------------------------------------------
// RMSE (R13): per-group fp32 dot, per-lane-0 fp64 accumulation, fixed-order block
// reduction to one partial per CTA; k_rmse_final sums the partials in a fixed order.
// ---------------------------------------------------------------------------------------------
template <typename T, int K, int L>
// loss = 1: Eq. 2 instead: per sample (r - p.q)^2 + lp ||p_u||^2 + lq ||q_v||^2.
__global__ void __launch_bounds__(256) k_rmse_partial(const Rating* __restrict__ test, int64_t N,
                                                      const T* __restrict__ P,
                                                      const T* __restrict__ Q,
                                                      double* __restrict__ partial, int loss,
                                                      float lp, float lq) {
  using G = Geo<T, K, L>;
  constexpr int PW = Pack<T>::kPerWord;
  const int lane = threadIdx.x & 31;
  const int grp = lane / L, gl = lane % L, gbase = grp * L;
  const unsigned gmask = (L == 32) ? 0xffffffffu : (((1u << L) - 1u) << gbase);
  const int gpb = blockDim.x / L;
  const int64_t stride = (int64_t)gridDim.x * gpb;
  double acc = 0.0;
  for (int64_t x = (int64_t)blockIdx.x * gpb + threadIdx.x / L; x < N; x += stride) {
    const int* tp = reinterpret_cast<const int*>(test + x);
    const int u = __ldcs(tp), v = __ldcs(tp + 1);
    const float r = __int_as_float(__ldcs(tp + 2));
    if (u < 0) continue;  // sentinel pad slot (group-uniform)
    Words<G::NW> pw, qw;
    load_row(row_ptr<T, K>(P, u, gl, G::VEC), pw);
    load_row(row_ptr<T, K>(Q, v, gl, G::VEC), qw);
    float p[G::VEC], q[G::VEC];
#pragma unroll
    for (int i = 0; i < G::NW; ++i) {
      Pack<T>::unpack(pw.w[i], p + i * PW);
      Pack<T>::unpack(qw.w[i], q + i * PW);
    }
    float d = 0.f, pp = 0.f, qq = 0.f;
#pragma unroll
    for (int e = 0; e < G::VEC; ++e) {
      d = fmaf(p[e], q[e], d);
      pp = fmaf(p[e], p[e], pp);
      qq = fmaf(q[e], q[e], qq);
    }
#pragma unroll
    for (int o = L / 2; o > 0; o >>= 1) {
      d += __shfl_xor_sync(gmask, d, o);
      if (loss) {
        pp += __shfl_xor_sync(gmask, pp, o);
        qq += __shfl_xor_sync(gmask, qq, o);
      }
    }
    const float e = r - d;
    if (gl == 0) {
      acc += (double)e * (double)e;
      if (loss) acc += (double)lp * (double)pp + (double)lq * (double)qq;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  __shared__ double wsum[32];
  if (lane == 0) wsum[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
    for (int i = 0; i < (int)(blockDim.x >> 5); ++i) s += wsum[i];
    partial[blockIdx.x] = s;
  }
}

__global__ void k_rmse_final(const double* __restrict__ partial, int n, double* __restrict__ out) {
  __shared__ double sm[256];
  double s = 0.0;
  for (int i = threadIdx.x; i < n; i += blockDim.x) s += partial[i];
  sm[threadIdx.x] = s;
  __syncthreads();
  for (int w = blockDim.x / 2; w > 0; w >>= 1) {
    if ((int)threadIdx.x < w) sm[threadIdx.x] += sm[threadIdx.x + w];
    __syncthreads();
  }
  if (threadIdx.x == 0) out[0] = sm[0];
}

// Exactly-once check (Eq. 7: an epoch is N updates): count the work units (Hogwild chunks,
// wavefront sub-blocks, LIBMF blocks) whose claim counter differs from the expected number of
// epochs.  Together with the device update count this shows every sample is updated once per
// epoch: units are disjoint slot ranges, each run over all of its slots.
__global__ void k_visit_check(const unsigned* __restrict__ v, int64_t n, unsigned expect,
                              unsigned long long* __restrict__ out) {
  unsigned long long bad = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    bad += v[i] != expect;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) bad += __shfl_xor_sync(0xffffffffu, bad, o);
  if ((threadIdx.x & 31) == 0 && bad) atomicAdd(out, bad);
}

cudaError_t launch_visit_check(const unsigned* visits, int64_t n, unsigned expect,
                               unsigned long long* out, int num_sms, cudaStream_t st) {
  if (n == 0) return cudaSuccess;   // accumulates into *out (the caller zeroes it)
  int64_t blocks = (n + 255) / 256;
  if (blocks > (int64_t)num_sms * 8) blocks = (int64_t)num_sms * 8;
  k_visit_check<<<(unsigned)blocks, 256, 0, st>>>(visits, n, expect, out);
  return cudaGetLastError();
}

// ---------------------------------------------------------------------------------------------
// Dispatch
// ---------------------------------------------------------------------------------------------
// 1.0f and -0.0f come from here (host), opaque to the device compiler (see Step)
template <typename Launch>
static Step step_of(const Launch& a) {
  return Step{a.g, a.lp, a.lq, 1.0f, -0.0f};
}

template <typename T, int K, int L, int D, bool ADA = false, bool EX = false, int SRC = 0,
          bool GRP = false, int LC = 0>
static cudaError_t launch_hogwild_t(const HogwildLaunch& a) {
  auto kern = k_hogwild<T, K, L, D, ADA, EX, SRC, GRP, LC>;
  if (a.out_q_l1) *a.out_q_l1 = (LC & 1);
  const int threads = 256;
  const int groups = threads / 32 * (32 / L);
  const size_t smem = SRC == 1   ? (size_t)groups * (16 + 2 * kSubBytes)
                      : SRC == 2 ? (size_t)groups * 4 * 2 * K * sizeof(T)
                                 : 0;
  cudaError_t e;
  if (SRC != 0) {
    if (SRC == 1 && a.f % kSub != 0) return cudaErrorInvalidValue;   // mf_create rejects it first
    e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    // the rings need the shared-memory carveout that keeps MF_HOG_MINB blocks resident
    e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout,
                             cudaSharedmemCarveoutMaxShared);
    if (e != cudaSuccess) return e;
  }
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, threads, smem);
  if (e != cudaSuccess) return e;
  const int gpw = 32 / L;
  const int resident_workers = per_sm * a.num_sms * (threads / 32) * gpw;
  int workers = a.workers > 0 ? a.workers : resident_workers;
  int blocks = (int)cdiv64((int64_t)workers, (int64_t)(threads / 32) * gpw);
  if (a.out_workers) *a.out_workers = workers;
  if (a.out_lanes) *a.out_lanes = L;
  if (a.out_grid) *a.out_grid = blocks;
  kern<<<blocks, threads, smem, a.stream>>>(a.slots, a.chunks, a.segs, a.counter, workers,
                                         reinterpret_cast<T*>(a.P), reinterpret_cast<T*>(a.Q), a.f,
                                         step_of(a), a.ada, a.visits, a.upd);
  return cudaGetLastError();
}

template <typename T, int K, int L, bool ADA = false, bool EX = false>
static cudaError_t launch_wavefront_t(const WavefrontLaunch& a) {
  auto kern = k_wavefront<T, K, L, ADA, EX>;
  const int threads = 128;
  const int64_t total_threads = (int64_t)a.s * a.blocks.n * L;
  const int blocks = (int)cdiv64(total_threads, threads);
  int per_sm = 0;
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, threads, 0);
  if (e != cudaSuccess) return e;
  if ((int64_t)per_sm * a.num_sms < blocks) return cudaErrorCooperativeLaunchTooLarge;
  if (a.out_lanes) *a.out_lanes = L;
  if (a.out_grid) *a.out_grid = blocks;
  const Rating* slots = a.slots;
  const int64_t* sub_off = a.sub_off;
  const int32_t* seq = a.seq;
  const int32_t* rank = a.rank;
  int* tickets = a.tickets;
  int s = a.s, c = a.c;
  T* P = reinterpret_cast<T*>(a.P);
  T* Q = reinterpret_cast<T*>(a.Q);
  Step st = step_of(a);
  WfBlocks bl = a.blocks;
  AdaArgs ada = a.ada;
  unsigned* visits = a.visits;
  unsigned long long* upd = a.upd;
  int* owners = a.owners;
  unsigned* viol = a.viol;
  void* args[] = {&slots, &sub_off, &seq, &rank, &tickets, &s, &c, &P, &Q, &st, &bl,
                  &ada, &visits, &upd, &owners, &viol};
  return cudaLaunchCooperativeKernel(reinterpret_cast<void*>(kern), blocks, threads, args, 0,
                                     a.stream);
}



template <typename T, int K, int L, int RS_ = 0, int F_ = 0, bool EX = false>
static cudaError_t launch_wavefront2_t(const WavefrontLaunch& a) {
  constexpr int S = (int)sizeof(T);
  constexpr int RS = RS_ ? RS_ : ring_slots(K, S), F = F_ ? F_ : ring_ahead(K, S);
  auto kern = k_wavefront2<T, K, L, RS, F, EX>;
  constexpr int ROWB = K * S;
  const int threads = 32;                                    // one warp = one worker
  const int wpc = 1;
  const size_t smem = (size_t)wpc * RS * 2 * ROWB;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  const int blocks = (int)cdiv64((int64_t)a.s * a.blocks.n, wpc);
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, threads, smem);
  if (e != cudaSuccess) return e;
  if ((int64_t)per_sm * a.num_sms < blocks) return cudaErrorCooperativeLaunchTooLarge;
  if (a.out_lanes) *a.out_lanes = L;
  if (a.out_grid) *a.out_grid = blocks;
  const Rating* slots = a.slots;
  const uint16_t* dup = a.dup;
  const int64_t* sub_off = a.sub_off;
  const int32_t* seq = a.seq;
  const int32_t* rank = a.rank;
  int* tickets = a.tickets;
  int s = a.s, c = a.c;
  T* P = reinterpret_cast<T*>(a.P);
  T* Q = reinterpret_cast<T*>(a.Q);
  Step st = step_of(a);
  WfBlocks bl = a.blocks;
  long long* prof = a.prof;
  unsigned* visits = a.visits;
  unsigned long long* upd = a.upd;
  int* owners = a.owners;
  unsigned* viol = a.viol;
  void* args[] = {&slots, &dup, &sub_off, &seq, &rank, &tickets, &s, &c, &P, &Q, &st,
                  &bl, &prof, &visits, &upd, &owners, &viol};
  return cudaLaunchCooperativeKernel(reinterpret_cast<void*>(kern), blocks, threads, args, smem,
                                     a.stream);
}

template <typename T, int K, int L>
static cudaError_t launch_libmf_t(const LibmfLaunch& a) {
  if (a.out_lanes) *a.out_lanes = L;
  k_libmf<T, K, L><<<a.workers, 32, 0, a.stream>>>(
      a.slots, a.blk_off, a.blk_len, a.a, a.lock, a.row_busy, a.col_busy, a.done, a.remaining,
      a.workers, reinterpret_cast<T*>(a.P), reinterpret_cast<T*>(a.Q), step_of(a), a.seed,
      a.visits, a.upd);
  return cudaGetLastError();
}

template <typename T, int K, int L>
static cudaError_t launch_rmse_t(const RmseLaunch& a) {
  const int threads = 256;
  const int blocks = a.num_sms * 4;
  if (a.N > 0)
    k_rmse_partial<T, K, L><<<blocks, threads, 0, a.stream>>>(
        a.test, a.N, reinterpret_cast<const T*>(a.P), reinterpret_cast<const T*>(a.Q), a.partial,
        a.loss, a.lp, a.lq);
  else
    cudaMemsetAsync(a.partial, 0, sizeof(double) * blocks, a.stream);
  k_rmse_final<<<1, 256, 0, a.stream>>>(a.partial, blocks, a.out);
  return cudaGetLastError();
}

// the quarter-lane ring (lane_bytes = 64): L = ring_lanes / 4 lanes, RS = 16, F = 7 < L
constexpr bool quarter_ring_ok(int K, int S) {
  return ring_lanes(K, S) / 4 > 7 && (K * S / (ring_lanes(K, S) / 4)) % 16 == 0;
}

// lanes per sample for a given bytes-per-lane target: L = clamp(k*S/lane_bytes, 1, 32)
static constexpr int lanes_for(int K, int S, int LB) {
  return (K * S / LB) >= 32 ? 32 : ((K * S / LB) < 1 ? 1 : (K * S / LB));
}

template <typename T, int K, int LB>
static cudaError_t hogwild_kl(const HogwildLaunch& a) {
  constexpr int S = (int)sizeof(T);
  constexpr bool l1ok = true;                   // q_v through L1 (R28): plain and grouped paths
  if (a.group) {                                 // column-grouped batches (R24), depth 1
    if (a.ada.GP) return launch_hogwild_t<T, K, lanes_for(K, S, LB), 1, true, false, 0, true>(a);
    if (a.exact) return launch_hogwild_t<T, K, lanes_for(K, S, LB), 1, false, true, 0, true>(a);
    if constexpr (l1ok)
      if (a.q_l1) return launch_hogwild_t<T, K, lanes_for(K, S, LB), 1, false, false, 0, true, kLcQ>(a);
    return launch_hogwild_t<T, K, lanes_for(K, S, LB), 1, false, false, 0, true>(a);
  }
  if (a.ada.GP) return launch_hogwild_t<T, K, lanes_for(K, S, LB), 1, true>(a);
  if (a.exact) return launch_hogwild_t<T, K, lanes_for(K, S, LB), 1, false, true>(a);  // depth 1
  if (a.rating_stage == 1 && LB == 16)
    return launch_hogwild_t<T, K, lanes_for(K, S, LB), 1, false, false, 1>(a);        // TMA stream
  if constexpr ((K * S) / lanes_for(K, S, LB) == 16)
    if (a.rating_stage == 2) return launch_hogwild_t<T, K, lanes_for(K, S, LB), 1, false, false, 2>(a);
  if constexpr (l1ok)
    if (a.prefetch == 1 && a.q_l1)
      return launch_hogwild_t<T, K, lanes_for(K, S, LB), 1, false, false, 0, false, kLcQ>(a);
  if (a.prefetch == 1) return launch_hogwild_t<T, K, lanes_for(K, S, LB), 1>(a);
  if (a.q_l1) return launch_hogwild_t<T, K, lanes_for(K, S, LB), 2, false, false, 0, false, kLcQ>(a);
  return launch_hogwild_t<T, K, lanes_for(K, S, LB), 2>(a);
}
template <typename T, int K>
static cudaError_t hogwild_k(const HogwildLaunch& a) {
  if (a.lane_bytes == 32) return hogwild_kl<T, K, 32>(a);
  if (a.lane_bytes == 8) return hogwild_kl<T, K, 8>(a);
  return hogwild_kl<T, K, 16>(a);
}
template <typename T, int K>
static cudaError_t libmf_k(const LibmfLaunch& a) {
  constexpr int S = (int)sizeof(T);
  return launch_libmf_t<T, K, lanes_for(K, S, 16)>(a);
}
template <typename T, int K>
static cudaError_t rmse_k(const RmseLaunch& a) {
  constexpr int S = (int)sizeof(T);
  return launch_rmse_t<T, K, lanes_for(K, S, 16)>(a);
}
template <typename T, int K, bool EX>
static cudaError_t wavefront_kx(const WavefrontLaunch& a) {
  constexpr int S = (int)sizeof(T);
  if (a.ada.GP) return launch_wavefront_t<T, K, lanes_for(K, S, 8), true>(a);  // register kernel
  constexpr int L2 = ring_lanes(K, S);
  constexpr int L3 = L2 / 2;                 // lane_bytes = 32: half the lanes, 32 B per lane
  if constexpr (L3 > ring_ahead(K, S) && (K * S / L3) % 16 == 0)
    if (a.variant == 1 && a.dup && a.lane_bytes == 32) return launch_wavefront2_t<T, K, L3, 0, 0, EX>(a);
  constexpr int L4 = L2 / 4;                 // lane_bytes = 64: a quarter of the lanes
  if constexpr (quarter_ring_ok(K, S))
    if (a.variant == 1 && a.dup && a.lane_bytes == 64) return launch_wavefront2_t<T, K, L4, 16, 7, EX>(a);
  // narrow slices on a full warp (lane_bytes = 0); lane_bytes = 16 keeps 16-B lanes
  if constexpr (narrow_ring(K, S))
    if (a.variant == 1 && a.dup && a.lane_bytes == 0) return launch_wavefront2_t<T, K, 32, 32, 15, EX>(a);
  if constexpr (narrow16_ring(K, S))
    if (a.variant == 1 && a.dup && a.lane_bytes == 0) return launch_wavefront2_t<T, K, 16, 16, 7, EX>(a);
  if constexpr (L2 > ring_ahead(K, S) && (K * S / L2) % 16 == 0)  // needs F < L, 16-B pieces
    if (a.variant == 1 && a.dup) return launch_wavefront2_t<T, K, L2, 0, 0, EX>(a);
  return launch_wavefront_t<T, K, lanes_for(K, S, 8), false, EX>(a);
}
template <typename T, int K>
static cudaError_t wavefront_k(const WavefrontLaunch& a) {
  return a.exact ? wavefront_kx<T, K, true>(a) : wavefront_kx<T, K, false>(a);
}

#define MF_DISPATCH(FN, ARG)                                                         \
  switch (ARG.storage) {                                                             \
    case 0:                                                                          \
      switch (ARG.k) {                                                               \
        case 16: return FN<float, 16>(ARG);                                          \
        case 32: return FN<float, 32>(ARG);                                          \
        case 64: return FN<float, 64>(ARG);                                          \
        case 128: return FN<float, 128>(ARG);                                        \
        case 256: return FN<float, 256>(ARG);                                        \
      }                                                                              \
      break;                                                                         \
    case 1:                                                                          \
      switch (ARG.k) {                                                               \
        case 16: return FN<__half, 16>(ARG);                                         \
        case 32: return FN<__half, 32>(ARG);                                         \
        case 64: return FN<__half, 64>(ARG);                                         \
        case 128: return FN<__half, 128>(ARG);                                       \
        case 256: return FN<__half, 256>(ARG);                                       \
      }                                                                              \
      break;                                                                         \
    case 2:                                                                          \
      switch (ARG.k) {                                                               \
        case 16: return FN<__nv_bfloat16, 16>(ARG);                                  \
        case 32: return FN<__nv_bfloat16, 32>(ARG);                                  \
        case 64: return FN<__nv_bfloat16, 64>(ARG);                                  \
        case 128: return FN<__nv_bfloat16, 128>(ARG);                                \
        case 256: return FN<__nv_bfloat16, 256>(ARG);                                \
      }                                                                              \
      break;                                                                         \
  }                                                                                  \
  return cudaErrorInvalidValue;

cudaError_t launch_hogwild(const HogwildLaunch& a) { MF_DISPATCH(hogwild_k, a) }
cudaError_t launch_wavefront(const WavefrontLaunch& a) { MF_DISPATCH(wavefront_k, a) }
cudaError_t launch_rmse(const RmseLaunch& a) { MF_DISPATCH(rmse_k, a) }
cudaError_t launch_libmf(const LibmfLaunch& a) { MF_DISPATCH(libmf_k, a) }
template <int K, int S>
static int ring_window_t(int lane_bytes) {
  if (lane_bytes == 64 && quarter_ring_ok(K, S)) return 16 - 7 - 1;  // RS = 16, F = 7
  if (lane_bytes == 0 && narrow_ring(K, S)) return 32 - 15 - 1;        // RS = 32, F = 15
  if (lane_bytes == 0 && narrow16_ring(K, S)) return 16 - 7 - 1;        // RS = 16, F = 7
  return ring_slots(K, S) - ring_ahead(K, S) - 1;
}

int ring_window(int k, int storage, int lane_bytes) {
  const bool h = storage != 0;
  switch (k) {
    case 16: return h ? ring_window_t<16, 2>(lane_bytes) : ring_window_t<16, 4>(lane_bytes);
    case 32: return h ? ring_window_t<32, 2>(lane_bytes) : ring_window_t<32, 4>(lane_bytes);
    case 64: return h ? ring_window_t<64, 2>(lane_bytes) : ring_window_t<64, 4>(lane_bytes);
    case 128: return h ? ring_window_t<128, 2>(lane_bytes) : ring_window_t<128, 4>(lane_bytes);
    default: return h ? ring_window_t<256, 2>(lane_bytes) : ring_window_t<256, 4>(lane_bytes);
  }
}

}  // namespace mfb
