/*
 * include/mf.h -- C ABI of libmf_b200.so, the B200-native hot path of cuMF_SGD
 * (Xie, Tan, Fong, Liang, "CuMF_SGD: Parallelized Stochastic Gradient Descent for Matrix
 * Factorization on GPUs", HPDC'17).  "P:L<n>" cites a line of the paper text
 * (/root/reference/PAPER.md), "A:" the index/RNG specification of SURVEY.md Appendix A, and
 * "R<n>" a reading of a silent or garbled passage listed in DESIGN.md section 3.
 *
 * Problem (Eq. 1-3): R (m x n, N observed ratings r_{u,v}) ~ P (m x k) x Q (k x n).
 * Per rating, Algorithm 1 lines 8-10:
 *     e = r - p_u . q_v ;  p_u += gamma_t (e q_v - lambda_p p_u) ;  q_v += gamma_t (e p_u - lambda_q q_v)
 * (both from the pre-update p_u, q_v -- R1), gamma_t = alpha / (1 + beta t^1.5)  (Eq. 9),
 * scheduled by batch-Hogwild! (section 5.1) or by the deterministic wavefront
 * (section 5.2) inside DSGD-style strata across GPUs (section 6.1).
 *
 * Conventions (all entry points):
 *  - Every call returns mf_status (0 = MF_OK, < 0 = error); nothing throws or aborts across the
 *    ABI.  mf_last_error(ctx) returns a NUL-terminated message for the last error of a ctx.
 *  - A CUDA error is sticky: the call returns MF_E_CUDA and every later call on that ctx
 *    returns MF_E_STATE.  NCCL errors likewise (MF_E_NCCL).
 *  - Ownership: the caller owns every buffer it passes in or receives results into (host or
 *    device, see each on_device flag); the ctx owns all of its device state, allocated through
 *    params.alloc when given (else cudaMallocAsync on the ctx stream), freed by mf_destroy.
 *  - One ctx per device (per rank); a ctx is not thread-safe.
 *  - Call order: mf_create -> mf_load_coo(MF_TRAIN) [-> mf_load_coo(MF_TEST)] ->
 *    { mf_train_epoch | mf_rmse | mf_get_factors | mf_set_factors | mf_export_schedule }*
 *    -> mf_destroy.  Out of order, or a second load of the same set, returns MF_E_STATE.
 *  - Work is enqueued on params.stream (a cudaStream_t, e.g. torch.cuda.current_stream()),
 *    or on a ctx-created stream when NULL.  mf_train_epoch does not synchronise; mf_rmse,
 *    mf_get_factors, mf_export_schedule and mf_get_stats do.
 *  - Index types: N is int64 (Hugewiki-shaped N = 3.07e9 > 2^31); u, v are int32.
 */
#ifndef MF_B200_H
#define MF_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MF_ABI_VERSION 6

typedef struct mf_ctx mf_ctx; /* opaque, owned by the library */

typedef int32_t mf_status;
enum {
  MF_OK = 0,
  MF_E_INVAL = -1,       /* bad argument / parameter                                  */
  MF_E_NOMEM = -2,       /* device or host allocation failed                          */
  MF_E_CUDA = -3,        /* CUDA runtime error (sticky)                               */
  MF_E_NCCL = -4,        /* NCCL error or NCCL unavailable for world > 1 (sticky)     */
  MF_E_STATE = -5,       /* call out of order, or ctx already in an error state        */
  MF_E_RANGE = -6,       /* rating index out of [0,m)x[0,n), non-finite r, NaN RMSE    */
  MF_E_UNSUPPORTED = -7  /* k not in {16,32,64,128,256}, too many workers, no device  */
};

typedef enum { MF_FP32 = 0, MF_FP16 = 1, MF_BF16 = 2 } mf_storage;   /* P:L242 feature storage */
typedef enum {
  MF_HOGWILD = 0,   /* batch-Hogwild! (section 5.1)                                           */
  MF_WAVEFRONT = 1, /* deterministic wavefront (section 5.2)                                  */
  MF_LIBMF = 2      /* BASELINE: LIBMF-GPU global-table block scheduler (section 5, Fig. 5a,
                       P:L258-268); grid_a x grid_a blocks (0 = 64), workers = warps (0 = a/2);
                       one GPU, resident ratings only                                          */
} mf_schedule;
typedef enum { MF_TRAIN = 0, MF_TEST = 1 } mf_set;

/* Device-memory hooks (e.g. torch's caching allocator).  alloc returns NULL on failure. */
typedef struct mf_allocator {
  void* (*alloc)(size_t bytes, void* stream, void* user);
  void (*free)(void* ptr, size_t bytes, void* stream, void* user);
  void* user;
} mf_allocator;

typedef struct mf_params {
  uint32_t struct_size;   /* = sizeof(mf_params) (ABI check)                                   */
  int64_t m, n;           /* R is m x n                                                */
  int32_t k;              /* feature dimension (Table 2 k = 128); {16,32,64,128,256}     */
  float lambda_p;         /* Eq. 2 regularisers; the paper uses one lambda (R3)          */
  float lambda_q;
  float alpha, beta;      /* Eq. 9 learning-rate schedule (Table 3)                 */
  float init_scale;       /* Alg. 1 l.3 scale_factor: P,Q ~ U[0, sqrt(1/(k*init_scale))) (R5)    */
  float rating_scale;     /* r' = r / rating_scale for training; RMSE reported x rating_scale   */
  uint64_t seed;          /* keys every random choice (A: streams S_SHUF ... S_ST)              */
  int32_t schedule;       /* mf_schedule                                                        */
  int32_t storage;        /* mf_storage of P and Q; arithmetic is always fp32                   */
  int32_t workers;        /* s: Hogwild = concurrent sample groups (0 = all resident);
                             wavefront = row sub-blocks per strata block (0 = min(768/(a/world),
                             m/(4a)): one launch runs the a/world blocks of a stratum together) */
  int32_t batch_f;        /* Eq. 8 batch f (0 = 256)                                    */
  int32_t wf_cols;        /* wavefront column sub-blocks c (0 = 2*s, R9)                        */
  int32_t grid_a;         /* strata grid a x a (0 = 1 if world == 1 else 8); a % world == 0
                             and a / world <= 16                                                */
  int32_t cyclic;         /* wavefront: 1 = cyclic column order (A: cyclic variant), needs c >= s */
  int32_t lane_bytes;     /* Hogwild kernel: bytes of p_u (and q_v) per lane, 8, 16 or 32 (0 = 16).
                             Ring wavefront: 0 = default geometry (fp16/bf16 k = 128: 8 B on 32
                             lanes), 16 = 16-B lanes, 32 / 64 = half / quarter of the lanes   */
  int32_t prefetch;       /* Hogwild software-pipeline depth: samples in flight per worker, 1 or 2 (0 = 1) */
  int32_t lr_rule;        /* 0 = Eq. 9 schedule (the paper); 1 = ADAGRAD (P:L419 future work,
                             Duchi et al. [20]; R23): per-coordinate fp32 accumulators
                             G += g^2, step alpha*g/sqrt(G + ada_eps); Hogwild and register
                             wavefront kernels                                                  */
  float ada_eps;          /* ADAGRAD epsilon (0 = 1e-8)                                         */
  int32_t staged;         /* 2 = ratings AND P out of core (section 6.1 step 3, and the
                             three streams of section 6.3): P's row segments live in
                             pinned host memory and the strata blocks run one at a time, each
                             with its segment copied in on a copy stream, trained, and written
                             back on a D2H stream while the next block computes; Q stays
                             resident.  One GPU, Eq. 9 step; same result as resident.
                             1 = out-of-core ratings (section 6.2): the bucketed
                             ratings live in pinned host memory (a host train set is
                             preprocessed in chunks of stage_chunk samples, never whole in
                             HBM; a device set is preprocessed resident, then moved) and
                             each stratum's blocks stream into one of two HBM buffers on a copy
                             stream while the previous stratum computes; P, Q stay resident.
                             The host copy and the H2D stream carry packed records: (u, v) as
                             one integer of bits(m) + bits(n-1) bits in 5 bytes (<= 40 bits) or
                             6 (<= 48), plus r fp32 -- 9 or 10 B per rating, expanded on the GPU
                             (12-B slots beyond 48 bits).
                             Same order and result as resident.  0 = ratings resident in HBM */
  int32_t wf_kernel;      /* wavefront kernel: 0 = auto = 1 = ring-staged (cp.async smem ring),
                             2 = register pipeline; both give the same result                   */
  int32_t device;         /* CUDA device ordinal                                                */
  int32_t rank, world;    /* world > 1: DSGD strata over `world` GPUs, one ctx per rank         */
  int32_t transport;      /* world > 1: 0 = NCCL (one process per GPU); 1 = loopback (all ranks
                             in one process, one host thread each, device-to-device copies;
                             tests the multi-rank path on one GPU)                              */
  const void* nccl_id;    /* 128 bytes identical on all ranks (world > 1): the ncclUniqueId, or
                             for loopback any key naming the group                              */
  void* stream;           /* cudaStream_t or NULL                                               */
  const mf_allocator* alloc; /* NULL = cudaMallocAsync                                          */
  int32_t launch_blocks;  /* Hogwild: strata blocks per SGD launch (0 = every block the rank
                             trains in the sub-epoch, interleaved in one launch).  B > 0 runs
                             them B at a time, in row-segment order: with world = 1 and B = a/G
                             each launch is exactly what one of G GPUs runs in that sub-epoch
                             (tools/scale_emulation.py).  Same result either way: a stratum's
                             blocks touch disjoint P and Q rows                                 */
  int32_t exact_order;    /* 1 = evaluate Alg. 1 l.8-10 in the paper's operation order, every
                             operation rounded once (err = r - p.q; p + g((err q) - (lp p))),
                             as the oracle does: bit-identical to it whenever the dot product is
                             exact.  0 (default) = the fast form p' = fma(g err, q, (1-g lp) p),
                             which rounds differently by an ulp of fp32 now and then and is
                             8-21% faster                                 */
  int32_t rating_stage;   /* Hogwild rating stream (north_star (2), Eq. 8 batches): 0 = per-lane
                             streaming loads + warp shuffles; 1 = TMA: one lane per worker
                             bulk-copies its chunk into shared memory in 768-B sub-chunks
                             (cp.async.bulk + mbarrier, double buffered).  1 needs f % 64 == 0,
                             prefetch 1 and the default 16-B lanes (else MF_E_UNSUPPORTED).
                             2 = the next 2 samples' p/q rows copied into a per-worker shared-
                             memory ring by cp.async (a deeper row pipeline without registers;
                             16-B lane slices: k S <= 512, prefetch 1).  1 and 2 are Hogwild
                             with the Eq. 9 step in the fast form only (exact_order, ADAGRAD or
                             another schedule: MF_E_UNSUPPORTED).  All three: same order and
                             result                                                          */
  int64_t stage_chunk;    /* staged = 1 with a HOST train set: samples per chunk of the
                             out-of-core preprocessing (0 = 2^26).  Device memory then holds one
                             chunk (~68 B per sample) or one strata block (~60 B per sample) at a
                             time instead of the whole set (section 6)            */
  int32_t group_cols;     /* batch-Hogwild, reading R24: every batch of f consecutive samples
                             (Eq. 8; "fetch f consecutive samples and update them serially",
                             P:L272) is updated in order of (relabelled column, storage
                             position) instead of storage order, so repeated -- power-law-hot --
                             columns of a batch run back to back and their q_v stays in
                             registers (no load, no intermediate store).  The oracle runs the
                             same order (or_params.group_cols).  Hogwild only                */
  int32_t check_owners;   /* debug (deterministic wavefront): tag each column block with its
                             holder on acquire (atomicCAS) and check the tag on release; any
                             overlap of two holders is counted (mf_owner_violations) -- the
                             mutual exclusion of the ticket protocol on the global P/Q rows,
                             which compute-sanitizer's racecheck (shared memory only) cannot
                             see.  One atomic per wave when on, nothing when off             */
  int32_t grid_cols;      /* column segments of the grid: 0 = grid_a (the a x a strata grid),
                             1 = the paper's a x 1 row blocks (Hugewiki in 64 x 1
                             blocks; reading R27): block r holds the ratings of relabelled row
                             segment r and all columns, and an epoch trains the a blocks one
                             after another in the order perm(S_STRATA(t), a), each by batch-
                             Hogwild.  a <= m (a may exceed n), a <= 256; grid_a = 0 picks a
                             = ceil(|P| / 32 MiB) (a segment of P stays L2-resident while its
                             block trains: Netflix 4, Yahoo 8, Hugewiki 256).  One GPU, Hogwild,
                             Eq. 9 (else MF_E_UNSUPPORTED).  With staged = 2 every P row
                             segment crosses the host link twice per epoch instead of 2a times */
  int32_t q_cache;        /* batch-Hogwild: cache policy of the q_v row loads (reading R28; the
                             per-instruction "cache or bypass" choice of section 4, P:L234,
                             made for the feature row with temporal reuse).  0 = auto: q_v rows
                             are read through the SM's L1 (ld.ca, write-back stores) in the
                             Hogwild kernels on the Eq. 9 fast-form path (plain batches at
                             prefetch 1 or 2, column-grouped batches): a hot column is then read from
                             L1 by every worker of the SM instead of by an L2 load that
                             serialises with other SMs' stores to the same line.  L1 is not
                             coherent across SMs, so a read may miss other SMs' latest store --
                             a racy read, which Hogwild permits (R19).  Every other kernel and
                             path reads through L2.  1 = L2 only (.cg loads, .cg stores)
                             everywhere.  mf_stats.q_l1 reports which one ran                 */
} mf_params;

/* Fill *p with defaults (Table 3 Netflix lambda/alpha/beta, k = 128, fp32, Hogwild, f = 256). */
mf_status mf_params_default(mf_params* p);

/* Validate parameters, select the device, create/adopt the stream; world > 1 also initialises
 * the NCCL communicator from nccl_id (libnccl.so.2 is dlopen'ed; missing -> MF_E_NCCL).
 * Returns MF_E_INVAL / MF_E_UNSUPPORTED for bad params; *out is NULL on error. */
mf_status mf_create(const mf_params* p, mf_ctx** out);

/* Load a rating set in COO form: nnz triples (u[i], v[i], r[i]) (2 ints + 1 float),
 * host or device pointers (on_device = 0/1); the library copies them and never keeps the
 * caller's pointers.  MF_TRAIN runs the one-time preprocessing on the GPU:
 *   validation (MF_E_RANGE if u or v out of range or r non-finite; the ctx stays usable),
 *   Alg. 1 l.2 random_shuffle (storage order = perm(S_SHUF, nnz), A),
 *   row/column relabel (A: S_ROW, S_COL) and bucketing into strata blocks / wavefront
 *   sub-blocks, Alg. 1 l.3 initialisation of P, Q (A: S_P, S_Q).
 * world > 1: every rank passes the FULL set; a rank keeps only the blocks it owns.
 * MF_TEST stores the test set (relabelled, scaled) for mf_rmse. */
mf_status mf_load_coo(mf_ctx* ctx, int32_t set, int64_t nnz, const int32_t* u, const int32_t* v,
                      const float* r, int32_t on_device);

/* Enqueue one epoch t (t = ctx epoch counter, 0-based, R4) on the stream: gamma_t (Eq. 9),
 * the epoch schedule (chunk order / column sequences / tickets, A) and the SGD kernels; for
 * world > 1 the a sub-epochs each followed by the NCCL Q-segment rotation.  Increments t and
 * writes it to *epoch_done when non-NULL.  Does not synchronise. */
mf_status mf_train_epoch(mf_ctx* ctx, int32_t* epoch_done);

/* RMSE of the chosen set (R13): rating_scale * sqrt(sum (r' - p_u.q_v)^2 / N), fp32 dots,
 * fp64 accumulation, deterministic reduction order.  world > 1: global value (all ranks).
 * Synchronises.  MF_E_RANGE if the result is NaN (divergence). */
mf_status mf_rmse(mf_ctx* ctx, int32_t set, double* out);

/* Eq. 2 over the training set: sum over train ratings of (r' - p_u.q_v)^2 +
 * lambda_p ||p_u||^2 + lambda_q ||q_v||^2, in the scaled rating units r' = r / rating_scale the
 * model trains on; fp32 dots and norms per sample, fp64 accumulation.  world > 1: the global
 * value on every rank.  Resident ratings only (MF_E_UNSUPPORTED when staged).  Synchronises. */
mf_status mf_loss(mf_ctx* ctx, double* out);

/* Copy the model out in ORIGINAL ids as fp32 (Alg. 1 l.15 model_shuffle): P is m x k
 * row-major, Q is n x k row-major (row v = q_v, R14).  Either pointer may be NULL.
 * world > 1: gathers all segments; every rank receives the full P and Q.  Synchronises. */
mf_status mf_get_factors(mf_ctx* ctx, float* P, float* Q, int32_t on_device);

/* Overwrite P and/or Q (same layout as mf_get_factors), rounded to the storage type (RNE). */
mf_status mf_set_factors(mf_ctx* ctx, const float* P, const float* Q, int32_t on_device);

/* Set / get the epoch counter t (checkpoint-resume). */
mf_status mf_set_epoch(mf_ctx* ctx, int32_t t);
mf_status mf_get_epoch(const mf_ctx* ctx, int32_t* t);

/* Export an index structure for bit-exact comparison (tests).  Host int64 buffer; with
 * buf == NULL only *len is set to the required element count; otherwise *len must be >= it.
 * Layouts are identical to the oracle's exports. */
enum {
  MF_EX_PERM = 0,       /* [N]  caller index of storage position j                     */
  MF_EX_RHO_R = 1,      /* [m]  row relabel rank                                       */
  MF_EX_RHO_C = 2,      /* [n]  column relabel rank                                    */
  MF_EX_BLOCKID = 3,    /* [N]  per storage position: block b (Hogwild) or
                                b*(s*c) + i*c + j (wavefront)                           */
  MF_EX_CHUNKORDER = 4, /* [sum_b nchunks_b] Hogwild chunk order per block, b ascending (epoch) */
  MF_EX_WFSEQ = 5,      /* [a*a*s*c] seq_i[w] per block b, worker i, wave w (epoch)     */
  MF_EX_TICKETS = 6,    /* [a*a*s*c] ticket rank of visit (w,i), stored [b][i][w] (epoch) */
  MF_EX_STRATA = 7      /* [a]  pi_t (epoch)                                            */
};
mf_status mf_export_schedule(mf_ctx* ctx, int32_t what, int32_t epoch, int64_t* buf, int64_t* len);

/* Timing of the last mf_train_epoch, from CUDA events recorded on the ctx stream around the
 * work (synchronises).  sgd_ms: SGD kernel launches only; sched_ms: schedule build;
 * comm_ms: Q rotation; launches: kernels launched by the epoch. */
typedef struct mf_stats {
  double epoch_ms, sgd_ms, sched_ms, comm_ms;
  int64_t sgd_launches, launches;
  int64_t updates;          /* samples updated by this rank in the epoch, counted ON THE DEVICE
                               by the SGD kernels (non-sentinel samples each worker ran; Eq. 7,
                               P:L253: an epoch is N updates)                                  */
  int64_t bytes_per_update; /* algorithmic: 12 + 4*k*sizeof(storage) (north_star; Eq. 5)  */
  int32_t workers, lanes, grid, block;
  int64_t h2d_bytes;        /* staged mode: bytes copied host -> device for the epoch's ratings
                               (9 or 10 per rating packed, see params.staged; 12 unpacked; +2
                               with the wavefront's duplicate distances; + P's row segments
                               when staged = 2)                                                 */
  int32_t q_l1;             /* 1 if the last SGD launch read q_v rows through L1 (q_cache) */
} mf_stats;
mf_status mf_get_stats(mf_ctx* ctx, mf_stats* out);

/* Exactly-once evidence (Eq. 7; SURVEY 8(c) "each sample exactly once per epoch").
 * Every SGD kernel records, on the device, one claim per work unit it runs: a Hogwild chunk of
 * f consecutive slots, a wavefront sub-block, a LIBMF block.  Units are disjoint slot ranges
 * and a worker runs every slot of the unit it claimed, so "every unit claimed exactly once per
 * epoch" plus mf_stats.updates == N (the kernels' own count of non-sentinel samples) means
 * every sample was updated exactly once.  This call compares each unit's claim count since
 * mf_load_coo with the number of epochs run since then (0 for wavefront sub-blocks of blocks
 * this rank does not train) and writes the number of mismatching units to *bad_units, the
 * number of units to *units and the epochs to *epochs (either may be NULL).  Synchronises. */
mf_status mf_check_visits(mf_ctx* ctx, int64_t* bad_units, int64_t* units, int32_t* epochs);

/* Ownership-checker violations counted since load (params.check_owners = 1, wavefront;
 * MF_E_STATE otherwise).  0 = no two workers ever held a column block at the same time. */
mf_status mf_owner_violations(mf_ctx* ctx, int64_t* violations);

/* Per-launch device times (ms, CUDA events) of the SGD launches of the last epoch, in launch
 * order (synchronises).  With ms == NULL only *n is set; otherwise *n must be >= the count and
 * receives it. */
mf_status mf_get_launch_ms(mf_ctx* ctx, double* ms, int64_t* n);

/* Host-only strata planner (no GPU needed): which rank trains block row-segment r in
 * sub-epoch j of epoch t, and which Q segments move before sub-epoch j.  For each segment
 * J in [0,a): holder[J] = rank that holds (trains with) segment J during sub-epoch j.
 * A: the stratum of sub-epoch j is {(r, (r + pi_t[j]) mod a)}; rank g owns row segments
 * [g*a/G, (g+1)*a/G).  Returns MF_E_INVAL if a % world != 0. */
mf_status mf_strata_holders(uint64_t seed, int32_t a, int32_t world, int32_t t, int32_t j,
                            int32_t* holder);

/* Host-only plan of sub-epoch j of epoch t for `rank` -- the function mf_train_epoch itself
 * uses (A: strata order; section 6.1 P:L305-316 adapted).  holders[a] is in/out: on entry the
 * rank holding each Q segment's valid copy (-1 = every rank holds one), on exit the holders
 * during sub-epoch j.  Outputs: blocks[*nblocks] (<= a/world) = the strata blocks b = r*a + J
 * the rank trains; xfers[5 * *nxfers] = {J, src, dst, lo, hi}: segment J (relabelled Q rows
 * [lo, hi), n = number of columns) moves src -> dst before the sub-epoch.  Caller allocates
 * blocks[a] and xfers[5a].  MF_E_INVAL for a % world != 0 or n < a. */
mf_status mf_strata_plan(uint64_t seed, int32_t a, int32_t world, int32_t rank, int64_t n,
                         int32_t t, int32_t j, int32_t* holders, int64_t* blocks,
                         int32_t* nblocks, int64_t* xfers, int32_t* nxfers);

/* Debug / test surface: run every primitive of the strata mode's transport (a12; section 6.1,
 * P:L305-316 adapted) outside a training context and check the results: the fp64 all-reduce
 * of the RMSE, a broadcast, one grouped send/recv set shaped like a Q-segment rotation
 * (segment r moves r -> (r+1) mod world), and the segment gather of mf_get_factors.  Each of
 * the `world` ranks calls it on its own `device` with the same 128-byte ncclUniqueId (transport
 * 0 = NCCL) or loopback group key (1, ranks = threads of one process).  world = 1 is valid and
 * runs every NCCL call on one GPU (the rotation becomes a send/recv to self).  Synchronises.
 * Returns MF_OK when every value checks, MF_E_NCCL / MF_E_CUDA on a failed call, MF_E_RANGE
 * on a wrong value; `msg` (msg_len bytes, may be NULL) receives a one-line report. */
mf_status mf_comm_selftest(const void* comm_id, int32_t world, int32_t rank, int32_t device,
                           int32_t transport, char* msg, int32_t msg_len);

void mf_destroy(mf_ctx* ctx);
const char* mf_last_error(const mf_ctx* ctx);
const char* mf_status_string(mf_status s);
int32_t mf_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* MF_B200_H */
