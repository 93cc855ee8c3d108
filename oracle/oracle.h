/*
 * oracle/oracle.h -- plain, single-threaded CPU oracle for the cuMF_SGD hot path
 * (Xie, Tan, Fong, Liang, "CuMF_SGD", HPDC'17).  Citations "P:L<n>" are lines of
 * /root/reference/PAPER.md; "A:<item>" is SURVEY.md Appendix A; "R<n>" is a reading
 * listed in DESIGN.md section 3.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_hpdc_xietfl17_b200/) never includes, links or calls it, and the two share
 * no source: this file and oracle.c were written from the paper and Appendix A alone.
 *
 * Every function here is pinned by a -m "not gpu" test in tests/test_oracle_*.py except
 * where its comment says "parity unpinned".
 */
#ifndef CUMF_ORACLE_H
#define CUMF_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- Appendix A counter-based hashing (bit-exact spec shared by specification only) ---- */
uint64_t or_mix(uint64_t z);                                     /* SplitMix64 finaliser */
uint64_t or_stream(uint64_t seed, uint64_t tag, uint64_t a, uint64_t b);
uint64_t or_key(uint64_t S, uint64_t i);                         /* mix(S + i*phi) */
int      or_perm(uint64_t S, int64_t n, int64_t* out);           /* [0,n) sorted by key(S,.) */

/* ---- storage rounding (P:L242 half-precision storage; R16 round-to-nearest-even) ---- */
uint16_t or_f16_bits(float x);
float    or_f16_value(uint16_t h);
uint16_t or_bf16_bits(float x);
float    or_bf16_value(uint16_t h);
float    or_round_storage(int32_t storage, float x);             /* 0 fp32, 1 fp16, 2 bf16 */

/* ---- the method's arithmetic ---- */
float  or_gamma(float alpha, float beta, int32_t t);             /* Eq. 9 */
void   or_update(int32_t k, float* p, float* q, float r, float gamma,
                 float lambda_p, float lambda_q, int32_t storage); /* Alg. 1 l.8-10 */
double or_sample_loss(int32_t k, const double* p, const double* q, double r,
                      double lambda_p, double lambda_q);           /* Eq. 3 */
/* ADAGRAD variant ("cuMF_SGD can also use ADAGRAD", Duchi et al. [20]; reading R23):
 * per coordinate, with pre-update values (R1):
 *   g_p = -(e q - lambda_p p);  G_p += g_p^2;  p <- p - alpha g_p / sqrt(G_p + eps)   (same for q)
 * gp, gq: the fp32 accumulators of p_u and q_v. */
void   or_update_adagrad(int32_t k, float* p, float* q, float* gp, float* gq, float r,
                         float alpha, float lambda_p, float lambda_q, float eps, int32_t storage);

/* ---- a whole training run, in the schedule's serial order ---- */
typedef struct or_params {
  int64_t m, n;
  int32_t k;
  float   lambda_p, lambda_q;
  float   alpha, beta;
  float   init_scale;      /* Alg. 1 l.3 scale_factor (R5) */
  float   rating_scale;    /* r' = r / rating_scale (R5) */
  uint64_t seed;
  int32_t schedule;        /* 0 batch-Hogwild (serial emulation), 1 wavefront */
  int32_t storage;         /* 0 fp32, 1 fp16, 2 bf16 */
  int32_t workers;         /* s: wavefront row sub-blocks per strata block */
  int32_t batch_f;         /* f (Eq. 8) */
  int32_t wf_cols;         /* c: wavefront column sub-blocks per strata block */
  int32_t grid_a;          /* a: strata grid a x a (1 = single block) */
  int32_t cyclic;          /* wavefront cyclic column order variant (A: cyclic) */
  int32_t lr_rule;         /* 0 = Eq. 9 schedule; 1 = ADAGRAD (or_update_adagrad, R23) */
  float   ada_eps;         /* ADAGRAD epsilon */
  int32_t group_cols;      /* batch-Hogwild, reading R24: inside each batch of f consecutive
                              samples, update them in order of (relabelled column, position) */
  int32_t grid_cols;       /* column segments of the grid: 0 = a (the a x a strata grid), 1 =
                              the paper's a x 1 row blocks (P:L379, 64 x 1 for Hugewiki; reading
                              R27): blocks one after another in the order perm(S_STRATA(t), a) */
} or_params;

typedef struct or_ctx or_ctx;

/* train arrays are in caller order; copied.  Returns NULL on invalid input. */
or_ctx* or_create(const or_params* prm, int64_t N, const int32_t* u, const int32_t* v,
                  const float* r);
void    or_destroy(or_ctx* c);
int     or_train_epoch(or_ctx* c);                       /* runs epoch t, then t++ */
int     or_run_block(or_ctx* c, int32_t t, int64_t b);   /* one strata block of epoch t */
int     or_set_epoch(or_ctx* c, int32_t t);
int32_t or_get_epoch(const or_ctx* c);
double  or_rmse(const or_ctx* c, int64_t N, const int32_t* u, const int32_t* v, const float* r);
double  or_loss(const or_ctx* c);                        /* Eq. 2 over the train set */
void    or_get_factors(const or_ctx* c, float* P, float* Q);
void    or_set_factors(or_ctx* c, const float* P, const float* Q);  /* rounds to storage */
/* Set the rows of Q whose relabelled column index lies in [lo, hi) (strata segment copy). */
void    or_copy_q_rows(or_ctx* dst, const or_ctx* src, int64_t lo, int64_t hi);

/* Schedule exports (bit-exact index parity).  `len` is in/out element count. */
enum {
  OR_EX_PERM = 0,      /* int64[N]  caller index of storage position j            */
  OR_EX_RHO_R = 1,     /* int64[m]  row relabel rank                              */
  OR_EX_RHO_C = 2,     /* int64[n]  column relabel rank                           */
  OR_EX_BLOCKID = 3,   /* int64[N]  per storage position: b*(s*c) + i*c + j (WF) or b (HW) */
  OR_EX_CHUNKORDER = 4,/* int64[sum_b nchunks_b] chunk order of every block, b ascending */
  OR_EX_WFSEQ = 5,     /* int64[a*a*s*c] seq_i[w] for b, i, w                      */
  OR_EX_TICKETS = 6,   /* int64[a*a*s*c] ticket rank of visit (w,i) stored [b][i][w] */
  OR_EX_STRATA = 7,    /* int64[a]      pi_t                                        */
  OR_EX_ORDER = 8      /* int64[N]  storage positions in the exact execution order  */
};
int or_export(const or_ctx* c, int32_t what, int32_t t, int64_t* buf, int64_t* len);

#ifdef __cplusplus
}
#endif
#endif
