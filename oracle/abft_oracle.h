/*
 * abft_oracle.h -- CPU ORACLE for ABFT-SpMV with implicit error localization
 * (Schoell, Braun, Kochte, Wunderlich, DSN 2016; /root/reference/PAPER.md).
 *
 * THIS IS TEST INFRASTRUCTURE, NOT PRODUCT CODE.  Only tests/, the
 * __graft_entry__.smoke() check and bench.py's cpu_baseline / --impl reference
 * legs may load liboracle.so.  The product path (libabft.so) shares no code,
 * header, table or constant generator with this file.
 *
 * Plain, slow, obviously-correct C99 in IEEE binary64, built with
 * -O2 -ffp-contract=off (no FMA contraction, no fast-math).  Every function
 * cites the paper passage (P:<line> = PAPER.md line) it follows; numeric
 * conventions the paper leaves open follow DESIGN.md "Readings" R1..R22
 * (= SURVEY.md §8(c) N1..N15 / Q1..Q22 with the deviations DESIGN.md lists).
 *
 * Notation (Fig. 1): A is N x N CSR, the SpMV operand is x (paper: b),
 * the result y (paper: r), b_s the row-block size, nb = ceil(N / b_s) blocks.
 * C is the sparse checksum matrix (nb rows), t1 = C x the operand checksums,
 * t2_k = w_k^T y_k the result checksums (w_k = all ones), s = t1 - t2 the
 * syndrome, beta = ||x||_2, tau_k = K_k * beta the per-block bound.
 */
#ifndef ABFT_ORACLE_H
#define ABFT_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  int64_t n;               /* rows = cols */
  const int32_t *row_ptr;  /* [n+1] */
  const int32_t *col;      /* [nnz], ascending within a row, no duplicates */
  const double *val;       /* [nnz] */
} or_csr;

enum { OR_INJ_NONE = 0, OR_INJ_LIST = 1, OR_INJ_RATE = 2 };
enum { OR_T_Y = 0, OR_T_T1 = 1, OR_T_T2 = 2 };

typedef struct {
  int32_t mode;            /* OR_INJ_* */
  uint64_t seed;           /* rate mode: Philox key */
  uint64_t call;           /* rate mode: SpMV call index (counter word 2) */
  double lambda;           /* rate mode: fault probability per arithmetic op */
  uint32_t targets;        /* rate mode: bit t set => target t receives faults */
  int64_t n_list;          /* list mode: entries */
  const int32_t *list_round;
  const int32_t *list_target;
  const int64_t *list_index;
  const uint64_t *list_mask;
  const int64_t *list_call; /* list mode, nullable: entry e applies only to SpMV call
                               list_call[e] (matched against `call`); NULL = every call */
} or_inject;

/* --- canonical pairwise sum (R2) --- */
double or_pw(const double *v, int64_t n);
double or_pw_slots(const double *v, const unsigned char *present, int64_t n);

/* --- plain SpMV y = A x (P:74 step 1) --- */
double or_row_dot(const or_csr *A, int64_t i, const double *x);
void or_spmv(const or_csr *A, const double *x, double *y);

/* --- encoding --- */
int64_t or_encode_structure(const or_csr *A, int32_t bs, int32_t *c_row_ptr, int32_t *c_col);
void or_encode_values(const or_csr *A, int32_t bs, const int32_t *c_row_ptr,
                      const int32_t *c_col, double *c_val);
void or_encode_bound(const or_csr *A, int32_t bs, const int32_t *c_row_ptr,
                     const double *c_val, double *K, double *row_norm, double *S, double *c_norm);

/* --- fault model --- */
void or_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
void or_burst_table(uint64_t T[65]);
uint64_t or_fault_mask(const or_inject *inj, int32_t round, int32_t target, int64_t index,
                       int64_t ops);
int64_t or_rate_chunk(double lambda);
int or_poisson_table(double mu, uint64_t *T, int cap);
int64_t or_rate_plan(const or_csr *A, int32_t bs, const int32_t *c_row_ptr, int32_t check,
                     const or_inject *inj, int32_t max_rounds, int32_t *o_round,
                     int32_t *o_target, int64_t *o_index, uint64_t *o_mask);

/* --- protected SpMV: steps 1-5 of Fig. 1 ---
 * flags: [(max_rounds+1) * nb], round r's sorted flagged blocks at flags + r*nb,
 * flag_counts[r] their number.  Round 0 = detection in the main pass; round
 * r >= 1 = blocks still failing after the r-th partial recomputation.
 * y_pre (nullable) receives y after the main pass (faults included).
 * Returns 0, or -6 when blocks remain flagged after max_rounds recomputations. */
int or_abft_spmv(const or_csr *A, int32_t bs, const int32_t *c_row_ptr, const int32_t *c_col,
                 const double *c_val, const double *K, const double *x, const or_inject *inj,
                 int32_t max_rounds, double *y, double *y_pre, double *t1, double *t2,
                 double *s, double *beta_out, int32_t *flag_counts, int32_t *flags);

/* --- related-work baseline: dense check [30, 31] + complete recomputation ---
 * (R23-R25)
 * c [n]: c_j = PW over column j in row order; *k35: the [35] constant (m = N).
 * or_dense_spmv: bound35 = 0 -> tau = ||x||_2 (norm-based), 1 -> tau =
 * k35 ||x||_2.  flag_rounds [max_rounds+1]: 1 where round r's check failed
 * (round r >= 1 = r-th complete recomputation).  out [4] (nullable): round 0's
 * t1, t2, beta, tau.  List faults: index 0 for t1 / t2; rate mode: the plan
 * over the SpMV's y ops of round 0 (R25).  Returns 0, -6 if still flagged
 * after max_rounds recomputations. */
void or_dense_encode(const or_csr *A, double *c, double *k35);
int or_dense_spmv(const or_csr *A, const double *c, double k35, int32_t bound35,
                  const double *x, const or_inject *inj, int32_t max_rounds, double *y,
                  double *y_pre, double *out, int32_t *flag_rounds);

/* --- Jacobi-PCG with the protected SpMV (Saad Alg. 9.1) ---
 * res_hist [max_iter+1].  stats: [0] iters, [1] spmv calls, [2] flagged blocks
 * (round 0, summed), [3] recomputed blocks (summed over rounds), [4] uncorrected
 * calls.  Returns 0 converged, -5 not converged, -7 breakdown.
 * check: 0 plain SpMV, 1 protected; | OR_PCG_LITERAL_STOP: stop when
 * r^T r < tol (P:296 read literally, R16*) instead of ||r|| <= tol ||b||. */
#define OR_PCG_LITERAL_STOP 0x100
int or_pcg(const or_csr *A, int32_t bs, const int32_t *c_row_ptr, const int32_t *c_col,
           const double *c_val, const double *K, const double *b, double *x,
           const double *diag, double tol, int64_t max_iter, const or_inject *inj,
           int32_t max_rounds, int32_t check, double *res_hist, int64_t *stats);

/* --- related-work baseline for the PCG case study: checkpoint-rollback ---
 * (R26-R27) Jacobi-PCG whose every SpMV
 * is checked by the dense check with tau = ||v||_2; the state
 * (x, r, z, p, rho, it) is sampled every ckpt_every iterations (20)
 * and restored on a detection.  c: or_dense_encode's checksum.  Rate faults
 * hit y only (call j = inj->call + j-th executed SpMV).  max_iter bounds
 * executed iterations (<= 0 -> 10 N).  stats [5]: iterations of the result,
 * SpMV calls, rollbacks, executed iterations, 0.  Returns 0 / -5 / -7. */
int or_pcg_cr(const or_csr *A, const double *c, const double *b, double *x, const double *diag,
              double tol, int64_t max_iter, const or_inject *inj, int32_t ckpt_every,
              double *res_hist, int64_t *stats);

#ifdef __cplusplus
}
#endif
#endif
