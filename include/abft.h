/*
 * abft.h -- C ABI of the B200-native ABFT-SpMV library (libabft.so).
 *
 * Method: Schoell, Braun, Kochte, Wunderlich, "Efficient Algorithm-Based Fault
 * Tolerance for Sparse Matrix Operations", DSN 2016 (PAPER.md; P:<n> = line).
 *
 *   abft_encode  -- build the sparse checksum matrix C and the bound constants
 *                   once per matrix (SIII-B/C/D, P:94, P:108, P:128-130,
 *                   P:156-160, Fig. 2/3).
 *   abft_spmv    -- y = A x with detection and implicit localization in the
 *                   same pass (Fig. 1 steps 1-4).
 *   abft_correct -- partial recomputation of the flagged blocks only
 *                   (Fig. 1 step 5), re-verified each round.
 *   abft_pcg     -- Jacobi-preconditioned CG whose every SpMV is protected
 *                   (SVI-A; success within 10 N iterations).
 *
 * Conventions (all entry points):
 *  - Pointers are DEVICE pointers unless marked (host).  FP64 values, int32
 *    indices, row-major CSR with columns ascending within each row and no
 *    duplicates (square matrices in CSR).
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *    stream).  abft_spmv / abft_correct are stream-ordered and asynchronous:
 *    they never synchronise with the host.  abft_encode synchronises once (to
 *    size C); abft_pcg and abft_spmv_host synchronise before returning.
 *  - No exception crosses the boundary.  Host-detectable argument errors
 *    return ABFT_EINVAL immediately; CUDA errors return ABFT_ECUDA.
 *  - Numerics: IEEE binary64, round-to-nearest, no FMA contraction; every
 *    sum uses the canonical pairwise order PW of DESIGN.md (R2), so results
 *    are bit-reproducible and bit-identical to the CPU oracle.
 *  - A handle is not thread-safe; use it from one stream at a time.
 */
#ifndef ABFT_H
#define ABFT_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  ABFT_OK = 0,
  ABFT_EINVAL = -1,        /* bad argument (host-detected) */
  ABFT_ECUDA = -2,         /* CUDA runtime error (see abft_last_cuda_error) */
  ABFT_ENOMEM = -3,        /* device allocation failed */
  ABFT_ENOTSUP = -4,       /* unsupported configuration (e.g. block_size > 1024) */
  ABFT_ENOCONV = -5,       /* PCG: not converged within max_iter */
  ABFT_EUNCORRECTED = -6,  /* blocks still flagged after max_rounds recomputations */
  ABFT_EBREAKDOWN = -7,    /* PCG: p.q <= 0 or NaN residual */
  ABFT_ENCCL = -8          /* NCCL error (multi-GPU; see abft_last_cuda_error) */
} abft_status;

/* CSR matrix, DEVICE arrays. row_ptr[n+1], col_idx[nnz], val[nnz].
 * The caller owns the arrays; they must outlive the handle (correction and
 * PCG re-read A; it is never copied).
 * Square (n_cols == 0 or n_cols == n, x_offset == 0), or -- for a row-block
 * shard of a distributed matrix -- n rows over n_cols >= x_offset + n local
 * columns: the operand x then has n_cols entries and the shard's own rows'
 * entries are x[x_offset .. x_offset + n) (halo columns before and after,
 * numbered in global order so every sum keeps the single-GPU order). */
typedef struct {
  int64_t n;
  int64_t nnz;
  const int32_t *row_ptr;
  const int32_t *col_idx;
  const double *val;
  int64_t n_cols;    /* 0 -> n */
  int64_t x_offset;  /* 0 for a square matrix */
} abft_csr_t;

typedef struct abft_ctx *abft_handle_t;

/* Fault injection (PAPER.md SIV-A, and the rate model of P:284).
 * Test/experiment harness only; mode NONE (or inj == NULL) selects kernels
 * compiled without any injection code.
 *  LIST: entry e XORs list_mask[e] into the value produced for element
 *        list_index[e] of target list_target[e] (0 = y row, 1 = t1 block,
 *        2 = t2 block) in round list_round[e] (0 = main pass, r >= 1 = r-th
 *        correction round).  The list arrays are HOST arrays, copied.
 *  RATE: the paper's Poisson process with rate lambda per arithmetic
 *        operation (R13).  The call's operations are
 *        numbered y first (2 per A entry, row order), then t1 (2 per C
 *        entry, block order), then t2 (1 per row), and cut into chunks of
 *        CH = abft_rate_chunk(lambda) operations.  Chunk c of round r draws
 *        its event count from the Poisson(lambda * len) CDF table of
 *        abft_poisson_table with Philox4x32-10 (key {seed lo, seed hi},
 *        counter {c, 0, call, r<<8 | 0x80}) word 0; event e takes its offset
 *        floor(w0 * len / 2^32) and its burst from counter {c, e, call,
 *        r<<8 | 0x40}: start bit w1 & 63, length from w2 through the table of
 *        abft_burst_table.  An event hits the element its operation produces
 *        (row of y, block of t1 / t2); events on one element compose by XOR.
 *        `targets` masks the targets that receive events.  The plan is built
 *        on the device (5 short launches) by every call that injects. */
enum { ABFT_INJ_NONE = 0, ABFT_INJ_LIST = 1, ABFT_INJ_RATE = 2, ABFT_INJ_RESIDENT = 3 };
enum { ABFT_TARGET_Y = 0, ABFT_TARGET_T1 = 1, ABFT_TARGET_T2 = 2 };
typedef struct {
  uint32_t mode;
  uint64_t seed;
  uint64_t call;       /* SpMV call index (rate mode counter word 2) */
  double lambda;       /* rate mode: fault probability per arithmetic op */
  uint32_t targets;    /* rate mode: bit t => target t receives faults */
  int64_t n_list;      /* list mode */
  const int32_t *list_round;   /* (host) */
  const int32_t *list_target;  /* (host) */
  const int64_t *list_index;   /* (host) */
  const uint64_t *list_mask;   /* (host) */
} abft_inject_t;

/* RESIDENT (mode 3): reuse the device fault list the handle's last injecting
 * call (or abft_inject_prepare) built -- same faults, no plan generation: the
 * method's cost under faults is then timed without the injector's.
 * abft_inject_prepare: build the device list of `inj` (list upload, or the
 *   rate plan of inj->call, for the op counts of `mode`: CHECK or not)
 *   without running an SpMV; stream-ordered.
 * abft_inject_list: device pointers to that list: keys ((round << 58) |
 *   (target << 56) | index, ascending), XOR masks, its length (a device int32
 *   for rate plans, else *n_host) and capacity; valid until the next
 *   injecting call. */
abft_status abft_inject_prepare(abft_handle_t h, const abft_inject_t *inj, uint32_t mode,
                                void *stream);
abft_status abft_inject_list(abft_handle_t h, const uint64_t **keys, const uint64_t **masks,
                             const int32_t **n_dev, int32_t *n_host, int32_t *cap);
/* Zero the masks of the resident list (keys kept): RESIDENT calls then do
 * the injector's every lookup but change no value -- the harness control of
 * an overhead measurement (bench.py --lam-sweep).  Stream-ordered. */
abft_status abft_inject_clear_masks(abft_handle_t h, void *stream);

/* abft_spmv mode bits */
enum {
  ABFT_NOCHECK = 0,          /* plain y = A x (the unprotected baseline) */
  ABFT_CHECK = 1,            /* steps 1-4: y, t1, t2, s, beta, tau, flags */
  ABFT_AUTOCORRECT = 2,      /* + step 5: up to max_rounds correction rounds */
  ABFT_DEBUG_CHECKSUMS = 4,  /* also store t1, t2 per block (abft_debug_checksums) */
  ABFT_DEFER_FINISH = 8      /* distributed: run steps 1-3 only; beta comes from all
                                ranks (abft_beta_partial + abft_finish) */
};

/* Build C (CSR: nb rows, ascending columns = the non-empty columns of A_k,
 * values = column sums of A_k) and K_k = ((n_k + 2 b_s - 2)
 * * sum_{i in k} ||a_i||_2 + n_k ||c_k||_2) * 2^-53 (eps_M of P:154),
 * so that tau_k = K_k * ||x||_2.  block_size: power of two in [1, 1024]
 * (default 32 = the paper's choice; 64 .. 1024 run the
 * block-size sweep kernels of kernels_bigblock.cuh, one warp per block, for
 * Fig. 4 / Fig. 7 of P:248-270, not a tuned path); larger: ABFT_ENOTSUP.
 * max_rounds: correction rounds for ABFT_AUTOCORRECT / abft_pcg (>= 1, <= 16;
 * 0 -> 4).  flags: 0, or ABFT_ENCODE_C_CSR to stream C in the paper's plain
 * CSR form (FP64 values, int32 columns) instead of the lossless compact form
 * the encoder picks by default (values in the narrowest type that holds every
 * c_kj exactly -- int8 / int16 / float / double -- and columns as uint16
 * offsets from each row's first column, when every row spans < 65536
 * columns).  Both give bit-identical results.
 * Synchronises `stream` (sizes C, picks the format).
 * On success *out owns C, K and all scratch (device). */
enum { ABFT_ENCODE_C_CSR = 1 };
abft_status abft_encode(const abft_csr_t *A, int32_t block_size, int32_t max_rounds,
                        uint32_t flags, void *stream, abft_handle_t *out);

/* Encoding facts (host struct): sizes, the checksum-matrix format the fused
 * kernel streams and its byte count, and how the groups of 32 rows split
 * between the staged fast path and the general path. */
enum { ABFT_CFMT_CSR = 0, ABFT_CFMT_I8 = 1, ABFT_CFMT_I16 = 2, ABFT_CFMT_F32 = 3,
       ABFT_CFMT_F64 = 4,
       /* position-map records (row-regular matrices) */
       ABFT_CFMT_POS_I8 = 5, ABFT_CFMT_POS_I16 = 6, ABFT_CFMT_POS_F32 = 7, ABFT_CFMT_POS_F64 = 8 };
typedef struct {
  int64_t n, nnz, nb, nnz_c;
  int32_t block_size, c_format;
  int64_t c_bytes;          /* bytes of C (+ row pointers, bases) streamed per call */
  int64_t groups, general_groups;  /* 32-row groups; those on the general path */
  int32_t lean;             /* staged (TMA) path available */
  int32_t max_rounds;
  int64_t irr_groups;       /* 32-row groups on the irregular-row path (k_irr) */
  int32_t lean_short;       /* k_lean SHORT instantiation (all its rows <= 8 entries) */
  int32_t lean_runs;        /* k_lean walks interleaved runs of groups (large matrices) */
  int32_t stream;           /* warp-specialized kernel (position-map records) in use */
  int32_t stream_g;         /* its groups per chunk (consumer warps per CTA) */
  int32_t stream_stages;    /* its ring stages */
  int32_t col_perm;         /* irregular path gathers x through a popularity-ordered copy
                               (renumbered column arrays, one scatter of x per call;
                               DESIGN.md §6.10) */
  int64_t pos_exc_rows;     /* exception rows over all position-map records */
  int64_t stream_plain_bytes;  /* bytes the warp-specialized kernel streams per call with the
                                  check off (A values and columns, structure records, x, y),
                                  0 if unused */
  int64_t stream_check_bytes;  /* bytes the check adds (checksum records) */
  int64_t hub_chunks;       /* aligned 1024-entry chunks of hub rows (k_hub items) */
} abft_info_t;
abft_status abft_info(abft_handle_t h, abft_info_t *info);

/* Protected SpMV y = A x (steps 1-4), optionally with correction
 * (mode | ABFT_AUTOCORRECT, step 5).  x and y: device [n], must not alias.
 * x_norm: nullable DEVICE scalar holding ||x||_2 if the caller already has it
 * (PW-exact value required for oracle parity); NULL -> computed in-pass.
 * inj: nullable (no injection).  Flagged blocks stay on the device
 * (abft_flags); nothing is copied to the host. */
abft_status abft_spmv(abft_handle_t h, const double *x, double *y, const double *x_norm,
                      const abft_inject_t *inj, uint32_t mode, void *stream);

/* Distributed protected SpMV (row-block shards).  After
 * abft_spmv(..., mode | ABFT_DEFER_FINISH), abft_beta_partial enqueues the
 * PW of this shard's sum of x_i^2 over its own rows into the caller's device
 * scalar *partial.  Gather the partials of all ranks in rank order (e.g. an NCCL
 * all-gather) into a device array and call abft_finish: beta =
 * sqrt(PW(parts)) -- bit-identical to the single-GPU beta when every shard
 * owns an aligned power-of-two row range -- then step 4 (flags) and up to
 * `rounds` correction rounds (step 5). */
abft_status abft_beta_partial(abft_handle_t h, double *partial, void *stream);
abft_status abft_finish(abft_handle_t h, const double *x, double *y, const double *parts,
                        int32_t nparts, int32_t rounds, const abft_inject_t *inj, void *stream);

/* Step 5 alone: rounds r = 1..max_rounds recompute the rows of
 * the blocks flagged in round r-1, recompute t1/t2 and re-check; blocks that
 * still fail form round r's list.  Uses beta of the last abft_spmv.  `inj`
 * must describe the same call as that abft_spmv (rate mode: the same seed,
 * lambda, targets and call index); the rate plan it built is reused from the
 * device list when those match (abft_finish likewise), else rebuilt. */
abft_status abft_correct(abft_handle_t h, const double *x, double *y, int32_t max_rounds,
                         const abft_inject_t *inj, void *stream);

/* Device pointers to round `round`'s flagged-block list (unordered set of
 * 0-based block indices) and its length (device int32).  Round 0 = detection;
 * round r = blocks still failing after correction round r.  Valid until the
 * next call on the handle.  round in [0, max_rounds]. */
abft_status abft_flags(abft_handle_t h, int32_t round, const int32_t **flagged,
                       const int32_t **n_flagged);

/* Device pointer to beta = ||x||_2 of the last abft_spmv (device
 * double).  The fused kernel completes beta only when a block needs it (a
 * detection candidate) or x_norm was given; otherwise this call enqueues the
 * PW reduction of the per-group partial sums on `stream` first. */
abft_status abft_beta(abft_handle_t h, void *stream, const double **beta);

/* Device pointers to the encoded checksum matrix and bound constants. */
abft_status abft_checksum_matrix(abft_handle_t h, const int32_t **c_row_ptr,
                                 const int32_t **c_col, const double **c_val, const double **K,
                                 int64_t *nnz_c, int64_t *nb);

/* Device pointers to t1 / t2 of the last abft_spmv run with
 * ABFT_DEBUG_CHECKSUMS (values after injection, before correction). */
abft_status abft_debug_checksums(abft_handle_t h, const double **t1, const double **t2);

/* End-to-end call with HOST buffers: copies x (host, pinned recommended) to
 * the device, runs abft_spmv(mode), copies y back to y_host and the round-0
 * flag count to *n_flagged_host (nullable), then synchronises `stream`. */
abft_status abft_spmv_host(abft_handle_t h, const double *x_host, double *y_host,
                           int32_t *n_flagged_host, uint32_t mode, void *stream);

/* The same for a stream of nsteps products with HOST buffers: step k copies
 * x_hosts[k] (n_cols doubles, pinned recommended) in, runs abft_spmv(mode)
 * and copies y_hosts[k] (n doubles) and n_flagged_hosts[k] (nullable array,
 * round-0 flag count) out.  Two device buffer slots and separate copy-in /
 * copy-out streams overlap step k's copies with steps k-1 / k+1 (x_k's
 * upload, y_{k-1}'s download and the products run concurrently).  No
 * injection.  Synchronises before returning. */
/* Page-locked host memory from the library's own CUDA runtime (the host
 * buffers of the two calls above: the library's runtime then sees them as
 * pinned, so its copies are asynchronous and overlap; memory pinned by
 * another runtime instance may be staged synchronously).  abft_host_free
 * releases it. */
abft_status abft_host_alloc(int64_t bytes, void **p);
abft_status abft_host_free(void *p);

abft_status abft_spmv_host_pipelined(abft_handle_t h, const double *const *x_hosts,
                                     double *const *y_hosts, int32_t nsteps,
                                     int32_t *n_flagged_hosts, uint32_t mode, void *stream);

/* PCG statistics (host struct). */
typedef struct {
  int64_t iters;
  int64_t spmv_calls;
  int64_t flagged_blocks;    /* sum over SpMV calls of round-0 flags */
  int64_t recomputed_blocks; /* sum over calls and rounds of recomputed blocks */
  int64_t uncorrected_calls; /* calls that ended with blocks still flagged */
  int32_t converged;
  double final_residual;     /* ||r||_2 of the recursive residual */
} abft_pcg_stats_t;

/* Jacobi-PCG (Saad Alg. 9.1) for SPD A: solves A x = b from the
 * initial guess in x (overwritten with the solution).  diag: nullable device
 * [n] (NULL -> the diagonal of A).  Stops when ||r||_2 <= tol * ||b||_2
 * (R16) or after max_iter iterations (<= 0 -> 10 N);
 * check | ABFT_PCG_LITERAL_STOP: stops when r^T r < tol instead (P:296's
 * "||r_k|| = r_k^T r_k < eps" read literally, R16*; not with check == 2).
 * check == 1 protects every SpMV (detect + correct); check == 0 runs the
 * unprotected baseline with the same kernels; check == 2 runs the related-work
 * CHECKPOINTING baseline: every SpMV checked by
 * the dense check with tau = ||v||_2 (needs abft_dense_encode), the
 * state (x, r, z, p, rho) sampled every 20 iterations and restored
 * on a detection; rate faults hit y only; max_iter bounds executed
 * iterations; stats: flagged_blocks = rollbacks, recomputed_blocks =
 * discarded iterations (R26-R27).  inj: nullable; its `call`
 * is the index of the first SpMV (call + j for the j-th).  res_hist:
 * nullable device [max_iter + 1] of ||r_j||_2.  stats: nullable (host).
 * b, x, diag and res_hist must be 16-byte aligned (128-bit vector accesses;
 * ABFT_EINVAL otherwise).
 * Synchronises the stream.  Returns ABFT_OK, ABFT_ENOCONV or ABFT_EBREAKDOWN. */
enum { ABFT_PCG_LITERAL_STOP = 0x100 };
abft_status abft_pcg(abft_handle_t h, const double *b, double *x, const double *diag,
                     double tol, int64_t max_iter, const abft_inject_t *inj, int32_t check,
                     double *res_hist, abft_pcg_stats_t *stats, void *stream);

/* --- Distributed Jacobi-PCG (Saad Alg. 9.1) ---
 * The rows are sharded across ranks (one process per GPU); the handle is the
 * rank's shard (abft_encode of the local rows, n_cols / x_offset set).  The
 * iteration is abft_pcg's, split at its global reductions so the caller can
 * all-gather the per-rank partials between the kernels (NCCL; 24 bytes per
 * rank per phase) and then finish them on the device in rank order:
 *   begin; SpMV q = A x0 (the caller's distributed protected SpMV over the
 *   halo-extended operand); local(INIT) -> gather -> combine(INIT);
 *   per iteration j = 1, 2, ...: SpMV q = A p; local(DOT) -> gather ->
 *   combine(DOT); local(UPDATE, j) -> gather -> combine(UPDATE, j);
 *   local(P, j); poll abft_pcg_dist_status every few iterations.
 * A global sum is PW over the ranks (padded with absent slots) of each rank's
 * PW over its own rows (R2, R28): for equal power-of-two row ranges
 * aligned to 2048 rows, the single-GPU sums bit for bit.
 * abft_pcg_dist_begin: b, x (in x0, out x), q (the SpMV result, [n]) and diag
 *   (nullable: the diagonal of A at local column row + x_offset) are the
 *   rank's own rows, 16-byte aligned; pext is the own slice of the SpMV's
 *   halo-extended operand (any alignment; p is written there too); max_iter
 *   > 0 (the caller passes 10 N of the global matrix); check 0 | 1 as
 *   abft_pcg; res_hist nullable device [max_iter + 1].  Stream-ordered.
 * abft_pcg_dist_local: phase 0 INIT (r = b - q, z = r/d, p = z; partials
 *   r.z, r.r, b.b), 1 DOT (p.q), 2 UPDATE (x, r, z; partials r.z, r.r),
 *   3 P (p = z + beta p; no partial).  send: device double[3] (unused for P).
 *   Kernels of a finished solve are no-ops.
 * abft_pcg_dist_combine: recv = device double[3 * world] (rank r at 3r);
 *   1 <= world <= 64; phases 0-2; updates the device scalars.
 * abft_pcg_dist_status: host copies of the state (0 running, 1 converged, 2
 *   breakdown, 3 max_iter) and rank-local stats; synchronises the stream. */
#define ABFT_PCG_PHASE_INIT 0
#define ABFT_PCG_PHASE_DOT 1
#define ABFT_PCG_PHASE_UPDATE 2
#define ABFT_PCG_PHASE_P 3
/* Single-reduction (Chronopoulos-Gear) variant (DESIGN.md
 * R29; beyond the paper): s = A p is carried by recurrence, so each
 * iteration needs ONE gather of (r.u, r.r, w.u) instead of two.  Sequence
 * after begin: SpMV q = A x0; local(INIT) -> gather -> combine(INIT); SpMV
 * w = A u0 (the operand's own slice holds u0); local(CG1_DOT, 0) -> gather ->
 * combine(CG1_DOT, 0); per iteration j >= 1: local(CG1_UPDATE, j) (p, s, x,
 * r, u; partials r.u, r.r in send[0..2)); SpMV w = A u; local(CG1_DOT, j)
 * (partial w.u in send[2]); gather -> combine(CG1_DOT, j).  q is w. */
#define ABFT_PCG_PHASE_CG1_UPDATE 4
#define ABFT_PCG_PHASE_CG1_DOT 5
abft_status abft_pcg_dist_begin(abft_handle_t h, const double *b, double *x, double *pext,
                                double *q, const double *diag, double tol, int64_t max_iter,
                                int32_t check, double *res_hist, void *stream);
abft_status abft_pcg_dist_local(abft_handle_t h, int32_t phase, int64_t iter, double *send,
                                void *stream);
abft_status abft_pcg_dist_combine(abft_handle_t h, int32_t phase, int64_t iter,
                                  const double *recv, int32_t world, void *stream);
abft_status abft_pcg_dist_status(abft_handle_t h, int32_t *state, abft_pcg_stats_t *stats,
                                 void *stream);

/* --- Multi-GPU: row-block shards inside the library (
 * DESIGN.md §8) ---
 * The paper runs one GPU; the split follows north_star: contiguous
 * row ranges, one rank per GPU, one exchange per SpMV (the x halo) plus the
 * all-gather of each rank's ||x||^2 partial (8 bytes per rank) that makes
 * beta = sqrt(PW over the ranks, in rank order, of each rank's PW over its own
 * rows) -- bit-identical to one GPU for equal power-of-two ranges (R28).
 * Row blocks never straddle ranks (row boundaries multiples of block_size),
 * so C, detection and correction stay rank-local.
 *
 * abft_dist_unique_id: a 128-byte NCCL unique id (host); rank 0 makes it and
 *   the caller broadcasts it (torch.distributed, MPI, a file ...).
 * abft_dist_create: ranges = host int64 [world + 1] row boundaries (ranges[0]
 *   = 0, ranges[world] = n_global, non-decreasing); nccl_id = the 128-byte id
 *   (host) -> an NCCL communicator over the `world` ranks (collective: every
 *   rank calls it; the current device is this rank's GPU), or NULL -> no
 *   communicator: the caller moves the exchange buffers itself
 *   (abft_dist_begin / abft_dist_buffers / abft_dist_end; tests, other
 *   transports).  The dist object must outlive its handles.
 * abft_dist_encode: this rank's rows as CSR with GLOBAL column indices (n =
 *   ranges[rank+1] - ranges[rank] rows, n_cols / x_offset ignored).  Builds
 *   the local column order [halo below | own | halo above] (global order, so
 *   every sum sees the single-GPU operands in the single-GPU order), a
 *   handle-owned copy of the renumbered columns (row_ptr and values stay the
 *   caller's and must outlive the handle), the halo plan (per peer: the
 *   contiguous slice of the extended operand it fills, and the own entries
 *   it needs), the checksum encoding of the local rows (as abft_encode), and
 *   the split of the blocks into interior (no halo column) and boundary
 *   ones.  With a communicator the ranks exchange their needs over NCCL
 *   (collective); without one the caller reads abft_dist_needs and sets
 *   abft_dist_set_send for every peer.  Synchronises.
 * abft_dist_operand: device pointer to the handle's halo-extended operand
 *   (n_cols doubles) and the offset of the own slice; a caller (the PCG) may
 *   write its own x there directly.
 * abft_dist_spmv (communicator only): one distributed protected SpMV of the
 *   own x (device [n_own]; NULL = already in the operand's own slice) into
 *   y (device [n_own]); mode / inj as abft_spmv (fault indices rank-local).
 *   Enqueues on `stream`: the pack kernel (send buffer + x^2 partial), the
 *   NCCL group (halo send/recv + partial all-gather) on the handle's comm
 *   stream, the interior blocks meanwhile, then beta, the boundary blocks,
 *   the finish and the corrections.  Asynchronous; collective.
 * abft_dist_begin / abft_dist_end (either mode; abft_dist_spmv = begin +
 *   exchange + end): begin copies x_own into the operand (unless NULL) and
 *   packs the send buffers and the partial; the caller then delivers, for
 *   every peer p, p's send buffer for this rank into this rank's receive
 *   slice for p (abft_dist_buffers, device pointers, counts in doubles) and
 *   all ranks' partials, in rank order, into a device array parts[world]
 *   (abft_dist_partial); end runs the fused kernels, the finish and the
 *   corrections with beta = sqrt(PW(parts)).
 * abft_dist_pcg (communicator only): the distributed Jacobi-PCG of
 *   abft_pcg_dist_* with every exchange (halo, beta, dot partials) inside
 *   the library; b, x own rows (device), diag nullable, max_iter <= 0 -> 10 N
 *   of the global matrix; inj->call counts this rank's SpMVs (rate mode: the
 *   seed is the caller's, e.g. distinct per rank); variant 0 = textbook
 *   PCG (two reductions per iteration), 1 = single reduction (R29).
 *   Fault-free solves replay a CUDA graph of 16 captured iterations (kernels,
 *   NCCL calls, cross-stream events), cached per buffer set; faulty solves
 *   are sequenced eagerly (ABFT_DIST_PCG_EAGER=1 forces eager sequencing).
 *   Synchronises; every rank returns the same status.
 * abft_halo_plan (host only, no GPU): the local column order of abft_dist_
 *   encode for host arrays -- local_col [nnz], *n_below / *n_above, per peer
 *   recv_start / recv_count [world], halo = the global index of every halo
 *   column in operand order (capacity cap; NULL with cap 0 to count only). */
typedef struct abft_dist *abft_dist_t;
abft_status abft_dist_unique_id(void *nccl_id);
abft_status abft_dist_create(int32_t rank, int32_t world, const int64_t *ranges,
                             const void *nccl_id, abft_dist_t *out);
abft_status abft_dist_destroy(abft_dist_t d);
abft_status abft_dist_encode(abft_dist_t d, const abft_csr_t *A_rows, int32_t block_size,
                             int32_t max_rounds, uint32_t flags, void *stream, abft_handle_t *out);
abft_status abft_dist_needs(abft_handle_t h, int32_t peer, int64_t *count, int64_t *global_idx);
abft_status abft_dist_set_send(abft_handle_t h, int32_t peer, const int64_t *global_idx,
                               int64_t count);
abft_status abft_dist_operand(abft_handle_t h, double **x_ext, int64_t *n_cols,
                              int64_t *own_offset);
abft_status abft_dist_spmv(abft_handle_t h, const double *x_own, double *y,
                           const abft_inject_t *inj, uint32_t mode, void *stream);
abft_status abft_dist_begin(abft_handle_t h, const double *x_own, void *stream);
abft_status abft_dist_buffers(abft_handle_t h, int32_t peer, const double **send,
                              int64_t *send_count, double **recv, int64_t *recv_count);
abft_status abft_dist_partial(abft_handle_t h, const double **part);
abft_status abft_dist_end(abft_handle_t h, double *y, const double *parts,
                          const abft_inject_t *inj, uint32_t mode, void *stream);
abft_status abft_dist_pcg(abft_handle_t h, const double *b, double *x, const double *diag,
                          double tol, int64_t max_iter, const abft_inject_t *inj, int32_t check,
                          int32_t variant, double *res_hist, abft_pcg_stats_t *stats,
                          void *stream);
abft_status abft_halo_plan(int32_t rank, int32_t world, const int64_t *ranges, const int32_t *col,
                           int64_t nnz, int32_t *local_col, int64_t *n_below, int64_t *n_above,
                           int64_t *recv_start, int64_t *recv_count, int64_t *halo, int64_t cap);

/* --- Related-work baseline: DENSE CHECK [30, 31] + COMPLETE RECOMPUTATION ---
 * (eq. (1), P:148-152 [35]'s bound, P:240, P:250-252,
 * P:258, R23-R25.)  One checksum
 * over all N rows: c = 1^T A (c_j = PW over column j in row order), t1 = PW_j
 * c_j x_j, t2 = PW_i y_i, flag iff NOT(|t1 - t2| <= tau) with tau = ||x||_2
 * (the norm-based bound of [30]) or, with ABFT_DENSE_BOUND35,
 * tau = K35 ||x||_2, K35 = ((n + 2N - 2) PW_i ||a_i||_2 + n ||c||_2) 2^-53.
 * A flag under ABFT_AUTOCORRECT recomputes ALL of y and re-checks, at most
 * max_rounds times (complete recomputation).  Square handles only
 * (ABFT_ENOTSUP for shards).  List injection: target 0 = y row, target 1 / 2
 * index 0 = t1 / t2 of the check.  Rate mode: the plan of R13 over the
 * SpMV's y operations of round 0 only (the 3N operations of the check are not
 * injected; R25).
 * abft_dense_encode: builds c and K35 on the device (owned by the handle;
 *   temporaries of ~17 B per nonzero during the call); synchronises.
 * abft_spmv_dense: the method's SpMV kernels with the check off, then one
 *   persistent check/recompute kernel; asynchronous, results stay on device.
 * abft_dense_result: host copies of round 0's (t1, t2, beta, tau) [4], the
 *   per-round flags [max_rounds+1] (1 = round r's check failed) and K35;
 *   each pointer nullable; synchronises. */
#define ABFT_DENSE_BOUND35 16u
abft_status abft_dense_encode(abft_handle_t h, void *stream);
abft_status abft_spmv_dense(abft_handle_t h, const double *x, double *y,
                            const abft_inject_t *inj, uint32_t mode, void *stream);
abft_status abft_dense_result(abft_handle_t h, double *out, int32_t *flag_rounds, double *k35,
                              void *stream);
/* Device pointer to c [n] (valid until abft_destroy). */
abft_status abft_dense_checksum(abft_handle_t h, const double **c);

abft_status abft_destroy(abft_handle_t h);

/* Device-side health of a handle.  The finish / correction and dense-check
 * kernels synchronise their CTAs with a software grid barrier that needs all
 * CTAs (one per SM) co-resident; when other work holds SMs the barrier times
 * out after about a second instead of hanging, and the calls that hit it
 * leave incomplete results.  abft_health synchronises
 * `stream`, sets *err = 1 if a barrier timed out since the last call (else
 * 0) and then clears the error word and resets the barrier.  abft_pcg checks
 * it before returning (ABFT_ECUDA on a timeout). */
abft_status abft_health(abft_handle_t h, void *stream, int32_t *err);

/* Plumbing for bindings: cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDefault)
 * on `stream`, then synchronise it.  Used to read the device-resident results
 * above (flags, counts, C, K, beta) without a second CUDA binding. */
abft_status abft_memcpy(void *dst, const void *src, int64_t bytes, void *stream);

/* Host helpers (no GPU needed). */
const char *abft_status_string(abft_status st);
const char *abft_last_cuda_error(void);
/* Fault-model tables (R13), host only:
 * abft_burst_table: T[l] = floor(2^32 P(L <= l)) for the burst length
 *   L = max(1, round(3 + sqrt(2) Z)), from the C library's erfc.
 * abft_poisson_table: the Poisson(mu) event-count CDF table of rate mode
 *   (floor(2^32 F(k)), last entry 2^32); returns its length (<= cap), 0 on a
 *   bad argument.
 * abft_rate_chunk: operations per chunk of rate mode for lambda. */
void abft_burst_table(uint64_t T[65]);
int32_t abft_poisson_table(double mu, uint64_t *T, int32_t cap);
int64_t abft_rate_chunk(double lambda);
/* Library version string. */
const char *abft_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ABFT_H */
