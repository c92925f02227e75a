// kernels_pcg.cuh -- Jacobi-PCG vector kernels (SVI-A; Saad
// Alg. 9.1).  The SpMV q = A p is the protected k_lean/k_general/k_finish
// set; these kernels fuse the vector updates with their dot products.
//
// Every dot is PW over the global index (R2): a CTA owns an aligned chunk of
// kPcgRows = 2048 rows; thread t holds rows 8t..8t+7 of it (vector loads),
// reduces them with an 8-leaf register tree, the warp's 32 sums by the xor
// butterfly (an aligned 256-row node) and the 8 warp sums by a tree -- the
// chunk's PW node.  The last CTA (atomic ticket) completes the tree over the
// chunk sums and updates the scalars, so an iteration needs no host round
// trip.  A device `state` word turns every kernel of a finished solve into a
// no-op.
#pragma once
#include "abft_device.cuh"

namespace abft {

constexpr int kPcgThreads = 256;
constexpr int kPcgPer = 8;                         // rows per thread
constexpr int kPcgRows = kPcgThreads * kPcgPer;    // rows per CTA (aligned)

enum { PCG_RUN = 0, PCG_CONVERGED = 1, PCG_BREAKDOWN = 2, PCG_MAXITER = 3 };

struct PcgScalars {
  double rho, pq, alpha, beta, res, thr;
  int64_t it, max_iter;
  int64_t flagged, recomputed, uncorrected, calls;
  int32_t state;
  int32_t skip_it;           // checkpoint mode: this iteration was rolled back
  int64_t upd;               // host iteration index of the last executed update
  double ck_rho, ck_res;     // checkpoint mode: sampled scalars
  int64_t ck_it;
  int64_t j;                 // device-resident loop: the next iteration's index (1-based)
};

struct PcgArgs {
  int64_t n;
  int64_t ns;  // stride of the scratch vectors (n rounded up to even: 16-B aligned)
  const double *__restrict__ b;
  double *x, *r, *z, *p, *q;
  const double *__restrict__ d;
  double *part0, *part1, *part2;  // per-CTA chunk sums
  unsigned *ticket;
  PcgScalars *sc;
  double *hist;                   // nullable
  double tol;
  const int32_t *n_flags;         // protected-SpMV flag counts (stats)
  int32_t max_rounds;
  int32_t check;
  // checkpoint-rollback baseline: dense-check flag of the
  // iteration's SpMV, sampled x | r | z | p (4 n), sampling interval
  int32_t cr;
  int32_t ckpt_every;
  const int32_t *dflag;
  double *ck;
  // distributed PCG (abft_pcg_dist_*): nullable.  dsend: the last CTA writes
  // this rank's chunk-tree sums here instead of updating the scalars (the
  // combine kernel finishes them over all ranks); pext: p is also written to
  // the own slice of the halo-extended SpMV operand (any alignment).
  double *dsend;
  double *pext;
  double *s;  // single-reduction variant (cg1): s = A p, updated by recurrence
  // stopping rule: 0 = ||r|| <= tol ||b|| (R16); 1 = r^T r < tol (P:296 read
  // literally, R16*)
  int32_t literal;
};

// The stopping test on res = ||r|| (R16) or RR = r^T r (R16*); thr is
// tol ||b|| resp. tol.
__device__ __forceinline__ bool pcg_done(const PcgArgs &a, double res, double RR, double thr) {
  return a.literal ? (RR < thr) : (res <= thr);
}

// Eight consecutive doubles v[0..8) at p + 8t (or absent past n).
__device__ __forceinline__ void ld8(double (&v)[8], const double *p, int64_t i0, int64_t n) {
  if (i0 + 8 <= n) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const double2 w = *reinterpret_cast<const double2 *>(p + i0 + 2 * u);
      v[2 * u] = w.x;
      v[2 * u + 1] = w.y;
    }
  } else {
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = i0 + u < n ? p[i0 + u] : 0.0;
  }
}
__device__ __forceinline__ void st8(double *p, const double (&v)[8], int64_t i0, int64_t n) {
  if (i0 + 8 <= n) {
#pragma unroll
    for (int u = 0; u < 4; ++u)
      *reinterpret_cast<double2 *>(p + i0 + 2 * u) = make_double2(v[2 * u], v[2 * u + 1]);
  } else {
#pragma unroll
    for (int u = 0; u < 8; ++u)
      if (i0 + u < n) p[i0 + u] = v[u];
  }
}

// CTA chunk sum: per-thread 8-leaf tree (absent past n), warp butterfly,
// tree over the 8 warps.  All threads get the result.
__device__ __forceinline__ double cta_pw(double (&v)[8], int64_t i0, int64_t n, double *s_w) {
#pragma unroll
  for (int u = 0; u < 8; ++u)
    if (i0 + u >= n) v[u] = kAbsent;
  double t = bfly32(tree<8>(v));
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  __syncthreads();
  if (lane == 0) s_w[warp] = t;
  __syncthreads();
  double w[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) w[q] = s_w[q];
  return tree<8>(w);
}

// Two chunk sums at once (one barrier pair): s_w holds 16 doubles.
__device__ __forceinline__ void cta_pw2(double (&v)[8], double (&w)[8], int64_t i0, int64_t n,
                                        double *s_w, double &out_v, double &out_w) {
#pragma unroll
  for (int u = 0; u < 8; ++u)
    if (i0 + u >= n) v[u] = w[u] = kAbsent;
  double t = tree<8>(v), q = tree<8>(w);
#pragma unroll
  for (int m = 1; m < 32; m <<= 1) {
    t = dadd(t, __shfl_xor_sync(kFull, t, m));
    q = dadd(q, __shfl_xor_sync(kFull, q, m));
  }
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  __syncthreads();
  if (lane == 0) {
    s_w[warp] = t;
    s_w[8 + warp] = q;
  }
  __syncthreads();
  double a[8], b[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    a[k] = s_w[k];
    b[k] = s_w[8 + k];
  }
  out_v = tree<8>(a);
  out_w = tree<8>(b);
}

// Last-CTA completion of PW over partials[0..ncta) (aligned chunk nodes):
// thread t reduces an aligned run of m partials in registers (m <= 16; a
// PwSeq beyond), the ascending xor butterfly joins the 32 runs of a warp and
// an 8-leaf tree the 8 warps -- the PW tree over 256 m slots with absent
// padding (R2).  Two arrays at once (their latency chains overlap); p1 may
// be null.  All threads get the results.
__device__ __forceinline__ void grid_pw2(const double *p0, const double *p1, int ncta, double *s_red,
                                         double &o0, double &o1) {
  int m = 1;
  while (m * kPcgThreads < ncta) m <<= 1;
  const int b = threadIdx.x * m;
  double t0, t1 = kAbsent;
  if (m <= 16) {
    double v0[16], v1[16];
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      const bool in = q < m && b + q < ncta;
      v0[q] = in ? __ldcg(p0 + b + q) : kAbsent;
      v1[q] = (in && p1) ? __ldcg(p1 + b + q) : kAbsent;
    }
    t0 = tree<16>(v0);
    t1 = tree<16>(v1);
  } else {
    PwSeq a0, a1;
    for (int q = b; q < min(b + m, ncta); ++q) {
      a0.push(__ldcg(p0 + q));
      if (p1) a1.push(__ldcg(p1 + q));
    }
    t0 = a0.finish();
    if (p1) t1 = a1.finish();
  }
#pragma unroll
  for (int sft = 1; sft < 32; sft <<= 1) {
    t0 = dadd(t0, __shfl_xor_sync(kFull, t0, sft));
    t1 = dadd(t1, __shfl_xor_sync(kFull, t1, sft));
  }
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  __syncthreads();
  if (lane == 0) {
    s_red[warp] = t0;
    s_red[8 + warp] = t1;
  }
  __syncthreads();
  double w0[8], w1[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    w0[k] = s_red[k];
    w1[k] = s_red[8 + k];
  }
  o0 = tree<8>(w0);
  o1 = tree<8>(w1);
}
__device__ __forceinline__ double grid_pw(const double *partials, int ncta, double *s_red) {
  double o0, o1;
  grid_pw2(partials, nullptr, ncta, s_red, o0, o1);
  return o0;
}

// Ticket: true in the last CTA to finish (after its partials are written).
__device__ __forceinline__ bool last_cta(unsigned *ticket, int *s_flag) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned t = atomicAdd(ticket, 1u);
    *s_flag = (t == gridDim.x - 1);
  }
  __syncthreads();
  if (*s_flag) __threadfence();
  return *s_flag;
}

__device__ __forceinline__ bool pcg_skip(const PcgScalars *sc) {
  return *(volatile const int32_t *)&sc->state != PCG_RUN ||
         *(volatile const int32_t *)&sc->skip_it != 0;
}

__device__ __forceinline__ void pcg_stats(const PcgArgs &a, PcgScalars *sc) {
  if (a.cr) return;  // checkpoint mode counts in k_pcg_cr
  sc->calls += 1;
  if (a.check) {
    const int32_t *nf = a.n_flags;
    sc->flagged += nf[0];
    for (int r = 0; r < a.max_rounds; ++r) sc->recomputed += nf[r];
    if (nf[a.max_rounds] > 0) sc->uncorrected += 1;
  }
}

// diag(A) (R21; missing diagonal -> 0, as the oracle)
__global__ void k_pcg_diag(int64_t n, int64_t off, const int32_t *__restrict__ rp,
                           const int32_t *__restrict__ ci, const double *__restrict__ va,
                           double *d) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  double v = 0.0;
  for (int32_t q = rp[i]; q < rp[i + 1]; ++q)
    if (ci[q] == i + off) v = va[q];
  d[i] = v;
}

// Scalar steps of each kernel's last CTA, shared with the distributed
// combine (k_pcg_comb), which calls them with the all-rank sums.
__device__ __forceinline__ void init_scalars(const PcgArgs &a, double RZ, double RR, double BB) {
  PcgScalars *sc = a.sc;
  pcg_stats(a, sc);  // the SpMV q = A x0
  sc->rho = RZ;
  sc->res = __dsqrt_rn(RR);
  sc->thr = a.literal ? a.tol : dmul(a.tol, __dsqrt_rn(BB));
  sc->it = 0;
  if (a.hist) a.hist[0] = sc->res;
  sc->state = pcg_done(a, sc->res, RR, sc->thr) ? PCG_CONVERGED
                                                : (sc->max_iter <= 0 ? PCG_MAXITER : PCG_RUN);
  if (!(sc->res == sc->res)) sc->state = PCG_BREAKDOWN;
  if (a.cr) {
    sc->calls += 1;
    sc->skip_it = 0;
    sc->ck_rho = sc->rho;
    sc->ck_res = sc->res;
    sc->ck_it = 0;
  }
}

__device__ __forceinline__ void dot_scalars(const PcgArgs &a, double PQ) {
  PcgScalars *sc = a.sc;
  pcg_stats(a, sc);
  sc->pq = PQ;
  if (!(PQ > 0.0))
    sc->state = PCG_BREAKDOWN;
  else
    sc->alpha = __ddiv_rn(sc->rho, PQ);
}

__device__ __forceinline__ void update_scalars(const PcgArgs &a, int64_t iter, double RZ,
                                               double RR) {
  PcgScalars *sc = a.sc;
  const double res = __dsqrt_rn(RR);
  sc->it += 1;
  sc->res = res;
  if (a.hist) a.hist[sc->it] = res;
  sc->beta = __ddiv_rn(RZ, sc->rho);
  sc->rho = RZ;
  sc->upd = iter;
  if (pcg_done(a, res, RR, sc->thr)) sc->state = PCG_CONVERGED;
  else if (!(res == res)) sc->state = PCG_BREAKDOWN;
  else if (sc->it >= sc->max_iter) sc->state = PCG_MAXITER;
}

// p's copy in the halo-extended operand (distributed PCG): scalar stores,
// the own slice need not be 16-byte aligned.
__device__ __forceinline__ void st8_ext(double *p, const double (&v)[8], int64_t i0, int64_t n) {
  if (!p) return;
#pragma unroll
  for (int u = 0; u < 8; ++u)
    if (i0 + u < n) p[i0 + u] = v[u];
}

// r = b - q; z = r / d; p = z; rho = PW(r.z); res = ||r||; thr = tol ||b||
__global__ void __launch_bounds__(kPcgThreads) k_pcg_init(const PcgArgs a) {
  __shared__ double s_w[8];
  __shared__ double s_red[kPcgThreads];
  __shared__ int s_flag;
  const int64_t i0 = (int64_t)blockIdx.x * kPcgRows + threadIdx.x * kPcgPer;
  double bv[8], qv[8], dv[8], r[8], z[8], rz[8], rr[8], bb[8];
  ld8(bv, a.b, i0, a.n);
  ld8(qv, a.q, i0, a.n);
  ld8(dv, a.d, i0, a.n);
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    r[u] = dsub(bv[u], qv[u]);
    z[u] = __ddiv_rn(r[u], dv[u]);
    rz[u] = dmul(r[u], z[u]);
    rr[u] = dmul(r[u], r[u]);
    bb[u] = dmul(bv[u], bv[u]);
  }
  st8(a.r, r, i0, a.n);
  st8(a.z, z, i0, a.n);
  st8(a.p, z, i0, a.n);
  st8_ext(a.pext, z, i0, a.n);
  if (a.cr) {  // sample 0: x0, r0, z0, p0
    double xv[8];
    ld8(xv, a.x, i0, a.n);
    st8(a.ck, xv, i0, a.n);
    st8(a.ck + a.ns, r, i0, a.n);
    st8(a.ck + 2 * a.ns, z, i0, a.n);
    st8(a.ck + 3 * a.ns, z, i0, a.n);
  }
  const double RZc = cta_pw(rz, i0, a.n, s_w);
  const double RRc = cta_pw(rr, i0, a.n, s_w);
  const double BBc = cta_pw(bb, i0, a.n, s_w);
  if (threadIdx.x == 0) {
    a.part0[blockIdx.x] = RZc;
    a.part1[blockIdx.x] = RRc;
    a.part2[blockIdx.x] = BBc;
  }
  if (!last_cta(a.ticket, &s_flag)) return;
  double RZ, RR, BB, unused;
  grid_pw2(a.part0, a.part1, gridDim.x, s_red, RZ, RR);
  grid_pw2(a.part2, nullptr, gridDim.x, s_red, BB, unused);
  if (threadIdx.x == 0) {
    if (a.dsend) {
      a.dsend[0] = RZ;
      a.dsend[1] = RR;
      a.dsend[2] = BB;
    } else {
      init_scalars(a, RZ, RR, BB);
    }
    *a.ticket = 0u;
  }
}

// pq = PW(p.q); alpha = rho / pq; protected-SpMV statistics.
__global__ void __launch_bounds__(kPcgThreads) k_pcg_dot(const PcgArgs a) {
  __shared__ double s_w[8];
  __shared__ double s_red[kPcgThreads];
  __shared__ int s_flag;
  if (pcg_skip(a.sc)) return;
  const int64_t i0 = (int64_t)blockIdx.x * kPcgRows + threadIdx.x * kPcgPer;
  double pv[8], qv[8];
  ld8(pv, a.p, i0, a.n);
  ld8(qv, a.q, i0, a.n);
#pragma unroll
  for (int u = 0; u < 8; ++u) pv[u] = dmul(pv[u], qv[u]);
  const double PQc = cta_pw(pv, i0, a.n, s_w);
  if (threadIdx.x == 0) a.part0[blockIdx.x] = PQc;
  if (!last_cta(a.ticket, &s_flag)) return;
  const double PQ = grid_pw(a.part0, gridDim.x, s_red);
  if (threadIdx.x == 0) {
    if (a.dsend)
      a.dsend[0] = PQ;
    else
      dot_scalars(a, PQ);
    *a.ticket = 0u;
  }
}

// pq = PW(p.q) from the SpMV's per-group partials (SpmvArgs::pq: aligned
// 32-row nodes; a CTA's 2048 groups are an aligned node, the last CTA
// completes the tree -- the same PW as k_pcg_dot over the n products).
__global__ void __launch_bounds__(kPcgThreads) k_pcg_dotg(const PcgArgs a, const double *pqg,
                                                          int64_t ngroups) {
  __shared__ double s_w[8];
  __shared__ double s_red[kPcgThreads];
  __shared__ int s_flag;
  if (pcg_skip(a.sc)) return;
  const int64_t i0 = (int64_t)blockIdx.x * kPcgRows + threadIdx.x * kPcgPer;
  double v[8];
  ld8(v, pqg, i0, ngroups);
  const double PQc = cta_pw(v, i0, ngroups, s_w);
  if (threadIdx.x == 0) a.part0[blockIdx.x] = PQc;
  if (!last_cta(a.ticket, &s_flag)) return;
  const double PQ = grid_pw(a.part0, gridDim.x, s_red);
  if (threadIdx.x == 0) {
    if (a.dsend)
      a.dsend[0] = PQ;
    else
      dot_scalars(a, PQ);
    *a.ticket = 0u;
  }
}

// r -= alpha q; z = r / d; rho' = PW(r.z); res = ||r||; beta = rho'/rho;
// convergence test (R15, R16).  x += alpha p moved to k_pcg_p, which reads
// p anyway (one vector stream less per iteration; the same bits).
#ifndef ABFT_PCG_UPD_MINB
#define ABFT_PCG_UPD_MINB 4  // 64 registers, 4 CTAs per SM: 192^3 PCG 48.5 -> 46.9 ms (same box)
#endif
__global__ void __launch_bounds__(kPcgThreads, ABFT_PCG_UPD_MINB) k_pcg_update(const PcgArgs a, int64_t iter) {
  __shared__ double s_w[16];
  __shared__ double s_red[kPcgThreads];
  __shared__ int s_flag;
  if (pcg_skip(a.sc)) return;
  const double alpha = a.sc->alpha;
  const int64_t i0 = (int64_t)blockIdx.x * kPcgRows + threadIdx.x * kPcgPer;
  double rv[8], qv[8], dv[8], rz[8], rr[8];
  ld8(rv, a.r, i0, a.n);
  ld8(qv, a.q, i0, a.n);
  ld8(dv, a.d, i0, a.n);
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    rv[u] = dsub(rv[u], dmul(alpha, qv[u]));
#if ABFT_EXP == 9  // timing experiment only: no division (wrong z)
    dv[u] = dmul(rv[u], dv[u]);
#else
    dv[u] = __ddiv_rn(rv[u], dv[u]);  // z
#endif
    rz[u] = dmul(rv[u], dv[u]);
    rr[u] = dmul(rv[u], rv[u]);
  }
  st8(a.r, rv, i0, a.n);
  st8(a.z, dv, i0, a.n);
  double RZc, RRc;
  cta_pw2(rz, rr, i0, a.n, s_w, RZc, RRc);
  if (threadIdx.x == 0) {
    a.part0[blockIdx.x] = RZc;
    a.part1[blockIdx.x] = RRc;
  }
  if (!last_cta(a.ticket, &s_flag)) return;
  double RZ, RR;
  grid_pw2(a.part0, a.part1, gridDim.x, s_red, RZ, RR);
  if (threadIdx.x == 0) {
    if (a.dsend) {
      a.dsend[0] = RZ;
      a.dsend[1] = RR;
    } else {
      update_scalars(a, iter >= 0 ? iter : a.sc->j, RZ, RR);
    }
    *a.ticket = 0u;
  }
}

// x += alpha p; p = z + beta p (old p for both).  Runs in the iteration
// that converged too (as the oracle); skipped only when this iteration's
// update was skipped.
#ifndef ABFT_PCG_P_MINB
#define ABFT_PCG_P_MINB 1
#endif
__global__ void __launch_bounds__(kPcgThreads, ABFT_PCG_P_MINB) k_pcg_p(const PcgArgs a, int64_t iter) {
  // iter < 0: the device-resident loop's counter (CUDA graph while node)
  if (iter < 0) iter = *(volatile const int64_t *)&a.sc->j;
  if (*(volatile const int64_t *)&a.sc->upd != iter) return;  // this iteration did not execute
  const double beta = a.sc->beta, alpha = a.sc->alpha;
  const int64_t i0 = (int64_t)blockIdx.x * kPcgRows + threadIdx.x * kPcgPer;
  double zv[8], pv[8], xv[8];
  ld8(zv, a.z, i0, a.n);
  ld8(pv, a.p, i0, a.n);
  ld8(xv, a.x, i0, a.n);
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    xv[u] = dadd(xv[u], dmul(alpha, pv[u]));
    pv[u] = dadd(zv[u], dmul(beta, pv[u]));
  }
  st8(a.x, xv, i0, a.n);
  st8(a.p, pv, i0, a.n);
  st8_ext(a.pext, pv, i0, a.n);
  // checkpoint mode: sample (x, r, z, p, rho, it) every ckpt_every iterations
  const int64_t it = a.sc->it;
  if (a.cr && a.ckpt_every > 0 && it % a.ckpt_every == 0) {
    double rv[8];
    ld8(rv, a.r, i0, a.n);
    st8(a.ck, xv, i0, a.n);
    st8(a.ck + a.ns, rv, i0, a.n);
    st8(a.ck + 2 * a.ns, zv, i0, a.n);
    st8(a.ck + 3 * a.ns, pv, i0, a.n);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      a.sc->ck_rho = a.sc->rho;
      a.sc->ck_res = a.sc->res;
      a.sc->ck_it = it;
    }
  }
}

// Device-resident loop (CUDA graph while node): the loop's condition --
// the solve still runs and the next iteration is within max_iter (executed
// iterations, as the host loop counts them); bump: advance the counter
// first (end of an iteration's body).
__global__ void k_pcg_cond(const PcgArgs a, cudaGraphConditionalHandle hnd, int bump) {
  PcgScalars *sc = a.sc;
  if (bump) sc->j += 1;
  cudaGraphSetConditional(hnd, (sc->state == PCG_RUN && sc->j <= sc->max_iter) ? 1u : 0u);
}

// Checkpoint mode: after the dense check of this iteration's
// SpMV, either continue (skip_it = 0) or restore the last sample and mark
// the iteration rolled back (its dot / update / p kernels then return).
__global__ void __launch_bounds__(kPcgThreads) k_pcg_cr(const PcgArgs a) {
  if (*(volatile const int32_t *)&a.sc->state != PCG_RUN) return;
  const bool flagged = *(volatile const int32_t *)a.dflag != 0;
  if (flagged) {
    const int64_t i0 = (int64_t)blockIdx.x * kPcgRows + threadIdx.x * kPcgPer;
    double v[8];
    ld8(v, a.ck, i0, a.n);
    st8(a.x, v, i0, a.n);
    ld8(v, a.ck + a.ns, i0, a.n);
    st8(a.r, v, i0, a.n);
    ld8(v, a.ck + 2 * a.ns, i0, a.n);
    st8(a.z, v, i0, a.n);
    ld8(v, a.ck + 3 * a.ns, i0, a.n);
    st8(a.p, v, i0, a.n);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    PcgScalars *sc = a.sc;
    sc->calls += 1;
    sc->skip_it = flagged ? 1 : 0;
    if (flagged) {
      sc->rho = sc->ck_rho;
      sc->res = sc->ck_res;
      sc->recomputed += sc->it - sc->ck_it;  // advanced iterations discarded
      sc->it = sc->ck_it;
      sc->flagged += 1;                      // detections = rollbacks
    }
  }
}


// ---------------------------------------------------------------------------
// Single-reduction PCG (Chronopoulos-Gear, R29):
// the iteration recurs s = A p so that (r.u), (r.r) and (w.u) with w = A u
// are ONE all-gather per iteration instead of two.  Vectors: x, r, u (the z
// slot), w (the SpMV output q), p, s; scalars: gamma (rho), delta (pq),
// alpha, beta.  Distributed API only (phases 4 and 5).
// ---------------------------------------------------------------------------
enum { PCG_PHASE_CG1_UPDATE = 4, PCG_PHASE_CG1_DOT = 5 };

// p = u + beta p; s = w + beta s; x += alpha p; r -= alpha s; u = r / d;
// partials (r.u, r.r) -> dsend[0..2)
__global__ void __launch_bounds__(kPcgThreads, 2) k_cg1_update(const PcgArgs a) {
  __shared__ double s_w[8];
  __shared__ double s_red[kPcgThreads];
  __shared__ int s_flag;
  if (pcg_skip(a.sc)) return;
  const double alpha = a.sc->alpha, beta = a.sc->beta;
  const int64_t i0 = (int64_t)blockIdx.x * kPcgRows + threadIdx.x * kPcgPer;
  double uv[8], wv[8], pv[8], sv[8], xv[8], rv[8], dv[8], ru[8], rr[8];
  ld8(uv, a.z, i0, a.n);
  ld8(wv, a.q, i0, a.n);
  ld8(pv, a.p, i0, a.n);
  ld8(sv, a.s, i0, a.n);
  ld8(xv, a.x, i0, a.n);
  ld8(rv, a.r, i0, a.n);
  ld8(dv, a.d, i0, a.n);
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    pv[u] = dadd(uv[u], dmul(beta, pv[u]));
    sv[u] = dadd(wv[u], dmul(beta, sv[u]));
    xv[u] = dadd(xv[u], dmul(alpha, pv[u]));
    rv[u] = dsub(rv[u], dmul(alpha, sv[u]));
    uv[u] = __ddiv_rn(rv[u], dv[u]);
    ru[u] = dmul(rv[u], uv[u]);
    rr[u] = dmul(rv[u], rv[u]);
  }
  st8(a.p, pv, i0, a.n);
  st8(a.s, sv, i0, a.n);
  st8(a.x, xv, i0, a.n);
  st8(a.r, rv, i0, a.n);
  st8(a.z, uv, i0, a.n);
  st8_ext(a.pext, uv, i0, a.n);  // the next SpMV's operand is u
  const double RUc = cta_pw(ru, i0, a.n, s_w);
  const double RRc = cta_pw(rr, i0, a.n, s_w);
  if (threadIdx.x == 0) {
    a.part0[blockIdx.x] = RUc;
    a.part1[blockIdx.x] = RRc;
  }
  if (!last_cta(a.ticket, &s_flag)) return;
  double RU, RR;
  grid_pw2(a.part0, a.part1, gridDim.x, s_red, RU, RR);
  if (threadIdx.x == 0) {
    a.dsend[0] = RU;
    a.dsend[1] = RR;
    *a.ticket = 0u;
  }
}

// partial (w.u) -> dsend[2]; first call (iter 0): also s = w (s_0 = A p_0
// with p_0 = u_0)
__global__ void __launch_bounds__(kPcgThreads) k_cg1_dot(const PcgArgs a, int64_t iter) {
  __shared__ double s_w[8];
  __shared__ double s_red[kPcgThreads];
  __shared__ int s_flag;
  if (pcg_skip(a.sc)) return;
  const int64_t i0 = (int64_t)blockIdx.x * kPcgRows + threadIdx.x * kPcgPer;
  double wv[8], uv[8];
  ld8(wv, a.q, i0, a.n);
  ld8(uv, a.z, i0, a.n);
  if (iter == 0) st8(a.s, wv, i0, a.n);
#pragma unroll
  for (int u = 0; u < 8; ++u) uv[u] = dmul(wv[u], uv[u]);
  const double WUc = cta_pw(uv, i0, a.n, s_w);
  if (threadIdx.x == 0) a.part2[blockIdx.x] = WUc;
  if (!last_cta(a.ticket, &s_flag)) return;
  const double WU = grid_pw(a.part2, gridDim.x, s_red);
  if (threadIdx.x == 0) {
    a.dsend[2] = WU;
    *a.ticket = 0u;
  }
}

// Scalars after the iteration's single reduction.  iter 0: delta_0 = (w.u),
// alpha_0 = gamma_0 / delta_0, beta_0 = 0.  iter j > 0: gamma' = (r.u),
// res = sqrt(r.r) (convergence), beta = gamma'/gamma,
// alpha = gamma' / (delta - beta gamma' / alpha).
__device__ __forceinline__ void cg1_scalars(const PcgArgs &a, int64_t iter, double RU, double RR,
                                            double WU) {
  PcgScalars *sc = a.sc;
  pcg_stats(a, sc);  // the SpMV w = A u of this step
  if (iter == 0) {
    sc->pq = WU;
    if (!(WU > 0.0)) {
      sc->state = PCG_BREAKDOWN;
      return;
    }
    sc->alpha = __ddiv_rn(sc->rho, WU);
    sc->beta = 0.0;
    return;
  }
  const double res = __dsqrt_rn(RR);
  sc->it += 1;
  sc->res = res;
  if (a.hist) a.hist[sc->it] = res;
  sc->upd = iter;
  if (pcg_done(a, res, RR, sc->thr)) {
    sc->state = PCG_CONVERGED;
    return;
  }
  if (!(res == res)) {
    sc->state = PCG_BREAKDOWN;
    return;
  }
  if (sc->it >= sc->max_iter) {
    sc->state = PCG_MAXITER;
    return;
  }
  const double beta = __ddiv_rn(RU, sc->rho);
  const double den = dsub(WU, __ddiv_rn(dmul(beta, RU), sc->alpha));
  sc->pq = WU;
  if (!(den > 0.0)) {
    sc->state = PCG_BREAKDOWN;
    return;
  }
  sc->beta = beta;
  sc->alpha = __ddiv_rn(RU, den);
  sc->rho = RU;
}

// Distributed PCG: finish a phase's dot products over all ranks.  recv holds
// world x 3 partials (rank r at [3r, 3r+3), gathered in rank order); each
// component is PW over the ranks (R2: pad with absent slots to a power of
// two).  One thread; the scalar steps are the single-GPU ones.
__device__ __forceinline__ double pw_ranks(const double *recv, int world, int c) {
  double v[64];
  int m = 1;
  while (m < world) m <<= 1;
  for (int q = 0; q < m; ++q) v[q] = q < world ? recv[3 * q + c] : kAbsent;
  for (int s = 1; s < m; s <<= 1)
    for (int q = 0; q + s < m; q += 2 * s) v[q] = dadd(v[q], v[q + s]);
  return v[0];
}

enum { PCG_PHASE_INIT = 0, PCG_PHASE_DOT = 1, PCG_PHASE_UPDATE = 2, PCG_PHASE_P = 3 };

__global__ void k_pcg_comb(const PcgArgs a, int phase, int64_t iter, const double *recv,
                           int world) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  if (phase != PCG_PHASE_INIT && pcg_skip(a.sc)) return;
  const double s0 = pw_ranks(recv, world, 0);
  if (phase == PCG_PHASE_INIT)
    init_scalars(a, s0, pw_ranks(recv, world, 1), pw_ranks(recv, world, 2));
  else if (phase == PCG_PHASE_DOT)
    dot_scalars(a, s0);
  else if (phase == PCG_PHASE_UPDATE)
    update_scalars(a, iter, s0, pw_ranks(recv, world, 1));
  else  // PCG_PHASE_CG1_DOT
    cg1_scalars(a, iter, iter ? s0 : 0.0, iter ? pw_ranks(recv, world, 1) : 0.0,
                pw_ranks(recv, world, 2));
}

}  // namespace abft
