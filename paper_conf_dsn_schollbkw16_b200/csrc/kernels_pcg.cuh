// kernels_pcg.cuh -- Jacobi-PCG vector kernels (SVI-A; Saad
// Alg. 9.1).  The SpMV q = A p is the protected k_fused/k_correct pair; these
// kernels fuse the vector updates with their dot products.  Every dot is PW
// over the global index (R2): each CTA reduces its aligned 256-row subtree,
// the last CTA (atomic ticket) completes the tree and updates the scalars, so
// the iteration runs without host round trips.  A device `state` word makes
// every kernel of a converged / broken-down solve a no-op.
#pragma once
#include "abft_device.cuh"

namespace abft {

constexpr int kPcgThreads = 256;

enum { PCG_RUN = 0, PCG_CONVERGED = 1, PCG_BREAKDOWN = 2, PCG_MAXITER = 3 };

struct PcgScalars {
  double rho, pq, alpha, beta, res, thr;
  int64_t it, max_iter;
  int64_t flagged, recomputed, uncorrected, calls;
  int32_t state;
  int32_t pad;
};

struct PcgArgs {
  int64_t n;
  const double *__restrict__ b;
  double *x, *r, *z, *p, *q;
  const double *__restrict__ d;
  double *part0, *part1, *part2;  // per-CTA partial sums
  unsigned *ticket;
  PcgScalars *sc;
  double *hist;                   // nullable
  double tol;
  const int32_t *n_flags;         // protected-SpMV flag counts (stats)
  int32_t max_rounds;
  int32_t check;
};

// CTA-level PW of one value per thread (thread t <-> row base + t): butterfly
// in each warp, tree over the 8 warp sums.  All threads get the result.
__device__ __forceinline__ double cta_pw256(double v, double *s_w) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  v = bfly32(v);
  __syncthreads();
  if (lane == 0) s_w[warp] = v;
  __syncthreads();
  double w[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) w[q] = s_w[q];
  return tree<8>(w);
}

// Last-CTA completion of PW over partials[0..ncta) (aligned 256-row
// subtrees).  Called by all threads of the last CTA.
__device__ __forceinline__ double grid_pw(const double *partials, int ncta, double *s_red) {
  int m = 1;
  while (m * kPcgThreads < ncta) m <<= 1;
  PwSeq acc;
  const int b = threadIdx.x * m;
  for (int q = b; q < min(b + m, ncta); ++q) acc.push(__ldcg(partials + q));
  __syncthreads();
  s_red[threadIdx.x] = acc.finish();
  __syncthreads();
  for (int s = 1; s < kPcgThreads; s <<= 1) {
    if ((threadIdx.x & (2 * s - 1)) == 0)
      s_red[threadIdx.x] = dadd(s_red[threadIdx.x], s_red[threadIdx.x + s]);
    __syncthreads();
  }
  return s_red[0];
}

// Ticket: returns true in the last CTA to finish (after its partials are
// written).  The last CTA resets the ticket for the next kernel.
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
  return *(volatile const int32_t *)&sc->state != PCG_RUN;
}

// diag(A) (R21; missing diagonal -> 0, as the oracle)
__global__ void k_pcg_diag(int64_t n, const int32_t *__restrict__ rp,
                           const int32_t *__restrict__ ci, const double *__restrict__ va,
                           double *d) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  double v = 0.0;
  for (int32_t q = rp[i]; q < rp[i + 1]; ++q)
    if (ci[q] == i) v = va[q];
  d[i] = v;
}

// r = b - q; z = r / d; p = z; rho = PW(r.z); res = ||r||; thr = tol ||b||
__global__ void __launch_bounds__(kPcgThreads) k_pcg_init(const PcgArgs a) {
  __shared__ double s_w[8];
  __shared__ double s_red[kPcgThreads];
  __shared__ int s_flag;
  const int64_t i = (int64_t)blockIdx.x * kPcgThreads + threadIdx.x;
  double rz = kAbsent, rr = kAbsent, bb = kAbsent;
  if (i < a.n) {
    const double bi = a.b[i];
    const double ri = dsub(bi, a.q[i]);
    const double zi = __ddiv_rn(ri, a.d[i]);
    a.r[i] = ri;
    a.z[i] = zi;
    a.p[i] = zi;
    rz = dmul(ri, zi);
    rr = dmul(ri, ri);
    bb = dmul(bi, bi);
  }
  rz = cta_pw256(rz, s_w);
  rr = cta_pw256(rr, s_w);
  bb = cta_pw256(bb, s_w);
  if (threadIdx.x == 0) {
    a.part0[blockIdx.x] = rz;
    a.part1[blockIdx.x] = rr;
    a.part2[blockIdx.x] = bb;
  }
  if (!last_cta(a.ticket, &s_flag)) return;
  const double RZ = grid_pw(a.part0, gridDim.x, s_red);
  const double RR = grid_pw(a.part1, gridDim.x, s_red);
  const double BB = grid_pw(a.part2, gridDim.x, s_red);
  if (threadIdx.x == 0) {
    PcgScalars *sc = a.sc;
    sc->calls += 1;  // the SpMV q = A x0
    if (a.check) {
      const int32_t *nf = a.n_flags;
      sc->flagged += nf[0];
      for (int r = 0; r < a.max_rounds; ++r) sc->recomputed += nf[r];
      if (nf[a.max_rounds] > 0) sc->uncorrected += 1;
    }
    sc->rho = RZ;
    sc->res = __dsqrt_rn(RR);
    sc->thr = dmul(a.tol, __dsqrt_rn(BB));
    sc->it = 0;
    if (a.hist) a.hist[0] = sc->res;
    sc->state = (sc->res <= sc->thr) ? PCG_CONVERGED : (sc->max_iter <= 0 ? PCG_MAXITER : PCG_RUN);
    if (!(sc->res == sc->res)) sc->state = PCG_BREAKDOWN;
    *a.ticket = 0u;
  }
}

// pq = PW(p.q); alpha = rho / pq; protected-SpMV statistics.
__global__ void __launch_bounds__(kPcgThreads) k_pcg_dot(const PcgArgs a) {
  __shared__ double s_w[8];
  __shared__ double s_red[kPcgThreads];
  __shared__ int s_flag;
  if (pcg_skip(a.sc)) return;
  const int64_t i = (int64_t)blockIdx.x * kPcgThreads + threadIdx.x;
  double pq = kAbsent;
  if (i < a.n) pq = dmul(a.p[i], a.q[i]);
  pq = cta_pw256(pq, s_w);
  if (threadIdx.x == 0) a.part0[blockIdx.x] = pq;
  if (!last_cta(a.ticket, &s_flag)) return;
  const double PQ = grid_pw(a.part0, gridDim.x, s_red);
  if (threadIdx.x == 0) {
    PcgScalars *sc = a.sc;
    sc->calls += 1;
    if (a.check) {
      const int32_t *nf = a.n_flags;
      sc->flagged += nf[0];
      for (int r = 0; r < a.max_rounds; ++r) sc->recomputed += nf[r];
      if (nf[a.max_rounds] > 0) sc->uncorrected += 1;
    }
    sc->pq = PQ;
    if (!(PQ > 0.0)) {
      sc->state = PCG_BREAKDOWN;
    } else {
      sc->alpha = __ddiv_rn(sc->rho, PQ);
    }
    *a.ticket = 0u;
  }
}

// x += alpha p; r -= alpha q; z = r / d; rho' = PW(r.z); res = ||r||;
// beta = rho'/rho; convergence test (R15, R16).
__global__ void __launch_bounds__(kPcgThreads) k_pcg_update(const PcgArgs a) {
  __shared__ double s_w[8];
  __shared__ double s_red[kPcgThreads];
  __shared__ int s_flag;
  if (pcg_skip(a.sc)) return;
  const double alpha = a.sc->alpha;
  const int64_t i = (int64_t)blockIdx.x * kPcgThreads + threadIdx.x;
  double rz = kAbsent, rr = kAbsent;
  if (i < a.n) {
    const double pi = a.p[i];
    a.x[i] = dadd(a.x[i], dmul(alpha, pi));
    const double ri = dsub(a.r[i], dmul(alpha, a.q[i]));
    const double zi = __ddiv_rn(ri, a.d[i]);
    a.r[i] = ri;
    a.z[i] = zi;
    rz = dmul(ri, zi);
    rr = dmul(ri, ri);
  }
  rz = cta_pw256(rz, s_w);
  rr = cta_pw256(rr, s_w);
  if (threadIdx.x == 0) {
    a.part0[blockIdx.x] = rz;
    a.part1[blockIdx.x] = rr;
  }
  if (!last_cta(a.ticket, &s_flag)) return;
  const double RZ = grid_pw(a.part0, gridDim.x, s_red);
  const double RR = grid_pw(a.part1, gridDim.x, s_red);
  if (threadIdx.x == 0) {
    PcgScalars *sc = a.sc;
    const double res = __dsqrt_rn(RR);
    sc->it += 1;
    sc->res = res;
    if (a.hist) a.hist[sc->it] = res;
    sc->beta = __ddiv_rn(RZ, sc->rho);
    sc->rho = RZ;
    if (res <= sc->thr) sc->state = PCG_CONVERGED;
    else if (!(res == res)) sc->state = PCG_BREAKDOWN;
    else if (sc->it >= sc->max_iter) sc->state = PCG_MAXITER;
    *a.ticket = 0u;
  }
}

// p = z + beta p.  Runs in the iteration that converged too (as the oracle);
// skipped only when this iteration's update was skipped.
__global__ void __launch_bounds__(kPcgThreads) k_pcg_p(const PcgArgs a, int64_t iter) {
  const int64_t it = *(volatile const int64_t *)&a.sc->it;
  if (it != iter) return;  // this iteration did not execute
  const int64_t i = (int64_t)blockIdx.x * kPcgThreads + threadIdx.x;
  if (i < a.n) a.p[i] = dadd(a.z[i], dmul(a.sc->beta, a.p[i]));
}

}  // namespace abft
