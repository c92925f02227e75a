// kernels_dense.cuh -- related-work baseline: the DENSE
// CHECK of [30, 31] (one checksum over all N rows, eq. (1)) with the
// norm-based bound tau = ||x||_2 of [30] or the analytical bound of
// [35], and COMPLETE RECOMPUTATION [31] on a flag.
// It runs on the same SpMV kernels as the method (CHECK = false), so the
// comparison of Fig. 5-7 isolates the checking scheme.  DESIGN.md "Dense
// check baseline" and readings R23-R25.
//
// Encode (once): c = 1^T A with c_j = PW over column j's entries in ascending
// row order -- a stable radix sort of the entries by column (CUB) gives the
// column lists in row order; short columns are reduced lane-private, long
// ones by the warp.  K35 = ((n + 2N - 2) PW_i ||a_i|| + n ||c||) 2^-53.
// Per call: the SpMV, then ONE persistent kernel (PDL launch, one CTA per SM,
// software grid barrier): aligned 2048-row chunk partials of y, c o x and x^2,
// every CTA finishes the three PW totals from the partials (so all CTAs agree
// on the flag without another barrier), flag iff NOT(|t1 - t2| <= tau); on a
// flag it recomputes all of y (round r + 1) and checks again, <= R rounds.
#pragma once
#include "kernels_spmv.cuh"

namespace abft {

constexpr int kDenseChunk = 8192;  // rows per aligned partial of the encode-time sums
constexpr int kDenseRows = 2048;   // rows per aligned partial of the per-call sums (one CTA)

// Column id of every entry (rows expanded), the sort key.
__global__ void k_dense_keys(int64_t n, const int32_t *__restrict__ rp,
                             const int32_t *__restrict__ ci, int32_t *keys, int32_t *idx) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = gw; i < n; i += nw)
    for (int32_t e = rp[i] + lane; e < rp[i + 1]; e += 32) {
      keys[e] = ci[e];
      idx[e] = e;
    }
}

// cstart[j] = first sorted position of column j (empty columns: the next
// column's start); cstart[n] = nnz.
__global__ void k_dense_starts(int64_t n, int64_t nnz, const int32_t *__restrict__ skeys,
                               int32_t *cstart) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e <= nnz;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t lo = e == 0 ? -1 : skeys[e - 1];
    const int64_t hi = e == nnz ? n - 1 : skeys[e];
    for (int64_t j = lo + 1; j <= hi; ++j) cstart[j] = (int32_t)e;
    if (e == nnz) cstart[n] = (int32_t)nnz;
  }
}

// c_j = PW over column j's values in row order (R23); +0.0 for an empty column.
__global__ void __launch_bounds__(256) k_dense_colsum(int64_t n, const int32_t *__restrict__ cstart,
                                                      const int32_t *__restrict__ perm,
                                                      const double *__restrict__ va, double *c) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t j0 = gw * 32; j0 < n; j0 += nw * 32) {
    const int64_t j = j0 + lane;
    int32_t b = 0, L = 0;
    if (j < n) {
      b = cstart[j];
      L = cstart[j + 1] - b;
    }
    double r = 0.0;
    if (j < n && L <= 32) {  // lane-private: aligned 8-leaf subtrees, tree over 4
      double q[4];
#pragma unroll 1
      for (int t = 0; t < 4; ++t) {
        double v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const int e = 8 * t + u;
          v[u] = e < L ? __ldg(va + __ldg(perm + b + e)) : kAbsent;
        }
        q[t] = tree<8>(v);
      }
      r = L > 0 ? tree<4>(q) : 0.0;
    }
    unsigned longm = __ballot_sync(kFull, j < n && L > 32);
    while (longm) {  // long columns: the warp, 256-entry chunks (binary counter == PW)
      const int l = __ffs(longm) - 1;
      longm &= longm - 1;
      const int32_t bl = __shfl_sync(kFull, b, l), Ll = __shfl_sync(kFull, L, l);
      PwSeq acc;
      for (int32_t o = 0; o < Ll; o += 256) {
        double v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const int e = o + 32 * u + lane;
          v[u] = e < Ll ? __ldg(va + __ldg(perm + bl + e)) : kAbsent;
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = bfly32(v[u]);
        acc.push(tree<8>(v));
      }
      const double t = acc.finish();
      if (lane == l) r = t;
    }
    if (j < n) c[j] = r;
  }
}

// ||a_i||_2 = sqrt(PW(a_ij^2)) per row (R6), lane per row.
__global__ void k_dense_rownorm(int64_t n, const int32_t *__restrict__ rp,
                                const double *__restrict__ va, double *out) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t b = rp[i], L = rp[i + 1] - b;
    PwSeq acc;  // aligned 8-leaf subtrees
    for (int32_t o = 0; o < L; o += 8) {
      double v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const double a = o + u < L ? va[b + o + u] : 0.0;
        v[u] = o + u < L ? dmul(a, a) : kAbsent;
      }
      acc.push(tree<8>(v));
    }
    out[i] = __dsqrt_rn(L > 0 ? acc.finish() : 0.0);
  }
}

// PW over 1024 staged values (absent-padded) by a CTA of 256 threads: thread t
// sums the aligned 4-run 4t..4t+3, then a shared-memory tree over the runs.
// Called by all threads; s is read after a __syncthreads by the caller.
__device__ __forceinline__ double cta_pw_smem1024(const double *s, double *s_red) {
  double v[4];
#pragma unroll
  for (int u = 0; u < 4; ++u) v[u] = s[4 * threadIdx.x + u];
  s_red[threadIdx.x] = tree<4>(v);
  __syncthreads();
  for (int st = 1; st < 256; st <<= 1) {
    if ((threadIdx.x & (2 * st - 1)) == 0)
      s_red[threadIdx.x] = dadd(s_red[threadIdx.x], s_red[threadIdx.x + st]);
    __syncthreads();
  }
  const double r = s_red[0];
  __syncthreads();
  return r;
}

// PW over v[0..n) (sq: of v_i^2) in aligned chunks of kDenseChunk, one CTA
// each: eight aligned 1024-slices, then a tree over the slices.
__global__ void __launch_bounds__(256) k_dense_chunks(const double *__restrict__ v, int64_t n,
                                                      int sq, double *part) {
  __shared__ double s_red[256];
  __shared__ double s_tmp[1024];
  const int64_t nch = (n + kDenseChunk - 1) / kDenseChunk;
  for (int64_t ch = blockIdx.x; ch < nch; ch += gridDim.x) {
    double q[8];
    for (int sl = 0; sl < 8; ++sl) {
      const int64_t b = ch * kDenseChunk + sl * 1024;
      const int64_t m = b < n ? min64(1024, n - b) : 0;
      for (int t = threadIdx.x; t < 1024; t += blockDim.x) {
        const double a = t < m ? v[b + t] : 0.0;
        s_tmp[t] = t < m ? (sq ? dmul(a, a) : a) : kAbsent;
      }
      __syncthreads();
      q[sl] = cta_pw_smem1024(s_tmp, s_red);
    }
    if (threadIdx.x == 0) part[ch] = tree<8>(q);
  }
}

// k35 = fl(fl(fl(m S) + fl(n ||c||)) 2^-53), m = n + 2N - 2 (R24);
// S = PW over the chunk partials of the row norms, ||c||^2 likewise.
__global__ void __launch_bounds__(256) k_dense_k35(int64_t n, const double *spart,
                                                   const double *cpart, int64_t nch,
                                                   double *k35) {
  __shared__ double s_red[256];
  const double S = cta_pw_array(spart, nch, s_red);
  const double c2 = cta_pw_array(cpart, nch, s_red);
  if (threadIdx.x == 0) {
    const double m = (double)(n + 2 * n - 2);
    *k35 = dmul(dadd(dmul(m, S), dmul((double)n, __dsqrt_rn(c2))), 0x1p-53);
  }
}

struct DenseArgs {
  SpmvArgs a;             // SpMV operands (rp, ci, va, x, y, inj, gbar ...)
  const double *c;        // [n]
  const double *k35;      // device scalar
  int bound35;
  int rounds;             // complete recomputations allowed
  double *part;           // [3 * nch]: y, c o x, x^2 chunk partials
  double *res;            // [(rounds+1) * 4]: t1, t2, beta, tau per round
  int32_t *flag_rounds;   // [max_rounds + 1]
};

// Recompute all of y (round r of the complete recomputation), warp per group.
template <bool INJECT>
__device__ __forceinline__ void dense_recompute(const SpmvArgs &a, int round) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const LdgSrc As{a.va, a.ci};
  for (int64_t g = gw; g < a.ngroups; g += nw) {
    const int64_t r0 = g * 32, i = r0 + lane;
    const bool valid = i < a.n;
    int32_t rs = 0, len = 0;
    if (valid) {
      rs = __ldg(a.rp + i);
      len = __ldg(a.rp + i + 1) - rs;
    }
    const int maxlen = warp_max_i(len);
    double yv = 0.0;
    if (maxlen <= 32) {
      if (valid) yv = lane_dot_any(As, rs, len, maxlen, a.x);
    } else {
      for (int j = 0; j < 32 && r0 + j < a.n; ++j) {
        const double t = warp_dot(As, __shfl_sync(kFull, rs, j), __shfl_sync(kFull, len, j), a.x, lane);
        if (lane == j) yv = t;
      }
    }
    if (len == 0) yv = 0.0;
    if (INJECT) {
      const uint64_t m = group_y_mask(a.inj, round, r0, i, lane);
      if (valid) yv = apply_mask(yv, m);
    }
    if (valid) a.y[i] = yv;
  }
}

// Aligned 2048-row partial of the three dense-check sums (rows b .. b+2047,
// absent past n) by a CTA of 256 threads: lane l of warp w owns the aligned
// 8-run b + 256 w + 8 l, an 8-leaf tree in registers, the butterfly joins the
// warp's 256, a tree over the 8 warps (shared memory) the CTA's 2048 -- the
// PW tree of the chunk (R2).  Called by all threads; valid in thread 0.
__device__ __forceinline__ void dense_chunk(const DenseArgs &d, int64_t b, double (*s_w)[8],
                                            double out[3]) {
  const SpmvArgs &a = d.a;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t r0 = b + 256 * warp + 8 * lane;
  double vy[8], vc[8], vx[8];
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    const bool in = r0 + u < a.n;
    vy[u] = in ? __ldcg(a.y + r0 + u) : kAbsent;
    vx[u] = in ? __ldg(a.x + r0 + u) : 0.0;
    vc[u] = in ? __ldg(d.c + r0 + u) : 0.0;
  }
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    const bool in = r0 + u < a.n;
    vc[u] = in ? dmul(vc[u], vx[u]) : kAbsent;
    vx[u] = in ? dmul(vx[u], vx[u]) : kAbsent;
  }
  double w[3] = {bfly32(tree<8>(vy)), bfly32(tree<8>(vc)), bfly32(tree<8>(vx))};
  if (lane == 0)
    for (int k = 0; k < 3; ++k) s_w[k][warp] = w[k];
  __syncthreads();
  if (threadIdx.x == 0)
    for (int k = 0; k < 3; ++k) {
      double v[8];
      for (int q = 0; q < 8; ++q) v[q] = s_w[k][q];
      out[k] = tree<8>(v);
    }
  __syncthreads();
}

template <bool INJECT>
__global__ void __launch_bounds__(256) k_dense(const DenseArgs d) {
  __shared__ double s_red[256];
  __shared__ double s_w[3][8];
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const SpmvArgs &a = d.a;
  if (skip_call(a)) return;  // PCG: solver no longer running
  const int64_t n = a.n;
  const int64_t nch = (n + kDenseRows - 1) / kDenseRows;
  double beta = 0.0, tau = 0.0;
  if (blockIdx.x == 0 && threadIdx.x == 0)
    for (int q = 0; q <= a.max_rounds; ++q) d.flag_rounds[q] = 0;
  for (int r = 0; r <= d.rounds; ++r) {
    if (r > 0) {
      dense_recompute<INJECT>(a, r);
      if (!grid_sync(a.gbar)) return;
    }
    for (int64_t ch = blockIdx.x; ch < nch; ch += gridDim.x) {
      double o[3];
      dense_chunk(d, ch * kDenseRows, s_w, o);
      if (threadIdx.x == 0)
        for (int k = 0; k < 3; ++k) d.part[k * nch + ch] = o[k];
    }
    if (!grid_sync(a.gbar)) return;
    // every CTA finishes the totals itself (same bits everywhere)
    const double t2raw = cta_pw_array(d.part, nch, s_red);
    const double t1raw = cta_pw_array(d.part + nch, nch, s_red);
    if (r == 0) {
      beta = __dsqrt_rn(cta_pw_array(d.part + 2 * nch, nch, s_red));  // R10
      tau = d.bound35 ? dmul(__ldg(d.k35), beta) : beta;  // [35] / [30]
    }
    double t1 = t1raw, t2 = t2raw;
    if (INJECT) {
      t1 = apply_mask(t1, fault_mask(a.inj, r, 1, 0, 2 * n));
      t2 = apply_mask(t2, fault_mask(a.inj, r, 2, 0, n));
    }
    const bool flagged = !(fabs(dsub(t1, t2)) <= tau);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      d.res[4 * r + 0] = t1;
      d.res[4 * r + 1] = t2;
      d.res[4 * r + 2] = beta;
      d.res[4 * r + 3] = tau;
      d.flag_rounds[r] = flagged ? 1 : 0;
    }
    if (!flagged) break;
    if (!grid_sync(a.gbar)) return;  // partials consumed before the next round rewrites them
  }
}

}  // namespace abft
