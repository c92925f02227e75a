// kernels_perm.cuh -- popularity-ordered copy of x for irregular matrices
// (DESIGN.md §6.10).
//
// Power-law matrices (R-MAT, configs[2]) gather x at random columns, and a
// random vertex permutation scatters the popular columns over all of x: at
// scale 24, 1% of the columns take 62% of the gathers and 10% take 92%, but
// they sit one per 32-byte sector across 134 MB (> L2).  At encode time the
// columns are renumbered by descending reference count (a stable sort, ties
// in column order); the handle keeps renumbered copies of A's and C's column
// arrays, and every call first scatters x into that order (xp[inv[j]] =
// x[j]) -- then the hot columns share sectors and stay in L1/L2.  Only where
// x_j is read from changes: every product fl(a_ij x_j) and every sum keeps
// its operands and order, so y, t1, t2 and the flags are bit-identical.
#pragma once
#include "abft_device.cuh"

namespace abft {

// reference count of every column of A
__global__ void k_col_hist(int64_t nnz, const int32_t *__restrict__ ci, int32_t *cnt) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz;
       e += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(cnt + __ldg(ci + e), 1);
}

__global__ void k_iota(int64_t n, int32_t *v) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    v[i] = (int32_t)i;
}

// inv[perm[k]] = k
__global__ void k_perm_inv(int64_t n, const int32_t *__restrict__ perm, int32_t *inv) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n;
       k += (int64_t)gridDim.x * blockDim.x)
    inv[__ldg(perm + k)] = (int32_t)k;
}

// out[e] = inv[in[e]] (column arrays in the new numbering; 4 per thread)
__global__ void k_remap_cols(int64_t m, const int32_t *__restrict__ in, const int32_t *__restrict__ inv,
                             int32_t *out) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < m;
       e += (int64_t)gridDim.x * blockDim.x)
    out[e] = __ldg(inv + __ldg(in + e));
}

// Per call: xp[inv[j]] = x[j].  x and inv are read coalesced (four 16-B /
// 8-B pairs per thread in flight before the first store, when x is 16-B
// aligned); the writes scatter, and L2 merges the partial sectors before they
// reach DRAM.
__global__ void __launch_bounds__(256) k_xperm(int64_t n, const double *__restrict__ x,
                                               const int32_t *__restrict__ inv,
                                               double *__restrict__ xp) {
  constexpr int U = 4;
  const bool vec = (reinterpret_cast<uintptr_t>(x) & 15u) == 0;
  const int64_t n2 = vec ? n / 2 : 0;
  const int64_t nt = (int64_t)gridDim.x * blockDim.x;
  const double2 *x2 = reinterpret_cast<const double2 *>(x);
  const int2 *i2 = reinterpret_cast<const int2 *>(inv);
  for (int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t0 < n2; t0 += U * nt) {
    double2 v[U];
    int2 k[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t t = t0 + u * nt;
      if (t < n2) {
        v[u] = __ldcs(x2 + t);
        k[u] = __ldcs(i2 + t);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (t0 + u * nt < n2) {
        xp[k[u].x] = v[u].x;
        xp[k[u].y] = v[u].y;
      }
  }
  for (int64_t j = 2 * n2 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += nt)
    xp[__ldg(inv + j)] = __ldg(x + j);
}

}  // namespace abft
