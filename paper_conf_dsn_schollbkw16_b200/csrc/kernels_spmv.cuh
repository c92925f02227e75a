// kernels_spmv.cuh -- the hot path: fused multiply + detect (Fig. 1 steps
// 1-4) with in-kernel finalize, and the correction relaunch (step 5,
// P:76).  See DESIGN.md "Kernels".
//
// Mapping.  One warp owns a group of 32 consecutive rows (= 32 / b_s row
// blocks); a CTA of kWarps warps owns an aligned range of 32*kWarps rows.
//  * A's segment of the group is streamed with coalesced, warp-strided loads
//    (evict-first in L2), multiplied by the gathered x (read-only path, L2
//    resident), and the products are staged in shared memory; lane l then
//    reduces row r0+l with an in-register PW tree of P = 2^ceil(log2 maxlen)
//    leaves read from shared memory.  Groups whose segment exceeds the
//    staging capacity or whose longest row exceeds 32 fall back to one
//    warp-cooperative reduction per row.
//  * t2_k = PW over the b_s slots of y (xor butterfly over b_s lanes).
//  * t1_k = c_k . x: C's row is streamed warp-strided; each 32-element chunk
//    is reduced by a butterfly, chunks by an in-register tree (== PW).
//  * s_k = t1_k - t2_k is compared with K_k * beta_local, beta_local = the
//    norm of the CTA's aligned slice of x.  Monotone rounding makes
//    beta_local <= beta exactly (R12'), so |s| <= K beta_local
//    proves the block clean; only the rest become candidates.
//  * The CTA's x^2 subtree goes to `partials`; the last CTA to finish (atomic
//    ticket) completes beta = sqrt(PW(partials)), confirms the candidates
//    against tau_k = K_k beta and writes the flagged list + count: steps 2-4
//    finish without a second launch and without a host round trip.
#pragma once
#include "abft_device.cuh"

namespace abft {

constexpr int kWarps = 8;            // warps per CTA in the fused kernel
constexpr int kThreads = kWarps * 32;

struct SpmvArgs {
  int64_t n;
  int32_t bs;        // block size, power of two <= 32
  int32_t log2bs;
  int64_t nb;
  const int32_t *__restrict__ rp;
  const int32_t *__restrict__ ci;
  const double *__restrict__ va;
  const int32_t *__restrict__ crp;
  const int32_t *__restrict__ ccol;
  const double *__restrict__ cval;
  const double *__restrict__ K;
  const double *__restrict__ x;
  double *__restrict__ y;
  const double *x_norm;   // nullable device scalar
  double *partials;       // [gridDim.x]
  unsigned *done;         // ticket counter (reset by the last CTA)
  int32_t *n_cand;        // candidate count (reset by the last CTA)
  int32_t *cand;          // [nb]
  double *cand_s;         // [nb]
  int32_t *flags;         // [(max_rounds+1) * nb]; round r at flags + r*nb
  int32_t *n_flags;       // [max_rounds+1]
  int32_t max_rounds;
  double *beta;           // device scalar out
  double *dbg_t1, *dbg_t2;  // nullable
  const int32_t *skip;      // nullable device flag: != 0 -> kernel is a no-op (PCG)
  InjDev inj;
};

__device__ __forceinline__ bool skip_call(const SpmvArgs &a) {
  return a.skip && *(volatile const int32_t *)a.skip != 0;
}

// PW over the products val[b+e] * x[col[b+e]], e in [0, cnt), cnt <= 256,
// computed by the whole warp: lane l holds chunk elements u*32 + l; each
// 32-chunk is reduced by the butterfly, the 8 chunk sums by a tree.
__device__ __forceinline__ double warp_dot256(const double *__restrict__ val,
                                              const int32_t *__restrict__ col, int64_t b,
                                              int cnt, const double *__restrict__ x, int lane) {
  double v[8];
  int c[8];
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    int e = u * 32 + lane;
    if (u * 32 < cnt && e < cnt) {
      v[u] = ld_stream(val + b + e);
      c[u] = ld_stream(col + b + e);
    }
  }
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    int e = u * 32 + lane;
    if (u * 32 < cnt && e < cnt) v[u] = dmul(v[u], ld_x(x + c[u])); else v[u] = kAbsent;
  }
#pragma unroll
  for (int u = 0; u < 8; ++u)
    if (u * 32 < cnt) v[u] = bfly32(v[u]);
  return tree<8>(v);
}

// PW over an arbitrary-length dot product, whole warp; +0.0 when empty.
__device__ __noinline__ double warp_dot(const double *__restrict__ val,
                                        const int32_t *__restrict__ col, int64_t b, int64_t n,
                                        const double *__restrict__ x, int lane) {
  if (n <= 0) return 0.0;
  if (n <= 256) return warp_dot256(val, col, b, (int)n, x, lane);
  PwSeq acc;  // binary counter over aligned 256-chunks (== PW)
  for (int64_t o = 0; o < n; o += 256)
    acc.push(warp_dot256(val, col, b + o, (int)min64(256, n - o), x, lane));
  return acc.finish();
}

// Lane-private PW dot over a short row (len <= P) with direct loads.
template <int P>
__device__ __forceinline__ double lane_dot_direct(const double *__restrict__ val,
                                                  const int32_t *__restrict__ col, int64_t b,
                                                  int len, const double *__restrict__ x) {
  double v[P];
  int c[P];
#pragma unroll
  for (int j = 0; j < P; ++j)
    if (j < len) {
      v[j] = __ldg(val + b + j);
      c[j] = __ldg(col + b + j);
    }
#pragma unroll
  for (int j = 0; j < P; ++j) v[j] = j < len ? dmul(v[j], ld_x(x + c[j])) : kAbsent;
  return tree<P>(v);
}

__device__ __forceinline__ double lane_dot_direct_any(const double *__restrict__ val,
                                                      const int32_t *__restrict__ col,
                                                      int64_t b, int len, int maxlen,
                                                      const double *__restrict__ x) {
  if (maxlen <= 1) return lane_dot_direct<1>(val, col, b, len, x);
  if (maxlen <= 2) return lane_dot_direct<2>(val, col, b, len, x);
  if (maxlen <= 4) return lane_dot_direct<4>(val, col, b, len, x);
  if (maxlen <= 8) return lane_dot_direct<8>(val, col, b, len, x);
  if (maxlen <= 16) return lane_dot_direct<16>(val, col, b, len, x);
  return lane_dot_direct<32>(val, col, b, len, x);
}

// Lane-private PW tree over staged products s[off .. off+len), P leaves.
template <int P>
__device__ __forceinline__ double lane_tree_smem(const double *s, int off, int len) {
  double v[P];
#pragma unroll
  for (int j = 0; j < P; ++j) v[j] = j < len ? s[off + j] : kAbsent;
  return tree<P>(v);
}

__device__ __forceinline__ double lane_tree_smem_any(const double *s, int off, int len,
                                                     int maxlen) {
  if (maxlen <= 1) return lane_tree_smem<1>(s, off, len);
  if (maxlen <= 2) return lane_tree_smem<2>(s, off, len);
  if (maxlen <= 4) return lane_tree_smem<4>(s, off, len);
  if (maxlen <= 8) return lane_tree_smem<8>(s, off, len);
  if (maxlen <= 16) return lane_tree_smem<16>(s, off, len);
  return lane_tree_smem<32>(s, off, len);
}

// y for the 32 rows r0 .. r0+31 (lane l -> row r0+l); rows past n get len 0.
// Returns y_i (+0.0 for empty rows); rs/len out for the caller.
template <int CAP>
__device__ __forceinline__ double group_rows(const SpmvArgs &a, int64_t r0, int lane,
                                             double *s_prod, int &len_out) {
  const int64_t n = a.n;
  const int64_t i = r0 + lane;
  const int32_t rs = ld_stream(a.rp + min(i, n));
  int32_t rlast = 0;
  if (lane == 31) rlast = ld_stream(a.rp + min(r0 + 32, n));
  int32_t re = __shfl_down_sync(kFull, rs, 1);
  if (lane == 31) re = rlast;
  const int len = re - rs;
  len_out = len;
  const int32_t seg_b = __shfl_sync(kFull, rs, 0);
  const int32_t seg_e = __shfl_sync(kFull, re, 31);
  const int nseg = seg_e - seg_b;
  const int maxlen = warp_max_i(len);
  double yv;
  if (nseg <= CAP && maxlen <= 32) {
    // Stage the products of the whole segment (coalesced, warp-strided).
    for (int base = 0; base < nseg; base += 256) {
      double v[8];
      int c[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        int e = base + u * 32 + lane;
        if (e < nseg) {
          v[u] = ld_stream(a.va + seg_b + e);
          c[u] = ld_stream(a.ci + seg_b + e);
        }
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        int e = base + u * 32 + lane;
        if (e < nseg) s_prod[e] = dmul(v[u], ld_x(a.x + c[u]));
      }
    }
    __syncwarp();
    yv = lane_tree_smem_any(s_prod, rs - seg_b, len, maxlen);
    __syncwarp();
  } else {
    // Fallback: one warp-cooperative PW reduction per row.
    yv = 0.0;
    for (int j = 0; j < 32; ++j) {
      const int32_t rb = __shfl_sync(kFull, rs, j);
      const int rl = __shfl_sync(kFull, len, j);
      if (r0 + j >= n) break;
      const double t = warp_dot(a.va, a.ci, rb, rl, a.x, lane);
      if (lane == j) yv = t;
    }
  }
  if (len == 0) yv = 0.0;  // PW of an empty row is +0.0 (R2)
  return yv;
}

template <bool CHECK, bool INJECT, int CAP>
__global__ void __launch_bounds__(kThreads) k_fused(const SpmvArgs a) {
  extern __shared__ double s_dyn[];  // kWarps * CAP staged products
  __shared__ double s_red[kThreads];
  __shared__ int s_last;
  __shared__ int s_nflag;
  if (skip_call(a)) return;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t n = a.n;
  const int64_t r0 = ((int64_t)blockIdx.x * kWarps + warp) * 32;
  const int64_t i = r0 + lane;
  const bool valid = i < n;

  double s_syn = 0.0;
  int64_t k = 0;
  bool leader = false;
  if (r0 < n) {
    int len;
    double yv = group_rows<CAP>(a, r0, lane, s_dyn + warp * CAP, len);
    if (INJECT && valid) yv = apply_mask(yv, fault_mask(a.inj, 0, 0, i, 2 * (int64_t)len));
    if (valid) a.y[i] = yv;
    if (CHECK) {
      // step 2: t2_k = w_k^T y_k over the b_s slots; absent past n.
      double t2 = bfly(valid ? yv : kAbsent, a.bs);
      // step 1: t1_k = c_k . x
      const int bl = lane >> a.log2bs;        // block slot within the warp
      k = (r0 >> a.log2bs) + bl;
      leader = ((lane & (a.bs - 1)) == 0) && valid;
      double t1;
      int nk;
      if (a.bs == 32) {
        const int32_t cb = ld_stream(a.crp + k), ce = ld_stream(a.crp + k + 1);
        nk = ce - cb;
        t1 = warp_dot(a.cval, a.ccol, cb, nk, a.x, lane);
      } else {
        const int nblk = 32 >> a.log2bs;
        int32_t cb = 0, ce = 0;
        const int64_t kl = (r0 >> a.log2bs) + lane;
        if (lane < nblk && kl < a.nb) {
          cb = ld_stream(a.crp + kl);
          ce = ld_stream(a.crp + kl + 1);
        }
        const int nkl = ce - cb;
        const int maxnk = warp_max_i(nkl);
        double t1l = 0.0;
        if (maxnk <= 32) {
          if (lane < nblk) t1l = lane_dot_direct_any(a.cval, a.ccol, cb, nkl, maxnk, a.x);
          if (nkl == 0) t1l = 0.0;
        } else {
          for (int l = 0; l < nblk; ++l) {
            const int32_t b = __shfl_sync(kFull, cb, l);
            const int m = __shfl_sync(kFull, nkl, l);
            const double t = warp_dot(a.cval, a.ccol, b, m, a.x, lane);
            if (lane == l) t1l = t;
          }
        }
        t1 = __shfl_sync(kFull, t1l, bl);
        nk = __shfl_sync(kFull, nkl, bl);
      }
      if (INJECT && leader) {
        t1 = apply_mask(t1, fault_mask(a.inj, 0, 1, k, 2 * (int64_t)nk));
        const int64_t rows = min64(a.bs, n - (k << a.log2bs));
        t2 = apply_mask(t2, fault_mask(a.inj, 0, 2, k, rows));
      }
      if (leader && a.dbg_t1) {
        a.dbg_t1[k] = t1;
        a.dbg_t2[k] = t2;
      }
      s_syn = dsub(t1, t2);  // step 3
    }
  }
  if (!CHECK) return;

  // beta: the CTA's aligned x^2 subtree (a node of the global PW tree).
  {
    double sq = kAbsent;
    if (valid) {
      const double xv = ld_x(a.x + i);
      sq = dmul(xv, xv);
    }
    sq = bfly32(sq);
    if (lane == 0) s_red[warp] = sq;
  }
  __syncthreads();
  double cta;
  {
    double w[kWarps];
#pragma unroll
    for (int q = 0; q < kWarps; ++q) w[q] = s_red[q];
    cta = tree<kWarps>(w);
  }
  // step 4 pre-filter: |s| <= K * beta_local  =>  |s| <= K * beta (exact).
  if (leader) {
    const double beta_loc = a.x_norm ? __ldg(a.x_norm) : __dsqrt_rn(cta);
    const double tau_loc = dmul(__ldg(a.K + k), beta_loc);
    if (!(fabs(s_syn) <= tau_loc)) {
      const int pos = atomicAdd(a.n_cand, 1);
      a.cand[pos] = (int32_t)k;
      a.cand_s[pos] = s_syn;
      __threadfence();
    }
  }
  __syncthreads();  // all candidate writes of this CTA precede its ticket
  if (threadIdx.x == 0) {
    a.partials[blockIdx.x] = cta;
    __threadfence();
    const unsigned t = atomicAdd(a.done, 1u);
    s_last = (t == gridDim.x - 1);
    s_nflag = 0;
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();

  // ---- last CTA: beta = sqrt(PW over the CTA partials), confirm candidates.
  const int ncta = gridDim.x;
  int m = 1;
  while (m * kThreads < ncta) m <<= 1;
  {
    PwSeq acc;
    const int b = threadIdx.x * m;
    for (int q = b; q < min(b + m, ncta); ++q) acc.push(__ldcg(a.partials + q));
    s_red[threadIdx.x] = acc.finish();
  }
  __syncthreads();
  for (int s = 1; s < kThreads; s <<= 1) {
    if ((threadIdx.x & (2 * s - 1)) == 0) s_red[threadIdx.x] = dadd(s_red[threadIdx.x], s_red[threadIdx.x + s]);
    __syncthreads();
  }
  const double beta = a.x_norm ? __ldcg(a.x_norm) : __dsqrt_rn(s_red[0]);
  const int nc = __ldcg(a.n_cand);
  for (int c = threadIdx.x; c < nc; c += kThreads) {
    const int32_t kk = __ldcg(a.cand + c);
    const double s = __ldcg(a.cand_s + c);
    const double tau = dmul(__ldg(a.K + kk), beta);   // tau_k = K_k * beta
    if (!(fabs(s) <= tau)) a.flags[atomicAdd(&s_nflag, 1)] = kk;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    *a.beta = beta;
    a.n_flags[0] = s_nflag;
    for (int r = 1; r <= a.max_rounds; ++r) a.n_flags[r] = 0;
    *a.n_cand = 0;
    *a.done = 0u;
  }
}

// Step 5: round `round` recomputes the rows of every block in
// round (round-1)'s list, recomputes t1/t2 and re-checks; survivors form
// round `round`'s list.  One warp per flagged block; grid-stride.
template <bool INJECT>
__global__ void __launch_bounds__(256) k_correct(const SpmvArgs a, int round) {
  if (skip_call(a)) return;
  const int32_t nprev = __ldcg(a.n_flags + round - 1);
  if (nprev == 0) return;
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int32_t *prev = a.flags + (int64_t)(round - 1) * a.nb;
  int32_t *next = a.flags + (int64_t)round * a.nb;
  const double beta = __ldcg(a.beta);
  const int64_t n = a.n;
  for (int64_t q = gw; q < nprev; q += nw) {
    const int64_t k = __ldcg(prev + q);
    const int64_t i = (k << a.log2bs) + lane;
    const bool valid = lane < a.bs && i < n;
    int32_t rs = 0, len = 0;
    if (valid) {
      rs = __ldg(a.rp + i);
      len = __ldg(a.rp + i + 1) - rs;
    }
    const int maxlen = warp_max_i(len);
    double yv = 0.0;
    if (maxlen <= 32) {
      if (valid) yv = lane_dot_direct_any(a.va, a.ci, rs, len, maxlen, a.x);
    } else {
      for (int j = 0; j < a.bs; ++j) {
        const int32_t rb = __shfl_sync(kFull, rs, j);
        const int rl = __shfl_sync(kFull, len, j);
        if ((k << a.log2bs) + j >= n) break;
        const double t = warp_dot(a.va, a.ci, rb, rl, a.x, lane);
        if (lane == j) yv = t;
      }
    }
    if (len == 0) yv = 0.0;
    if (INJECT && valid) yv = apply_mask(yv, fault_mask(a.inj, round, 0, i, 2 * (int64_t)len));
    if (valid) a.y[i] = yv;
    double t2 = bfly32(valid ? yv : kAbsent);
    const int32_t cb = __ldg(a.crp + k), ce = __ldg(a.crp + k + 1);
    double t1 = warp_dot(a.cval, a.ccol, cb, ce - cb, a.x, lane);
    if (lane == 0) {
      if (INJECT) {
        t1 = apply_mask(t1, fault_mask(a.inj, round, 1, k, 2 * (int64_t)(ce - cb)));
        const int64_t rows = min64(a.bs, n - (k << a.log2bs));
        t2 = apply_mask(t2, fault_mask(a.inj, round, 2, k, rows));
      }
      const double s = dsub(t1, t2);
      if (!(fabs(s) <= dmul(__ldg(a.K + k), beta))) next[atomicAdd(a.n_flags + round, 1)] = (int32_t)k;
    }
  }
}

}  // namespace abft
