// kernels_encode.cuh -- checksum-matrix construction, once per matrix
// (SIII-D, Fig. 3; structure P:128-130; values P:94, P:108;
// bound constants P:156-160).  Not on the per-call path.
//
// One warp per row block k; lane l walks row k*b_s + l (columns ascending).
// Each step takes the warp minimum of the lanes' current column heads: that
// is the next column of C's row k (a b_s-way merge with de-duplication, so
// C's columns come out ascending).  Lanes whose head equals it
// contribute a_ij to the column sum, reduced over the b_s row slots by the
// butterfly (PW over slots, absent where the row lacks the column).
#pragma once
#include "abft_device.cuh"

namespace abft {

struct EncodeArgs {
  int64_t n;
  int32_t bs;
  int64_t nb;
  const int32_t *__restrict__ rp;
  const int32_t *__restrict__ ci;
  const double *__restrict__ va;
  int32_t *counts;   // [nb] (count pass)
  int32_t *crp;      // [nb+1] (fill pass)
  int32_t *ccol;
  double *cval;
  double *K;
};

// Largest A and C segment over the 32-row groups (sizes the staging buffers).
__global__ void k_group_stats(int64_t n, int32_t log2bs, int64_t nb,
                              const int32_t *__restrict__ rp, const int32_t *__restrict__ crp,
                              int32_t *out /* [2]: max A seg, max C seg */) {
  const int64_t ng = (n + 31) / 32;
  int32_t ma = 0, mc = 0;
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < ng;
       g += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r0 = g * 32, r1 = min64(r0 + 32, n);
    ma = max(ma, rp[r1] - rp[r0]);
    const int64_t kb = r0 >> log2bs, ke = ((r1 - 1) >> log2bs) + 1;
    mc = max(mc, crp[min64(ke, nb)] - crp[kb]);
  }
  ma = warp_max_i(ma);
  mc = warp_max_i(mc);
  if ((threadIdx.x & 31) == 0) {
    atomicMax(out, ma);
    atomicMax(out + 1, mc);
  }
}

template <bool FILL>
__global__ void __launch_bounds__(256) k_encode(const EncodeArgs a) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  constexpr int kEnd = 0x7fffffff;
  for (int64_t k = gw; k < a.nb; k += nw) {
    const int64_t i = k * a.bs + lane;
    const bool valid = lane < a.bs && i < a.n;
    int32_t p = 0, e = 0;
    if (valid) {
      p = __ldg(a.rp + i);
      e = __ldg(a.rp + i + 1);
    }
    int head = p < e ? __ldg(a.ci + p) : kEnd;
    int32_t cnt = 0;
    int32_t pos = FILL ? a.crp[k] : 0;
    PwSeq csq;  // ||c_k||^2 over the ascending columns (lane 0)
    while (true) {
      const int mcol = warp_min_i(head);
      if (mcol == kEnd) break;
      if (FILL) {
        const double v = (head == mcol) ? __ldg(a.va + p) : kAbsent;
        const double c = bfly32(v);   // c_kj = PW over the b_s row slots
        if (lane == 0) {
          a.ccol[pos] = mcol;
          a.cval[pos] = c;
          csq.push(dmul(c, c));
        }
        ++pos;
      }
      ++cnt;
      if (head == mcol) {
        ++p;
        head = p < e ? __ldg(a.ci + p) : kEnd;
      }
    }
    if (!FILL) {
      if (lane == 0) a.counts[k] = cnt;
    } else {
      // ||a_i||_2 = sqrt(PW(a_ij^2)) over the row (R6); S_k over the slots.
      double rn = kAbsent;
      if (valid) {
        PwSeq rsq;
        const int32_t b0 = __ldg(a.rp + i), e0 = __ldg(a.rp + i + 1);
        for (int32_t q = b0; q < e0; ++q) {
          const double v = __ldg(a.va + q);
          rsq.push(dmul(v, v));
        }
        rn = e0 > b0 ? __dsqrt_rn(rsq.finish()) : 0.0;
      }
      const double S = bfly32(rn);
      if (lane == 0) {
        const double cn = cnt > 0 ? __dsqrt_rn(csq.finish()) : 0.0;
        const double nk = (double)cnt;
        const double mk = (double)(cnt + 2 * a.bs - 2);   // n_k + 2 b_s - 2
        a.K[k] = dmul(dadd(dmul(mk, S), dmul(nk, cn)), 0x1p-53);  // eps_M = 2^-53
      }
    }
  }
}

// Compact checksum matrix: the values of C in the
// narrowest type that holds every one of them exactly, and per entry a uint16
// index of an A entry of the same block with the same column (so the kernel
// reuses that entry's gathered x_j).  Rows start on 16-entry boundaries so
// every staged piece is 16-B aligned.  Lossless: the kernels recover
// bit-identical c_kj and x_j.
enum { CF_CSR = 0, CF_I8 = 1, CF_I16 = 2, CF_F32 = 3, CF_F64 = 4 };
constexpr int kCRowAlign = 16;  // compact row alignment (entries)

// props bits: 1 = some value is not an integer in [-128,127], 2 = not in
// [-32768,32767], 4 = not exactly representable in float.
__global__ void k_cformat_scan(int64_t nb, const int32_t *__restrict__ crp,
                               const int32_t *__restrict__ ccol, const double *__restrict__ cval,
                               int32_t *props) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  int32_t pr = 0;
  for (int64_t k = gw; k < nb; k += nw) {
    const int32_t b = crp[k], e = crp[k + 1];
    for (int32_t q = b + lane; q < e; q += 32) {
      const double v = cval[q];
      if (!(v == rint(v)) || v < -128.0 || v > 127.0) pr |= 1;
      if (!(v == rint(v)) || v < -32768.0 || v > 32767.0) pr |= 2;
      if (!((double)(float)v == v) && v == v) pr |= 4;
      if (v != v) pr |= 7;  // NaN: keep f64
    }
  }
  pr = __reduce_or_sync(kFull, pr);
  if (lane == 0) atomicOr(props, pr);
}

__global__ void k_cformat_padlen(int64_t nb, const int32_t *__restrict__ crp, int32_t *plen) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nb;
       k += (int64_t)gridDim.x * blockDim.x)
    plen[k] = (crp[k + 1] - crp[k] + kCRowAlign - 1) & ~(kCRowAlign - 1);
}

// Compact C for the staged fast path (b_s = 32), stored as one record per
// 32-row group so the fused kernel stages all of a group's handle-owned data
// with ONE bulk copy:
//
//   [0, 8)    K_g (double)
//   [8, 74)   ro[0..32]: row starts relative to rp[32g] (uint16)
//   [74, 76)  max row length of the group (uint16)
//   [76, 80)  zero
//   [80, ..)  plen values c_kj in the narrow type T (plen = row length of C
//             padded to 16 entries; padding values 0)
//   [.., ..)  plen uint16 A-slot indices + 1 (0 = padding)
//
// Record g starts at byte 80 g + crp_c[g] (sizeof(T) + 2); every part is
// 16-B aligned.  Instead of its column, an entry stores the staging slot of
// an A entry of the same block with that column (slot = position in A's
// arrays - (rp[32k] & ~3)), so the kernel multiplies c_kj with the x_j it
// already gathered for A; slot index 0 selects a -0.0 sentinel, so padded
// products are -0.0, the exact identity of the sum (R2).
constexpr int kRecHead = 80;  // record header bytes

__device__ __forceinline__ int64_t rec_offset(int64_t k, const int32_t *crp_c, int tsize) {
  return (int64_t)kRecHead * k + (int64_t)crp_c[k] * (tsize + 2);
}

template <typename T>
__global__ void k_cformat_fill(int64_t nb, int64_t n, const int32_t *__restrict__ rp,
                               const int32_t *__restrict__ ci, const int32_t *__restrict__ crp,
                               const int32_t *__restrict__ crp_c, const int32_t *__restrict__ ccol,
                               const double *__restrict__ cval, unsigned char *rec,
                               int32_t *bad) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t k = gw; k < nb; k += nw) {
    const int32_t b = crp[k], e = crp[k + 1];
    const int32_t plen = crp_c[k + 1] - crp_c[k];
    unsigned char *rk = rec + rec_offset(k, crp_c, (int)sizeof(T));
    T *cv = reinterpret_cast<T *>(rk + kRecHead);
    uint16_t *cmap = reinterpret_cast<uint16_t *>(rk + kRecHead + (int64_t)plen * sizeof(T));
    const int64_t r0 = k * 32, r1 = min64(r0 + 32, n);
    const int32_t s0 = rp[r0] & ~3;
    // blocks whose A segment exceeds the uint16 slot range (hub blocks) are
    // never taken by the compact-C kernels (k_lean / k_irr stage at most 1024
    // entries; k_general streams CSR C): their record is left unmapped
    const bool mapped = (int64_t)rp[r1] - s0 <= 65534;
    for (int32_t q = b + lane; q < e; q += 32) {
      const int32_t j = ccol[q];
      cv[q - b] = (T)cval[q];
      if (!mapped) {
        cmap[q - b] = 0;
        continue;
      }
      int64_t slot = -1;
      for (int64_t r = r0; r < r1 && slot < 0; ++r) {  // first row of the block holding j
        int32_t lo = rp[r], hi = rp[r + 1];
        while (lo < hi) {
          const int32_t mid = (lo + hi) >> 1;
          if (ci[mid] < j) lo = mid + 1; else hi = mid;
        }
        if (lo < rp[r + 1] && ci[lo] == j) slot = lo - s0;
      }
      if (slot < 0 || slot > 65534) atomicOr(bad, 1);
      cmap[q - b] = (uint16_t)(slot < 0 ? 0 : slot + 1);  // 0 = row padding (value 0)
    }
  }
}

// Record headers: K_g, the group's relative row starts and its longest row
// (one warp per group; values past 65535 only occur in groups the fused
// kernel does not take).
__global__ void k_cformat_head(int64_t nb, int64_t n, const int32_t *__restrict__ rp,
                               const double *__restrict__ K, const int32_t *__restrict__ crp_c,
                               int tsize, unsigned char *rec) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t k = gw; k < nb; k += nw) {
    unsigned char *rk = rec + rec_offset(k, crp_c, tsize);
    uint16_t *ro = reinterpret_cast<uint16_t *>(rk + 8);
    const int64_t r0 = k * 32;
    const int32_t base = rp[r0];
    const int32_t s = rp[min64(r0 + lane, n)] - base, e = rp[min64(r0 + lane + 1, n)] - base;
    ro[lane] = (uint16_t)min(s, 65535);
    const int ml = warp_max_i(e - s);
    if (lane == 0) {
      *reinterpret_cast<double *>(rk) = K[k];
      ro[32] = (uint16_t)min(rp[min64(r0 + 32, n)] - base, 65535);
      ro[33] = (uint16_t)min(ml, 65535);
      ro[34] = 0;
      ro[35] = 0;
    }
  }
}

// Exclusive scan of counts[0..nb) into crp[0..nb], crp[nb] = total.
// Three phases: per-CTA scan (1024 elements), scan of CTA totals (one CTA,
// sequential chunks), add offsets.
__global__ void __launch_bounds__(1024) k_scan_local(const int32_t *in, int32_t *out, int64_t n,
                                                      int32_t *totals) {
  __shared__ int32_t s_w[32];
  const int64_t g = (int64_t)blockIdx.x * 1024 + threadIdx.x;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  int32_t v = g < n ? in[g] : 0;
  int32_t inc = v;
#pragma unroll
  for (int m = 1; m < 32; m <<= 1) {
    int32_t t = __shfl_up_sync(kFull, inc, m);
    if (lane >= m) inc += t;
  }
  if (lane == 31) s_w[warp] = inc;
  __syncthreads();
  if (warp == 0) {
    int32_t w = s_w[lane];
#pragma unroll
    for (int m = 1; m < 32; m <<= 1) {
      int32_t t = __shfl_up_sync(kFull, w, m);
      if (lane >= m) w += t;
    }
    s_w[lane] = w;
  }
  __syncthreads();
  const int32_t off = warp > 0 ? s_w[warp - 1] : 0;
  if (g < n) out[g] = off + inc - v;
  if (threadIdx.x == 1023) totals[blockIdx.x] = off + inc;
}

__global__ void __launch_bounds__(1024) k_scan_totals(int32_t *totals, int64_t nt,
                                                       int32_t *out_last) {
  __shared__ int32_t s_w[32];
  __shared__ int32_t s_carry;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) s_carry = 0;
  __syncthreads();
  for (int64_t base = 0; base < nt; base += 1024) {
    const int64_t g = base + threadIdx.x;
    int32_t v = g < nt ? totals[g] : 0;
    int32_t inc = v;
#pragma unroll
    for (int m = 1; m < 32; m <<= 1) {
      int32_t t = __shfl_up_sync(kFull, inc, m);
      if (lane >= m) inc += t;
    }
    if (lane == 31) s_w[warp] = inc;
    __syncthreads();
    if (warp == 0) {
      int32_t w = s_w[lane];
#pragma unroll
      for (int m = 1; m < 32; m <<= 1) {
        int32_t t = __shfl_up_sync(kFull, w, m);
        if (lane >= m) w += t;
      }
      s_w[lane] = w;
    }
    __syncthreads();
    const int32_t off = (warp > 0 ? s_w[warp - 1] : 0) + s_carry;
    if (g < nt) totals[g] = off + inc - v;  // exclusive
    __syncthreads();
    if (threadIdx.x == 1023) s_carry = off + inc;
    __syncthreads();
  }
  if (threadIdx.x == 0) *out_last = s_carry;
}

__global__ void k_scan_add(int32_t *out, int64_t n, const int32_t *totals) {
  const int64_t g = (int64_t)blockIdx.x * 1024 + threadIdx.x;
  if (g < n) out[g] += totals[blockIdx.x];
}

}  // namespace abft
