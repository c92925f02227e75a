// kernels_irr.cuh -- fused multiply + detect (Fig. 1 steps 1-4) for
// IRREGULAR 32-row groups (b_s = 32): rows of any length up to kHubLen, i.e.
// the power-law rows of configs[2] (R-MAT) that k_lean's lane-per-row pass
// cannot take.  DESIGN.md "Irregular groups".
//
// One warp per group (grid-stride over an encode-time list).  Per group:
//  * A pass: the group's CSR segment [rp[32g], rp[32g+32]) is ONE contiguous
//    run, loaded lane-strided and coalesced (16 values + 16 columns in flight
//    per lane), x_j gathered (16 in flight), and a_ij x_j and x_j written to
//    the warp's shared scratch on the compact-C staging grid (slot = element
//    - (rp[32g] & ~3)) -- one memory round trip for the whole group instead
//    of one per row;
//  * rows <= 32 entries: lane l reduces row 32g+l from the scratch with an
//    aligned in-register tree (PW, R3);
//  * rows 33..1024: the warp reads the row lane-strided (conflict-free) and
//    reduces 8 aligned 32-subtrees at a time with ONE reduce-scatter
//    butterfly (12 shuffles instead of 40), chunks by a 4-leaf tree (== PW);
//  * t1 (compact C): c_kj times the x_j the A pass left in the scratch at the
//    entry's A slot (no second gather); CSR C: coalesced loads + gathers;
//  * t2, t1's chunk sums and the x^2 subtree by one reduce-scatter butterfly,
//    then the exact pre-filter of R12 (as k_lean).
// Groups with hub rows (> kHubLen entries), hub C rows or segments beyond the
// scratch stay with k_general.
#pragma once
#include "kernels_spmv.cuh"

namespace abft {

#ifndef ABFT_IRR_CAP
#define ABFT_IRR_CAP 1024
#endif
#ifndef ABFT_IRR_U
#define ABFT_IRR_U 16
#endif
#ifndef ABFT_IRR_MINB
#define ABFT_IRR_MINB 3
#endif
constexpr int kIrrWarps = 4;             // warps per CTA
constexpr int kIrrCap = ABFT_IRR_CAP;    // staging-grid slots per group (segment + (rp & 3))
constexpr int kIrrU = ABFT_IRR_U;        // A entries in flight per lane
constexpr int kIrrMinB = ABFT_IRR_MINB;  // resident CTAs per SM the budget targets
constexpr size_t kIrrSmemPerWarp = 2 * (size_t)kIrrCap * sizeof(double);  // products + x_j

// PW of 8 aligned 32-subtrees held lane-strided (v[u] = element 32u + lane of
// a 256-entry chunk), returned to every lane.  Levels 1-3 of the xor butterfly
// are a reduce-scatter (a lane keeps the subtrees whose index bits match its
// own lane bits and sends the others), levels 4-5 are plain; subtree (lane &
// 7) then sits in lane l and three more levels (xor 1, 2, 4) form the 8-leaf
// tree over the subtrees.  Every addition pairs the operands PW pairs
// (fl(a+b) == fl(b+a)), so the bits equal 8 butterflies and a tree<8>.
__device__ __forceinline__ double rs_bfly8(const double (&v)[8], int lane) {
  const bool b0 = lane & 1, b1 = lane & 2, b2 = lane & 4;
  double w4[4], w2[2];
#pragma unroll
  for (int j = 0; j < 4; ++j)
    w4[j] = dadd(b0 ? v[2 * j + 1] : v[2 * j],
                 __shfl_xor_sync(kFull, b0 ? v[2 * j] : v[2 * j + 1], 1));  // subtree 2j + b0
#pragma unroll
  for (int j = 0; j < 2; ++j)
    w2[j] = dadd(b1 ? w4[2 * j + 1] : w4[2 * j],
                 __shfl_xor_sync(kFull, b1 ? w4[2 * j] : w4[2 * j + 1], 2));  // 4j + 2b1 + b0
  double w = dadd(b2 ? w2[1] : w2[0], __shfl_xor_sync(kFull, b2 ? w2[0] : w2[1], 4));
  w = dadd(w, __shfl_xor_sync(kFull, w, 8));
  w = dadd(w, __shfl_xor_sync(kFull, w, 16));  // subtree (lane & 7), all 32 lanes
  w = dadd(w, __shfl_xor_sync(kFull, w, 1));
  w = dadd(w, __shfl_xor_sync(kFull, w, 2));
  return dadd(w, __shfl_xor_sync(kFull, w, 4));
}

// Eight consecutive compact-C values from global memory (16-B aligned rows).
template <typename T>
__device__ __forceinline__ void ldg8(T (&v)[8], const unsigned char *p) {
  if constexpr (sizeof(T) == 1) {
    const uint2 w = __ldg(reinterpret_cast<const uint2 *>(p));
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      v[u] = (int8_t)((w.x >> (8 * u)) & 0xff);
      v[u + 4] = (int8_t)((w.y >> (8 * u)) & 0xff);
    }
  } else if constexpr (sizeof(T) == 2) {
    const uint4 w = __ldg(reinterpret_cast<const uint4 *>(p));
    const uint32_t ww[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = (int16_t)((ww[u >> 1] >> (16 * (u & 1))) & 0xffff);
  } else if constexpr (sizeof(T) == 4) {
    const float4 a = __ldg(reinterpret_cast<const float4 *>(p));
    const float4 b = __ldg(reinterpret_cast<const float4 *>(p + 16));
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
    v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
  } else {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const double2 d = __ldg(reinterpret_cast<const double2 *>(p + 16 * u));
      v[2 * u] = d.x;
      v[2 * u + 1] = d.y;
    }
  }
}

template <bool CHECK, bool INJECT, int CF>
__device__ __forceinline__ void group_irr(const SpmvArgs &a, int64_t g, int32_t rs, int32_t re,
                                          int lane, double *P, double *X) {
  using CT = typename CType<CF>::T;
  constexpr bool KEEPX = CHECK && CF != CF_CSR;
  const int64_t r0 = g * 32, i = r0 + lane;
  const int len = re - rs;
  const int32_t sa = __shfl_sync(kFull, rs, 0), ea = __shfl_sync(kFull, re, 31);
  const int32_t sa4 = sa & ~3;
  const int seg = ea - sa, off = sa - sa4;  // scratch slot of element e: e - sa4
  const double xv = CHECK ? __ldg(a.xr + i) : 0.0;
  // compact C: the record's first 256-entry chunk is loaded up front, so its
  // latency overlaps the A pass
  int nC = 0;
  const unsigned char *cvb = nullptr;
  const uint16_t *cm = nullptr;
  double Kk = 0.0;
  CT c0[8];
  uint4 m0 = make_uint4(0, 0, 0, 0);
  if (CHECK && CF != CF_CSR) {
    const int32_t cc = __ldg(a.crp_c + g);
    nC = __ldg(a.crp_c + g + 1) - cc;
    const unsigned char *rec = a.grec + (int64_t)kRecHead * g + (int64_t)cc * (sizeof(CT) + 2);
    Kk = __ldg(reinterpret_cast<const double *>(rec));
    cvb = rec + kRecHead;
    cm = reinterpret_cast<const uint16_t *>(cvb + (size_t)nC * sizeof(CT));
    if (lane * 8 < nC) {
      ldg8(c0, cvb + (size_t)lane * 8 * sizeof(CT));
      m0 = __ldg(reinterpret_cast<const uint4 *>(cm + lane * 8));
    }
  }

  // A pass: 16 values + 16 columns in flight per lane, then 16 gathers
#pragma unroll 1
  for (int w = 0; w < seg; w += 32 * kIrrU) {
    double v[kIrrU], xj[kIrrU];
    int c[kIrrU];
#pragma unroll
    for (int u = 0; u < kIrrU; ++u) {
      const int e = w + u * 32 + lane;
      if (e < seg) {
        v[u] = ld_stream(a.va + sa + e);
        c[u] = ld_stream(a.ci + sa + e);
      }
    }
#pragma unroll
    for (int u = 0; u < kIrrU; ++u)
      if (w + u * 32 + lane < seg) xj[u] = ld_x(a.x + c[u]);
#pragma unroll
    for (int u = 0; u < kIrrU; ++u) {
      const int e = w + u * 32 + lane;
      if (e < seg) {
        P[off + e] = dmul(v[u], xj[u]);
        if (KEEPX) X[off + e] = xj[u];
      }
    }
  }
  __syncwarp();

  // rows <= 32 entries: lane-private aligned tree from the scratch
  const int q0 = rs - sa4;
  const int plen = len <= 32 ? len : 0;
  const int pmax = warp_max_i(plen);
  double yv = 0.0;
  if (pmax > 0) yv = lane_sum_smem_any(smem_u32(P + q0), plen, pmax);
  // rows 33 .. kHubLen: the warp, 256-entry chunks of 8 aligned 32-subtrees
  unsigned longm = __ballot_sync(kFull, len > 32);
  while (longm) {
    const int j = __ffs(longm) - 1;
    longm &= longm - 1;
    const int o = __shfl_sync(kFull, q0, j), L = __shfl_sync(kFull, len, j);
    double q[4];
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      if (t * 256 < L) {
        double v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const int e = t * 256 + u * 32 + lane;
          v[u] = e < L ? P[o + e] : kAbsent;
        }
        q[t] = rs_bfly8(v, lane);
      } else {
        q[t] = kAbsent;
      }
    }
    const double t = tree<4>(q);
    if (lane == j) yv = t;
  }
  if (len == 0) yv = 0.0;  // PW of an empty row is +0.0 (R2)
  if (INJECT) yv = apply_mask(yv, group_y_mask(a.inj, 0, r0, i, lane));
  a.y[i] = yv;
  if (!CHECK) return;

  // step 1: t1_k = c_k . x; chunk sums per aligned 256 entries
  double q[4];
  int nk;  // n_k (unpadded) for the fault model
  if (CF != CF_CSR) {
    const double *xm1 = X - 1;  // slot + 1 indexing; 0 = padding (absent)
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      const int j0 = t * 256 + lane * 8;
      double qt = kAbsent;  // rows are padded to 16 entries: a lane's 8 are all in or all out
      if (t * 256 < nC && j0 < nC) {
        CT cvv[8];
        uint4 o4 = m0;
        if (t == 0) {
#pragma unroll
          for (int u = 0; u < 8; ++u) cvv[u] = c0[u];
        } else {
          ldg8(cvv, cvb + (size_t)j0 * sizeof(CT));
          o4 = __ldg(reinterpret_cast<const uint4 *>(cm + j0));
        }
        const uint32_t ow[4] = {o4.x, o4.y, o4.z, o4.w};
        double v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const int slot = (int)((ow[u >> 1] >> (16 * (u & 1))) & 0xffffu);
          v[u] = slot ? dmul((double)cvv[u], xm1[slot]) : kAbsent;
        }
        qt = tree<8>(v);
      }
      q[t] = qt;
    }
    nk = INJECT ? __ldg(a.crp + g + 1) - __ldg(a.crp + g) : 0;
    if (nC > 256) {
#pragma unroll
      for (int t = 0; t < 4; ++t) q[t] = bfly32(q[t]);
    } else {
      q[0] = bfly32(q[0]);
    }
  } else {
    const int32_t cb = __ldg(a.crp + g), ce = __ldg(a.crp + g + 1);
    nk = ce - cb;
    const GlobalSrc Cs{a.cval, a.ccol};
    q[0] = warp_dot(Cs, cb, nk, a.x, lane);  // PW of the whole row (+0.0 when empty)
    q[1] = q[2] = q[3] = kAbsent;
    Kk = __ldg(a.K + g);
    nC = nk;
  }
  double t1 = nC == 0 ? 0.0 : tree<4>(q);
  // step 2: t2_k = w_k^T y_k; the group's x^2 subtree (beta, R10)
  double t2 = bfly32(yv);
  const double gs = bfly32(dmul(xv, xv));
  if (INJECT && lane == 0) {
    t1 = apply_mask(t1, fault_mask(a.inj, 0, 1, g, 2 * (int64_t)nk));
    t2 = apply_mask(t2, fault_mask(a.inj, 0, 2, g, 32));
  }
  if (lane == 0 && a.dbg_t1) {
    a.dbg_t1[g] = t1;
    a.dbg_t2[g] = t2;
  }
  if (lane == 0) {
    a.gsum[g] = gs;
    test_block_lo(a, g, dsub(t1, t2), gs, Kk);  // steps 3-4
  }
}

__device__ __forceinline__ void prefetch_l2(const void *p, uint32_t bytes) {
  if (bytes) asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}

// Bounds of a group ahead of the current one and the L2 prefetch of its
// A segment (values, columns: 16-B aligned 4-element grid) and C record.
struct IrrBounds {
  int64_t g = 0;
  int32_t sa = 0, ea = 0, cc = 0, ce = 0;
  template <bool CHECK, int CF>
  __device__ __forceinline__ void load(const SpmvArgs &a, int64_t grp) {
    g = grp;
    sa = __ldg(a.rp + grp * 32);
    ea = __ldg(a.rp + grp * 32 + 32);
    if (CHECK && CF != CF_CSR) {
      cc = __ldg(a.crp_c + grp);
      ce = __ldg(a.crp_c + grp + 1);
    }
  }
  template <bool CHECK, int CF>
  __device__ __forceinline__ void prefetch(const SpmvArgs &a) const {
    using CT = typename CType<CF>::T;
    const int64_t nnz4 = a.nnz & ~3ll;
    const int64_t s4 = sa & ~3, e4 = min64((ea + 3) & ~3, nnz4);
    if (e4 > s4) {
      prefetch_l2(a.va + s4, (uint32_t)(e4 - s4) * 8);
      prefetch_l2(a.ci + s4, (uint32_t)(e4 - s4) * 4);
    }
    if (CHECK && CF != CF_CSR)
      prefetch_l2(a.grec + (int64_t)kRecHead * g + (int64_t)cc * (sizeof(CT) + 2),
                  (uint32_t)(kRecHead + (ce - cc) * (int)(sizeof(CT) + 2)));
  }
};

template <bool CHECK, bool INJECT, int CF>
__global__ void __launch_bounds__(kIrrWarps * 32, kIrrMinB) k_irr(const SpmvArgs a) {
  extern __shared__ __align__(16) double irr_smem[];
  if (skip_call(a)) return;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  double *P = irr_smem + (size_t)warp * 2 * kIrrCap;
  double *X = P + kIrrCap;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  // L2 prefetch one group ahead (lane 0): that group's bounds are loaded one
  // iteration earlier still, so its A segment and C record are already being
  // pulled into L2 while the current group is computed (DRAM latency off the
  // per-group critical path; the group's own loads then hit L2).
  const int64_t n = a.n_ilist;
  IrrBounds nb1, nb2;
  if (lane == 0 && gw + nw < n) nb1.load<CHECK, CF>(a, __ldg(a.ilist + gw + nw));
  // row bounds of the next group are loaded while the current one is computed
  int64_t g = gw < n ? __ldg(a.ilist + gw) : 0;
  int32_t rs = 0, re = 0;
  if (gw < n) {
    rs = __ldg(a.rp + g * 32 + lane);
    re = __ldg(a.rp + g * 32 + lane + 1);
  }
  for (int64_t q = gw; q < n; q += nw) {
    if (lane == 0) {
      if (q + nw < n) nb1.prefetch<CHECK, CF>(a);
      if (q + 2 * nw < n) nb2.load<CHECK, CF>(a, __ldg(a.ilist + q + 2 * nw));
    }
    int64_t gn = 0;
    int32_t rsn = 0, ren = 0;
    if (q + nw < n) {
      gn = __ldg(a.ilist + q + nw);
      rsn = __ldg(a.rp + gn * 32 + lane);
      ren = __ldg(a.rp + gn * 32 + lane + 1);
    }
    group_irr<CHECK, INJECT, CF>(a, g, rs, re, lane, P, X);
    __syncwarp();  // scratch reusable
    nb1 = nb2;
    g = gn;
    rs = rsn;
    re = ren;
  }
}

}  // namespace abft
