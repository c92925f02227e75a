// kernels_bigblock.cuh -- row blocks LARGER than a warp: b_s = 64 .. 1024
// (the block-size sweep of Fig. 4 / Fig. 7).
// Same definitions as b_s <= 32 (R4-R9): c_kj = PW over the b_s row slots,
// t2_k = PW over the b_s slots of y, t1_k = PW over C's row, K_k with the
// literal b_s.  These are the sweep's kernels, not a tuned path: b_s = 32 is
// the paper's optimum and the staged kernels serve it.
//
// Encode: one CTA of b_s threads per block, thread t walks row k b_s + t; each
// step a CTA-wide minimum of the column heads (per-warp REDUX, then over the
// warps) gives C's next column; the slot values are reduced by the butterfly
// per warp and a tree over the warps (aligned 32-slot subtrees -> PW).
// SpMV: one warp per block, its b_s / 32 groups in order -- y rows as in the
// correction pass (lane per row, warp per long row), t2 and the block's x^2
// from the groups' aligned 32-subtrees by a binary counter (== PW), t1 by the
// warp over C's row.
#pragma once
#include "kernels_spmv.cuh"

namespace abft {

template <bool FILL>
__global__ void __launch_bounds__(1024) k_encode_big(const EncodeArgs a) {
  __shared__ int s_min[32];
  __shared__ double s_v[32];
  const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
  const int nw = blockDim.x >> 5;  // b_s / 32 (a power of two)
  constexpr int kEnd = 0x7fffffff;
  for (int64_t k = blockIdx.x; k < a.nb; k += gridDim.x) {
    const int64_t i = k * a.bs + t;
    const bool valid = i < a.n;
    int32_t p = 0, e = 0;
    if (valid) {
      p = __ldg(a.rp + i);
      e = __ldg(a.rp + i + 1);
    }
    int head = p < e ? __ldg(a.ci + p) : kEnd;
    int32_t cnt = 0;
    int32_t pos = FILL ? a.crp[k] : 0;
    PwSeq csq;  // ||c_k||^2 (thread 0)
    while (true) {
      const int wm = warp_min_i(head);
      if (lane == 0) s_min[warp] = wm;
      __syncthreads();
      int mcol = kEnd;
      for (int w = 0; w < nw; ++w) mcol = min(mcol, s_min[w]);
      if (mcol == kEnd) break;  // uniform
      if (FILL) {
        const double v = bfly32((head == mcol) ? __ldg(a.va + p) : kAbsent);
        if (lane == 0) s_v[warp] = v;
        __syncthreads();
        if (t == 0) {
          double c = s_v[0];  // tree over the warps' aligned 32-slot subtrees
          for (int st = 1; st < nw; st <<= 1)
            for (int w = 0; w + st < nw; w += 2 * st) s_v[w] = dadd(s_v[w], s_v[w + st]);
          c = s_v[0];
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
      __syncthreads();  // s_min / s_v reusable
    }
    __syncthreads();
    if (!FILL) {
      if (t == 0) a.counts[k] = cnt;
    } else {
      double rn = kAbsent;  // ||a_i||_2 (R6); S_k = PW over the b_s slots
      if (valid) {
        PwSeq rsq;
        const int32_t b0 = __ldg(a.rp + i), e0 = __ldg(a.rp + i + 1);
        for (int32_t q = b0; q < e0; ++q) {
          const double v = __ldg(a.va + q);
          rsq.push(dmul(v, v));
        }
        rn = e0 > b0 ? __dsqrt_rn(rsq.finish()) : 0.0;
      }
      const double ws = bfly32(rn);
      if (lane == 0) s_v[warp] = ws;
      __syncthreads();
      if (t == 0) {
        for (int st = 1; st < nw; st <<= 1)
          for (int w = 0; w + st < nw; w += 2 * st) s_v[w] = dadd(s_v[w], s_v[w + st]);
        const double S = s_v[0];
        const double cn = cnt > 0 ? __dsqrt_rn(csq.finish()) : 0.0;
        const double mk = (double)(cnt + 2 * a.bs - 2);  // n_k + 2 b_s - 2
        a.K[k] = dmul(dadd(dmul(mk, S), dmul((double)cnt, cn)), 0x1p-53);
      }
      __syncthreads();
    }
  }
}

template <bool CHECK, bool INJECT>
__global__ void __launch_bounds__(128) k_bigblock(const SpmvArgs a) {
  if (skip_call(a)) return;
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t k = gw; k < a.nb; k += nw) {
    double gs = 0.0;
    const double s = big_block<CHECK, INJECT>(a, k, 0, lane, &gs);
    if (CHECK && lane == 0) test_block(a, k, s, gs);  // steps 3-4 (pre-filter, R12)
  }
}

}  // namespace abft
