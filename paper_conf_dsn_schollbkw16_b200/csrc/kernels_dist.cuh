// kernels_dist.cuh -- row-block sharding across GPUs (DESIGN.md
// §8): the per-call pack of a rank's halo send buffer, fused with the rank's
// ||x||^2 partial over its own rows (R28: PW over the own rows, an aligned
// node of the global tree when ranges are equal powers of two), so the
// partial can travel in the same NCCL group as the halo.
#pragma once
#include "kernels_spmv.cuh"

namespace abft {

constexpr int kDistRows = 2048;  // own rows per CTA chunk of the x^2 partial (aligned subtree)

struct DistPackArgs {
  const double *__restrict__ xo;     // own slice of the extended operand
  int64_t n_own;
  const int32_t *__restrict__ sidx;  // [n_send] own-local index of each send slot
  int64_t n_send;
  double *sbuf;                      // [n_send]
  double *chunk;                     // [ceil(n_own / kDistRows)] chunk partials
  unsigned *ticket;                  // last-CTA election (reset by the last CTA)
  double *part;                      // out: PW over the own rows of x_i^2
  int32_t want_part;
};

// One launch: every CTA gathers a grid-strided share of the send slots and
// reduces one or more aligned kDistRows-row chunks of x^2 (8 rows per thread,
// an 8-leaf tree, a CTA tree of 256 leaves == the chunk's PW); the last CTA
// to finish reduces the chunk partials (aligned runs and a CTA tree == PW).
__global__ void __launch_bounds__(256) k_dist_pack(const DistPackArgs a) {
  __shared__ double s_red[256];
  __shared__ bool s_last;
  for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < a.n_send;
       q += (int64_t)gridDim.x * blockDim.x)
    a.sbuf[q] = a.xo[__ldg(a.sidx + q)];
  if (!a.want_part) return;
  const int64_t nch = (a.n_own + kDistRows - 1) / kDistRows;
  for (int64_t c = blockIdx.x; c < nch; c += gridDim.x) {
    const int64_t r0 = c * kDistRows + (int64_t)threadIdx.x * 8;
    double v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int64_t i = r0 + u;
      v[u] = i < a.n_own ? dmul(a.xo[i], a.xo[i]) : kAbsent;
    }
    s_red[threadIdx.x] = tree<8>(v);
    __syncthreads();
    for (int st = 1; st < 256; st <<= 1) {
      if ((threadIdx.x & (2 * st - 1)) == 0)
        s_red[threadIdx.x] = dadd(s_red[threadIdx.x], s_red[threadIdx.x + st]);
      __syncthreads();
    }
    if (threadIdx.x == 0) a.chunk[c] = s_red[0];
    __syncthreads();
  }
  // last CTA: PW over the chunk partials (aligned subtrees, in order)
  if (threadIdx.x == 0) {
    __threadfence();
    s_last = atomicAdd(a.ticket, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  const double tot = cta_pw_array(a.chunk, nch, s_red);  // aligned runs + CTA tree == PW
  if (threadIdx.x == 0) {
    *a.part = nch > 0 ? tot : 0.0;
    *a.ticket = 0u;
  }
}

}  // namespace abft
