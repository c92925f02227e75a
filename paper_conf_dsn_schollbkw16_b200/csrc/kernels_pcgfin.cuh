// kernels_pcgfin.cuh -- the PCG's p.q completion inside k_finish (abft_pcg,
// protected SpMV): PW over the group partials the fused pass wrote (and the
// corrections rewrote), in the chunking of k_pcg_dotg -- aligned 2048-group
// CTA chunks (cta_pw), then grid_pw over the chunk sums -- so the bits are
// k_pcg_dotg's; then the alpha step (dot_scalars).  Saves the separate
// k_pcg_dotg launch of every protected iteration.
#pragma once
#include "kernels_pcg.cuh"
#include "kernels_spmv.cuh"

namespace abft {

// All CTAs of k_finish (solo: CTA 0 alone, every chunk).  The last CTA to
// count (a.pcga->ticket) completes the grid sum.
__device__ void pcg_fin_dot(const SpmvArgs &a, double *s_red, bool solo) {
  __shared__ double s_w[8];
  __shared__ int s_flag;
  const PcgArgs &p = *a.pcga;
  const int64_t nch = (a.ngroups + kPcgRows - 1) / kPcgRows;
  const int64_t c0 = solo ? 0 : blockIdx.x, cs = solo ? 1 : gridDim.x;
  for (int64_t c = c0; c < nch; c += cs) {
    const int64_t i0 = c * kPcgRows + threadIdx.x * kPcgPer;
    double v[8];
    ld8(v, a.pq, i0, a.ngroups);
    const double PQc = cta_pw(v, i0, a.ngroups, s_w);
    if (threadIdx.x == 0) p.part0[c] = PQc;
  }
  if (!solo && !last_cta(p.ticket, &s_flag)) return;
  if (solo) __syncthreads();
  const double PQ = grid_pw(p.part0, (int)nch, s_red);
  if (threadIdx.x == 0) {
    if (p.dsend)
      p.dsend[0] = PQ;
    else
      dot_scalars(p, PQ);
    if (!solo) *p.ticket = 0u;
  }
}

}  // namespace abft
