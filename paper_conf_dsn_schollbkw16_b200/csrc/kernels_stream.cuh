// kernels_stream.cuh -- the fused multiply + detect pass (Fig. 1 steps 1-4,
// P:74-76) as a warp-specialized persistent kernel over
// position-map records.
//
// Encoding (once per matrix, row-regular matrices, b_s = 32): every 32-row
// group g (= row block k) gets
//  * a STRUCTURE record: the row ends and the C positions of the group's A
//    entries (entry j of a regular row l has C position W[j] + l; the few
//    exception rows -- stencil boundary rows -- carry their own W);
//  * a CHECKSUM record: K_g and the c_kj of C's row in the narrowest exact
//    type (C's columns are never stored: every column of C's row k occurs in
//    A_k, R5, so each position receives its x_j from the A pass).
//
// Kernel: a CTA = G consumer warps + a TMA warp sharing a ring of NS
// shared-memory stages, one CHUNK of G consecutive groups per stage (chunks
// grid-strided over the eligible list: all CTAs work on nearby rows, so the
// gathered x stays in L2).  The TMA warp issues one bulk copy per array and
// chunk: structure records, checksum records (CHECK), A values, A columns
// (L2 evict-first).  Consumer warp w computes group w of each chunk, lane l
// = row 32g + l, in two phases so the x gathers of its next group are in
// flight while it finishes the current one:
//  * y_i = PW over the row of fl(a_ij x_j) (R3), an aligned 8-leaf tree;
//  * each gathered x_j is stored at its C position W[j] + l in the warp's
//    scratch; lane l then multiplies positions 8l..8l+7 with the c_kj and
//    reduces them with an 8-leaf tree and the butterfly: t1 = PW over C's
//    row of fl(c_kj x_j) (R8);
//  * t2 (R9) and the group's x^2 subtree share one reduce-scatter butterfly
//    with t1; s = t1 - t2 against the exact pre-filter K_k beta_lo (R12).
// The plain kernel (CHECK = false) is the same pipeline without the checksum
// records, the scratch, the C pass and the test.
#pragma once
#include "kernels_spmv.cuh"

namespace abft {

// ---------------------------------------------------------------------------
// Records.
//  structure record (16-B aligned):
//   [0, 64)   ro[l], l = 0..31: end of row l relative to the group's first A
//             entry (uint16); row l spans [ro[l-1], ro[l]) (ro[-1] = 0)
//   [64, 66)  nC = entries of C's row (uint16)
//   [66, 68)  zero
//   [68, 72)  exception lane mask (uint32)
//   [72, 80)  zero
//   [80, ..)  W: S int32 (S = slots per row, a multiple of 8), then one
//             block of S int32 per exception row (ascending lane); entries
//             past a row's length point at the trash positions R8 + l
//             (R8 = nC rounded up to 8), so every slot is stored unpredicated
//  checksum record (16-B aligned): [0, 8) K_g, [8, 16) zero, [16, ..) nCpad =
//   roundup(nC, 16) values c_kj of type T, ascending column order, padding 0
// ---------------------------------------------------------------------------
constexpr int kPosHead = 80;

__host__ __device__ __forceinline__ int pos_srec_bytes(int S, int n_exc) {
  return (kPosHead + 4 * S * (1 + n_exc) + 15) & ~15;
}

// One warp per group g.  Pass 0 (!FILL) writes the record sizes (16-B units;
// 0 = not eligible), and counts exception rows / eligible
// groups; pass FILL writes the records at the scanned offsets.  Eligible: a
// full group, rows <= S entries (S <= 32), C row of 1..1024 entries.
template <typename T, bool FILL>
__global__ void __launch_bounds__(256) k_pos_encode(
    int64_t n, int64_t ngroups, int32_t S, const int32_t *__restrict__ rp,
    const int32_t *__restrict__ ci, const int32_t *__restrict__ crp,
    const int32_t *__restrict__ ccol, const double *__restrict__ cval,
    const double *__restrict__ K, uint32_t *ssz, uint32_t *csz,
    const uint32_t *__restrict__ soff, const uint32_t *__restrict__ coff,
    unsigned char *srec, unsigned char *crec, unsigned long long *stats) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t g = gw; g < ngroups; g += nw) {
    const int64_t r0 = g * 32;
    bool ok = r0 + 32 <= n;
    int32_t rs = 0, re = 0;
    if (ok) {
      rs = rp[r0 + lane];
      re = rp[r0 + lane + 1];
    }
    const int len = re - rs;
    const int32_t cb = ok ? crp[g] : 0, ce = ok ? crp[g + 1] : 0;
    const int nC = ce - cb;
    ok = ok && warp_max_i(len) <= S && nC <= 1024 && nC > 0;
    if (!ok) {
      if (!FILL && lane == 0) {
        ssz[g] = 0;
        csz[g] = 0;
      }
      continue;
    }
    // positions: W_l[j] = rank of column ci[rs + j] in C's row, minus l
    int32_t W[32];
#pragma unroll 1
    for (int j = 0; j < 32; ++j) {
      W[j] = 0;
      if (j < len) {
        const int32_t col = ci[rs + j];
        int lo = cb, hi = ce;
        while (lo < hi) {
          const int mid = (lo + hi) >> 1;
          if (ccol[mid] < col) lo = mid + 1; else hi = mid;
        }
        W[j] = (lo - cb) - lane;
      }
    }
    // typical row: the candidate lane (1, 15, 16 or 30) with the fewest
    // exceptions; lane l is regular iff len_l <= len_c and its W agrees on
    // its own entries
    int best_c = 1, best = 33;
    const int cand[4] = {1, 15, 16, 30};
#pragma unroll 1
    for (int t = 0; t < 4; ++t) {
      const int c = cand[t];
      const int lc = __shfl_sync(kFull, len, c);
      bool reg = len <= lc;
#pragma unroll 1
      for (int j = 0; j < 32; ++j) {
        const int32_t wc = __shfl_sync(kFull, W[j], c);
        if (j < len && W[j] != wc) reg = false;
      }
      const int ne = __popc(__ballot_sync(kFull, !reg));
      if (ne < best) {
        best = ne;
        best_c = c;
      }
    }
    const int lc = __shfl_sync(kFull, len, best_c);
    bool reg = len <= lc;
    int32_t Wt[32];
#pragma unroll 1
    for (int j = 0; j < 32; ++j) {
      Wt[j] = __shfl_sync(kFull, W[j], best_c);
      if (j < len && W[j] != Wt[j]) reg = false;
    }
    const uint32_t mask = __ballot_sync(kFull, !reg);
    const int n_exc = __popc(mask);
    const uint32_t sbytes = (uint32_t)pos_srec_bytes(S, n_exc);
    const int nCpad = (nC + 15) & ~15;
    const uint32_t cbytes = 16u + (((uint32_t)nCpad * (uint32_t)sizeof(T) + 15u) & ~15u);
    if (!FILL) {
      if (lane == 0) {
        ssz[g] = sbytes / 16u;
        csz[g] = cbytes / 16u;
        atomicAdd(stats, (unsigned long long)n_exc);
        atomicAdd(stats + 1, 1ull);
      }
      continue;
    }
    unsigned char *R = srec + (int64_t)soff[g] * 16;
    reinterpret_cast<uint16_t *>(R)[lane] = (uint16_t)(re - rp[r0]);
    if (lane == 0) {
      *reinterpret_cast<uint16_t *>(R + 64) = (uint16_t)nC;
      *reinterpret_cast<uint16_t *>(R + 66) = 0;
      *reinterpret_cast<uint32_t *>(R + 68) = mask;
      *reinterpret_cast<uint64_t *>(R + 72) = 0;
    }
    // entries past a row's length point at the trash positions R8 + l
    const int32_t R8 = (nC + 7) & ~7;
    int32_t *Wr = reinterpret_cast<int32_t *>(R + kPosHead);
    for (int j = lane; j < S; j += 32) {
      int32_t v = R8;
#pragma unroll 1
      for (int q = 0; q < 32; ++q)
        if (q == j && j < lc) v = Wt[q];
      Wr[j] = v;
    }
    if (!reg) {
      int32_t *We = Wr + S * (1 + __popc(mask & ((1u << lane) - 1u)));
      for (int j = 0; j < S; ++j) We[j] = j < len ? W[j] : R8;
    }
    for (int b = kPosHead + 4 * S * (1 + n_exc) + lane; b < (int)sbytes; b += 32) R[b] = 0;
    unsigned char *Cr = crec + (int64_t)coff[g] * 16;
    if (lane == 0) {
      *reinterpret_cast<double *>(Cr) = K[g];
      *reinterpret_cast<uint64_t *>(Cr + 8) = 0;
    }
    T *cv = reinterpret_cast<T *>(Cr + 16);
    for (int e = lane; e < nCpad; e += 32) cv[e] = e < nC ? (T)cval[cb + e] : (T)0;
    for (int b = 16 + nCpad * (int)sizeof(T) + lane; b < (int)cbytes; b += 32) Cr[b] = 0;
  }
}

// Longest row among the full 32-row groups (sizes S).
__global__ void k_pos_maxlen(int64_t n, const int32_t *__restrict__ rp, int32_t *out) {
  int m = 0;
  const int64_t nfull = (n / 32) * 32;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nfull;
       i += (int64_t)gridDim.x * blockDim.x)
    m = max(m, rp[i + 1] - rp[i]);
  m = warp_max_i(m);
  if ((threadIdx.x & 31) == 0) atomicMax(out, m);
}

// ---------------------------------------------------------------------------
// Kernel pieces.
// ---------------------------------------------------------------------------
// chunk header at the start of each stage (int32):
//   [0 .. G]          A staging slot of group g0 + w's first entry (w = 0..ng)
//   [G+1 .. 2G+1]     byte offset of group g0 + w's structure record
//   [2G+2 .. 3G+2]    byte offset of group g0 + w's checksum record
//   [3G+3] g0 (-1: no more chunks), [3G+4] ng
__host__ __device__ constexpr uint32_t stream_hdr_bytes(int G) {
  return (uint32_t)((4 * (3 * G + 5) + 15) & ~15);
}

// Physical slot of C position p in a warp's scratch: the 16-B pair index inside
// each 8-position block is XORed with bits 1-2 of the block index, so the
// 128-bit reads of the C pass (lane l: positions 8l..8l+7, pair u) hit 8
// distinct bank groups per quarter warp.
__device__ __forceinline__ uint32_t xs_phys(int p) { return (uint32_t)(p ^ ((p >> 3) & 6)); }

__device__ __forceinline__ void lds128(uint32_t addr, double &a, double &b) {
  asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(a), "=d"(b) : "r"(addr));
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
  asm volatile(
      "{\n\t.reg .b64 st;\n\t"
      "mbarrier.arrive.release.cta.shared::cta.b64 st, [%0];\n\t}" ::"r"(smem_u32(bar))
      : "memory");
}
// Eight c_kj of a record (16-B aligned row, 8 consecutive entries).
template <typename T>
__device__ __forceinline__ void cvals8(const unsigned char *p, double (&c)[8]) {
  T v[8];
  load8(v, p);
#pragma unroll
  for (int u = 0; u < 8; ++u) c[u] = (double)v[u];
}

// Scratch layout of the C positions.  Integer checksum types (int8 / int16):
// LINEAR (position p at 8p), so a lane stores x_j at xs + 8 (W[j] + lane) with
// one address add; the C pass's 128-bit reads stay conflict-free because lane
// l reads its pairs in the order u ^ sw (sw = bits 1-2 of l) and takes the
// c_kj pairs permuted the same way (a few integer ops on the packed values).
// The 8-leaf tree then sees the pairs in the order P_{u ^ sw}: the level-1
// pair sums are the same numbers (pairs are not split), and the two level-2
// sums pair {P0, P1} and {P2, P3} in either order -- IEEE addition is
// commutative, so the bits are those of PW (R8).  Float / double checksums
// keep the XOR-swizzled layout (xs_phys) and natural-order values.
template <int CF> struct XsLinear { static constexpr bool v = (CF == CF_I8 || CF == CF_I16); };
template <int CF>
__device__ __forceinline__ uint32_t xs_addr(uint32_t xs, int p) {
  if constexpr (XsLinear<CF>::v) return xs + 8u * (uint32_t)p;
  else return xs + 8u * xs_phys(p);
}
// c_kj pairs in the read order of the C pass: pair u of c = pair u ^ sw of the
// record (linear layout); natural order otherwise.
template <int CF>
__device__ __forceinline__ void cvals8_read(const unsigned char *p, int sw, double (&c)[8]) {
  using T = typename CType<CF>::T;
  if constexpr (CF == CF_I8) {
    uint2 w = *reinterpret_cast<const uint2 *>(p);   // pair q: word q >> 1, half q & 1
    if (sw & 2) { const uint32_t t = w.x; w.x = w.y; w.y = t; }
    const uint32_t sel = (sw & 1) ? 0x1032u : 0x3210u;
    w.x = __byte_perm(w.x, 0u, sel);
    w.y = __byte_perm(w.y, 0u, sel);
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      c[u] = (double)(int8_t)((w.x >> (8 * u)) & 0xff);
      c[u + 4] = (double)(int8_t)((w.y >> (8 * u)) & 0xff);
    }
  } else if constexpr (CF == CF_I16) {
    const uint4 w4 = *reinterpret_cast<const uint4 *>(p);  // pair q: word q
    uint32_t w[4] = {w4.x, w4.y, w4.z, w4.w};
    if (sw & 1) {
      uint32_t t = w[0]; w[0] = w[1]; w[1] = t;
      t = w[2]; w[2] = w[3]; w[3] = t;
    }
    if (sw & 2) {
      uint32_t t = w[0]; w[0] = w[2]; w[2] = t;
      t = w[1]; w[1] = w[3]; w[3] = t;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) c[u] = (double)(int16_t)((w[u >> 1] >> (16 * (u & 1))) & 0xffff);
  } else {
    cvals8<T>(p, c);
  }
}

#if ABFT_EXP == 8
// timing experiment 8: per-phase SM clock cycles of the SHORT consumers
// (summed over all consumer warps, lane 0), read by abft_debug_phases
__device__ unsigned long long g_phase[8];
#define PH_MARK(v) v = clock64()
#define PH_ADD(k, t0, t1) ph[k] += (unsigned long long)((t1) - (t0))
#else
#define PH_MARK(v) ((void)(v))
#define PH_ADD(k, t0, t1) ((void)(t0), (void)(t1))
#endif

// Consumer: group g from stage `st` (header hdr, warp w, scratch xs).
template <bool CHECK, bool INJECT, int CF, bool SHORT>
__device__ __forceinline__ void stream_group(const SpmvArgs &a, const StreamCfg &c, int64_t g,
                                             int w, const unsigned char *st, uint32_t xs,
                                             int lane) {
  using CT = typename CType<CF>::T;
  const int32_t *hdr = reinterpret_cast<const int32_t *>(st);
  const int a0 = hdr[w];
  const double *av = reinterpret_cast<const double *>(st + c.off_av);
  const int32_t *ac = reinterpret_cast<const int32_t *>(st + c.off_ac);
  const int64_t i = g * 32 + lane;
  double xi = 0.0;
  if (CHECK || a.pq) xi = ld_x(a.xr + i);  // own x_i for the x^2 subtree (L2; issued early)
  const unsigned char *rec = st + c.off_srec + hdr[c.G + 1 + w];
  const unsigned char *crec = st + c.off_crec + hdr[2 * c.G + 2 + w];
  const uint16_t *ro = reinterpret_cast<const uint16_t *>(rec);
  const int re = a0 + ro[lane];
  const int rs = lane ? a0 + ro[lane - 1] : a0;
  const int len = re - rs;
  const bool hit = INJECT && inj_group_hit(a.inj, g);

  // C positions of this lane's row (CHECK): the regular row's bases, or
  // the lane's own block when it is an exception row
  const int32_t *Wp = nullptr;
  int nC = 0;
  if (CHECK) {
    const uint32_t mask = *reinterpret_cast<const uint32_t *>(rec + 68);
    nC = *reinterpret_cast<const uint16_t *>(rec + 64);
    Wp = reinterpret_cast<const int32_t *>(rec + kPosHead);
    if ((mask >> lane) & 1u) Wp += c.S * (1 + __popc(mask & ((1u << lane) - 1u)));
  }
  double yv;
  if (SHORT) {
    double xj[8];
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if (j < len) xj[j] = ld_x(a.x + ac[rs + j]);
    double v[8];
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if (j < len) v[j] = dmul(av[rs + j], xj[j]);
    yv = tree8_len(v, len);
    if (CHECK) {
      const int4 w0 = *reinterpret_cast<const int4 *>(Wp);
      const int4 w1 = *reinterpret_cast<const int4 *>(Wp + 4);
      const int32_t W[8] = {w0.x, w0.y, w0.z, w0.w, w1.x, w1.y, w1.z, w1.w};
#pragma unroll
      for (int j = 0; j < 8; ++j)
        if (j < len) sts_f64(xs_addr<CF>(xs, W[j] + lane), xj[j]);
    }
  } else {
    // rows of 9..32 entries: aligned 8-leaf subtrees one at a time,
    // tree<4>((q0 + q1) + (q2 + q3)) with absent = -0.0 (R2)
    // software-pipelined: subtree t + 1's gathers are issued before subtree
    // t is multiplied, so a row of 9..32 entries waits for L2 about once
    // instead of once per subtree (27-pt: four dependent round trips)
    double s01 = kAbsent, s23 = kAbsent;
    double xn[8];
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if (j < len) xn[j] = ld_x(a.x + ac[rs + j]);
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      if (!(len > 8 * t)) break;
      const int lt = len - 8 * t;
      double xj[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) xj[j] = xn[j];
      if (t < 3) {
#pragma unroll
        for (int j = 0; j < 8; ++j)
          if (j < lt - 8) xn[j] = ld_x(a.x + ac[rs + 8 * (t + 1) + j]);
      }
      double v[8];
#pragma unroll
      for (int j = 0; j < 8; ++j)
        if (j < lt) v[j] = dmul(av[rs + 8 * t + j], xj[j]);
      const double qt = tree8_len(v, lt);
      if (t < 2)
        s01 = t == 0 ? qt : dadd(s01, qt);
      else
        s23 = t == 2 ? qt : dadd(s23, qt);
      if (CHECK) {
        const int4 w0 = *reinterpret_cast<const int4 *>(Wp + 8 * t);
        const int4 w1 = *reinterpret_cast<const int4 *>(Wp + 8 * t + 4);
        const int32_t W[8] = {w0.x, w0.y, w0.z, w0.w, w1.x, w1.y, w1.z, w1.w};
#pragma unroll
        for (int j = 0; j < 8; ++j)
          if (j < lt) sts_f64(xs_addr<CF>(xs, W[j] + lane), xj[j]);
      }
    }
    yv = dadd(s01, s23);
  }
  if (len == 0) yv = 0.0;  // PW of an empty row is +0.0 (R2)
  InjMasks M{0, 0, 0};
  if (INJECT && hit) {
    M = inj_masks(a.inj, g, i);
    yv = apply_mask(yv, M.y);
  }
  a.y[i] = yv;
  if (!CHECK) {
    if (a.pq) {
      const double t = bfly32(dmul(xi, yv));
      if (lane == 0) a.pq[g] = t;
    }
    return;
  }

  // padding positions nC .. roundup8(nC) - 1 hold -0.0 (their c is 0: the
  // product is -0.0, the exact identity of the sum, R2)
  const int npad = (-nC) & 7;
  if (lane < npad) sts_f64(xs_addr<CF>(xs, nC + lane), kAbsent);
  __syncwarp();
  // t1_k = PW over C's row of fl(c_kj x_j) (R8): lane l owns positions
  // 256 t + 8 l .. + 7 -- an 8-leaf tree, then the butterfly; chunks of 256
  // by a 4-leaf tree
  const unsigned char *cvb = crec + 16;
  const int sw = (lane >> 1) & 3;  // xs_phys swizzle of this lane's pairs
  double q[4] = {kAbsent, kAbsent, kAbsent, kAbsent};
  const int nt = (SHORT || nC <= 256) ? 1 : (nC + 255) >> 8;
#pragma unroll
  for (int t = 0; t < (SHORT ? 1 : 4); ++t) {
    if (t >= nt) continue;
    const int j0 = t * 256 + lane * 8;
    if (j0 < nC) {
      double cv[8], v[8];
      cvals8_read<CF>(cvb + (size_t)j0 * sizeof(CT), sw, cv);
      const uint32_t blk = xs + 8u * (uint32_t)j0;
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        double x0, x1;
        lds128(blk + 16u * (uint32_t)(u ^ sw), x0, x1);
        v[2 * u] = dmul(cv[2 * u], x0);
        v[2 * u + 1] = dmul(cv[2 * u + 1], x1);
      }
      q[t] = tree<8>(v);
    }
  }
  double t2 = yv;                // step 2: t2_k = w_k^T y_k, butterflied below
  double gs = dmul(xi, xi);      // the group's x^2 subtree, butterflied below
  if (SHORT || nC <= 256) {
    // one chunk: the three butterflies as one reduce-scatter (levels 1 and 2
    // split the values over lane pairs; every value keeps PW's pairing);
    // afterwards lane 4m holds t2, 4m+1 t1 and 4m+2 the x^2 sum
    const bool b0 = lane & 1, b1 = lane & 2;
    const double pq = a.pq ? dmul(xi, yv) : kAbsent;  // 4th value: x_i y_i (PCG p.q)
    const double s0 = b0 ? t2 : q[0], s1 = b0 ? gs : pq;
    const double k0 = b0 ? q[0] : t2, k1 = b0 ? pq : gs;
    const double r0 = dadd(k0, __shfl_xor_sync(kFull, s0, 1));
    const double r1 = dadd(k1, __shfl_xor_sync(kFull, s1, 1));
    double v = dadd(b1 ? r1 : r0, __shfl_xor_sync(kFull, b1 ? r0 : r1, 2));
#pragma unroll
    for (int m = 4; m < 32; m <<= 1) v = dadd(v, __shfl_xor_sync(kFull, v, m));
    t2 = v;
    q[0] = __shfl_sync(kFull, v, 1);
    gs = __shfl_sync(kFull, v, 2);
    if (a.pq && lane == 3) a.pq[g] = v;
  } else {
    t2 = bfly32(t2);
    gs = bfly32(gs);
    if (a.pq) {
      const double t = bfly32(dmul(xi, yv));
      if (lane == 0) a.pq[g] = t;
    }
#pragma unroll
    for (int t = 0; t < 4; ++t)
      if (t < nt) q[t] = bfly32(q[t]);
  }
  double t1 = (!SHORT && nC > 256) ? tree<4>(q) : q[0];  // nC > 0 (eligible groups)
  if (INJECT && hit) {
    t1 = apply_mask(t1, M.t1);
    t2 = apply_mask(t2, M.t2);
  }
  if (lane == 0) {
    if (a.dbg_t1) {
      a.dbg_t1[g] = t1;
      a.dbg_t2[g] = t2;
    }
    a.gsum[g] = gs;
    test_block_lo(a, g, dsub(t1, t2), gs, *reinterpret_cast<const double *>(crec));  // steps 3-4
  }
  __syncwarp();  // scratch reads done before the next group's stores
}

// SHORT (rows <= 8 entries) consumer in two phases, so a warp issues the
// x gathers of its next group before it finishes the current one (their L2
// latency overlaps the products, the C pass and the butterflies).
// Phase A: row bounds, the 8 column reads and x gathers (unpredicated: slots
// past a row read the next row's staged columns or the ring's zero-filled /
// stale tail, always valid indices; their products are not summed), x_i.
struct ShortA {
  const unsigned char *st, *rec, *crec;
  int64_t g;
  int rs, len;
  int ml;    // longest row of the group (uniform)
  bool uni;  // every row of the group has ml entries (uniform)
  bool hit;  // INJECT: the group may hold a round-0 fault (inj_group_hit)
  double xj[8];
  double xi;
};

template <bool CHECK, bool INJECT>
__device__ __forceinline__ void short_load(const SpmvArgs &a, const StreamCfg &c, const double *xg,
                                           int64_t g, int w, const unsigned char *st, int lane,
                                           ShortA &A) {
  const int32_t *hdr = reinterpret_cast<const int32_t *>(st);
  const int a0 = hdr[w];
  A.st = st;
  A.g = g;
  A.rec = st + c.off_srec + hdr[c.G + 1 + w];
  A.crec = st + c.off_crec + hdr[2 * c.G + 2 + w];
  const uint16_t *ro = reinterpret_cast<const uint16_t *>(A.rec);
  const int re = a0 + ro[lane];
  const int rs = lane ? a0 + ro[lane - 1] : a0;
  A.xi = (CHECK || a.pq) ? ld_x(a.xr + g * 32 + lane) : 0.0;
  A.hit = INJECT && inj_group_hit(a.inj, g);
  A.rs = rs;
  A.len = re - rs;
  A.ml = warp_max_i(A.len);
  A.uni = warp_min_i(A.len) == A.ml;
  const int32_t *ac = reinterpret_cast<const int32_t *>(st + c.off_ac) + rs;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    if (j == 7 && A.ml <= 7) {  // uniform: the 8th slot only when some row has 8 entries
      A.xj[7] = 0.0;
      break;
    }
    if (ABFT_EXP == 6)  // timing experiment only: no x gathers (wrong results)
      A.xj[j] = (double)ac[j];
    else
      A.xj[j] = ld_x(xg + ac[j]);
  }
}

// Phase B: products and y, the C positions, t1, t2, x^2, the test.
// A finished group's values between its C pass and its butterfly.
struct ShortP {
  int64_t g;
  double t2, q0, gs, pq, K;
  uint64_t mt1, mt2;
  bool hit, on;
};

template <bool CHECK, bool INJECT, int CF>
__device__ __forceinline__ void short_finish(const SpmvArgs &a, const StreamCfg &c, const ShortA &A,
                                             uint32_t xs, int lane, ShortP &P,
                                             unsigned long long *ph) {
  long long f0 = 0, f1 = 0, f2 = 0;
  PH_MARK(f0);
  using CT = typename CType<CF>::T;
  const int64_t g = A.g, i = g * 32 + lane;
  const double *av = reinterpret_cast<const double *>(A.st + c.off_av) + A.rs;
  double v[8];
  double yv;
  if (A.uni && A.ml == 7) {  // every row 7 entries (7-pt interior): PW of 7 leaves
#pragma unroll
    for (int j = 0; j < 7; ++j) v[j] = dmul(av[j], A.xj[j]);
    yv = dadd(dadd(dadd(v[0], v[1]), dadd(v[2], v[3])), dadd(dadd(v[4], v[5]), v[6]));
  } else {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const double pr = dmul(av[j], A.xj[j]);
      v[j] = j < A.len ? pr : kAbsent;  // absent leaves (R2): no branches
    }
    yv = A.len > 0 ? tree<8>(v) : 0.0;  // PW of an empty row is +0.0 (R2)
  }
  InjMasks M{0, 0, 0};
  if (INJECT && A.hit) {
    M = inj_masks(a.inj, g, i);
    yv = apply_mask(yv, M.y);
  }
  a.y[i] = yv;
  PH_MARK(f1);
  PH_ADD(3, f0, f1);
  if (!CHECK) {
    if (a.pq) {
      const double t = bfly32(dmul(A.xi, yv));
      if (lane == 0) a.pq[g] = t;
    }
    return;
  }
  const unsigned char *rec = A.rec;
  const uint32_t mask = *reinterpret_cast<const uint32_t *>(rec + 68);
  const int nC = *reinterpret_cast<const uint16_t *>(rec + 64);
  const int32_t *Wp = reinterpret_cast<const int32_t *>(rec + kPosHead);
  if (mask != 0u && ((mask >> lane) & 1u)) Wp += 8 * (1 + __popc(mask & ((1u << lane) - 1u)));
  const int4 w0 = *reinterpret_cast<const int4 *>(Wp);
  const int4 w1 = *reinterpret_cast<const int4 *>(Wp + 4);
  const int32_t W[8] = {w0.x, w0.y, w0.z, w0.w, w1.x, w1.y, w1.z, w1.w};
  double q0 = kAbsent;
  // x_j -> C position W[j] + lane (slots past the row land in the trash)
#pragma unroll
  for (int j = 0; j < 7; ++j) sts_f64(xs_addr<CF>(xs, W[j] + lane), A.xj[j]);
  if (A.ml > 7) sts_f64(xs_addr<CF>(xs, W[7] + lane), A.xj[7]);
  const int npad = (-nC) & 7;  // positions nC .. roundup8(nC)-1 hold -0.0 (R2)
  if (lane < npad) sts_f64(xs_addr<CF>(xs, nC + lane), kAbsent);
  __syncwarp();
  const int j0 = lane * 8;
  if (j0 < nC) {
    double cv[8], u8[8];
    const int sw = (lane >> 1) & 3;
    cvals8_read<CF>(A.crec + 16 + (size_t)j0 * sizeof(CT), sw, cv);
    const uint32_t blk = xs + 8u * (uint32_t)j0;
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      double x0, x1;
      lds128(blk + 16u * (uint32_t)(u ^ sw), x0, x1);
      u8[2 * u] = dmul(cv[2 * u], x0);
      u8[2 * u + 1] = dmul(cv[2 * u + 1], x1);
    }
    q0 = tree<8>(u8);
  }
  PH_MARK(f2);
  PH_ADD(4, f1, f2);
  // hand the four values to the (possibly deferred) reduce-scatter + test
  P.g = g;
  P.t2 = yv;
  P.q0 = q0;
  P.gs = dmul(A.xi, A.xi);
  P.pq = a.pq ? dmul(A.xi, yv) : kAbsent;  // 4th value: x_i y_i (PCG p.q)
  P.K = *reinterpret_cast<const double *>(A.crec);
  P.mt1 = M.t1;
  P.mt2 = M.t2;
  P.hit = INJECT && A.hit;
  P.on = true;
  __syncwarp();  // scratch reads done before the next group's stores
}

// Steps 2-4 of a finished group (ShortP): t2 (R9), t1 (R8), the x^2 subtree
// and the p.q partial as ONE reduce-scatter butterfly (levels 1-2 split the
// four values over lane pairs, each keeping PW's pairing), then the exact
// pre-filter (R12) on lane 0.  Deferred (StreamCfg::defer): a warp runs it
// for group g after issuing the next group's gathers and before it needs
// them, so the shuffle chain overlaps their latency.
template <bool INJECT>
__device__ __forceinline__ void short_bfly(const SpmvArgs &a, ShortP &P, int lane,
                                           unsigned long long *ph) {
  long long f2 = 0, f3 = 0;
  PH_MARK(f2);
  const int64_t g = P.g;
  double t2 = P.t2, q0 = P.q0, gs = P.gs;
  {
    const bool b0 = lane & 1, b1 = lane & 2;
    const double pq = P.pq;
    const double s0 = b0 ? t2 : q0, s1 = b0 ? gs : pq;
    const double k0 = b0 ? q0 : t2, k1 = b0 ? pq : gs;
    const double r0 = dadd(k0, __shfl_xor_sync(kFull, s0, 1));
    const double r1 = dadd(k1, __shfl_xor_sync(kFull, s1, 1));
    double vv = dadd(b1 ? r1 : r0, __shfl_xor_sync(kFull, b1 ? r0 : r1, 2));
#pragma unroll
    for (int m = 4; m < 32; m <<= 1) vv = dadd(vv, __shfl_xor_sync(kFull, vv, m));
    t2 = vv;
    q0 = __shfl_sync(kFull, vv, 1);
    gs = __shfl_sync(kFull, vv, 2);
    if (a.pq && lane == 3) a.pq[g] = vv;
  }
  double t1 = q0;
  if (INJECT && P.hit) {
    t1 = apply_mask(t1, P.mt1);
    t2 = apply_mask(t2, P.mt2);
  }
  if (lane == 0) {
    if (a.dbg_t1) {
      a.dbg_t1[g] = t1;
      a.dbg_t2[g] = t2;
    }
    a.gsum[g] = gs;
    test_block_lo(a, g, dsub(t1, t2), gs, P.K);  // steps 3-4
  }
  P.on = false;
  PH_MARK(f3);
  PH_ADD(5, f2, f3);
}

#ifndef ABFT_STREAM_MINB
#define ABFT_STREAM_MINB 2  // resident CTAs per SM the register budget targets
#endif

#ifdef ABFT_STREAM_MAXNREG
#define ABFT_STREAM_BOUNDS __maxnreg__(ABFT_STREAM_MAXNREG)
#else
#define ABFT_STREAM_BOUNDS __launch_bounds__((kStreamMaxG + 1) * 32, ABFT_STREAM_MINB)
#endif

// DEFER (SHORT only): a group's reduce-scatter + test one step later
// (StreamCfg::defer picks the instantiation; a runtime branch cost 7-pt 128^3
// 5% in registers and scheduling)
template <bool CHECK, bool INJECT, int CF, bool SHORT, bool DEFER = false>
__global__ void ABFT_STREAM_BOUNDS k_stream(const SpmvArgs a) {
  extern __shared__ __align__(128) unsigned char smem[];
  pdl_trigger();  // the next kernel's CTAs may take SMs this grid leaves
  const StreamCfg c = a.stc;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int G = c.G, NS = c.NS;
  uint64_t *full = reinterpret_cast<uint64_t *>(smem);
  uint64_t *empty = full + NS;
  unsigned char *ring = smem + c.ring_off;
  // zero-fill the ring once: slots past a chunk's copy hold valid column
  // indices (0, or a previous chunk's) for the unpredicated SHORT gathers
  {
    const uint32_t words = (c.stage_bytes - c.off_ac) / 16u;
    for (int s = 0; s < NS; ++s) {
      int4 *r4 = reinterpret_cast<int4 *>(ring + (size_t)s * c.stage_bytes + c.off_ac);
      for (uint32_t q = threadIdx.x; q < words; q += blockDim.x) r4[q] = make_int4(0, 0, 0, 0);
    }
  }
  if (threadIdx.x == 0) {
    for (int s = 0; s < NS; ++s) {
      mbar_init(full + s, 1);
      mbar_init(empty + s, G);
    }
    fence_mbar_init();
  }
  fence_proxy_async_smem();  // the zero fill precedes the bulk writes into the ring
  __syncthreads();
  // the prologue above overlaps the preceding kernel (PDL); everything below
  // may read its results (x, the PCG state) or write what it reads (y, lists)
  pdl_wait();
  if (skip_call(a)) return;
  if (warp == G) {
    // ---------------- producer ----------------
    const uint64_t pol = policy_evict_first();
    const int64_t nnz4 = a.nnz & ~3ll;
    int s = 0;
    uint32_t eph = 0;   // parity of the next completion of empty[s] to wait for
    bool wrapped = false;
    int64_t t = blockIdx.x;
    int32_t q = t < a.n_clist ? __ldg(a.clist + t) : -1;
    for (;;) {
      unsigned char *st = ring + (size_t)s * c.stage_bytes;
      int32_t *hdr = reinterpret_cast<int32_t *>(st);
      // metadata of chunk q: group starts (lanes 0..ng) and record offsets
      int64_t g0 = 0;
      int ng = 0;
      int32_t arp = 0;
      uint32_t aso = 0, aco = 0;
      if (q >= 0) {
        g0 = (int64_t)q * G;
        ng = (int)min64((int64_t)G, a.ngroups - g0);
        if (lane <= ng) {
          arp = __ldg(a.rp + (g0 + lane) * 32);
          aso = __ldg(a.soff + g0 + lane);
          if (CHECK) aco = __ldg(a.coff + g0 + lane);
        }
      }
      // next chunk index (its load overlaps this chunk's issue)
      t += gridDim.x;
      const int32_t qn = (q >= 0 && t < a.n_clist) ? __ldg(a.clist + t) : -1;
      if (wrapped)  // stage reuse: wait until its consumers released it
        mbar_wait_sleep(empty + s, eph);
      if (q < 0) {
        if (lane == 0) {
          hdr[3 * G + 3] = -1;
          mbar_arrive(full + s);
        }
        break;
      }
      const int32_t sa = __shfl_sync(kFull, arp, 0), ea = __shfl_sync(kFull, arp, ng);
      const uint32_t so0 = __shfl_sync(kFull, aso, 0), so1 = __shfl_sync(kFull, aso, ng);
      const uint32_t co0 = __shfl_sync(kFull, aco, 0), co1 = __shfl_sync(kFull, aco, ng);
      const int64_t sa4 = sa & ~3, ea4 = min64(((int64_t)ea + 3) & ~3ll, nnz4);
      if (lane <= ng) {
        hdr[lane] = (int32_t)(arp - sa4);
        hdr[G + 1 + lane] = (int32_t)((aso - so0) * 16u);
        hdr[2 * G + 2 + lane] = (int32_t)((aco - co0) * 16u);
      }
      if (lane == 0) {
        hdr[3 * G + 3] = (int32_t)g0;
        hdr[3 * G + 4] = ng;
      }
      // A slots past the arrays' last 4-element boundary (the bulk copy
      // covers whole 16-B units only)
      if (ea > nnz4 && lane < 4) {
        const int64_t e = nnz4 + lane;
        if (e < a.nnz && e >= sa4) {
          reinterpret_cast<int32_t *>(st + c.off_ac)[e - sa4] = __ldg(a.ci + e);
          reinterpret_cast<double *>(st + c.off_av)[e - sa4] = __ldg(a.va + e);
        }
      }
      __syncwarp();
      if (lane == 0) {
        const uint32_t bav = ea4 > sa4 ? (uint32_t)(ea4 - sa4) * 8u : 0u;
        const uint32_t bac = ea4 > sa4 ? (uint32_t)(ea4 - sa4) * 4u : 0u;
        const uint32_t bsr = (so1 - so0) * 16u;
        const uint32_t bcr = CHECK ? (co1 - co0) * 16u : 0u;
        mbar_arrive_expect_tx(full + s, bav + bac + bsr + bcr);
        bulk_g2s(st + c.off_srec, a.srec + (int64_t)so0 * 16, bsr, full + s, pol);
        if (CHECK) bulk_g2s(st + c.off_crec, a.grec + (int64_t)co0 * 16, bcr, full + s, pol);
        if (bav) bulk_g2s(st + c.off_av, a.va + sa4, bav, full + s, pol);
        if (bac) bulk_g2s(st + c.off_ac, a.ci + sa4, bac, full + s, pol);
      }
      q = qn;
      if (++s == NS) {
        s = 0;
        if (wrapped) eph ^= 1u;
        wrapped = true;
      }
    }
    return;
  }
  // ---------------- consumers ----------------
  const uint32_t xs = smem_u32(smem + c.xs_off + (size_t)warp * c.xs_bytes);
  int s = 0;
  uint32_t fph = 0;  // parity of the next completion of full[s]
  if constexpr (SHORT) {
    // ping-pong between two phase-A states (no register copies): each step
    // loads the next stage's group into one state and finishes the other
    const double *xg = a.x;
    ShortA sa, sb;
    ShortP P;
    P.on = false;
    unsigned long long ph[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    (void)ph;
    mbar_wait_sleep(full + s, fph);
    {
      const int32_t *hdr = reinterpret_cast<const int32_t *>(ring + (size_t)s * c.stage_bytes);
      const int32_t g0 = hdr[3 * G + 3];
      if (g0 < 0) return;
      if (warp < hdr[3 * G + 4])
        short_load<CHECK, INJECT>(a, c, xg, (int64_t)g0 + warp, warp, ring + (size_t)s * c.stage_bytes, lane, sa);
      else
        sa.g = -1;
    }
    // one step: wait for the next stage, phase A of its group into `nx`,
    // phase B of `cu`, release the current stage; false at the end
    auto step = [&](ShortA &cu, ShortA &nx) -> bool {
      long long t0 = 0, t1 = 0, t2 = 0, t3 = 0;
      PH_MARK(t0);
      int s1 = s + 1;
      uint32_t fph1 = fph;
      if (s1 == NS) {
        s1 = 0;
        fph1 ^= 1u;
      }
      const unsigned char *st1 = ring + (size_t)s1 * c.stage_bytes;
      mbar_wait_sleep(full + s1, fph1);
      PH_MARK(t1);
      PH_ADD(0, t0, t1);
      const int32_t *hdr1 = reinterpret_cast<const int32_t *>(st1);
      const int32_t g0n = hdr1[3 * G + 3];
      nx.g = -1;
      if (g0n >= 0 && warp < hdr1[3 * G + 4])
        short_load<CHECK, INJECT>(a, c, xg, (int64_t)g0n + warp, warp, st1, lane, nx);
      PH_MARK(t2);
      PH_ADD(1, t1, t2);
      if (CHECK && DEFER && P.on) short_bfly<INJECT>(a, P, lane, ph);
      if (cu.g >= 0) short_finish<CHECK, INJECT, CF>(a, c, cu, xs, lane, P, ph);
      if (CHECK && !DEFER && P.on) short_bfly<INJECT>(a, P, lane, ph);
      __syncwarp();
      if (lane == 0) mbar_arrive(empty + s);
      PH_MARK(t3);
      PH_ADD(2, t2, t3);
      ph[6] += 1;
      s = s1;
      fph = fph1;
      return g0n >= 0;
    };
    while (step(sa, sb) && step(sb, sa)) {
    }
    if (CHECK && P.on) short_bfly<INJECT>(a, P, lane, ph);
#if ABFT_EXP == 8
    if (lane == 0)
      for (int k = 0; k < 7; ++k) atomicAdd(&g_phase[k], ph[k]);
#endif
  } else {
    for (;;) {
      const unsigned char *st = ring + (size_t)s * c.stage_bytes;
      mbar_wait_sleep(full + s, fph);
      const int32_t *hdr = reinterpret_cast<const int32_t *>(st);
      const int32_t g0 = hdr[3 * G + 3];
      if (g0 < 0) break;
      const int ng = hdr[3 * G + 4];
      if (warp < ng) stream_group<CHECK, INJECT, CF, false>(a, c, (int64_t)g0 + warp, warp, st, xs, lane);
      fence_proxy_async_smem();  // generic accesses of this stage precede its next bulk write
      __syncwarp();
      if (lane == 0) mbar_arrive(empty + s);
      if (++s == NS) {
        s = 0;
        fph ^= 1u;
      }
    }
  }
}

}  // namespace abft
