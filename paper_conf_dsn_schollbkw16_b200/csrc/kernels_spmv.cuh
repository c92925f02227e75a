// kernels_spmv.cuh -- the hot path: fused multiply + detect (Fig. 1 steps
// 1-4) with an in-kernel finalize, and the correction pass (step 5,
// P:76).  DESIGN.md "Kernels" has the derivations.
//
// Work unit: a GROUP of 32 consecutive rows (= 32/b_s row blocks).
//
// Which kernel runs a group (plan at encode, abft.cu plan_fused):
//  * k_stream (kernels_stream.cuh): row-regular matrices --
//    position-map records, a warp-specialized TMA ring; the default for
//    every stencil;
//  * k_lean (below): the slot-map compact-C records (ABFT_NO_POS, or when
//    the position map cannot describe the matrix);
//  * k_irr (kernels_irr.cuh): groups with rows of 33..1024 entries;
//  * k_hub (below): aligned 1024-entry chunks of hub rows / hub C rows;
//  * k_general (below): everything else (b_s < 32, the ragged last group,
//    groups owning hub rows, unaligned operands) -- one warp per group,
//    operands read directly from global memory.
//
// k_lean (b_s = 32): a persistent grid; each warp owns a contiguous range of
// groups and pipelines them through per-warp shared-memory stages filled by
// TMA 1-D bulk copies (cp.async.bulk + mbarrier transaction counts, L2
// evict-first) of the group's record, x slice, A values and columns.  Per
// group: lane l = row 32g + l computes y_i as an in-register PW tree of its
// gathered products (rows <= 32 entries); each gathered x_j replaces a_ij in
// the staged values, where the C pass finds it through the record's slot
// map (t1 = PW over C's row); t2, t1 and the group's x^2 subtree share one
// reduce-scatter butterfly; s = t1 - t2 is compared with K_k * beta_lo,
// beta_lo <= beta exactly (an aligned node of the PW tree of ||x||^2,
// rounded down; R12): |s| <= K beta_lo proves the block clean,
// anything else becomes a candidate; the x^2 subtree goes to gsum[g].
// k_finish (one PDL launch after them) confirms the candidates against
// tau_k = K_k beta, beta = sqrt(PW(gsum)) computed by all SMs only when a
// candidate exists (or taken from x_norm), writes the flagged-block list and
// runs the correction rounds.
#pragma once
#include "abft_device.cuh"
#include "bulk.cuh"
#include "kernels_encode.cuh"

namespace abft {

// Element type of the compact checksum matrix for each format (CF_*).
template <int CF> struct CType { using T = double; };
template <> struct CType<CF_I8> { using T = int8_t; };
template <> struct CType<CF_I16> { using T = int16_t; };
template <> struct CType<CF_F32> { using T = float; };

constexpr int kLeanWarps = 4;  // warps per CTA of k_lean (<= 4)
// Timing experiments only (scripts/exp_libs.sh; results are NOT the method):
// 1 = no C products, 2 = C neither staged nor multiplied, 3 = no butterflies,
// 4 = no test, 5 = 1 + 3 + 4, 6 = k_stream without x gathers, 8 = k_stream
// SHORT per-phase cycle counters (scripts/phase_probe.py), 9 = PCG update
// without the division.  0 (the default)
// = the method.
#ifndef ABFT_EXP
#define ABFT_EXP 0
#endif
#ifndef ABFT_LEAN_MINB
#define ABFT_LEAN_MINB 5  // min resident CTAs per SM the register budget targets (measured best)
#endif
// SHORT instantiation (every k_lean row <= 8 entries: 5-/7-point stencils):
// the 16/32-leaf row path is compiled out, which lets the budget target 7
// CTAs per SM for the protected kernel (72 registers, no spills) and 6 for
// the plain one -- measured on 7-pt 128^3: protected 0.0594 -> 0.0550 ms,
// plain 0.0370 -> 0.0371 ms (7 CTAs: 0.0378).  The general instantiation
// keeps 5 (6 costs 27-pt 128^3 9%).
#ifndef ABFT_LEAN_MINB_SHORT
#define ABFT_LEAN_MINB_SHORT 7
#endif
#ifndef ABFT_LEAN_MINB_SHORT_PLAIN
#define ABFT_LEAN_MINB_SHORT_PLAIN 6
#endif

struct StageCfg {
  int32_t capA, capC;     // staged capacity (elements) of a group's A / C segment
  int32_t nstage;         // stages per warp (prefetch distance nstage-1)
  int32_t warps;          // warps per CTA
  uint32_t stage_bytes;   // bytes per stage
  uint32_t bar_bytes;     // mbarrier region at the start of dynamic smem
  uint32_t off_rp, off_x, off_k, off_av, off_ac, off_cv, off_cc, off_cp, off_xg;
  int32_t colg;           // A columns read from global memory, not staged (COLG)
};

// k_stream (kernels_stream.cuh): producer / consumer ring configuration.
constexpr int kStreamMaxG = 8;  // consumer warps per CTA (groups per chunk), at most
struct StreamCfg {
  int32_t G;             // groups per chunk = consumer warps per CTA
  int32_t NS;            // ring stages
  int32_t S;             // W slots per row of the structure records (multiple of 8)
  uint32_t stage_bytes;  // bytes per stage
  uint32_t off_srec;     // stage: structure records
  uint32_t off_crec;     // stage: checksum records (CHECK)
  uint32_t off_av, off_ac;  // stage: A values / columns (4-element grid from the chunk's first entry)
  uint32_t ring_off;     // dynamic smem: ring start (after the barriers)
  uint32_t xs_off;       // dynamic smem: per-consumer-warp C-position scratch
  uint32_t xs_bytes;     // per warp
  int32_t defer;         // SHORT consumers: a group's butterfly runs one step later
};

struct PcgArgs;  // kernels_pcg.cuh

struct SpmvArgs {
  int64_t n;
  int64_t nnz;
  int64_t nnz_c;     // entries of C (CSR arrays; k_hub's prefetch bound)
  int32_t bs;        // block size, power of two <= 1024 (> 32: kernels_bigblock.cuh)
  int32_t log2bs;
  int64_t nb;
  int64_t ngroups;
  const int32_t *__restrict__ rp;
  const int32_t *__restrict__ ci;
  const double *__restrict__ va;
  const int32_t *__restrict__ crp;
  const int32_t *__restrict__ ccol;
  const double *__restrict__ cval;
  const unsigned char *__restrict__ grec;  // compact C: per-group records (kernels_encode.cuh)
  const int32_t *__restrict__ crp_c;    // compact row starts (16-entry aligned)
  const double *__restrict__ K;
  const double *__restrict__ x;   // gather base: column j reads x[j]
  const double *__restrict__ xr;  // row-aligned view: row i's own entry is xr[i]
  double *__restrict__ y;
  const double *x_norm;   // nullable device scalar
  double *gsum;           // [ngroups] x^2 subtree of each group
  // nullable: [ngroups] PW over the group's rows of x_i y_i (PCG's p.q fused
  // into the SpMV epilogue, a 32-row aligned node of the global PW tree;
  // correction rounds rewrite it for the blocks they recompute, b_s = 32)
  double *pq;
  // abft_pcg, protected: k_finish also completes PW over the p.q group
  // partials and the PCG's alpha step (no separate k_pcg_dotg launch)
  const PcgArgs *pcga;
  double *bpart;          // [ceil(ngroups / 1024)] beta partials (k_finish)
  int32_t *n_cand;        // candidate count (reset by k_finish)
  int32_t *cand;          // [nb]
  double *cand_s;         // [nb]
  int32_t *flags;         // [(max_rounds+1) * nb]; round r at flags + r*nb
  int32_t *n_flags;       // [max_rounds+1]
  int32_t max_rounds;
  double *beta;           // device scalar out
  int32_t *beta_valid;    // 1 when *beta holds ||x|| of the last call
  unsigned *gbar;         // [2] grid barrier of the correction pass
  const int32_t *glist;   // k_general: groups to process (nullptr: all groups)
  int64_t n_glist;
  const int32_t *ilist;   // k_irr: irregular groups (kernels_irr.cuh)
  int64_t n_ilist;
  double *dbg_t1, *dbg_t2;  // nullable
  const int32_t *skip;      // nullable device flag: != 0 -> kernels are no-ops (PCG)
  const uint8_t *lean_ok;   // [ngroups] bit 0: k_lean takes the group; bit 1: it owns hub rows
  // hub rows: A rows / C rows longer than kHubLen are
  // split into aligned kHubLen-entry chunks, summed by k_hub before the fused
  // pass; the group kernels combine the chunk sums (PW: aligned subtrees).
  const int64_t *hub_beg;   // [n_hub] first entry of the chunk (A or C arrays)
  const uint32_t *hub_len;  // [n_hub] entries | (1u << 31 for a C row)
  double *hub_part;         // [n_hub] PW of the chunk's products
  int32_t n_hub;
  const int32_t *own_key;   // [n_own] sorted: g * 64 + (C ? 32 : 0) + row / block index in group
  const int32_t *own_first; // [n_own] first chunk item
  const int32_t *own_n;     // [n_own] chunk items
  int32_t n_own;
  StageCfg sc;
  InjDev inj;
  // k_stream (position-map records, kernels_stream.cuh); grec = checksum records
  const unsigned char *srec;  // structure records
  const uint32_t *soff;     // [ngroups + 1] structure record offsets (16-B units)
  const uint32_t *coff;     // [ngroups + 1] checksum record offsets (16-B units)
  const int32_t *clist;     // eligible chunks
  int64_t n_clist;
  StreamCfg stc;
};

__device__ __forceinline__ bool skip_call(const SpmvArgs &a) {
  return a.skip && *(volatile const int32_t *)a.skip != 0;
}

// ---------------------------------------------------------------------------
// Operand accessors and PW reductions over them.
// ---------------------------------------------------------------------------
struct GlobalSrc {  // streamed (L1 no-allocate, L2 evict-first)
  const double *v;
  const int32_t *c;
  __device__ __forceinline__ double val(int64_t e) const { return ld_stream(v + e); }
  __device__ __forceinline__ int32_t col(int64_t e) const { return ld_stream(c + e); }
};
struct LdgSrc {  // L1-cached (correction pass)
  const double *v;
  const int32_t *c;
  __device__ __forceinline__ double val(int64_t e) const { return __ldg(v + e); }
  __device__ __forceinline__ int32_t col(int64_t e) const { return __ldg(c + e); }
};

// PW over products of elements [b, b+cnt), cnt <= 256, whole warp: lane l
// holds elements u*32 + l; each 32-chunk by the butterfly, chunks by a tree.
template <class Src>
__device__ __forceinline__ double warp_dot256(const Src &s, int64_t b, int cnt,
                                              const double *__restrict__ x, int lane) {
  double v[8];
  int c[8];
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    const int e = u * 32 + lane;
    if (e < cnt) {
      v[u] = s.val(b + e);
      c[u] = s.col(b + e);
    }
  }
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    const int e = u * 32 + lane;
    v[u] = e < cnt ? dmul(v[u], ld_x(x + c[u])) : kAbsent;
  }
#pragma unroll
  for (int u = 0; u < 8; ++u)
    if (u * 32 < cnt) v[u] = bfly32(v[u]);
  return tree<8>(v);
}

// PW over an arbitrary-length dot product, whole warp; +0.0 when empty.
template <class Src>
__device__ __forceinline__ double warp_dot(const Src &s, int64_t b, int64_t n,
                                           const double *__restrict__ x, int lane) {
  if (n <= 0) return 0.0;
  if (n <= 256) return warp_dot256(s, b, (int)n, x, lane);
  PwSeq acc;  // binary counter over aligned 256-chunks (== PW)
  for (int64_t o = 0; o < n; o += 256)
    acc.push(warp_dot256(s, b + o, (int)min64(256, n - o), x, lane));
  return acc.finish();
}

// Lane-private PW dot over a short row (len <= P <= 8).
template <int P, class Src>
__device__ __forceinline__ double lane_dot8(const Src &s, int64_t b, int len,
                                            const double *__restrict__ x) {
  double v[P];
  int c[P];
#pragma unroll
  for (int j = 0; j < P; ++j)
    if (j < len) {
      v[j] = s.val(b + j);
      c[j] = s.col(b + j);
    }
#pragma unroll
  for (int j = 0; j < P; ++j) v[j] = j < len ? dmul(v[j], ld_x(x + c[j])) : kAbsent;
  return tree<P>(v);
}

// P = 16/32: aligned 8-leaf subtrees one at a time, then a tree over them.
template <int P, class Src>
__device__ __forceinline__ double lane_dot(const Src &s, int64_t b, int len,
                                           const double *__restrict__ x) {
  if constexpr (P <= 8) {
    return lane_dot8<P>(s, b, len, x);
  } else {
    // aligned 8-leaf subtrees one at a time (bounded register use):
    // tree<4>((q0 + q1) + (q2 + q3)), absent subtrees = -0.0 (P = 16: q2 = q3 absent)
    double s01 = kAbsent, s23 = kAbsent;
#pragma unroll 1
    for (int t = 0; t < P / 8 && t * 8 < len; ++t) {
      const double qt = lane_dot8<8>(s, b + t * 8, len - t * 8, x);
      if (t < 2)
        s01 = t == 0 ? qt : dadd(s01, qt);
      else
        s23 = t == 2 ? qt : dadd(s23, qt);
    }
    return dadd(s01, s23);
  }
}

template <class Src>
__device__ __noinline__ double lane_dot_any(const Src &s, int64_t b, int len, int maxlen,
                                               const double *__restrict__ x) {
  if (maxlen <= 1) return lane_dot<1>(s, b, len, x);
  if (maxlen <= 2) return lane_dot<2>(s, b, len, x);
  if (maxlen <= 4) return lane_dot<4>(s, b, len, x);
  if (maxlen <= 8) return lane_dot<8>(s, b, len, x);
  if (maxlen <= 16) return lane_dot<16>(s, b, len, x);
  return lane_dot<32>(s, b, len, x);
}

// Lane-private PW over P staged products at a shared address (len <= P).
template <int P>
__device__ __forceinline__ double lane_sum_smem(uint32_t addr, int len) {
  if constexpr (P <= 8) {
    double v[P];
#pragma unroll
    for (int j = 0; j < P; ++j) v[j] = j < len ? lds_f64(addr + 8u * j) : kAbsent;
    return tree<P>(v);
  } else {
    double q[P / 8];
#pragma unroll
    for (int t = 0; t < P / 8; ++t)
      q[t] = (t * 8 < len) ? lane_sum_smem<8>(addr + 64u * t, len - 8 * t) : kAbsent;
    return tree<P / 8>(q);
  }
}

__device__ __forceinline__ double lane_sum_smem_any(uint32_t addr, int len, int maxlen) {
  if (maxlen <= 1) return lane_sum_smem<1>(addr, len);
  if (maxlen <= 2) return lane_sum_smem<2>(addr, len);
  if (maxlen <= 4) return lane_sum_smem<4>(addr, len);
  if (maxlen <= 8) return lane_sum_smem<8>(addr, len);
  if (maxlen <= 16) return lane_sum_smem<16>(addr, len);
  return lane_sum_smem<32>(addr, len);
}

// Whole-warp PW over n <= 1024 staged products at addr (+0.0 when empty).
__device__ __forceinline__ double warp_sum_smem(uint32_t addr, int n, int lane) {
  if (n <= 0) return 0.0;
  double q[4];
#pragma unroll
  for (int t = 0; t < 4; ++t) {
    if (t * 256 < n) {
      double v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int e = t * 256 + u * 32 + lane;
        v[u] = e < n ? lds_f64(addr + 8u * e) : kAbsent;
      }
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (t * 256 + u * 32 < n) v[u] = bfly32(v[u]);
      q[t] = tree<8>(v);
    } else {
      q[t] = kAbsent;
    }
  }
  return tree<4>(q);
}

// ---------------------------------------------------------------------------
// Long rows.  kHubLen = the longest row a warp reduces
// through its scratch in one pass; longer rows are hub rows (k_hub chunks).
// ---------------------------------------------------------------------------
constexpr int kHubLen = 1024;
constexpr int kScr = kHubLen + kHubLen / 32;  // padded scratch (doubles per warp)
constexpr int kGenWarps = 4;                  // warps per CTA of k_general / k_hub

// PW over the products of entries [b, b+n), n <= kHubLen, whole warp: 32U-entry
// windows of coalesced lane-strided loads and gathers, products into the
// warp's scratch at e + e/32 (conflict-free both ways); lane l then reduces
// the aligned 32-entry subtree 32l..32l+31 (four 8-leaf trees and a 4-leaf
// tree) and the butterfly joins the 32 subtrees: the PW tree of the row.
// +0.0 when n == 0 (R2).
template <int U, class Src>
__device__ __noinline__ double warp_row_pw(const Src &s, int64_t b, int n,
                                              const double *__restrict__ x, double *scr,
                                              int lane) {
  if (n <= 0) return 0.0;
#pragma unroll 1
  for (int w = 0; w < n; w += 32 * U) {  // U loads, then U gathers in flight per lane
    double v[U];
    int c[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int e = w + u * 32 + lane;
      if (e < n) {
        v[u] = s.val(b + e);
        c[u] = s.col(b + e);
      }
    }
    // all U gathers in flight before the first product is stored: the
    // stores go through a generic pointer the compiler cannot separate from
    // x, so gathers issued after a store would wait for it (one DRAM round
    // trip per entry -- R-MAT hub rows ran 4x slower)
    double xj[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int e = w + u * 32 + lane;
      xj[u] = e < n ? ld_x(x + c[u]) : 0.0;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int e = w + u * 32 + lane;
      if (e < n) scr[e + (e >> 5)] = dmul(v[u], xj[u]);
    }
  }
  __syncwarp();
  const int e0 = lane * 32;
  const double *p = scr + lane * 33;
  double q[4];
#pragma unroll
  for (int t = 0; t < 4; ++t) {
    double v[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) v[j] = e0 + 8 * t + j < n ? p[8 * t + j] : kAbsent;
    q[t] = tree<8>(v);
  }
  const double r = bfly32(tree<4>(q));
  __syncwarp();  // scratch reusable
  return r;
}

// Chunk sums of hub items (one warp per item; items are independent).
#ifndef ABFT_HUB_MINB
#define ABFT_HUB_MINB 1  // resident CTAs per SM the register budget targets
#endif
#ifndef ABFT_HUB_U
#define ABFT_HUB_U 16  // entries in flight per lane
#endif
__global__ void __launch_bounds__(kGenWarps * 32, ABFT_HUB_MINB) k_hub(const SpmvArgs a) {
  __shared__ double scr_all[kGenWarps][kScr];
  if (a.skip && *(volatile const int32_t *)a.skip != 0) return;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const bool pf = ((reinterpret_cast<uintptr_t>(a.va) | reinterpret_cast<uintptr_t>(a.ci) |
                    reinterpret_cast<uintptr_t>(a.cval) | reinterpret_cast<uintptr_t>(a.ccol)) & 15u) == 0;
  for (int64_t q = gw; q < a.n_hub; q += nw) {
    // the warp's next item: its values and columns on their way into L2
    // while this one is reduced (the stream loads then wait for L2, not DRAM)
    if (pf && lane == 0 && q + nw < a.n_hub) {
      const uint32_t Ln = __ldg(a.hub_len + q + nw);
      const int64_t bn = __ldg(a.hub_beg + q + nw);
      const bool cn = Ln >> 31;
      const int64_t lim = (cn ? a.nnz_c : a.nnz) & ~3ll;
      const int64_t s4 = bn & ~3ll, e4 = min64((bn + (int64_t)(Ln & 0x7fffffffu) + 3) & ~3ll, lim);
      if (e4 > s4) {
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"((cn ? a.cval : a.va) + s4),
                     "r"((uint32_t)(e4 - s4) * 8u) : "memory");
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"((cn ? a.ccol : a.ci) + s4),
                     "r"((uint32_t)(e4 - s4) * 4u) : "memory");
      }
    }
    const uint32_t L = __ldg(a.hub_len + q);
    const int64_t b = __ldg(a.hub_beg + q);
    const int n = (int)(L & 0x7fffffffu);
    double r;
    if (L >> 31) {
      struct { const double *v; const int32_t *c;
        __device__ double val(int64_t e) const { return ld_stream(v + e); }
        __device__ int32_t col(int64_t e) const { return ld_stream(c + e); } } Cs{a.cval, a.ccol};
      r = warp_row_pw<ABFT_HUB_U>(Cs, b, n, a.x, scr_all[warp], lane);
    } else {
      struct { const double *v; const int32_t *c;
        __device__ double val(int64_t e) const { return ld_stream(v + e); }
        __device__ int32_t col(int64_t e) const { return ld_stream(c + e); } } As{a.va, a.ci};
      r = warp_row_pw<ABFT_HUB_U>(As, b, n, a.x, scr_all[warp], lane);
    }
    if (lane == 0) a.hub_part[q] = r;
  }
}

// PW over a hub row's chunk sums (aligned kHubLen-subtrees, in order).
__device__ __noinline__ double hub_sum(const SpmvArgs &a, int32_t first, int32_t cnt) {
  PwSeq acc;
  for (int32_t t = 0; t < cnt; ++t) acc.push(__ldcg(a.hub_part + first + t));
  return acc.finish();
}

// The same PW with the whole warp: lanes load 32 consecutive chunk sums at a
// time and the ascending xor butterfly reduces them (an aligned 32-chunk
// subtree; absent slots past cnt), the subtrees join by the binary counter --
// PW over the chunks again (R2: padding independence).  Warp-uniform.
__device__ __forceinline__ double hub_sum_warp(const SpmvArgs &a, int32_t first, int32_t cnt,
                                               int lane) {
  PwSeq acc;
  for (int32_t b = 0; b < cnt; b += 32)
    acc.push(bfly32(lane < cnt - b ? __ldcg(a.hub_part + first + b + lane) : kAbsent));
  return acc.finish();
}

// Range [lo, hi) of the group's entries in the sorted owner table.
__device__ __forceinline__ void own_range(const SpmvArgs &a, int64_t g, int &lo, int &hi) {
  lo = hi = 0;
  if (a.n_own == 0) return;
  const int32_t k0 = (int32_t)(g * 64), k1 = (int32_t)(g * 64 + 64);
  int l = 0, r = a.n_own;
  while (l < r) {
    const int m = (l + r) >> 1;
    if (__ldg(a.own_key + m) < k0) l = m + 1; else r = m;
  }
  lo = l;
  r = a.n_own;
  while (l < r) {
    const int m = (l + r) >> 1;
    if (__ldg(a.own_key + m) < k1) l = m + 1; else r = m;
  }
  hi = l;
}

// Owner-table entry with low key bits `low` (row index, or 32 + block index
// for a C row) among [lo, hi) of one group; -1 when absent.
__device__ __forceinline__ int own_find(const SpmvArgs &a, int lo, int hi, int low) {
  for (int e = lo; e < hi; ++e)
    if ((__ldg(a.own_key + e) & 63) == low) return e;
  return -1;
}

// ---------------------------------------------------------------------------
// Candidate test (step 4 pre-filter) shared by both kernels.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void test_block(const SpmvArgs &a, int64_t k, double s, double gs) {
  const double beta_g = a.x_norm ? __ldg(a.x_norm) : __dsqrt_rn(gs);
  if (!(fabs(s) <= dmul(__ldg(a.K + k), beta_g))) {
    const int pos = atomicAdd(a.n_cand, 1);
    a.cand[pos] = (int32_t)k;
    a.cand_s[pos] = s;
    __threadfence();
  }
}

// Same test with a cheaper exact lower bound of beta_g: for gs in [2^e,
// 2^(e+1)), beta_lo = 2^floor(e/2) <= sqrt(gs) <= beta (0 for zero,
// subnormal, Inf or NaN gs), so the pre-filter stays exact (a passing block
// provably passes against tau_k; the rest are confirmed by k_finish).
__device__ __forceinline__ double beta_lower(double gs) {
  const int hi = __double2hiint(gs);
  const int ef = (hi >> 20) & 0x7ff;
  const int h = (ef - 1023) >> 1;  // floor(e / 2)
  return (ef == 0 || ef == 0x7ff) ? 0.0 : __hiloint2double((h + 1023) << 20, 0);
}
__device__ __forceinline__ void test_block_lo(const SpmvArgs &a, int64_t k, double s, double gs,
                                              double Kk) {
  const double beta_lo = a.x_norm ? __ldg(a.x_norm) : beta_lower(gs);
  if (!(fabs(s) <= dmul(Kk, beta_lo))) {
    const int pos = atomicAdd(a.n_cand, 1);
    a.cand[pos] = (int32_t)k;
    a.cand_s[pos] = s;
    __threadfence();
  }
}

// ---------------------------------------------------------------------------
// General path: one group, operands from global memory (any b_s <= 32).
// ---------------------------------------------------------------------------
template <bool CHECK, bool INJECT>
__device__ __forceinline__ void group_general(const SpmvArgs &a, int64_t g, int lane, double *scr) {
  const int64_t n = a.n;
  const int64_t r0 = g * 32;
  const int64_t i = r0 + lane;
  const bool valid = i < n;
  int32_t rs = 0, re = 0;
  double xv = 0.0;
  if (valid) {
    rs = __ldg(a.rp + i);
    re = __ldg(a.rp + i + 1);
    xv = __ldg(a.xr + i);
  }
  const GlobalSrc As{a.va, a.ci}, Cs{a.cval, a.ccol};
  const int len = re - rs;
  // hub rows / hub C rows of this group (rare: an empty range almost always)
  int olo = 0, ohi = 0;
  if (a.lean_ok[g] & 2) own_range(a, g, olo, ohi);  // bit 1: the group owns hub rows
  bool hub = false;
  double yv = 0.0;
  for (int e = olo; e < ohi; ++e) {  // warp-uniform
    const int32_t key = __ldg(a.own_key + e);
    if (!(key & 32)) {  // A row 32g + (key & 31)
      const double t = hub_sum_warp(a, __ldg(a.own_first + e), __ldg(a.own_n + e), lane);
      if ((key & 31) == lane) {
        hub = true;
        yv = t;
      }
    }
  }
  // row-length-adaptive y: rows <= 32 entries lane-private (an aligned tree of
  // P = 2^ceil(log2 maxlen) leaves), longer ones by the warp (warp_row_pw)
  const bool small = !hub && len <= 32;
  const int maxs = warp_max_i(small ? len : 0);
  if (small && valid) yv = lane_dot_any(As, rs, len, maxs, a.x);
  unsigned longm = __ballot_sync(kFull, valid && !hub && len > 32);
  while (longm) {
    const int j = __ffs(longm) - 1;
    longm &= longm - 1;
    const double t = warp_row_pw<8>(As, __shfl_sync(kFull, rs, j), __shfl_sync(kFull, len, j), a.x,
                                 scr, lane);
    if (lane == j) yv = t;
  }
  if (len == 0) yv = 0.0;  // PW of an empty row is +0.0 (R2)
  if (INJECT) {
    const uint64_t m = group_y_mask(a.inj, 0, r0, i, lane);
    if (valid) yv = apply_mask(yv, m);
  }
  if (valid) a.y[i] = yv;
  if (a.pq) {
    const double t = bfly32(valid ? dmul(xv, yv) : kAbsent);
    if (lane == 0) a.pq[g] = t;
  }
  if (!CHECK) return;

  // step 2: t2_k = w_k^T y_k over the b_s slots; absent past n.
  double t2 = bfly(valid ? yv : kAbsent, a.bs);
  // step 1: t1_k = c_k . x: the 32/b_s C rows of the group,
  // lane-per-C-row when short, warp-cooperative otherwise, hub rows by chunks.
  const int bl = lane >> a.log2bs;
  const int64_t k = (r0 >> a.log2bs) + bl;
  const bool leader = ((lane & (a.bs - 1)) == 0) && valid;
  const int nblk = 32 >> a.log2bs;
  const int64_t kl = (r0 >> a.log2bs) + lane;
  int32_t cb = 0, ce = 0;
  if (lane < nblk && kl < a.nb) {
    cb = __ldg(a.crp + kl);
    ce = __ldg(a.crp + kl + 1);
  }
  const int nkl = ce - cb;
  bool chub = false;
  double t1l = 0.0;
  for (int e = olo; e < ohi; ++e) {  // warp-uniform
    const int32_t key = __ldg(a.own_key + e);
    if (key & 32) {  // C row of block (key & 31) of the group
      const double t = hub_sum_warp(a, __ldg(a.own_first + e), __ldg(a.own_n + e), lane);
      if ((key & 31) == lane) {
        chub = true;
        t1l = t;
      }
    }
  }
  const bool csmall = nblk > 1 && !chub && nkl <= 32;
  const int maxnk = warp_max_i(csmall ? nkl : 0);
  if (csmall && lane < nblk) t1l = lane_dot_any(Cs, cb, nkl, maxnk, a.x);
  unsigned cl = __ballot_sync(kFull, lane < nblk && !chub && !csmall);
  while (cl) {
    const int l = __ffs(cl) - 1;
    cl &= cl - 1;
    const int32_t b = __shfl_sync(kFull, cb, l);
    const int m = __shfl_sync(kFull, nkl, l);
    const double t = warp_row_pw<8>(Cs, b, m, a.x, scr, lane);
    if (lane == l) t1l = t;
  }
  if (nkl == 0) t1l = 0.0;
  double t1 = __shfl_sync(kFull, t1l, bl);
  const int nk = __shfl_sync(kFull, nkl, bl);
  if (INJECT && leader) {
    t1 = apply_mask(t1, fault_mask(a.inj, 0, 1, k, 2 * (int64_t)nk));
    t2 = apply_mask(t2, fault_mask(a.inj, 0, 2, k, min64(a.bs, n - (k << a.log2bs))));
  }
  if (leader && a.dbg_t1) {
    a.dbg_t1[k] = t1;
    a.dbg_t2[k] = t2;
  }
  const double gs = bfly32(valid ? dmul(xv, xv) : kAbsent);  // the group's x^2 subtree
  if (lane == 0) a.gsum[g] = gs;
  if (leader) test_block(a, k, dsub(t1, t2), gs);  // steps 3-4
}

template <bool CHECK, bool INJECT>
#ifndef ABFT_GEN_MINB
#define ABFT_GEN_MINB 4
#endif
__global__ void __launch_bounds__(kGenWarps * 32, ABFT_GEN_MINB) k_general(const SpmvArgs a) {
  __shared__ double scr_all[kGenWarps][kScr];
  if (skip_call(a)) return;
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t q = gw; q < a.n_glist; q += nw) {
    const int64_t g = a.glist ? (int64_t)__ldg(a.glist + q) : q;
    group_general<CHECK, INJECT>(a, g, lane, scr_all[threadIdx.x >> 5]);
  }
}

// ---------------------------------------------------------------------------
// Lean path: b_s = 32, full staged group, two stages per warp.  Shared memory
// is addressed through pointers derived from the kernel's shared array (so
// guarded accesses compile to predicated LDS/STS, not branches).
// ---------------------------------------------------------------------------

// Eight consecutive elements of a 16-B aligned staged compact-C row.
__device__ __forceinline__ void load8(int8_t (&v)[8], const unsigned char *p) {
  const uint2 w = *reinterpret_cast<const uint2 *>(p);
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    v[u] = (int8_t)((w.x >> (8 * u)) & 0xff);
    v[u + 4] = (int8_t)((w.y >> (8 * u)) & 0xff);
  }
}
__device__ __forceinline__ void load8(int16_t (&v)[8], const unsigned char *p) {
  const uint4 w = *reinterpret_cast<const uint4 *>(p);
  const uint32_t ww[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
  for (int u = 0; u < 8; ++u) v[u] = (int16_t)((ww[u >> 1] >> (16 * (u & 1))) & 0xffff);
}
__device__ __forceinline__ void load8(float (&v)[8], const unsigned char *p) {
  const float4 a = *reinterpret_cast<const float4 *>(p);
  const float4 b = *reinterpret_cast<const float4 *>(p + 16);
  v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
  v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}
__device__ __forceinline__ void load8(double (&v)[8], const unsigned char *p) {
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const double2 d = *reinterpret_cast<const double2 *>(p + 16 * u);
    v[2 * u] = d.x;
    v[2 * u + 1] = d.y;
  }
}

// Padded slot of C product e: one gap every 8 doubles, so lane l can read its
// 8 consecutive products e = 8l..8l+7 without bank conflicts.
__device__ __forceinline__ int cpad(int e) { return e + (e >> 3); }

// Fault-list ranges of a warp's contiguous group range (INJECT only): list
// positions [y0, y1) hold the y faults of its rows, [k0, k1) / [q0, q1) the
// t1 / t2 faults of its blocks (round 0).
struct InjRange {
  int y0, y1, k0, k1, q0, q1;
};

__device__ __forceinline__ InjRange inj_range(const InjDev &inj, int64_t g0, int64_t g1,
                                              int lane) {
  InjRange R{0, 0, 0, 0, 0, 0};
  if (lane == 0 && inj.mode == 1) {
    const int len = list_len(inj);
    if (len > 0) {
      R.y0 = list_lower(inj, len, list_key(0, 0, g0 * 32));
      R.y1 = list_lower(inj, len, list_key(0, 0, g1 * 32));
      R.k0 = list_lower(inj, len, list_key(0, 1, g0));
      R.k1 = list_lower(inj, len, list_key(0, 1, g1));
      R.q0 = list_lower(inj, len, list_key(0, 2, g0));
      R.q1 = list_lower(inj, len, list_key(0, 2, g1));
    }
  }
  R.y0 = __shfl_sync(kFull, R.y0, 0);
  R.y1 = __shfl_sync(kFull, R.y1, 0);
  R.k0 = __shfl_sync(kFull, R.k0, 0);
  R.k1 = __shfl_sync(kFull, R.k1, 0);
  R.q0 = __shfl_sync(kFull, R.q0, 0);
  R.q1 = __shfl_sync(kFull, R.q1, 0);
  return R;
}

// One aligned 8-leaf subtree of a lane-owned row: entries o .. o+min(len,8)-1
// of the staged arrays; PW with absent (-0.0) leaves past the row's end.
// KEEPX: the gathered x_j replaces a_ij in the staged values (xg == av; each
// slot belongs to one row, so only its owner lane touches it here).
__device__ __forceinline__ void tpr_gather8(const int32_t *ac, int o, int len,
                                            const double *__restrict__ x, double (&xj)[8]) {
  const int32_t *acp = ac + o;
#pragma unroll
  for (int j = 0; j < 8; ++j)
    if (j < len) xj[j] = ld_x(x + acp[j]);
}

// PW over the leaves v[0 .. len) of an 8-leaf tree: a node whose right
// subtree is absent passes its left one through (== -0.0 padding, R2), so
// absent leaves are never read and need no value.
__device__ __forceinline__ double tree8_len(double (&v)[8], int len) {
  if (len > 1) v[0] = dadd(v[0], v[1]);
  if (len > 3) v[2] = dadd(v[2], v[3]);
  if (len > 5) v[4] = dadd(v[4], v[5]);
  if (len > 7) v[6] = dadd(v[6], v[7]);
  if (len > 2) v[0] = dadd(v[0], v[2]);
  if (len > 6) v[4] = dadd(v[4], v[6]);
  if (len > 4) v[0] = dadd(v[0], v[4]);
  return v[0];  // meaningful when len > 0
}

template <bool KEEPX>
__device__ __forceinline__ double tpr_finish8(const double *av, double *xg, int o, int len,
                                              const double (&xj)[8]) {
  double v[8];
  const double *avp = av + o;
  double *xgp = xg + o;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    if (j < len) {
      v[j] = dmul(avp[j], xj[j]);  // a_ij read before x_j takes its slot (xg == av)
      if (KEEPX) xgp[j] = xj[j];
    }
  }
#pragma unroll
  for (int j = 0; j < 8; ++j)
    if (j >= len) v[j] = kAbsent;
  return tree<8>(v);
}
template <bool KEEPX>
__device__ __forceinline__ double tpr_chunk8(const double *av, const int32_t *ac, double *xg,
                                             int o, int len, const double *__restrict__ x) {
  double xj[8];
  tpr_gather8(ac, o, len, x, xj);
  return tpr_finish8<KEEPX>(av, xg, o, len, xj);
}

// A group's row bounds and, for rows of <= 8 entries, its x gathers already
// in flight (k_lean issues them one group ahead: their L2 latency overlaps
// the previous group's C pass and butterflies).
struct Pre {
  int32_t rs, re;
  int maxlen;
  double xj[8];
};

// Row bounds of staged group g (+ the gathers when every row has <= 8
// entries).  Also stages the A slots past the arrays' last 4-element
// boundary, which the bulk copy cannot cover.
// A columns of the group on the staging grid: staged, or (COLG) straight from
// global memory (L1-cached loads), which frees a third of each stage.
template <bool COLG>
__device__ __forceinline__ const int32_t *cols_base(const SpmvArgs &a, int32_t sa,
                                                    const unsigned char *st) {
  if (COLG) return a.ci + (sa & ~3);
  return reinterpret_cast<const int32_t *>(st + a.sc.off_ac);
}

template <int CF, bool SHORT, bool COLG>
__device__ __forceinline__ void pregather(const SpmvArgs &a, int32_t sa, int32_t ea,
                                          unsigned char *st, int lane, Pre &p) {
  const StageCfg &c = a.sc;
  if (ea > (a.nnz & ~3ll)) {  // A slots past the arrays' last 4-element boundary
    const int64_t nnz4 = a.nnz & ~3ll;
    const int64_t e = nnz4 + lane;  // slots of elements nnz4 .. nnz4+3
    if (lane < 4 && e >= (sa & ~3)) {
      const bool real = e < a.nnz;
      if (!COLG)
        reinterpret_cast<int32_t *>(st + c.off_ac)[e - (sa & ~3)] = real ? __ldg(a.ci + e) : 0;
      reinterpret_cast<double *>(st + c.off_av)[e - (sa & ~3)] = real ? __ldg(a.va + e) : 0.0;
    }
    __syncwarp();
  }
  // compact C: relative row starts and the longest row come with the record
  if (CF != CF_CSR) {
    const uint16_t *ro = reinterpret_cast<const uint16_t *>(st + c.off_rp + 8);
    p.rs = sa + ro[lane];
    p.re = sa + ro[lane + 1];
    p.maxlen = ro[33];
  } else {
    p.rs = reinterpret_cast<const int32_t *>(st + c.off_rp)[lane];
    p.re = __shfl_down_sync(kFull, p.rs, 1);
    if (lane == 31) p.re = ea;
    p.maxlen = warp_max_i(p.re - p.rs);
  }
  if (SHORT || p.maxlen <= 8)
    tpr_gather8(cols_base<COLG>(a, sa, st), p.rs - (sa & ~3), p.re - p.rs,
                a.x, p.xj);
}

template <bool CHECK, bool INJECT, int CF, bool SHORT, bool COLG>
__device__ __forceinline__ void group32(const SpmvArgs &a, int64_t g, int32_t sa, int32_t ea,
                                        int32_t sc, int32_t ec, unsigned char *st, int lane,
                                        const InjRange &R, const Pre &p) {
  using CT = typename CType<CF>::T;
  const StageCfg &c = a.sc;
  const int64_t i = g * 32 + lane;
  // A: values and columns staged on the same 4-element grid from sa & ~3, so
  // slot s holds element (sa & ~3) + s in both arrays.
  double *av = reinterpret_cast<double *>(st + c.off_av);
  const int32_t *ac = cols_base<COLG>(a, sa, st);
  const double *cv = reinterpret_cast<const double *>(st + c.off_cv) + (sc & 1);  // sc + e
  const int32_t *cc = reinterpret_cast<const int32_t *>(st + c.off_cc) + (sc & 3);
  double *cp = reinterpret_cast<double *>(st + c.off_cp);  // C products, padded
  double *xg = av;  // compact C, rows <= 32: gathered x_j per A slot, in place of a_ij
  const int nC = CHECK ? ec - sc : 0;
  const int32_t rs = p.rs;
  const int maxlen = p.maxlen;
  const int len = p.re - p.rs;
  double yv;
  {
    // rows of <= 32 entries (the encode-time plan gives k_lean no group with
    // a longer row): lane l computes row 32g + l on its own (staged
    // values and columns read at the row's slots -- conflict-free for the
    // near-constant row strides of stencils; x gathers of one instruction
    // hit 32 consecutive rows' j-th neighbours, i.e. a few lines), products
    // stay in registers, and (compact C) the gathered x_j replaces a_ij in
    // the staged values (xg[slot], read by the C pass).
    const int o = rs - (sa & ~3);  // staging slot of the row's first entry
    constexpr bool KEEPX = CHECK && CF != CF_CSR;
    if (SHORT || maxlen <= 8) {
      yv = tpr_finish8<KEEPX>(av, xg, o, len, p.xj);  // gathers issued by pregather
    } else {
      // 16 / 32 leaves: aligned 8-leaf subtrees one at a time (bounded
      // register use), tree<4>((q0 + q1) + (q2 + q3)) with absent = -0.0
      double s01 = kAbsent, s23 = kAbsent;
#pragma unroll 1
      for (int t = 0; t < 4 && len > 8 * t; ++t) {
        const double qt = tpr_chunk8<KEEPX>(av, ac, xg, o + 8 * t, len - 8 * t, a.x);
        if (t < 2)
          s01 = t == 0 ? qt : dadd(s01, qt);
        else
          s23 = t == 2 ? qt : dadd(s23, qt);
      }
      yv = dadd(s01, s23);
    }
  }
  // phase 1b (CSR C): C products into the padded layout (lane-strided, 8 gathers)
  if (CHECK && CF == CF_CSR) {
#pragma unroll 1
    for (int base = 0; base < nC; base += 256) {
      const double *cvl = cv + base + lane;
      const int32_t *ccl = cc + base + lane;
      double *cpl = cp + cpad(base + lane);  // cpad(e + 32u) = cpad(e) + 36u
      const int rc = nC - base - lane;
      double vc[8];
      int32_t ic[8];
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (u * 32 < rc) {
          vc[u] = cvl[u * 32];
          ic[u] = ccl[u * 32];
        }
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (u * 32 < rc) vc[u] = dmul(vc[u], ld_x(a.x + ic[u]));
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (u * 32 < rc) cpl[u * 36] = vc[u];
    }
  }
  if (CHECK) __syncwarp();  // xg / cp complete before the C pass reads them
  if (len == 0) yv = 0.0;  // PW of an empty row is +0.0 (R2)
  if (INJECT && R.y0 < R.y1) yv = apply_mask(yv, list_mask_in(a.inj, R.y0, R.y1, list_key(0, 0, i)));
  a.y[i] = yv;
  if (!CHECK) return;

  // the three warp butterflies (t2, chunk sums of t1, x^2) are independent:
  // they run interleaved in one loop below, so their latencies overlap
  double t2 = yv;  // step 2: t2_k = w_k^T y_k -- butterflied below
  const double xv = reinterpret_cast<const double *>(st + c.off_x)[lane];
  double gs = dmul(xv, xv);  // the group's x^2 subtree -- butterflied below
  // step 1: t1_k = c_k . x.  Lane l owns elements 8l..8l+7 of
  // each aligned 256-chunk: an 8-leaf tree in registers, then the butterfly
  // over lanes -- exactly the PW tree of the chunk; chunks by a 4-leaf tree.
  double q[4] = {kAbsent, kAbsent, kAbsent, kAbsent};
  if (ABFT_EXP == 1 || ABFT_EXP == 2 || ABFT_EXP == 5) {
    q[0] = q[1] = q[2] = q[3] = kAbsent;
  } else if (CF != CF_CSR) {
    // compact C: the row is staged 16-B aligned; values and A-slot indices
    // come in with vector loads, x_j from the A pass (in place of a_ij)
    const unsigned char *cvb = st + c.off_rp + kRecHead;
    const uint16_t *cm = reinterpret_cast<const uint16_t *>(cvb + (size_t)nC * sizeof(CT));
    const double *xgm1 = xg - 1;  // slot + 1 indexing; xg[-1] = -0.0 (padding)
    // uniform: one 256-chunk in the common case (SHORT: always -- the plan
    // takes SHORT only when every staged C row has <= 256 entries)
    const int nt = (SHORT || nC <= 256) ? 1 : 4;
#pragma unroll
    for (int t = 0; t < (SHORT ? 1 : 4); ++t) {
      if (t >= nt) {
        q[t] = kAbsent;
        continue;
      }
      const int j0 = t * 256 + lane * 8;
      double qt = kAbsent;  // rows are padded to 16 entries: a lane's 8 are all in or all out
      if (j0 < nC) {
        double v[8];
        CT cvv[8];
        load8(cvv, cvb + (size_t)j0 * sizeof(CT));
        const uint4 o4 = *reinterpret_cast<const uint4 *>(cm + j0);
        const uint32_t ow[4] = {o4.x, o4.y, o4.z, o4.w};
#pragma unroll
        for (int u = 0; u < 8; ++u) {  // slot + 1; 0 = padding -> -0.0 sentinel
          const int slot = (int)((ow[u >> 1] >> (16 * (u & 1))) & 0xffffu);
          v[u] = dmul((double)cvv[u], xgm1[slot]);
        }
        qt = tree<8>(v);
      }
      q[t] = qt;
    }
  } else {
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      if (t * 256 < nC) {
        const double *cpl = cp + t * 288 + lane * 9;  // cpad(t*256 + 8 lane + u)
        const int rc = nC - t * 256 - lane * 8;
        double v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = u < rc ? cpl[u] : kAbsent;
        q[t] = tree<8>(v);
      } else {
        q[t] = kAbsent;
      }
    }
  }
  if (ABFT_EXP == 3 || ABFT_EXP == 5) {
  } else if (SHORT || nC <= 256) {
    // the common case, one chunk: the three butterflies as one reduce-scatter
    // (levels 1 and 2 split the values over lane pairs, levels 3-5 are plain
    // butterflies) -- each value still sees the ascending-offset pairing of
    // PW; afterwards lane 4m holds t2, 4m+1 t1's chunk and 4m+2 the x^2 sum
    const bool b0 = lane & 1, b1 = lane & 2;
    const double s0 = b0 ? t2 : q[0], s1 = b0 ? gs : kAbsent;  // sent at level 1
    const double k0 = b0 ? q[0] : t2, k1 = b0 ? kAbsent : gs;  // kept
    const double r0 = dadd(k0, __shfl_xor_sync(kFull, s0, 1));
    const double r1 = dadd(k1, __shfl_xor_sync(kFull, s1, 1));
    double v = dadd(b1 ? r1 : r0, __shfl_xor_sync(kFull, b1 ? r0 : r1, 2));
#pragma unroll
    for (int m = 4; m < 32; m <<= 1) v = dadd(v, __shfl_xor_sync(kFull, v, m));
    t2 = v;
    q[0] = __shfl_sync(kFull, v, 1);
    gs = __shfl_sync(kFull, v, 2);
  } else {
    t2 = bfly32(t2);
    gs = bfly32(gs);
#pragma unroll
    for (int t = 0; t < 4; ++t)
      if (t * 256 < nC) q[t] = bfly32(q[t]);
  }
  // PW over the chunk sums (one chunk: q[0] itself; an empty row: +0.0)
  double t1 = (!SHORT && nC > 256) ? tree<4>(q) : nC > 0 ? q[0] : 0.0;
  if (INJECT && lane == 0) {
    if (R.k0 < R.k1) t1 = apply_mask(t1, list_mask_in(a.inj, R.k0, R.k1, list_key(0, 1, g)));
    if (R.q0 < R.q1) t2 = apply_mask(t2, list_mask_in(a.inj, R.q0, R.q1, list_key(0, 2, g)));
  }
  if (lane == 0 && a.dbg_t1) {
    a.dbg_t1[g] = t1;
    a.dbg_t2[g] = t2;
  }
  if (lane == 0) {
    a.gsum[g] = gs;
    if (ABFT_EXP != 4 && ABFT_EXP != 5) test_block_lo(a, g, dsub(t1, t2), gs,  // steps 3-4
                    CF != CF_CSR ? *reinterpret_cast<const double *>(st + c.off_rp)
                                 : reinterpret_cast<const double *>(st + c.off_k)[g & 1]);
  }
}

// Group bounds from the per-warp window: lane l holds rp[32 (wb+l)],
// crp[wb+l] and (compact C) crp_c[wb+l] (b_s = 32; clamped to n / nb).
template <int CF>
struct Window {
  int64_t wb;
  int32_t rpw, crpw, ccw;  // CSR C uses crpw, compact C ccw
  int32_t okw;             // lean_ok of group wb + lane
  __device__ __forceinline__ void load(const SpmvArgs &a, int64_t base, int lane) {
    wb = base;
    okw = a.lean_ok[min64(base + lane, a.ngroups - 1)];
    rpw = ld_stream(a.rp + min64((base + lane) * 32, a.n));
    if (CF == CF_CSR)
      crpw = ld_stream(a.crp + min64(base + lane, a.nb));
    else
      ccw = ld_stream(a.crp_c + min64(base + lane, a.nb));
  }
  __device__ __forceinline__ bool ok(int64_t g) const {
    return (__shfl_sync(kFull, okw, (int)(g - wb)) & 1) != 0;
  }
  // CSR C: sc/ec = C row bounds.  Compact C: sc = 0, ec = padded row length
  // (so ec - sc bounds the staged entries either way), cc = compact row start
  __device__ __forceinline__ void get(int64_t g, int32_t &sa, int32_t &ea, int32_t &sc,
                                      int32_t &ec, int32_t &cc) const {
    const int j = (int)(g - wb);
    sa = __shfl_sync(kFull, rpw, j);
    ea = __shfl_sync(kFull, rpw, j + 1);
    if (CF == CF_CSR) {
      sc = __shfl_sync(kFull, crpw, j);
      ec = __shfl_sync(kFull, crpw, j + 1);
      cc = 0;
    } else {
      cc = __shfl_sync(kFull, ccw, j);
      sc = 0;
      ec = __shfl_sync(kFull, ccw, j + 1) - cc;
    }
  }
};

// Issue the bulk copies of group g into stage `st` (lane 0 only).  The
// unprotected baseline (CHECK = false) does not touch C.
template <bool CHECK, int CF, bool COLG>
__device__ __forceinline__ void issue_stage(const SpmvArgs &a, int64_t g, int32_t sa, int32_t ea,
                                            int32_t sc, int32_t ec, int32_t cc, unsigned char *st,
                                            uint64_t *bar, uint64_t pol) {
  if (CF != CF_CSR) {  // compact C: record, x slice, A values, A columns
    using CT = typename CType<CF>::T;
    const StageCfg &c = a.sc;
    const int64_t r0 = g * 32;
    const int64_t nnz4 = a.nnz & ~3ll;
    const int64_t sa4 = sa & ~3, ea4 = min64((ea + 3) & ~3, nnz4);
    const uint32_t bav = ea4 > sa4 ? (uint32_t)(ea4 - sa4) * 8 : 0;
    const uint32_t bac = (!COLG && ea4 > sa4) ? (uint32_t)(ea4 - sa4) * 4 : 0;
    const uint32_t brec = kRecHead + (CHECK && ABFT_EXP != 2
                                          ? (uint32_t)ec * (uint32_t)(sizeof(CT) + 2) : 0u);
    const unsigned char *rec = a.grec + (int64_t)kRecHead * g + (int64_t)cc * (sizeof(CT) + 2);
    mbar_arrive_expect_tx(bar, brec + 256 + bav + bac);
    bulk_g2s(st + c.off_rp, rec, brec, bar, pol);
    bulk_g2s(st + c.off_x, a.xr + r0, 256, bar, pol);
    if (bav) bulk_g2s(st + c.off_av, a.va + sa4, bav, bar, pol);
    if (bac) bulk_g2s(st + c.off_ac, a.ci + sa4, bac, bar, pol);
    return;
  }
  const StageCfg &c = a.sc;
  const int64_t r0 = g * 32;
  const int64_t nnz4 = a.nnz & ~3ll;
  const int64_t sa4 = sa & ~3, ea4 = min64((ea + 3) & ~3, nnz4);  // A: 4-element grid
  const int64_t sc8 = sc & ~1, ec8 = (ec + 1) & ~1;  // C is padded: no clamp
  const int64_t sc4 = sc & ~3, ec4 = (ec + 3) & ~3;
  const uint32_t bav = ea4 > sa4 ? (uint32_t)(ea4 - sa4) * 8 : 0;
  const uint32_t bac = ea4 > sa4 ? (uint32_t)(ea4 - sa4) * 4 : 0;
  const uint32_t bcv = CHECK && ec8 > sc8 ? (uint32_t)(ec8 - sc8) * 8 : 0;
  const uint32_t bcc = CHECK && ec4 > sc4 ? (uint32_t)(ec4 - sc4) * 4 : 0;
  mbar_arrive_expect_tx(bar, 128 + 256 + (CHECK ? 16 : 0) + bav + bac + bcv + bcc);
  bulk_g2s(st + c.off_rp, a.rp + r0, 128, bar, pol);  // rp[r0 .. r0+31]; rp[r0+32] = ea
  bulk_g2s(st + c.off_x, a.xr + r0, 256, bar, pol);
  if (CHECK) bulk_g2s(st + c.off_k, a.K + (g & ~1ll), 16, bar, pol);
  if (bav) bulk_g2s(st + c.off_av, a.va + sa4, bav, bar, pol);
  if (bac) bulk_g2s(st + c.off_ac, a.ci + sa4, bac, bar, pol);
  if (bcv) bulk_g2s(st + c.off_cv, a.cval + sc8, bcv, bar, pol);
  if (bcc) bulk_g2s(st + c.off_cc, a.ccol + sc4, bcc, bar, pol);
}

// Work runs of k_lean (RUNS instantiation, NST = 2, chosen when ngroups >
// tw * kLeanRun): the groups are cut into super-chunks of tw * kLeanRun
// groups and warp gw takes the kLeanRun-group run at gw * kLeanRun of each;
// the last, partial super-chunk is split evenly.  Groups in flight at the same
// time then lie within ~tw * kLeanRun groups of each other, so the x entries
// they gather stay in L2 even when x does not fit (27-pt 256^3: 134 MB of x;
// the contiguous split spreads the warps over all of it).
#ifndef ABFT_LEAN_RUN
#define ABFT_LEAN_RUN 16
#endif
constexpr int64_t kLeanRun = ABFT_LEAN_RUN;
struct LeanRuns {
  int64_t full, rem, tw, gw;
  // run r of this warp: [b, e); false when there is none
  __device__ __forceinline__ bool get(int64_t r, int64_t &b, int64_t &e) const {
    if (r < full) {
      b = (r * tw + gw) * kLeanRun;
      e = b + kLeanRun;
      return true;
    }
    if (r == full && rem > 0) {
      b = full * tw * kLeanRun + gw * rem / tw;
      e = full * tw * kLeanRun + (gw + 1) * rem / tw;
      return b < e;
    }
    return false;
  }
  __device__ __forceinline__ int64_t last() const {
    int64_t b, e;
    return (rem > 0 && get(full, b, e)) ? full : full - 1;
  }
};

// NST = 2: double buffering, each group's gathers issued right before its
// products.  NST = 3 (small stages): prefetch distance 2, and group g+1's x
// gathers are issued before group g's products, C pass and butterflies.
template <bool CHECK, bool INJECT, int CF, int NST, bool SHORT = false, bool COLG = false,
          bool RUNS = false>
__global__ void __launch_bounds__(kLeanWarps * 32,
                                  SHORT ? (CHECK ? ABFT_LEAN_MINB_SHORT : ABFT_LEAN_MINB_SHORT_PLAIN)
                                        : ABFT_LEAN_MINB)
    k_lean(const SpmvArgs a) {
  extern __shared__ __align__(128) unsigned char smem[];
  if (skip_call(a)) return;
  const StageCfg &c = a.sc;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint64_t *bars = reinterpret_cast<uint64_t *>(smem) + warp * NST;
  unsigned char *wst = smem + c.bar_bytes + (size_t)warp * NST * c.stage_bytes;
  if (lane == 0) {
#pragma unroll
    for (int t = 0; t < NST; ++t) mbar_init(bars + t, 1);
    fence_mbar_init();
  }
  if (CHECK && CF != CF_CSR && lane < NST)  // -0.0 sentinel below each stage's A values (padding of C)
    reinterpret_cast<double *>(wst + (size_t)lane * c.stage_bytes + c.off_av)[-1] = -0.0;
  __syncwarp();
  const uint64_t pol = policy_evict_first();
  const int64_t tw = (int64_t)gridDim.x * c.warps;
  const int64_t gw = (int64_t)blockIdx.x * c.warps + warp;
  int64_t g0, g1;
  const LeanRuns runs{a.ngroups / (tw * kLeanRun), a.ngroups % (tw * kLeanRun), tw, gw};
  if constexpr (RUNS) {
    int64_t e0, bl;
    if (!runs.get(0, g0, e0)) return;
    runs.get(runs.last(), bl, g1);
  } else {
    g0 = gw * a.ngroups / tw;
    g1 = (gw + 1) * a.ngroups / tw;
  }
  if (g0 >= g1) return;
  InjRange R{0, 0, 0, 0, 0, 0};
  if (INJECT) R = inj_range(a.inj, g0, g1, lane);
  Window<CF> win;
  win.load(a, g0, lane);
  // bounds of groups g (and g + 1 for NST = 3), carried from their prefetch
  int32_t sa, ea, sc, ec, cc, sa1 = 0, ea1 = 0, sc1 = 0, ec1 = 0, cc1 = 0;
  win.get(g0, sa, ea, sc, ec, cc);
  bool elig = win.ok(g0), elig1 = false;
  if (lane == 0 && elig) issue_stage<CHECK, CF, COLG>(a, g0, sa, ea, sc, ec, cc, wst, bars, pol);
  uint32_t phase = 0;  // bit s = parity of stage s's next completion
  Pre pc;
  if (NST == 3) {
    if (g0 + 1 < g1) {
      win.get(g0 + 1, sa1, ea1, sc1, ec1, cc1);
      elig1 = win.ok(g0 + 1);
      if (lane == 0 && elig1)
        issue_stage<CHECK, CF, COLG>(a, g0 + 1, sa1, ea1, sc1, ec1, cc1, wst + c.stage_bytes, bars + 1, pol);
    }
    if (elig) {
      mbar_wait(bars, 0);
      phase ^= 1u;
      pregather<CF, SHORT, COLG>(a, sa, ea, wst, lane, pc);
    }
  }
  int s = 0;  // stage of group g
  if constexpr (RUNS && NST == 2) {
    int64_t r = 0, g = g0, re = 0;
    {
      int64_t b0;
      runs.get(0, b0, re);
    }
    while (true) {
      const int s1 = s + 1 == NST ? 0 : s + 1;
      // the next group: g + 1 in this run, else the first of the next run
      int64_t gn = g + 1, rn = r, ren = re;
      if (gn >= re) {
        ++rn;
        if (!runs.get(rn, gn, ren)) gn = -1;
      }
      int32_t nsa = 0, nea = 0, nsc = 0, nec = 0, ncc = 0;
      bool nelig = false;
      if (gn >= 0) {  // prefetch it into the other stage
        if (gn < win.wb || gn + 1 > win.wb + 31) win.load(a, gn, lane);
        win.get(gn, nsa, nea, nsc, nec, ncc);
        nelig = win.ok(gn);
        if (lane == 0 && nelig)
          issue_stage<CHECK, CF, COLG>(a, gn, nsa, nea, nsc, nec, ncc,
                                       wst + (size_t)s1 * c.stage_bytes, bars + s1, pol);
      }
      if (elig) {
        unsigned char *st = wst + (size_t)s * c.stage_bytes;
        mbar_wait(bars + s, (phase >> s) & 1u);
        phase ^= 1u << s;
        pregather<CF, SHORT, COLG>(a, sa, ea, st, lane, pc);
        group32<CHECK, INJECT, CF, SHORT, COLG>(a, g, sa, ea, sc, ec, st, lane, R, pc);
        __syncwarp();
        fence_proxy_async_smem();  // generic accesses of this stage precede its next bulk write
      }
      if (gn < 0) break;
      sa = nsa; ea = nea; sc = nsc; ec = nec; cc = ncc;
      elig = nelig;
      g = gn;
      r = rn;
      re = ren;
      s = s1;
    }
  } else {
  for (int64_t g = g0; g < g1; ++g) {
    const int s1 = s + 1 == NST ? 0 : s + 1;
    if (NST == 2) {
      int32_t nsa = 0, nea = 0, nsc = 0, nec = 0, ncc = 0;
      bool nelig = false;
      if (g + 1 < g1) {  // prefetch g + 1 into the other stage
        if (g + 2 > win.wb + 31) win.load(a, g, lane);
        win.get(g + 1, nsa, nea, nsc, nec, ncc);
        nelig = win.ok(g + 1);
        if (lane == 0 && nelig)
          issue_stage<CHECK, CF, COLG>(a, g + 1, nsa, nea, nsc, nec, ncc, wst + (size_t)s1 * c.stage_bytes,
                                 bars + s1, pol);
      }
      if (elig) {
        unsigned char *st = wst + (size_t)s * c.stage_bytes;
        mbar_wait(bars + s, (phase >> s) & 1u);
        phase ^= 1u << s;
        pregather<CF, SHORT, COLG>(a, sa, ea, st, lane, pc);
        group32<CHECK, INJECT, CF, SHORT, COLG>(a, g, sa, ea, sc, ec, st, lane, R, pc);
        __syncwarp();
        fence_proxy_async_smem();  // generic accesses of this stage precede its next bulk write
      }
      sa = nsa; ea = nea; sc = nsc; ec = nec; cc = ncc;
      elig = nelig;
    } else {
      const int s2 = s1 + 1 == NST ? 0 : s1 + 1;
      int32_t nsa = 0, nea = 0, nsc = 0, nec = 0, ncc = 0;
      bool nelig = false;
      if (g + 2 < g1) {  // prefetch g + 2 into the stage group g - 1 used
        if (g + 3 > win.wb + 31) win.load(a, g + 2, lane);
        win.get(g + 2, nsa, nea, nsc, nec, ncc);
        nelig = win.ok(g + 2);
        if (lane == 0 && nelig)
          issue_stage<CHECK, CF, COLG>(a, g + 2, nsa, nea, nsc, nec, ncc, wst + (size_t)s2 * c.stage_bytes,
                                 bars + s2, pol);
      }
      Pre pn;
      if (elig1) {  // group g + 1: row bounds and x gathers in flight
        unsigned char *st1 = wst + (size_t)s1 * c.stage_bytes;
        mbar_wait(bars + s1, (phase >> s1) & 1u);
        phase ^= 1u << s1;
        pregather<CF, SHORT, COLG>(a, sa1, ea1, st1, lane, pn);
      }
      if (elig) {
        unsigned char *st = wst + (size_t)s * c.stage_bytes;
        group32<CHECK, INJECT, CF, SHORT, COLG>(a, g, sa, ea, sc, ec, st, lane, R, pc);
        __syncwarp();
        fence_proxy_async_smem();  // generic accesses of this stage precede its next bulk write
      }
      pc = pn;
      sa = sa1; ea = ea1; sc = sc1; ec = ec1; cc = cc1;
      elig = elig1;
      sa1 = nsa; ea1 = nea; sc1 = nsc; ec1 = nec; cc1 = ncc;
      elig1 = nelig;
    }
    s = s1;
  }
  }
}

constexpr int kBetaChunk = 1024;  // groups per aligned beta partial (k_finish, k_bpart)
constexpr int kFewCand = 32;     // k_finish: up to this many candidates, CTA 0 alone confirms + corrects

// PW over n doubles at p by one CTA of 256 threads: thread t owns an aligned
// run of m = 2^k values, reduced 32 at a time in registers (32 loads in
// flight), runs by a shared-memory tree.  Called by all threads.
__device__ __forceinline__ double cta_pw_array(const double *p, int64_t n, double *s_red) {
  constexpr int T = 256;
  int64_t m = 1;
  while (m * T < n) m <<= 1;
  const int64_t b = (int64_t)threadIdx.x * m;
  double acc = kAbsent;
  if (m <= 32) {
    double v[32];
#pragma unroll
    for (int q = 0; q < 32; ++q) v[q] = (q < m && b + q < n) ? __ldcg(p + b + q) : kAbsent;
    acc = tree<32>(v);
  } else {
    PwSeq sub;  // runs of 32 (aligned nodes), combined by the binary counter
    for (int64_t o = 0; o < m && b + o < n; o += 32) {
      double v[32];
#pragma unroll
      for (int q = 0; q < 32; ++q) v[q] = (b + o + q < n) ? __ldcg(p + b + o + q) : kAbsent;
      sub.push(tree<32>(v));
    }
    acc = sub.finish();
  }
  __syncthreads();
  s_red[threadIdx.x] = acc;
  __syncthreads();
  for (int st = 1; st < T; st <<= 1) {
    if ((threadIdx.x & (2 * st - 1)) == 0)
      s_red[threadIdx.x] = dadd(s_red[threadIdx.x], s_red[threadIdx.x + st]);
    __syncthreads();
  }
  const double r = s_red[0];
  __syncthreads();
  return r;
}

// Local ||x||^2 partial of this handle's rows (distributed use): aligned
// 1024-group chunks by many CTAs, then the chunk sums by one CTA.
__global__ void __launch_bounds__(256) k_bpart(const SpmvArgs a) {
  __shared__ double s_red[256];
  const int64_t nch = (a.ngroups + kBetaChunk - 1) / kBetaChunk;
  for (int64_t c = blockIdx.x; c < nch; c += gridDim.x) {
    const double v = cta_pw_array(a.gsum + c * kBetaChunk,
                                  min64(kBetaChunk, a.ngroups - c * kBetaChunk), s_red);
    if (threadIdx.x == 0) a.bpart[c] = v;
  }
}
__global__ void __launch_bounds__(256) k_bpart_top(const SpmvArgs a, double *out) {
  __shared__ double s_red[256];
  const int64_t nch = (a.ngroups + kBetaChunk - 1) / kBetaChunk;
  const double v = cta_pw_array(a.bpart, nch, s_red);
  if (threadIdx.x == 0) *out = v;
}
// beta = sqrt(PW over per-rank partials, in rank order) -> *out (x_norm).
__global__ void __launch_bounds__(256) k_norm_parts(const double *parts, int64_t nparts,
                                                    double *out) {
  __shared__ double s_red[256];
  const double v = cta_pw_array(parts, nparts, s_red);
  if (threadIdx.x == 0) *out = __dsqrt_rn(v);
}

// beta on demand (abft_beta): PW over the group subtrees, one CTA.
__global__ void __launch_bounds__(256) k_beta(const SpmvArgs a) {
  __shared__ double s_red[256];
  if (*(volatile int32_t *)a.beta_valid) return;
  const double b2 = cta_pw_array(a.gsum, a.ngroups, s_red);
  if (threadIdx.x == 0) {
    *a.beta = __dsqrt_rn(b2);
    *a.beta_valid = 1;
  }
}

// ---------------------------------------------------------------------------
// Row blocks larger than a warp (b_s = 64 .. 1024; kernels_bigblock.cuh).
// ---------------------------------------------------------------------------
// y rows of group g (round `round` of the fault model), lane per row; rows
// longer than 32 entries by the warp.  Returns this lane's y (absent past n).
template <bool INJECT>
__device__ __forceinline__ double group_rows(const SpmvArgs &a, int64_t g, int round, int lane) {
  const int64_t r0 = g * 32, i = r0 + lane;
  const bool valid = i < a.n;
  const GlobalSrc As{a.va, a.ci};
  int32_t rs = 0, len = 0;
  if (valid) {
    rs = __ldg(a.rp + i);
    len = __ldg(a.rp + i + 1) - rs;
  }
  const int small = len <= 32 ? len : 0;
  const int maxs = warp_max_i(small);
  double yv = 0.0;
  if (valid && len <= 32 && maxs > 0) yv = lane_dot_any(As, rs, small, maxs, a.x);
  unsigned longm = __ballot_sync(kFull, valid && len > 32);
  while (longm) {
    const int j = __ffs(longm) - 1;
    longm &= longm - 1;
    const double t = warp_dot(As, __shfl_sync(kFull, rs, j), __shfl_sync(kFull, len, j), a.x, lane);
    if (lane == j) yv = t;
  }
  if (len == 0) yv = 0.0;
  if (INJECT) {
    const uint64_t m = group_y_mask(a.inj, round, r0, i, lane);
    if (valid) yv = apply_mask(yv, m);
  }
  if (valid) a.y[i] = yv;
  return valid ? yv : kAbsent;
}

// Block k (b_s > 32) of round `round`: y rows, t1, t2, and (round 0) the
// groups' x^2 subtrees; returns s_k = t1 - t2 on every lane, *gs_out the
// block's x^2 node (an aligned node of beta^2's tree).
template <bool CHECK, bool INJECT>
__device__ __forceinline__ double big_block(const SpmvArgs &a, int64_t k, int round, int lane,
                                           double *gs_out) {
  const int ngr = a.bs >> 5;
  const int64_t g0 = k * ngr;
  PwSeq t2s, gss;
  for (int sub = 0; sub < ngr; ++sub) {
    const int64_t g = g0 + sub;
    if (g * 32 >= a.n) break;  // trailing absent subtrees
    const double yv = group_rows<INJECT>(a, g, round, lane);
    if (CHECK) {
      t2s.push(bfly32(yv));
      if (round == 0) {
        const int64_t i = g * 32 + lane;
        const double xv = i < a.n ? __ldg(a.xr + i) : 0.0;
        const double gs = bfly32(i < a.n ? dmul(xv, xv) : kAbsent);
        if (lane == 0) a.gsum[g] = gs;
        gss.push(gs);
      }
    }
  }
  if (!CHECK) return 0.0;
  double t2 = t2s.finish();
  const int32_t cb = __ldg(a.crp + k), ce = __ldg(a.crp + k + 1);
  const GlobalSrc Cs{a.cval, a.ccol};
  double t1 = warp_dot(Cs, cb, ce - cb, a.x, lane);
  if (INJECT && lane == 0) {
    t1 = apply_mask(t1, fault_mask(a.inj, round, 1, k, 2 * (int64_t)(ce - cb)));
    t2 = apply_mask(t2, fault_mask(a.inj, round, 2, k, min64(a.bs, a.n - k * a.bs)));
  }
  if (round == 0 && lane == 0 && a.dbg_t1) {
    a.dbg_t1[k] = t1;
    a.dbg_t2[k] = t2;
  }
  if (gs_out) *gs_out = gss.finish();
  return dsub(t1, t2);
}

// Software grid barrier (all CTAs co-resident: grid <= SM count, one CTA per
// SM, checked against the occupancy at encode).  bar[0] = arrivals, bar[1] =
// generation, bar[2] = error word.  Co-residency is not guaranteed when other
// work holds SMs (another process, MPS limits, kernels on other streams), so
// the wait is bounded: after ~2^24 polls (about a second) the barrier sets
// bar[2] = 1 and every CTA returns false; a set error word makes every later
// barrier fail at once (the handle is poisoned until abft_health clears it),
// so a co-residency failure is reported instead of hanging the device.
__device__ __forceinline__ bool grid_sync(unsigned *bar) {
  __shared__ int s_ok;
  __syncthreads();
  if (threadIdx.x == 0) {
    int ok = *(volatile unsigned *)(bar + 2) == 0u;
    if (ok) {
      const unsigned gen = *(volatile unsigned *)(bar + 1);
      __threadfence();
      if (atomicAdd(bar, 1u) == gridDim.x - 1) {
        *(volatile unsigned *)bar = 0u;
        __threadfence();
        atomicAdd(bar + 1, 1u);
      } else {
        for (unsigned it = 0; *(volatile unsigned *)(bar + 1) == gen; ++it) {
          if (it >= (1u << 24) || *(volatile unsigned *)(bar + 2) != 0u) {
            atomicExch(bar + 2, 1u);
            ok = 0;
            break;
          }
          __nanosleep(64);
        }
      }
      __threadfence();
    }
    s_ok = ok;
  }
  __syncthreads();
  return s_ok != 0;
}

// Step 5 for one flagged block k in round `round`: recompute
// its rows and t1 / t2, re-check against tau_k = K_k beta.  Returns (warp-
// uniform) whether the block still fails.  [olo, ohi): the hub rows of the
// block's group whose chunk sums the CTA precomputed (solo hub rounds), or
// empty.  A block's rounds depend on no other block: the kernel runs each
// flagged block through all its rounds without grid barriers.
template <bool INJECT>
__device__ __forceinline__ bool fin_block(const SpmvArgs &a, int64_t k, int round, int lane,
                                          double beta, int olo, int ohi) {
  const int64_t n = a.n;
  if (a.bs > 32) {  // big blocks: recompute the block's groups, re-verify
    const double sv = big_block<true, INJECT>(a, k, round, lane, nullptr);
    return __shfl_sync(kFull, !(fabs(sv) <= dmul(__ldg(a.K + k), beta)), 0);
  }
  const LdgSrc As{a.va, a.ci}, Cs{a.cval, a.ccol};
  const int32_t cb = __ldg(a.crp + k), ce = __ldg(a.crp + k + 1);  // issued early
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
    if (valid) yv = lane_dot_any(As, rs, len, maxlen, a.x);
  } else {
    for (int j = 0; j < a.bs; ++j) {
      const int32_t rb = __shfl_sync(kFull, rs, j);
      const int rl = __shfl_sync(kFull, len, j);
      if ((k << a.log2bs) + j >= n) break;
      double t;
      const int e = rl > kHubLen ? own_find(a, olo, ohi, (int)(((k << a.log2bs) + j) & 31)) : -1;
      if (e >= 0)
        t = hub_sum(a, __ldg(a.own_first + e), __ldg(a.own_n + e));
      else
        t = warp_dot(As, rb, rl, a.x, lane);
      if (lane == j) yv = t;
    }
  }
  if (len == 0) yv = 0.0;
  if (INJECT) {
    const uint64_t m = group_y_mask(a.inj, round, k << a.log2bs, i, lane);
    if (valid) yv = apply_mask(yv, m);
  }
  if (valid) a.y[i] = yv;
  if (a.pq) {  // b_s = 32: the block is the group
    const double t = bfly32(valid ? dmul(__ldg(a.xr + i), yv) : kAbsent);
    if (lane == 0) a.pq[k] = t;
  }
  double t2 = bfly32(valid ? yv : kAbsent);
  const int ec = ce - cb > kHubLen
                     ? own_find(a, olo, ohi, 32 + (int)(k & ((32 >> a.log2bs) - 1))) : -1;
  double t1 = ec >= 0 ? hub_sum(a, __ldg(a.own_first + ec), __ldg(a.own_n + ec))
                      : warp_dot(Cs, cb, ce - cb, a.x, lane);
  bool fail = false;
  if (lane == 0) {
    if (INJECT) {
      t1 = apply_mask(t1, fault_mask(a.inj, round, 1, k, 2 * (int64_t)(ce - cb)));
      t2 = apply_mask(t2, fault_mask(a.inj, round, 2, k, min64(a.bs, n - (k << a.log2bs))));
    }
    fail = !(fabs(dsub(t1, t2)) <= dmul(__ldg(a.K + k), beta));
  }
  return __shfl_sync(kFull, fail, 0);
}

// Rounds 1..rounds of one block flagged in round 0: a round's failure puts
// the block on that round's list and runs the next round.
template <bool INJECT>
__device__ __forceinline__ void block_rounds(const SpmvArgs &a, int64_t k, int rounds, int lane,
                                             double beta) {
  for (int round = 1; round <= rounds; ++round) {
    if (!fin_block<INJECT>(a, k, round, lane, beta, 0, 0)) return;
    if (lane == 0) a.flags[(int64_t)round * a.nb + atomicAdd(a.n_flags + round, 1)] = (int32_t)k;
  }
}

// Steps 4-5 after the fused pass, one launch (programmatic dependent launch:
// its launch latency overlaps the fused kernels; griddepcontrol.wait orders
// it after them).  One CTA per SM, software grid barrier.
//  * CONFIRM: if the fused pass left candidates, beta = sqrt(PW(gsum))
//    (aligned 1024-group partials written by all CTAs; after one grid
//    barrier every CTA reduces them -- the same bits everywhere), and each
//    candidate is flagged iff NOT(|s_k| <= K_k beta).  No candidates:
//    flags are empty and the kernel returns at once.
//  * rounds r = 1..R (step 5): each block flagged in round 0 is
//    recomputed (rows, t1, t2) and re-checked by one warp until it passes or
//    R rounds are spent; round r's list holds the blocks failing round r.
//    No barrier between rounds (a block's rounds depend on no other block).
//    Matrices with hub rows and few candidates: CTA 0 alone runs the rounds
//    round by round, each round's hub chunk sums spread over its warps.
// kernels_pcgfin.cuh: the p.q completion k_finish runs for abft_pcg
__device__ void pcg_fin_dot(const SpmvArgs &a, double *s_red, bool solo);

template <bool INJECT, bool CONFIRM>
__global__ void __launch_bounds__(256) k_finish(const SpmvArgs a, int rounds) {
  __shared__ double s_red[256];
  pdl_trigger();
  pdl_wait();
  if (skip_call(a)) return;
  const int lane = threadIdx.x & 31;
  const bool hub_m = a.n_own > 0 && a.bs <= 32;
  bool hub_solo = false;
  double beta;
  int32_t nitems;
  const int32_t *items;
  if (CONFIRM) {
    const int nc = __ldcg(a.n_cand);
    if (nc == 0) {
      if (blockIdx.x == 0 && threadIdx.x == 0) {
        for (int r = 0; r <= a.max_rounds; ++r) a.n_flags[r] = 0;
        if (a.x_norm) *a.beta = __ldcg(a.x_norm);
        *a.beta_valid = a.x_norm ? 1 : 0;
      }
      if (a.pcga) pcg_fin_dot(a, s_red, false);  // every CTA takes part (no barrier)
      return;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0)
      for (int r = 0; r <= a.max_rounds; ++r) a.n_flags[r] = 0;
    hub_solo = hub_m && nc <= kFewCand && rounds > 0;
    const int64_t nch = (a.ngroups + kBetaChunk - 1) / kBetaChunk;
    if (!a.x_norm)
      for (int64_t c = blockIdx.x; c < nch; c += gridDim.x) {
        const double v = cta_pw_array(a.gsum + c * kBetaChunk,
                                      min64(kBetaChunk, a.ngroups - c * kBetaChunk), s_red);
        if (threadIdx.x == 0) a.bpart[c] = v;
      }
    // n_flags zeroed, partials written, n_cand read by every CTA
    if (!grid_sync(a.gbar)) return;
    if (hub_solo && blockIdx.x != 0) return;
    beta = a.x_norm ? __ldcg(a.x_norm) : __dsqrt_rn(cta_pw_array(a.bpart, nch, s_red));  // R10
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      *a.beta = beta;
      *a.beta_valid = 1;
      *a.n_cand = 0;
    }
    // one warp per candidate: confirm, then (not hub_solo) its rounds
    const int64_t gw = hub_solo ? (int64_t)(threadIdx.x >> 5)
                                : ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = hub_solo ? (int64_t)(blockDim.x >> 5) : ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t q = gw; q < nc; q += nw) {
      const int32_t kk = __ldcg(a.cand + q);
      const double sv = __ldcg(a.cand_s + q);
      if (fabs(sv) <= dmul(__ldg(a.K + kk), beta)) continue;  // tau_k = K_k * beta
      if (lane == 0) a.flags[atomicAdd(a.n_flags, 1)] = kk;
      if (!hub_solo) block_rounds<INJECT>(a, kk, rounds, lane, beta);
    }
    if (!hub_solo) {
      // the corrections rewrote the p.q partials of their groups
      if (a.pcga && grid_sync(a.gbar)) pcg_fin_dot(a, s_red, false);
      return;
    }
    __syncthreads();  // round 0's list complete
    nitems = __ldcg(a.n_flags);
    items = a.flags;
  } else {
    beta = __ldcg(a.beta);
    nitems = __ldcg(a.n_flags);
    items = a.flags;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t q = gw; q < nitems; q += nw)
      block_rounds<INJECT>(a, __ldcg(items + q), rounds, lane, beta);
    return;
  }
  // hub_solo: CTA 0, round by round
  const int64_t gw = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const LdgSrc As{a.va, a.ci}, Cs{a.cval, a.ccol};
  for (int round = 1; round <= rounds; ++round) {
    const int32_t nprev = round == 1 ? nitems : __ldcg(a.n_flags + round - 1);
    if (nprev == 0) break;
    const int32_t *prev = a.flags + (int64_t)(round - 1) * a.nb;
    int32_t *next = a.flags + (int64_t)round * a.nb;
    // the flagged blocks' hub chunk sums, spread over the CTA's warps (a hub
    // row of 40k entries is 40 chunks, not one warp's serial chain), then the
    // blocks below combine them (hub_sum: aligned subtrees == PW)
    {
      int item = 0;  // running chunk index over the flagged blocks (uniform)
      const int per_g = 32 >> a.log2bs;
      for (int q = 0; q < nprev; ++q) {
        const int64_t k = __ldcg(prev + q);
        const int64_t g = (k << a.log2bs) >> 5;
        if (!(__ldg(a.lean_ok + g) & 2)) continue;
        const int kb = (int)(k & (per_g - 1));
        int lo, hi;
        own_range(a, g, lo, hi);
        for (int e = lo; e < hi; ++e) {
          const int32_t key = __ldg(a.own_key + e);
          const bool crow = (key & 32) != 0;
          if ((crow ? (key & 31) : ((key & 31) >> a.log2bs)) != kb) continue;  // another block
          const int32_t f = __ldg(a.own_first + e), cnt = __ldg(a.own_n + e);
          for (int t = 0; t < cnt; ++t, ++item) {
            if (item % nw != gw) continue;
            const uint32_t L = __ldg(a.hub_len + f + t);
            const int64_t b = __ldg(a.hub_beg + f + t);
            const double r = (L >> 31) ? warp_dot(Cs, b, (int)(L & 0x7fffffffu), a.x, lane)
                                       : warp_dot(As, b, (int)(L & 0x7fffffffu), a.x, lane);
            if (lane == 0) a.hub_part[f + t] = r;
          }
        }
      }
      __syncthreads();
    }
    for (int64_t q = gw; q < nprev; q += nw) {
      const int64_t k = __ldcg(prev + q);
      int olo = 0, ohi = 0;
      if (__ldg(a.lean_ok + ((k << a.log2bs) >> 5)) & 2) own_range(a, (k << a.log2bs) >> 5, olo, ohi);
      if (fin_block<INJECT>(a, k, round, lane, beta, olo, ohi) && lane == 0)
        next[atomicAdd(a.n_flags + round, 1)] = (int32_t)k;
    }
    __syncthreads();
  }
  if (a.pcga) pcg_fin_dot(a, s_red, true);  // CTA 0 alone (the others left after the barrier)
}

}  // namespace abft
