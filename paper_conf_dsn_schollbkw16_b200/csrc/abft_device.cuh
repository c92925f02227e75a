// abft_device.cuh -- device-side building blocks for the sm_100a kernels.
//
// Numerics (R1/R2): every product and sum is an explicit
// round-to-nearest binary64 op (__dmul_rn / __dadd_rn; no FMA contraction,
// the TUs are also built with -fmad=false), and every sum follows the
// canonical pairwise tree PW: the list padded to a power of two with ABSENT
// slots.  On the device an absent slot is -0.0, the exact additive identity
// of IEEE round-to-nearest (x + -0 == x for every x, including +0 and -0),
// so a fixed-shape tree with -0.0 padding IS the absent-padded tree.  PW is
// padding-independent, so any aligned power-of-two split (lane tree, warp
// butterfly, CTA tree, grid tree) reproduces the same bits.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace abft {

constexpr double kAbsent = -0.0;
constexpr unsigned kFull = 0xffffffffu;

__device__ __forceinline__ int64_t min64(int64_t a, int64_t b) { return a < b ? a : b; }
__device__ __forceinline__ double dmul(double a, double b) { return __dmul_rn(a, b); }
__device__ __forceinline__ double dadd(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ double dsub(double a, double b) { return __dsub_rn(a, b); }

// Ascending-offset xor butterfly over aligned groups of `width` lanes
// (width a power of two <= 32): level m pairs lanes l and l^m, i.e. the
// adjacent pairs of PW; fl(a+b) == fl(b+a), so both lanes agree.
__device__ __forceinline__ double bfly(double v, int width) {
#pragma unroll
  for (int m = 1; m < 32; m <<= 1) {
    if (m >= width) break;
    v = dadd(v, __shfl_xor_sync(kFull, v, m));
  }
  return v;
}
__device__ __forceinline__ double bfly32(double v) {
#pragma unroll
  for (int m = 1; m < 32; m <<= 1) v = dadd(v, __shfl_xor_sync(kFull, v, m));
  return v;
}

__device__ __forceinline__ int warp_max_i(int v) {
#pragma unroll
  for (int m = 16; m > 0; m >>= 1) v = max(v, __shfl_xor_sync(kFull, v, m));
  return v;
}
__device__ __forceinline__ int warp_min_i(int v) {
#pragma unroll
  for (int m = 16; m > 0; m >>= 1) v = min(v, __shfl_xor_sync(kFull, v, m));
  return v;
}

// In-register PW tree over P leaves (P a power of two).
template <int P>
__device__ __forceinline__ double tree(double (&v)[P]) {
#pragma unroll
  for (int s = 1; s < P; s <<= 1)
#pragma unroll
    for (int j = 0; j + s < P; j += 2 * s) v[j] = dadd(v[j], v[j + s]);
  return v[0];
}

// PW over a sequential stream with a binary counter (merge pairs of equal
// size as they complete; merge the stack top-down at the end): identical to
// the absent-padded tree.  Used on tail paths only (stack lives in local mem).
struct PwSeq {
  double stk[40];
  int top = 0;
  int64_t cnt = 0;
  __device__ __forceinline__ void push(double v) {
    int64_t c = cnt++;
    while (c & 1) {
      v = dadd(stk[--top], v);
      c >>= 1;
    }
    stk[top++] = v;
  }
  // Returns kAbsent for an empty stream.
  __device__ __forceinline__ double finish() const {
    if (top == 0) return kAbsent;
    double r = stk[top - 1];
    for (int t = top - 2; t >= 0; --t) r = dadd(stk[t], r);
    return r;
  }
};

// Read-only streaming loads (A and C are read once per call: an evict-first
// L2 policy keeps x resident); x gathers go through the read-only path.
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t pol;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ double ld_stream(const double *p) {
  double v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;"
               : "=d"(v) : "l"(p), "l"(policy_evict_first()));
  return v;
}
__device__ __forceinline__ int ld_stream(const int *p) {
  int v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;"
               : "=r"(v) : "l"(p), "l"(policy_evict_first()));
  return v;
}
__device__ __forceinline__ double ld_x(const double *p) { return __ldg(p); }

// ---------------------------------------------------------------------------
// Fault injection (R12/R13).  Philox4x32-10
// implemented independently of the oracle.
// ---------------------------------------------------------------------------
struct InjDev {
  int mode;          // 0 none, 1 list, 2 rate
  uint32_t key0, key1, call;
  double lambda;
  uint32_t targets;
  int32_t n_list;
  const uint64_t *keys;   // sorted (round << 58) | (target << 56) | index
  const uint64_t *masks;
};

__device__ __forceinline__ void philox10(uint32_t c[4], uint32_t k0, uint32_t k1) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    uint32_t hi0 = __umulhi(0xD2511F53u, c[0]), lo0 = 0xD2511F53u * c[0];
    uint32_t hi1 = __umulhi(0xCD9E8D57u, c[2]), lo1 = 0xCD9E8D57u * c[2];
    uint32_t n0 = hi1 ^ c[1] ^ k0, n2 = hi0 ^ c[3] ^ k1;
    c[0] = n0;
    c[1] = lo1;
    c[2] = n2;
    c[3] = lo0;
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
}

// Single translation unit (abft.cu): the table is defined here.
__constant__ uint64_t c_burst_T[65];

__device__ __forceinline__ uint64_t list_key(int round, int target, int64_t index) {
  return ((uint64_t)round << 58) | ((uint64_t)target << 56) | (uint64_t)index;
}

__device__ __noinline__ uint64_t fault_mask(const InjDev &inj, int round, int target,
                                            int64_t index, int64_t ops) {
  if (inj.mode == 1) {
    uint64_t key = list_key(round, target, index);
    int lo = 0, hi = inj.n_list;
    while (lo < hi) {
      int mid = (lo + hi) >> 1;
      if (inj.keys[mid] < key) lo = mid + 1; else hi = mid;
    }
    uint64_t m = 0;
    for (int e = lo; e < inj.n_list && inj.keys[e] == key; ++e) m ^= inj.masks[e];
    return m;
  }
  if (inj.mode != 2 || !(inj.targets & (1u << target))) return 0;
  double p = dmul(inj.lambda, (double)ops);
  uint64_t thr = p >= 1.0 ? (1ull << 32) : __double2ull_rz(dmul(p, 4294967296.0));
  uint32_t c[4] = {(uint32_t)(uint64_t)index, (uint32_t)((uint64_t)index >> 32), inj.call,
                   ((uint32_t)round << 8) | (uint32_t)target};
  philox10(c, inj.key0, inj.key1);
  if ((uint64_t)c[0] >= thr) return 0;
  int start = (int)(c[1] & 63u);
  int len = 1;
  while (len < 64 && (uint64_t)c[2] >= c_burst_T[len]) ++len;
  int hi = min(start + len - 1, 63);
  uint64_t span = (hi - start + 1) == 64 ? ~0ull : ((1ull << (hi - start + 1)) - 1ull);
  return span << start;
}

__device__ __forceinline__ double apply_mask(double v, uint64_t m) {
  return __longlong_as_double((long long)((uint64_t)__double_as_longlong(v) ^ m));
}

}  // namespace abft
