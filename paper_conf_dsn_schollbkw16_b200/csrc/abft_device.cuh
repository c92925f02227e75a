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

// one REDUX instruction each (sm_80+), not a 5-step shuffle chain
__device__ __forceinline__ int warp_max_i(int v) { return __reduce_max_sync(kFull, v); }
__device__ __forceinline__ int warp_min_i(int v) { return __reduce_min_sync(kFull, v); }

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
  int mode;          // 0 none, 1 list
  int32_t n_list;    // list length (host-known), or
  const int32_t *n_list_dev;  // device-resident list length (rate-mode plans)
  int32_t cap;       // capacity of a device-generated list
  const uint64_t *keys;   // sorted (round << 58) | (target << 56) | index
  const uint64_t *masks;
  // bit g set <=> some round-0 entry touches 32-row group g (a y row of it,
  // or the t1 / t2 of a block starting in it); null = search every group
  const uint32_t *gbits;
  // [3][ngroups] first list position of a round-0 entry of (target, group);
  // read only for groups whose gbits bit is set (-1: no entry of that target)
  const int32_t *gstart;
  int64_t ngroups;
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

__device__ __forceinline__ int list_len(const InjDev &inj) {
  return inj.n_list_dev ? min(*inj.n_list_dev, inj.cap) : inj.n_list;
}

// Whether group g may hold a round-0 fault (the kernels skip the list
// search of every other group).
__device__ __forceinline__ bool inj_group_hit(const InjDev &inj, int64_t g) {
  return !inj.gbits || ((__ldg(inj.gbits + (g >> 5)) >> (g & 31)) & 1u);
}

// Build the group bitmap of a device list (round-0 entries only; the list
// is sorted, so the round-0 entries come first).
__device__ __forceinline__ int64_t inj_entry_group(uint64_t k, int32_t bs, int64_t ngroups,
                                                    int &t) {
  t = (int)((k >> 56) & 3u);
  const int64_t idx = (int64_t)(k & ((1ull << 56) - 1));
  if ((k >> 58) != 0) return ngroups;  // rounds >= 1: not the fused pass's
  return t == 0 ? min(idx >> 5, ngroups) : idx < ((int64_t)1 << 40) ? min((idx * bs) >> 5, ngroups) : ngroups;
}

__global__ void k_inj_bits(const InjDev inj, int32_t bs, int64_t ngroups, uint32_t *gbits,
                           int32_t *gstart) {
  const int len = list_len(inj);
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < len; e += gridDim.x * blockDim.x) {
    int t;
    const int64_t g = inj_entry_group(inj.keys[e], bs, ngroups, t);
    if (g >= ngroups) continue;
    int tp = -1;
    const int64_t gp = e > 0 ? inj_entry_group(inj.keys[e - 1], bs, ngroups, tp) : -1;
    if (gp != g || tp != t) {  // first entry of (target, group): sorted list
      gstart[(int64_t)t * ngroups + g] = e;
      atomicOr(gbits + (g >> 5), 1u << (g & 31));
    }
  }
}

// The masks of a group with round-0 entries (gbits set): y row i (every
// lane), t1 / t2 of block k (the stream kernel: bs = 32, k = g).  A few loads from the group's
// first entry instead of binary searches; not inlined (rare path).
struct InjMasks {
  uint64_t y, t1, t2;
};
__device__ __noinline__ InjMasks inj_group_masks(const uint64_t *keys, const uint64_t *masks,
                                                 const int32_t *n_dev, int n_list, int cap,
                                                 const int32_t *gstart, int64_t ngroups,
                                                 int64_t g, int64_t i, int64_t k) {
  // a start left by an earlier plan (this plan has no entry of that target
  // in g) points at an entry outside the range: the scans stop at once
  const int len = n_dev ? min(*n_dev, cap) : n_list;
  InjMasks m{0, 0, 0};
  const uint64_t y0 = list_key(0, 0, g * 32), y1 = list_key(0, 0, g * 32 + 32);
  for (int e = max(__ldg(gstart + g), 0); e < len; ++e) {
    const uint64_t key = __ldg(keys + e);
    if (key < y0 || key >= y1) break;
    if (key == list_key(0, 0, i)) m.y ^= __ldg(masks + e);
  }
  for (int e = max(__ldg(gstart + ngroups + g), 0); e < len && __ldg(keys + e) == list_key(0, 1, k); ++e)
    m.t1 ^= __ldg(masks + e);
  for (int e = max(__ldg(gstart + 2 * ngroups + g), 0); e < len && __ldg(keys + e) == list_key(0, 2, k); ++e)
    m.t2 ^= __ldg(masks + e);
  return m;
}
__device__ __forceinline__ InjMasks inj_masks(const InjDev &inj, int64_t g, int64_t i) {
  return inj_group_masks(inj.keys, inj.masks, inj.n_list_dev, inj.n_list, inj.cap, inj.gstart,
                         inj.ngroups, g, i, g);
}

// First list position with key >= k.
__device__ __forceinline__ int list_lower(const InjDev &inj, int len, uint64_t k) {
  int lo = 0, hi = len;
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (__ldg(inj.keys + mid) < k) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// XOR of the masks of every entry with key k (a search of its own; not
// inlined, so the rare faulty groups do not cost the others registers).
// (Arguments by value: a reference into the kernel's parameter block would
// force a stack copy of the whole argument struct.)
__device__ __noinline__ uint64_t list_mask_of_v(const uint64_t *keys, const uint64_t *masks,
                                                const int32_t *n_dev, int n_list, int cap,
                                                uint64_t k) {
  const int len = n_dev ? min(*n_dev, cap) : n_list;
  int lo = 0, hi = len;
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (__ldg(keys + mid) < k) lo = mid + 1; else hi = mid;
  }
  uint64_t m = 0;
  for (int e = lo; e < len && __ldg(keys + e) == k; ++e) m ^= __ldg(masks + e);
  return m;
}
__device__ __forceinline__ uint64_t list_mask_of(const InjDev &inj, uint64_t k) {
  return list_mask_of_v(inj.keys, inj.masks, inj.n_list_dev, inj.n_list, inj.cap, k);
}

// XOR of the masks of entries [lo, hi) whose key equals k.
__device__ __forceinline__ uint64_t list_mask_in(const InjDev &inj, int lo, int hi, uint64_t k) {
  uint64_t m = 0;
  for (int e = lo; e < hi; ++e)
    if (__ldg(inj.keys + e) == k) m ^= __ldg(inj.masks + e);
  return m;
}

// The XOR mask for one produced value (R13): the explicit fault list, or the
// list a rate-mode spec was expanded to before the launch.
__device__ __noinline__ uint64_t fault_mask(const InjDev &inj, int round, int target,
                                            int64_t index, int64_t ops) {
  (void)ops;
  if (inj.mode != 1) return 0;
  const int len = list_len(inj);
  if (len == 0) return 0;
  const uint64_t key = list_key(round, target, index);
  const int lo = list_lower(inj, len, key);
  uint64_t m = 0;
  for (int e = lo; e < len && __ldg(inj.keys + e) == key; ++e) m ^= __ldg(inj.masks + e);
  return m;
}

// Per-warp y-fault masks for rows r0 .. r0+31: one pair of binary searches
// for the group (lane 0), then each lane scans the (usually empty) range.
__device__ __forceinline__ uint64_t group_y_mask(const InjDev &inj, int round, int64_t r0,
                                                 int64_t i, int lane) {
  int lo = 0, hi = 0;
  if (lane == 0) {
    const int len = list_len(inj);
    if (len > 0) {
      lo = list_lower(inj, len, list_key(round, 0, r0));
      hi = list_lower(inj, len, list_key(round, 0, r0 + 32));
    }
  }
  lo = __shfl_sync(0xffffffffu, lo, 0);
  hi = __shfl_sync(0xffffffffu, hi, 0);
  return lo < hi ? list_mask_in(inj, lo, hi, list_key(round, 0, i)) : 0ull;
}

// ---------------------------------------------------------------------------
// Rate mode (R13): a Poisson process over the call's
// arithmetic operations, generated as an explicit sorted fault list.
// Op space per round: y_i owns 2 len_i ops, then t1_k 2 n_k, then t2_k
// rows-in-block (y only when unprotected).  Chunks of ch ops; chunk c holds
// K ~ Poisson(lambda len_c) events (inversion of a host-computed CDF table,
// Philox word 0 of {c, 0, call, r<<8 | 0x80}); event e (1..K) takes Philox
// {c, e, call, r<<8 | 0x40}: offset floor(w0 len_c / 2^32), burst from w1, w2.
// One thread per (round, chunk); pass 1 counts the kept events, pass 2
// writes them (ordered by offset) at the scanned positions.
// ---------------------------------------------------------------------------
constexpr int kRateTab = 32;  // table length cap: at most 31 events per chunk

struct RatePlanArgs {
  int64_t n, nb, ch, nch, y_ops, t1_ops, ops;
  int32_t bs, rounds;
  uint32_t key0, key1, call, targets;
  const int32_t *rp;
  const int32_t *crp;
  const uint64_t *tab;  // [2][kRateTab]: full chunks, last chunk
  int32_t nf, nl;
  int32_t *counts;      // [(rounds+1) * nch]
  const int32_t *offs;  // exclusive scan of counts
  uint64_t *keys, *masks;
  int64_t cap;          // capacity of keys/masks
  // op -> row lookup: bkt[b] = the row (block) holding op b << kOpBktShift
  // (largest i with 2 rp[i] <= op); the search then spans bkt[b]..bkt[b+1]
  const int32_t *ybkt, *cbkt;
};

constexpr int kOpBktShift = 8;  // ops per bucket of the op -> row lookup (256)

// bkt[b] = largest i in [0, n] with 2 rp[i] <= b << kOpBktShift, b in [0, nbkt)
__global__ void k_op_buckets(const int32_t *__restrict__ rp, int64_t n, int64_t nbkt,
                             int32_t *bkt) {
  const int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= nbkt) return;
  const int64_t p = b << kOpBktShift;
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    const int64_t mid = lo + (hi - lo + 1) / 2;
    if (2 * (int64_t)rp[mid] <= p) lo = mid; else hi = mid - 1;
  }
  bkt[b] = (int32_t)lo;
}

// largest i in [bkt[p >> s], bkt[(p >> s) + 1]] with 2 rp[i] <= p
__device__ __forceinline__ int64_t op_row(const int32_t *rp, const int32_t *bkt, int64_t p) {
  const int64_t b = p >> kOpBktShift;
  int64_t lo = __ldg(bkt + b), hi = __ldg(bkt + b + 1);
  while (lo < hi) {
    const int64_t mid = lo + (hi - lo + 1) / 2;
    if (2 * (int64_t)__ldg(rp + mid) <= p) lo = mid; else hi = mid - 1;
  }
  return lo;
}

template <bool WRITE>
__global__ void k_rate_plan(const RatePlanArgs a) {
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (tid >= (int64_t)(a.rounds + 1) * a.nch) return;
  const int r = (int)(tid / a.nch);
  const int64_t c = tid - (int64_t)r * a.nch;
  const bool lastc = c == a.nch - 1;
  const int64_t len = lastc ? a.ops - c * a.ch : a.ch;
  const uint64_t *T = a.tab + (lastc ? kRateTab : 0);
  const int tn = lastc ? a.nl : a.nf;
  uint32_t w[4] = {(uint32_t)c, 0u, a.call, ((uint32_t)r << 8) | 0x80u};
  philox10(w, a.key0, a.key1);
  int K = 0;
  while (K < tn - 1 && (uint64_t)w[0] >= T[K]) ++K;
  uint64_t ev[kRateTab], pay[kRateTab];
  for (int e = 1; e <= K; ++e) {
    uint32_t q[4] = {(uint32_t)c, (uint32_t)e, a.call, ((uint32_t)r << 8) | 0x40u};
    philox10(q, a.key0, a.key1);
    const uint64_t off = ((uint64_t)q[0] * (uint64_t)len) >> 32;
    uint64_t k0 = (off << 16) | (uint64_t)e, k1 = ((uint64_t)q[1] << 32) | q[2];
    int j = e - 2;  // insertion sort by (offset, e)
    while (j >= 0 && ev[j] > k0) {
      ev[j + 1] = ev[j];
      pay[j + 1] = pay[j];
      --j;
    }
    ev[j + 1] = k0;
    pay[j + 1] = k1;
  }
  int kept = 0;
  const int64_t base = WRITE ? a.offs[tid] : 0;
  for (int e = 0; e < K; ++e) {
    const int64_t p = c * a.ch + (int64_t)(ev[e] >> 16);
    int tgt;
    int64_t idx;
    if (p < a.y_ops) {  // largest row i with 2 rp[i] <= p
      tgt = 0;
      idx = op_row(a.rp, a.ybkt, p);
    } else if (p < a.y_ops + a.t1_ops) {  // largest block k with 2 crp[k] <= p - y_ops
      tgt = 1;
      idx = op_row(a.crp, a.cbkt, p - a.y_ops);
    } else {
      tgt = 2;
      idx = (p - a.y_ops - a.t1_ops) / a.bs;
    }
    if (!(a.targets & (1u << tgt))) continue;
    if (WRITE && base + kept < a.cap) {
      const uint32_t ws = (uint32_t)(pay[e] >> 32), wl = (uint32_t)pay[e];
      const int start = (int)(ws & 63u);
      int blen = 1;
      while (blen < 64 && (uint64_t)wl >= c_burst_T[blen]) ++blen;
      const int hib = min(start + blen - 1, 63);
      const uint64_t span = (hib - start + 1) == 64 ? ~0ull : ((1ull << (hib - start + 1)) - 1ull);
      a.keys[base + kept] = list_key(r, tgt, idx);
      a.masks[base + kept] = span << start;
    }
    ++kept;
  }
  if (!WRITE) a.counts[tid] = kept;
}

__device__ __forceinline__ double apply_mask(double v, uint64_t m) {
  return __longlong_as_double((long long)((uint64_t)__double_as_longlong(v) ^ m));
}

// Programmatic dependent launch (PDL): pdl_trigger lets the next kernel of
// the stream start launching (its CTAs are scheduled once every CTA of this
// grid has triggered or exited); pdl_wait blocks until the preceding grid has
// COMPLETED and its memory is visible -- every kernel calls it before it
// reads or writes anything a preceding kernel touches.  Both are no-ops
// without the launch attribute.
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

}  // namespace abft
