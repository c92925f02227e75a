/*
 * abft_oracle.c -- CPU ORACLE (test infrastructure only; see abft_oracle.h).
 *
 * Plain, slow, obviously correct.  No blocking, fusion or reordering beyond
 * what the paper (or a DESIGN.md reading) states.  Shares nothing with
 * paper_conf_dsn_schollbkw16_b200/csrc/.
 *
 * Build: gcc -std=c99 -O2 -ffp-contract=off -fno-fast-math -shared -fPIC -lm
 */
#include "abft_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------ */
/* R2: canonical pairwise summation PW.                                      */
/* PW(v_0..v_{n-1}) is the balanced binary tree over the list padded to the  */
/* next power of two, where padding slots are ABSENT (a node with one absent */
/* child is its other child, unchanged).  PW of an empty list is +0.0.       */
/* The paper fixes no order for its inner products ("reductions", */
/* P:164); this reading makes every result bit-reproducible.                 */
/* ------------------------------------------------------------------------ */
static int pw_node(const double *v, const unsigned char *present, int64_t n, int64_t lo,
                   int64_t size, double *out) {
  if (lo >= n) return 0; /* absent */
  if (size == 1) {
    if (present && !present[lo]) return 0;
    *out = v[lo];
    return 1;
  }
  double l = 0.0, r = 0.0;
  int hl = pw_node(v, present, n, lo, size / 2, &l);
  int hr = pw_node(v, present, n, lo + size / 2, size / 2, &r);
  if (hl && hr) {
    *out = l + r;
    return 1;
  }
  if (hl) {
    *out = l;
    return 1;
  }
  if (hr) {
    *out = r;
    return 1;
  }
  return 0;
}

double or_pw_slots(const double *v, const unsigned char *present, int64_t n) {
  int64_t size = 1;
  double out = 0.0;
  while (size < n) size *= 2;
  if (!pw_node(v, present, n, 0, size, &out)) return 0.0; /* empty sum */
  return out;
}

double or_pw(const double *v, int64_t n) { return or_pw_slots(v, NULL, n); }

/* ------------------------------------------------------------------------ */
/* SpMV (Fig. 1 step 1): y_i = sum_j a_ij * x_j, summed by PW over the */
/* row's entries in CSR order (R3).                                          */
/* ------------------------------------------------------------------------ */
double or_row_dot(const or_csr *A, int64_t i, const double *x) {
  int64_t b = A->row_ptr[i], e = A->row_ptr[i + 1];
  double *p = (double *)malloc(sizeof(double) * (size_t)(e > b ? e - b : 1));
  for (int64_t q = b; q < e; ++q) p[q - b] = A->val[q] * x[A->col[q]];
  double r = or_pw(p, e - b);
  free(p);
  return r;
}

void or_spmv(const or_csr *A, const double *x, double *y) {
  for (int64_t i = 0; i < A->n; ++i) y[i] = or_row_dot(A, i, x);
}

/* ------------------------------------------------------------------------ */
/* Encoding, structure (Fig. 2; Fig. 3 step 1): row k of C */
/* holds the columns of row block A_k that contain at least one element     */
/* (structural, R5), ascending.  Blocks are rows k*bs .. min((k+1)*bs,N)-1  */
/* (P:80, 0-based per R4).                                                    */
/* ------------------------------------------------------------------------ */
static int cmp_i32(const void *a, const void *b) {
  int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
  return (x > y) - (x < y);
}

int64_t or_encode_structure(const or_csr *A, int32_t bs, int32_t *c_row_ptr, int32_t *c_col) {
  int64_t n = A->n, nb = (n + bs - 1) / bs;
  int64_t *seen = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
  int32_t *tmp = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  for (int64_t j = 0; j < n; ++j) seen[j] = -1;
  int64_t total = 0;
  c_row_ptr[0] = 0;
  for (int64_t k = 0; k < nb; ++k) {
    int64_t cnt = 0;
    for (int64_t i = k * bs; i < (k + 1) * bs && i < n; ++i)
      for (int64_t q = A->row_ptr[i]; q < A->row_ptr[i + 1]; ++q) {
        int32_t j = A->col[q];
        if (seen[j] != k) {
          seen[j] = k;
          tmp[cnt++] = j;
        }
      }
    qsort(tmp, (size_t)cnt, sizeof(int32_t), cmp_i32);
    if (c_col) memcpy(c_col + total, tmp, sizeof(int32_t) * (size_t)cnt);
    total += cnt;
    c_row_ptr[k + 1] = (int32_t)total;
  }
  free(seen);
  free(tmp);
  return total;
}

/* Find a_ij in row i (binary search over the ascending columns); 1 if present. */
static int find_entry(const or_csr *A, int64_t i, int32_t j, double *out) {
  int64_t lo = A->row_ptr[i], hi = A->row_ptr[i + 1];
  while (lo < hi) {
    int64_t mid = lo + (hi - lo) / 2;
    if (A->col[mid] < j)
      lo = mid + 1;
    else
      hi = mid;
  }
  if (lo < A->row_ptr[i + 1] && A->col[lo] == j) {
    *out = A->val[lo];
    return 1;
  }
  return 0;
}

/* Encoding, values: c_k = w_k^T A_k with w_k = (1..1)  */
/* (R1), i.e. c_kj = sum over the b_s row slots of block k of a_ij,   */
/* summed by PW over the slots, absent where row i has no entry j or i >= N */
/* (R4').                                                                     */
void or_encode_values(const or_csr *A, int32_t bs, const int32_t *c_row_ptr,
                      const int32_t *c_col, double *c_val) {
  int64_t n = A->n, nb = (n + bs - 1) / bs;
  double *slot = (double *)malloc(sizeof(double) * (size_t)bs);
  unsigned char *pres = (unsigned char *)malloc((size_t)bs);
  for (int64_t k = 0; k < nb; ++k)
    for (int64_t q = c_row_ptr[k]; q < c_row_ptr[k + 1]; ++q) {
      for (int32_t s = 0; s < bs; ++s) {
        int64_t i = k * bs + s;
        pres[s] = 0;
        slot[s] = 0.0;
        if (i < n) pres[s] = (unsigned char)find_entry(A, i, c_col[q], &slot[s]);
      }
      c_val[q] = or_pw_slots(slot, pres, bs);
    }
  free(slot);
  free(pres);
}

/* Encoding, bound constants: the sparse bound                   */
/*   tau_k(beta) = ((n_k + 2 b_s - 2) * sum_{i in k} ||a_i||_2                 */
/*                  + n_k * ||c_k||_2) * eps_M * beta,   eps_M = 2^-53 */
/* is split into K_k (everything but beta, computed once per matrix) and    */
/* tau_k = K_k * beta (R7, R11).  The row sum runs over the b_s slots with  */
/* absent slots past N (R3'); ||.||_2 = sqrt(PW of squares) (R6).            */
void or_encode_bound(const or_csr *A, int32_t bs, const int32_t *c_row_ptr,
                     const double *c_val, double *K, double *row_norm, double *S_out,
                     double *c_norm) {
  int64_t n = A->n, nb = (n + bs - 1) / bs;
  double *rn = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
  for (int64_t i = 0; i < n; ++i) {
    int64_t b = A->row_ptr[i], e = A->row_ptr[i + 1];
    double *sq = (double *)malloc(sizeof(double) * (size_t)(e > b ? e - b : 1));
    for (int64_t q = b; q < e; ++q) sq[q - b] = A->val[q] * A->val[q];
    rn[i] = sqrt(or_pw(sq, e - b));
    free(sq);
    if (row_norm) row_norm[i] = rn[i];
  }
  double *slot = (double *)malloc(sizeof(double) * (size_t)bs);
  unsigned char *pres = (unsigned char *)malloc((size_t)bs);
  const double eps_m = ldexp(1.0, -53);
  for (int64_t k = 0; k < nb; ++k) {
    for (int32_t s = 0; s < bs; ++s) {
      int64_t i = k * bs + s;
      pres[s] = (unsigned char)(i < n);
      slot[s] = i < n ? rn[i] : 0.0;
    }
    double S = or_pw_slots(slot, pres, bs);
    int64_t cb = c_row_ptr[k], ce = c_row_ptr[k + 1];
    double *sq = (double *)malloc(sizeof(double) * (size_t)(ce > cb ? ce - cb : 1));
    for (int64_t q = cb; q < ce; ++q) sq[q - cb] = c_val[q] * c_val[q];
    double cn = sqrt(or_pw(sq, ce - cb));
    free(sq);
    double n_k = (double)(ce - cb);
    double m_k = n_k + 2.0 * (double)bs - 2.0;
    K[k] = (m_k * S + n_k * cn) * eps_m;
    if (S_out) S_out[k] = S;
    if (c_norm) c_norm[k] = cn;
  }
  free(slot);
  free(pres);
  free(rn);
}

/* ------------------------------------------------------------------------ */
/* Fault model.                                                               */
/* Philox4x32-10 (Salmon et al., SC'11), the counter-based generator both    */
/* sides implement independently (task rule ③).                              */
/* ------------------------------------------------------------------------ */
void or_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  uint32_t c0 = ctr[0], c1 = ctr[1], c2 = ctr[2], c3 = ctr[3];
  uint32_t k0 = key[0], k1 = key[1];
  for (int r = 0; r < 10; ++r) {
    uint64_t p0 = (uint64_t)0xD2511F53u * c0;
    uint64_t p1 = (uint64_t)0xCD9E8D57u * c2;
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c1 ^ k0;
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c3 ^ k1;
    uint32_t n3 = lo0;
    c0 = n0;
    c1 = n1;
    c2 = n2;
    c3 = n3;
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  out[0] = c0;
  out[1] = c1;
  out[2] = c2;
  out[3] = c3;
}

/* Burst length: "randomly chosen from a normal distribution with    */
/* mean = 3 and variance = 2", read as L = max(1, round(3 + sqrt(2) Z)) (R12).*/
/* T[l] = floor(2^32 * P(L <= l)), P(L <= l) = Phi((l + 0.5 - 3)/sqrt 2)     */
/*      = erfc(-(l - 2.5)/2) / 2 for l = 1..63; T[64] = 2^32; T[0] = 0.       */
void or_burst_table(uint64_t T[65]) {
  T[0] = 0;
  for (int l = 1; l < 64; ++l) {
    double p = 0.5 * erfc(-((double)l - 2.5) / 2.0);
    T[l] = (uint64_t)floor(ldexp(p, 32));
  }
  T[64] = (uint64_t)1 << 32;
}

static uint64_t burst_from_words(uint32_t w_start, uint32_t w_len) {
  static uint64_t T[65];
  static int init = 0;
  if (!init) {
    or_burst_table(T);
    init = 1;
  }
  int start = (int)(w_start & 63u);
  int len = 1;
  while (len < 64 && (uint64_t)w_len >= T[len]) ++len;
  int hi = start + len - 1;
  if (hi > 63) hi = 63;
  uint64_t m = 0;
  for (int b = start; b <= hi; ++b) m |= (uint64_t)1 << b;
  return m;
}

/* The XOR mask for the value produced for (round, target, index) under an
 * explicit fault list: XOR of all entries that match (R13, list mode). */
uint64_t or_fault_mask(const or_inject *inj, int32_t round, int32_t target, int64_t index,
                       int64_t ops) {
  (void)ops;
  if (!inj || inj->mode != OR_INJ_LIST) return 0;
  uint64_t m = 0;
  for (int64_t e = 0; e < inj->n_list; ++e)
    if (inj->list_round[e] == round && inj->list_target[e] == target &&
        inj->list_index[e] == index && (!inj->list_call || (uint64_t)inj->list_call[e] == inj->call))
      m ^= inj->list_mask[e];
  return m;
}

/* ------------------------------------------------------------------------ */
/* Rate mode (R13): "we determine the error events from an           */
/* exponential distribution with an error rate lambda ... 1/lambda [is] the  */
/* expected number of arithmetic operations between two consecutive error   */
/* events" -- a Poisson process over the call's arithmetic operations.       */
/* Op space of one call (per round): y_i owns 2 len_i ops, then t1_k owns    */
/* 2 n_k ops, then t2_k owns rows-in-block ops (y only when unprotected).    */
/* It is cut into chunks of CH ops (CH = 2^24 halved while lambda*CH > 4);   */
/* chunk c holds K ~ Poisson(lambda * len_c) events, K drawn by inversion of */
/* the CDF table T[k] = floor(2^32 P(K <= k)) with Philox word 0 of counter  */
/* {c, 0, call, r<<8 | 0x80}; event e in 1..K takes counter {c, e, call,     */
/* r<<8 | 0x40}: position = c*CH + floor(w0 * len_c / 2^32), burst start =   */
/* w1 & 63, burst length from w2 (R12).  Events of disabled targets are      */
/* dropped (thinning).  Output: list entries ordered by (round, op position).*/
/* ------------------------------------------------------------------------ */
int64_t or_rate_chunk(double lambda) {
  int64_t ch = (int64_t)1 << 24;
  while (ch > 1 && lambda * (double)ch > 4.0) ch /= 2;
  return ch;
}

/* Poisson(mu) CDF table; returns its length (last entry = 2^32). */
int or_poisson_table(double mu, uint64_t *T, int cap) {
  double p = exp(-mu), cdf = p;
  int k = 0;
  for (;;) {
    double c = cdf < 1.0 ? cdf : 1.0;
    T[k] = (uint64_t)floor(ldexp(c, 32));
    if (T[k] >= ((uint64_t)1 << 32) - 1 || k == cap - 1) {
      T[k] = (uint64_t)1 << 32;
      return k + 1;
    }
    ++k;
    p = p * mu / (double)k;
    cdf = cdf + p;
  }
}

/* Fill (round, target, index, mask) lists for rounds 0..max_rounds; returns
 * the number of events (call with NULL outputs to count). */
int64_t or_rate_plan(const or_csr *A, int32_t bs, const int32_t *c_row_ptr, int32_t check,
                     const or_inject *inj, int32_t max_rounds, int32_t *o_round,
                     int32_t *o_target, int64_t *o_index, uint64_t *o_mask) {
  int64_t n = A->n, nb = (n + bs - 1) / bs, nnz = A->row_ptr[n];
  int64_t nnzc = check ? c_row_ptr[nb] : 0;
  int64_t y_ops = 2 * nnz, t1_ops = check ? 2 * nnzc : 0, t2_ops = check ? n : 0;
  int64_t ops = y_ops + t1_ops + t2_ops;
  int64_t ch = or_rate_chunk(inj->lambda);
  int64_t nch = (ops + ch - 1) / ch;
  uint32_t key[2] = {(uint32_t)inj->seed, (uint32_t)(inj->seed >> 32)};
  uint64_t Tf[32], Tl[32];  /* mean <= 4 events per chunk: K <= 31 */
  int nf = or_poisson_table(inj->lambda * (double)ch, Tf, 32);
  int64_t last = ops - (nch - 1) * ch;
  int nl = or_poisson_table(inj->lambda * (double)last, Tl, 32);
  int64_t cnt = 0;
  int rounds = check ? max_rounds : 0;
  uint64_t *pos = (uint64_t *)malloc(sizeof(uint64_t) * 32 * 2);
  for (int32_t r = 0; r <= rounds; ++r)
    for (int64_t c = 0; c < nch; ++c) {
      int64_t len = c == nch - 1 ? last : ch;
      const uint64_t *T = c == nch - 1 ? Tl : Tf;
      int tn = c == nch - 1 ? nl : nf;
      uint32_t ctr[4] = {(uint32_t)c, 0u, (uint32_t)inj->call, ((uint32_t)r << 8) | 0x80u};
      uint32_t w[4];
      or_philox4x32_10(ctr, key, w);
      int K = 0;
      while (K < tn - 1 && (uint64_t)w[0] >= T[K]) ++K;
      /* events: (position << 16 | e) so equal positions keep event order */
      for (int e = 1; e <= K; ++e) {
        uint32_t c2[4] = {(uint32_t)c, (uint32_t)e, (uint32_t)inj->call, ((uint32_t)r << 8) | 0x40u};
        or_philox4x32_10(c2, key, w);
        uint64_t off = ((uint64_t)w[0] * (uint64_t)len) >> 32;
        pos[2 * (e - 1)] = (off << 16) | (uint64_t)e;
        pos[2 * (e - 1) + 1] = ((uint64_t)w[1] << 32) | w[2];
      }
      /* sort by (offset, e): pairs -- simple insertion sort on the keys */
      for (int i = 1; i < K; ++i) {
        uint64_t k0 = pos[2 * i], k1 = pos[2 * i + 1];
        int j = i - 1;
        while (j >= 0 && pos[2 * j] > k0) {
          pos[2 * (j + 1)] = pos[2 * j];
          pos[2 * (j + 1) + 1] = pos[2 * j + 1];
          --j;
        }
        pos[2 * (j + 1)] = k0;
        pos[2 * (j + 1) + 1] = k1;
      }
      for (int i = 0; i < K; ++i) {
        int64_t p = c * ch + (int64_t)(pos[2 * i] >> 16);
        int32_t tgt;
        int64_t idx;
        if (p < y_ops) { /* row i with 2 rp[i] <= p < 2 rp[i+1] */
          int64_t lo = 0, hi = n; /* largest i with 2 rp[i] <= p */
          while (lo < hi) {
            int64_t mid = lo + (hi - lo + 1) / 2;
            if (2 * (int64_t)A->row_ptr[mid] <= p) lo = mid; else hi = mid - 1;
          }
          tgt = OR_T_Y;
          idx = lo;
        } else if (p < y_ops + t1_ops) {
          int64_t q = p - y_ops, lo = 0, hi = nb;
          while (lo < hi) {
            int64_t mid = lo + (hi - lo + 1) / 2;
            if (2 * (int64_t)c_row_ptr[mid] <= q) lo = mid; else hi = mid - 1;
          }
          tgt = OR_T_T1;
          idx = lo;
        } else {
          tgt = OR_T_T2;
          idx = (p - y_ops - t1_ops) / bs;
        }
        if (!(inj->targets & (1u << tgt))) continue;
        if (o_round) {
          uint32_t ws = (uint32_t)(pos[2 * i + 1] >> 32), wl = (uint32_t)pos[2 * i + 1];
          o_round[cnt] = r;
          o_target[cnt] = tgt;
          o_index[cnt] = idx;
          o_mask[cnt] = burst_from_words(ws, wl);
        }
        ++cnt;
      }
    }
  free(pos);
  return cnt;
}

/* Expand a rate-mode spec into an explicit list (malloc'd; caller frees). */
static or_inject rate_to_list(const or_csr *A, int32_t bs, const int32_t *c_row_ptr,
                              int32_t check, const or_inject *inj, int32_t max_rounds,
                              void **keep) {
  or_inject L;
  memset(&L, 0, sizeof L);
  L.mode = OR_INJ_LIST;
  int64_t cnt = or_rate_plan(A, bs, c_row_ptr, check, inj, max_rounds, NULL, NULL, NULL, NULL);
  size_t m = (size_t)(cnt > 0 ? cnt : 1);
  char *buf = (char *)malloc(m * (4 + 4 + 8 + 8));
  int32_t *r = (int32_t *)buf, *t = (int32_t *)(buf + 4 * m);
  int64_t *ix = (int64_t *)(buf + 8 * m);
  uint64_t *mk = (uint64_t *)(buf + 16 * m);
  or_rate_plan(A, bs, c_row_ptr, check, inj, max_rounds, r, t, ix, mk);
  L.n_list = cnt;
  L.list_round = r;
  L.list_target = t;
  L.list_index = ix;
  L.list_mask = mk;
  *keep = buf;
  return L;
}

static double xor_double(double v, uint64_t m) {
  uint64_t u;
  memcpy(&u, &v, 8);
  u ^= m;
  memcpy(&v, &u, 8);
  return v;
}

/* ------------------------------------------------------------------------ */
/* Protected SpMV, Fig. 1:                                          */
/*  1. y = A x  and  t1 = C x                                                 */
/*  2. beta = ||x||_2  and  t2_k = w_k^T y_k                                  */
/*  3. s = t1 - t2                                                            */
/*  4. flag k iff NOT(|s_k| <= tau_k)   (pass condition R5'/Q5)       */
/*  5. recompute only the flagged blocks, re-verify (R11')     */
/* Faults are applied to the produced value before it is used.  */
/* ------------------------------------------------------------------------ */
static double block_t1(const int32_t *c_row_ptr, const int32_t *c_col, const double *c_val,
                       int64_t k, const double *x) {
  int64_t b = c_row_ptr[k], e = c_row_ptr[k + 1];
  double *p = (double *)malloc(sizeof(double) * (size_t)(e > b ? e - b : 1));
  for (int64_t q = b; q < e; ++q) p[q - b] = c_val[q] * x[c_col[q]];
  double r = or_pw(p, e - b);
  free(p);
  return r;
}

static double block_t2(const double *y, int64_t n, int32_t bs, int64_t k, double *slot,
                       unsigned char *pres) {
  for (int32_t s = 0; s < bs; ++s) {
    int64_t i = k * bs + s;
    pres[s] = (unsigned char)(i < n);
    slot[s] = i < n ? y[i] : 0.0;
  }
  return or_pw_slots(slot, pres, bs);
}

static int64_t rows_in_block(int64_t n, int32_t bs, int64_t k) {
  int64_t e = (k + 1) * bs < n ? (k + 1) * bs : n;
  return e - k * bs;
}

/* Compute y rows, t1_k, t2_k and the decision for block k in `round`. */
static int check_block(const or_csr *A, int32_t bs, const int32_t *c_row_ptr,
                       const int32_t *c_col, const double *c_val, const double *K,
                       const double *x, double beta, const or_inject *inj, int32_t round,
                       int64_t k, double *y, double *t1, double *t2, double *s, double *slot,
                       unsigned char *pres) {
  int64_t n = A->n;
  for (int64_t i = k * bs; i < (k + 1) * bs && i < n; ++i) {
    double v = or_row_dot(A, i, x);
    int64_t ops = 2 * (int64_t)(A->row_ptr[i + 1] - A->row_ptr[i]);
    y[i] = xor_double(v, or_fault_mask(inj, round, OR_T_Y, i, ops));
  }
  double a = block_t1(c_row_ptr, c_col, c_val, k, x);
  a = xor_double(a, or_fault_mask(inj, round, OR_T_T1, k,
                                  2 * (int64_t)(c_row_ptr[k + 1] - c_row_ptr[k])));
  double b = block_t2(y, n, bs, k, slot, pres);
  b = xor_double(b, or_fault_mask(inj, round, OR_T_T2, k, rows_in_block(n, bs, k)));
  double syn = a - b;
  double tau = K[k] * beta;
  if (t1) t1[k] = a;
  if (t2) t2[k] = b;
  if (s) s[k] = syn;
  return !(fabs(syn) <= tau);
}

int or_abft_spmv(const or_csr *A, int32_t bs, const int32_t *c_row_ptr, const int32_t *c_col,
                 const double *c_val, const double *K, const double *x, const or_inject *inj_in,
                 int32_t max_rounds, double *y, double *y_pre, double *t1, double *t2,
                 double *s, double *beta_out, int32_t *flag_counts, int32_t *flags) {
  int64_t n = A->n, nb = (n + bs - 1) / bs;
  void *keep = NULL;
  or_inject lst;
  const or_inject *inj = inj_in;
  if (inj_in && inj_in->mode == OR_INJ_RATE) {
    lst = rate_to_list(A, bs, c_row_ptr, 1, inj_in, max_rounds, &keep);
    inj = &lst;
  }
  /* step 2: beta = ||x||_2 = sqrt(PW(x_i^2)) (R10) */
  double *sq = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
  for (int64_t i = 0; i < n; ++i) sq[i] = x[i] * x[i];
  double beta = sqrt(or_pw(sq, n));
  free(sq);
  if (beta_out) *beta_out = beta;
  double *slot = (double *)malloc(sizeof(double) * (size_t)bs);
  unsigned char *pres = (unsigned char *)malloc((size_t)bs);
  /* steps 1-4 over all blocks (round 0) */
  int32_t cnt = 0;
  for (int64_t k = 0; k < nb; ++k)
    if (check_block(A, bs, c_row_ptr, c_col, c_val, K, x, beta, inj, 0, k, y, t1, t2, s, slot,
                    pres))
      flags[cnt++] = (int32_t)k;
  flag_counts[0] = cnt;
  if (y_pre) memcpy(y_pre, y, sizeof(double) * (size_t)n);
  /* step 5: partial recomputation of flagged blocks, re-verified each round */
  int rc = 0;
  for (int32_t r = 1; r <= max_rounds; ++r) {
    const int32_t *prev = flags + (int64_t)(r - 1) * nb;
    int32_t *next = flags + (int64_t)r * nb;
    int32_t nn = 0;
    for (int32_t q = 0; q < flag_counts[r - 1]; ++q) {
      int64_t k = prev[q];
      if (check_block(A, bs, c_row_ptr, c_col, c_val, K, x, beta, inj, r, k, y, t1, t2, s, slot,
                      pres))
        next[nn++] = (int32_t)k;
    }
    flag_counts[r] = nn;
  }
  if (max_rounds > 0 && flag_counts[max_rounds] > 0) rc = -6;
  free(slot);
  free(pres);
  free(keep);
  return rc;
}

/* ------------------------------------------------------------------------ */
/* Related-work baseline: the DENSE CHECK of [30, 31] (P:44-48,       */
/* P:250-252) with COMPLETE RECOMPUTATION [31].  One   */
/* checksum over all N rows: c = w^T A with w = 1 (eq. 1), so       */
/* c_j = sum of column j; t1 = c . x, t2 = w^T y.  Readings (DESIGN.md */
/* R23-R25): c_j = PW over column j's entries in ascending row order; t1 =   */
/* PW over the n columns of fl(c_j x_j) (c_j = +0.0 for an empty column);    */
/* t2 = PW over the N entries of y; the bound is either the norm-based       */
/* tau = ||x||_2 of [30] or the analytical bound of [35] */
/* with m = N rows and n columns: tau = K35 * ||x||_2,                        */
/* K35 = fl(fl(fl((n + 2N - 2) * PW_i ||a_i||_2) + fl(n * ||c||_2)) * 2^-53). */
/* Flag iff NOT(|t1 - t2| <= tau); a flag triggers a complete recomputation  */
/* of y (round r + 1), re-checked, at most max_rounds times.                  */
/* ------------------------------------------------------------------------ */
void or_dense_encode(const or_csr *A, double *c, double *k35) {
  int64_t n = A->n;
  int64_t nnz = A->row_ptr[n];
  /* column lists in ascending row order (a counting sort by column) */
  int64_t *cnt = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  for (int64_t e = 0; e < nnz; ++e) cnt[A->col[e] + 1]++;
  for (int64_t j = 0; j < n; ++j) cnt[j + 1] += cnt[j];
  double *cv = (double *)malloc(sizeof(double) * (size_t)(nnz > 0 ? nnz : 1));
  int64_t *pos = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
  for (int64_t j = 0; j < n; ++j) pos[j] = cnt[j];
  for (int64_t i = 0; i < n; ++i)
    for (int64_t q = A->row_ptr[i]; q < A->row_ptr[i + 1]; ++q) cv[pos[A->col[q]]++] = A->val[q];
  for (int64_t j = 0; j < n; ++j) c[j] = or_pw(cv + cnt[j], cnt[j + 1] - cnt[j]);
  if (k35) {
    double *tmp = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
    for (int64_t i = 0; i < n; ++i) {
      int64_t b = A->row_ptr[i], e = A->row_ptr[i + 1];
      double *sq = (double *)malloc(sizeof(double) * (size_t)(e > b ? e - b : 1));
      for (int64_t q = b; q < e; ++q) sq[q - b] = A->val[q] * A->val[q];
      tmp[i] = sqrt(or_pw(sq, e - b));
      free(sq);
    }
    double S = or_pw(tmp, n);
    for (int64_t j = 0; j < n; ++j) tmp[j] = c[j] * c[j];
    double cn = sqrt(or_pw(tmp, n));
    double m = (double)(n + 2 * n - 2); /* n columns + 2m - 2 with m = N = n rows */
    *k35 = ((m * S) + ((double)n * cn)) * 0x1p-53;
    free(tmp);
  }
  free(cnt);
  free(cv);
  free(pos);
}

int or_dense_spmv(const or_csr *A, const double *c, double k35, int32_t bound35,
                  const double *x, const or_inject *inj, int32_t max_rounds, double *y,
                  double *y_pre, double *out, int32_t *flag_rounds) {
  int64_t n = A->n;
  void *keep = NULL;
  or_inject lst;
  if (inj && inj->mode == OR_INJ_RATE) { /* rate mode: y ops of round 0 only (R25) */
    lst = rate_to_list(A, 32, NULL, 0, inj, 0, &keep);
    inj = &lst;
  }
  double *tmp = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
  for (int64_t i = 0; i < n; ++i) tmp[i] = x[i] * x[i];
  double beta = sqrt(or_pw(tmp, n)); /* ||x||_2, R10 */
  double tau = bound35 ? k35 * beta : beta;
  int rc = 0;
  for (int32_t r = 0; r <= max_rounds; ++r) {
    /* round 0: the SpMV; round r >= 1: the r-th complete recomputation */
    for (int64_t i = 0; i < n; ++i) {
      double v = or_row_dot(A, i, x);
      int64_t ops = 2 * (int64_t)(A->row_ptr[i + 1] - A->row_ptr[i]);
      y[i] = xor_double(v, or_fault_mask(inj, r, OR_T_Y, i, ops));
    }
    if (r == 0 && y_pre) memcpy(y_pre, y, sizeof(double) * (size_t)n);
    for (int64_t j = 0; j < n; ++j) tmp[j] = c[j] * x[j];
    double t1 = xor_double(or_pw(tmp, n), or_fault_mask(inj, r, OR_T_T1, 0, 2 * n));
    double t2 = xor_double(or_pw(y, n), or_fault_mask(inj, r, OR_T_T2, 0, n));
    int flagged = !(fabs(t1 - t2) <= tau);
    flag_rounds[r] = flagged;
    if (r == 0 && out) {
      out[0] = t1;
      out[1] = t2;
      out[2] = beta;
      out[3] = tau;
    }
    if (!flagged) {
      for (int32_t q = r + 1; q <= max_rounds; ++q) flag_rounds[q] = 0;
      break;
    }
    if (r == max_rounds) rc = -6;
  }
  free(tmp);
  free(keep);
  return rc;
}

/* ------------------------------------------------------------------------ */
/* Jacobi-preconditioned CG (Saad, Alg. 9.1) using the protected */
/* SpMV for every product with A.  Stop when ||r||_2 <= tol * ||b||_2 (R16)  */
/* or after max_iter iterations (10 N by default).  M = diag(A) and  */
/* z = r / d elementwise (R21).  Updates follow R15.                         */
/* ------------------------------------------------------------------------ */
static double dot_pw(const double *a, const double *b, int64_t n, double *tmp) {
  for (int64_t i = 0; i < n; ++i) tmp[i] = a[i] * b[i];
  return or_pw(tmp, n);
}

int or_pcg(const or_csr *A, int32_t bs, const int32_t *c_row_ptr, const int32_t *c_col,
           const double *c_val, const double *K, const double *b, double *x,
           const double *diag, double tol, int64_t max_iter, const or_inject *inj_in,
           int32_t max_rounds, int32_t check, double *res_hist, int64_t *stats) {
  int64_t n = A->n, nb = (n + bs - 1) / bs;
  if (max_iter <= 0) max_iter = 10 * n;
  /* P:296 read literally: stop when r^T r < eps (R16*); default: ||r|| <= eps ||b|| */
  const int literal = (check & OR_PCG_LITERAL_STOP) != 0;
  check &= ~OR_PCG_LITERAL_STOP;
  size_t vb = sizeof(double) * (size_t)(n > 0 ? n : 1);
  double *r = (double *)malloc(vb), *z = (double *)malloc(vb), *p = (double *)malloc(vb);
  double *q = (double *)malloc(vb), *tmp = (double *)malloc(vb), *d = (double *)malloc(vb);
  int32_t *fc = (int32_t *)malloc(sizeof(int32_t) * (size_t)(max_rounds + 1));
  int32_t *fl = (int32_t *)malloc(sizeof(int32_t) * (size_t)((max_rounds + 1) * nb + 1));
  or_inject inj;
  memset(&inj, 0, sizeof inj);
  if (inj_in) inj = *inj_in;
  uint64_t call0 = inj.call;
  int64_t calls = 0;
  for (int i = 0; i < 5; ++i) stats[i] = 0;
  for (int64_t i = 0; i < n; ++i) {
    if (diag) {
      d[i] = diag[i];
    } else {
      double v = 0.0;
      if (!find_entry(A, i, (int32_t)i, &v)) v = 0.0;
      d[i] = v;
    }
  }
  int rc = 0;
  /* protected SpMV wrapper: y = A v, counting flags and recomputations */
#define PROTECTED_SPMV(vin, yout)                                                          \
  do {                                                                                     \
    inj.call = call0 + (uint64_t)calls;                                                    \
    if (check) {                                                                           \
      int st = or_abft_spmv(A, bs, c_row_ptr, c_col, c_val, K, vin, &inj, max_rounds, yout, \
                            NULL, NULL, NULL, NULL, NULL, fc, fl);                         \
      stats[2] += fc[0];                                                                   \
      for (int32_t rr = 0; rr < max_rounds; ++rr) stats[3] += fc[rr];                      \
      if (st) stats[4] += 1;                                                               \
    } else {                                                                               \
      void *keep_ = NULL;                                                                  \
      or_inject l_ = inj;                                                                  \
      if (inj.mode == OR_INJ_RATE)                                                         \
        l_ = rate_to_list(A, bs, c_row_ptr, 0, &inj, 0, &keep_);                            \
      for (int64_t i_ = 0; i_ < n; ++i_) {                                                 \
        double v_ = or_row_dot(A, i_, vin);                                                \
        yout[i_] = xor_double(v_, or_fault_mask(&l_, 0, OR_T_Y, i_, 0));                   \
      }                                                                                    \
      free(keep_);                                                                         \
    }                                                                                      \
    calls++;                                                                               \
  } while (0)

  PROTECTED_SPMV(x, q); /* q = A x0 */
  for (int64_t i = 0; i < n; ++i) r[i] = b[i] - q[i];
  for (int64_t i = 0; i < n; ++i) z[i] = r[i] / d[i];
  for (int64_t i = 0; i < n; ++i) p[i] = z[i];
  double rho = dot_pw(r, z, n, tmp);
  double bnorm = sqrt(dot_pw(b, b, n, tmp));
  double thr = tol * bnorm;
  double rr = dot_pw(r, r, n, tmp);
  double res = sqrt(rr);
  res_hist[0] = res;
  int64_t it = 0;
#define PCG_DONE (literal ? (rr < tol) : (res <= thr))
  while (!PCG_DONE && it < max_iter) {
    if (res != res) {
      rc = -7;
      break;
    }
    PROTECTED_SPMV(p, q);
    double pq = dot_pw(p, q, n, tmp);
    if (!(pq > 0.0)) {
      rc = -7;
      break;
    }
    double alpha = rho / pq;
    for (int64_t i = 0; i < n; ++i) x[i] = x[i] + alpha * p[i];
    for (int64_t i = 0; i < n; ++i) r[i] = r[i] - alpha * q[i];
    for (int64_t i = 0; i < n; ++i) z[i] = r[i] / d[i];
    double rho_new = dot_pw(r, z, n, tmp);
    rr = dot_pw(r, r, n, tmp);
    res = sqrt(rr);
    ++it;
    res_hist[it] = res;
    double beta = rho_new / rho;
    rho = rho_new;
    for (int64_t i = 0; i < n; ++i) p[i] = z[i] + beta * p[i];
  }
#undef PROTECTED_SPMV
  if (rc == 0 && !PCG_DONE) rc = -5;
#undef PCG_DONE
  stats[0] = it;
  stats[1] = calls;
  free(r);
  free(z);
  free(p);
  free(q);
  free(tmp);
  free(d);
  free(fc);
  free(fl);
  return rc;
}

/* ------------------------------------------------------------------------ */
/* Related-work baseline for the PCG case study: the         */
/* CHECKPOINTING approach of P:286-292 -- every SpMV protected by the dense  */
/* check with the norm-based bound, the solver state sampled every   */
/* `ckpt_every` (20) iterations, and on a detection a rollback to the */
/* last sample and re-execution from there.  DESIGN.md R26-R27:              */
/*  * state = (x, r, z, p, rho, it); the first sample is taken after the     */
/*    initial residual; a flagged initial SpMV is simply redone;             */
/*  * SpMV call j (the j-th executed product, initial one = 0) draws its      */
/*    faults from the rate plan of call inj->call + j over y only (the       */
/*    dense check's own 3N detection ops are not injected);                  */
/*  * max_iter bounds EXECUTED iterations (re-executions count).      */
/* The updates are those of or_pcg (R15).  stats: [0] iterations of the     */
/* returned solution, [1] SpMV calls, [2] rollbacks, [3] executed            */
/* iterations, [4] 0.  Returns 0 converged, -5 not converged, -7 breakdown. */
/* ------------------------------------------------------------------------ */
int or_pcg_cr(const or_csr *A, const double *c, const double *b, double *x, const double *diag,
              double tol, int64_t max_iter, const or_inject *inj_in, int32_t ckpt_every,
              double *res_hist, int64_t *stats) {
  int64_t n = A->n;
  if (max_iter <= 0) max_iter = 10 * n;
  size_t vb = sizeof(double) * (size_t)(n > 0 ? n : 1);
  double *r = (double *)malloc(vb), *z = (double *)malloc(vb), *p = (double *)malloc(vb);
  double *q = (double *)malloc(vb), *tmp = (double *)malloc(vb), *d = (double *)malloc(vb);
  double *cx = (double *)malloc(vb), *cr = (double *)malloc(vb), *cz = (double *)malloc(vb);
  double *cp = (double *)malloc(vb);
  or_inject inj;
  memset(&inj, 0, sizeof inj);
  if (inj_in) inj = *inj_in;
  uint64_t call0 = inj.call;
  int64_t calls = 0, rollbacks = 0, executed = 0;
  for (int i = 0; i < 5; ++i) stats[i] = 0;
  for (int64_t i = 0; i < n; ++i) {
    double v = 0.0;
    if (diag) v = diag[i];
    else if (!find_entry(A, i, (int32_t)i, &v)) v = 0.0;
    d[i] = v;
  }
  /* y = A v with this call's y faults, then the dense check (t1 = c.v,
     t2 = sum y, tau = ||v||): returns 1 when flagged */
#define CHECKED_SPMV(vin, yout, flagged)                                         \
  do {                                                                           \
    inj.call = call0 + (uint64_t)calls;                                          \
    void *keep_ = NULL;                                                          \
    or_inject l_ = inj;                                                          \
    if (inj.mode == OR_INJ_RATE) l_ = rate_to_list(A, 32, NULL, 0, &inj, 0, &keep_); \
    for (int64_t i_ = 0; i_ < n; ++i_)                                           \
      yout[i_] = xor_double(or_row_dot(A, i_, vin), or_fault_mask(&l_, 0, OR_T_Y, i_, 0)); \
    free(keep_);                                                                 \
    for (int64_t i_ = 0; i_ < n; ++i_) tmp[i_] = c[i_] * vin[i_];               \
    double t1_ = or_pw(tmp, n);                                                  \
    double t2_ = or_pw(yout, n);                                                 \
    double bt_ = sqrt(dot_pw(vin, vin, n, tmp));                                 \
    flagged = !(fabs(t1_ - t2_) <= bt_);                                         \
    calls++;                                                                     \
  } while (0)

  int fl = 1, rc = 0;
  while (fl && calls < max_iter + 1) CHECKED_SPMV(x, q, fl); /* q = A x0 */
  for (int64_t i = 0; i < n; ++i) r[i] = b[i] - q[i];
  for (int64_t i = 0; i < n; ++i) z[i] = r[i] / d[i];
  for (int64_t i = 0; i < n; ++i) p[i] = z[i];
  double rho = dot_pw(r, z, n, tmp);
  double bnorm = sqrt(dot_pw(b, b, n, tmp));
  double thr = tol * bnorm;
  double res = sqrt(dot_pw(r, r, n, tmp));
  res_hist[0] = res;
  int64_t it = 0;
  /* sample 0 */
  memcpy(cx, x, vb); memcpy(cr, r, vb); memcpy(cz, z, vb); memcpy(cp, p, vb);
  double c_rho = rho, c_res = res;
  int64_t c_it = 0;
  while (!(res <= thr) && executed < max_iter) {
    if (res != res) {
      rc = -7;
      break;
    }
    ++executed;
    CHECKED_SPMV(p, q, fl);
    if (fl) { /* rollback to the last sample */
      memcpy(x, cx, vb); memcpy(r, cr, vb); memcpy(z, cz, vb); memcpy(p, cp, vb);
      rho = c_rho;
      res = c_res;
      it = c_it;
      ++rollbacks;
      continue;
    }
    double pq = dot_pw(p, q, n, tmp);
    if (!(pq > 0.0)) {
      rc = -7;
      break;
    }
    double alpha = rho / pq;
    for (int64_t i = 0; i < n; ++i) x[i] = x[i] + alpha * p[i];
    for (int64_t i = 0; i < n; ++i) r[i] = r[i] - alpha * q[i];
    for (int64_t i = 0; i < n; ++i) z[i] = r[i] / d[i];
    double rho_new = dot_pw(r, z, n, tmp);
    res = sqrt(dot_pw(r, r, n, tmp));
    ++it;
    res_hist[it] = res;
    double beta = rho_new / rho;
    rho = rho_new;
    for (int64_t i = 0; i < n; ++i) p[i] = z[i] + beta * p[i];
    if (ckpt_every > 0 && it % ckpt_every == 0) { /* sample the state */
      memcpy(cx, x, vb); memcpy(cr, r, vb); memcpy(cz, z, vb); memcpy(cp, p, vb);
      c_rho = rho;
      c_res = res;
      c_it = it;
    }
  }
#undef CHECKED_SPMV
  if (rc == 0 && !(res <= thr)) rc = -5;
  stats[0] = it;
  stats[1] = calls;
  stats[2] = rollbacks;
  stats[3] = executed;
  free(r); free(z); free(p); free(q); free(tmp); free(d);
  free(cx); free(cr); free(cz); free(cp);
  return rc;
}
