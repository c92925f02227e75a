"""ctypes wrapper around liboracle.so -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
--impl reference legs may import this module.  It never imports the product
package's CUDA code, and the product package never imports it.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "abft_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

CFLAGS = ["-std=c99", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fno-builtin",
          "-Wall", "-shared", "-fPIC"]


def build(force: bool = False) -> str:
    """Compile liboracle.so (gcc, no FMA contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "abft_oracle.h"))):
        subprocess.check_call(["gcc", *CFLAGS, "-o", _LIB, _SRC, "-lm"])
    return _LIB


_lib = None


class _Csr(C.Structure):
    _fields_ = [("n", C.c_int64), ("row_ptr", C.c_void_p), ("col", C.c_void_p),
                ("val", C.c_void_p)]


class _Inj(C.Structure):
    _fields_ = [("mode", C.c_int32), ("seed", C.c_uint64), ("call", C.c_uint64),
                ("lambda_", C.c_double), ("targets", C.c_uint32), ("n_list", C.c_int64),
                ("list_round", C.c_void_p), ("list_target", C.c_void_p),
                ("list_index", C.c_void_p), ("list_mask", C.c_void_p),
                ("list_call", C.c_void_p)]


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        L = _lib
        P, i64, i32, d = C.c_void_p, C.c_int64, C.c_int32, C.c_double
        L.or_pw.restype = d
        L.or_pw.argtypes = [P, i64]
        L.or_pw_slots.restype = d
        L.or_pw_slots.argtypes = [P, P, i64]
        L.or_spmv.argtypes = [P, P, P]
        L.or_encode_structure.restype = i64
        L.or_encode_structure.argtypes = [P, i32, P, P]
        L.or_encode_values.argtypes = [P, i32, P, P, P]
        L.or_encode_bound.argtypes = [P, i32, P, P, P, P, P, P]
        L.or_philox4x32_10.argtypes = [P, P, P]
        L.or_burst_table.argtypes = [P]
        L.or_fault_mask.restype = C.c_uint64
        L.or_fault_mask.argtypes = [P, i32, i32, i64, i64]
        L.or_rate_chunk.restype = i64
        L.or_rate_chunk.argtypes = [d]
        L.or_poisson_table.restype = C.c_int
        L.or_poisson_table.argtypes = [d, P, C.c_int]
        L.or_rate_plan.restype = i64
        L.or_rate_plan.argtypes = [P, i32, P, i32, P, i32, P, P, P, P]
        L.or_abft_spmv.restype = C.c_int
        L.or_abft_spmv.argtypes = [P, i32, P, P, P, P, P, P, i32, P, P, P, P, P, P, P, P]
        L.or_dense_encode.argtypes = [P, P, P]
        L.or_dense_spmv.restype = C.c_int
        L.or_dense_spmv.argtypes = [P, P, d, i32, P, P, i32, P, P, P, P]
        L.or_pcg_cr.restype = C.c_int
        L.or_pcg_cr.argtypes = [P, P, P, P, P, d, i64, P, i32, P, P]
        L.or_pcg.restype = C.c_int
        L.or_pcg.argtypes = [P, i32, P, P, P, P, P, P, P, d, i64, P, i32, i32, P, P]
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


class _CsrRef:
    """Keeps the numpy arrays alive while the C struct points into them."""

    def __init__(self, A):
        self.rp = np.ascontiguousarray(A.row_ptr, dtype=np.int32)
        self.col = np.ascontiguousarray(A.col, dtype=np.int32)
        self.val = np.ascontiguousarray(A.val, dtype=np.float64)
        self.s = _Csr(int(self.rp.shape[0] - 1), _p(self.rp).value, _p(self.col).value,
                      _p(self.val).value)

    def ref(self):
        return C.byref(self.s)


class Inject:
    """Fault injection spec shared by oracle calls (mirrors abft_inject_t)."""

    NONE, LIST, RATE = 0, 1, 2

    def __init__(self, mode=0, seed=0, call=0, lam=0.0, targets=0b001, plan=None):
        self.mode, self.seed, self.call, self.lam, self.targets = mode, seed, call, lam, targets
        self.plan = plan

    @staticmethod
    def from_plan(plan):
        return Inject(mode=Inject.LIST, plan=plan)

    @staticmethod
    def rate(seed, lam, targets=0b111, call=0):
        return Inject(mode=Inject.RATE, seed=seed, call=call, lam=lam, targets=targets)

    def _struct(self):
        s = _Inj()
        s.mode, s.seed, s.call, s.lambda_, s.targets = (self.mode, self.seed, self.call,
                                                        self.lam, self.targets)
        if self.mode == Inject.LIST and self.plan is not None and len(self.plan):
            self._keep = (np.ascontiguousarray(self.plan.round, np.int32),
                          np.ascontiguousarray(self.plan.target, np.int32),
                          np.ascontiguousarray(self.plan.index, np.int64),
                          np.ascontiguousarray(self.plan.mask, np.uint64))
            s.n_list = len(self.plan)
            s.list_round, s.list_target, s.list_index, s.list_mask = [
                _p(a).value for a in self._keep]
            call = getattr(self.plan, "call", None)
            if call is not None:  # per-call list (entry e only in SpMV call[e])
                self._keep_call = np.ascontiguousarray(call, np.int64)
                s.list_call = _p(self._keep_call).value
        else:
            s.n_list = 0
        return s


def pw(v, present=None) -> float:
    v = np.ascontiguousarray(v, dtype=np.float64)
    if present is None:
        return lib().or_pw(_p(v), v.shape[0])
    pr = np.ascontiguousarray(present, dtype=np.uint8)
    return lib().or_pw_slots(_p(v), _p(pr), v.shape[0])


def spmv(A, x) -> np.ndarray:
    r = _CsrRef(A)
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.empty(A.n)
    lib().or_spmv(r.ref(), _p(x), _p(y))
    return y


@dataclass
class Encoded:
    bs: int
    row_ptr: np.ndarray  # C row_ptr int32[nb+1]
    col: np.ndarray      # C col int32[nnz(C)]
    val: np.ndarray      # C val f64[nnz(C)]
    K: np.ndarray        # f64[nb]
    row_norm: np.ndarray
    S: np.ndarray
    c_norm: np.ndarray

    @property
    def nb(self):
        return int(self.row_ptr.shape[0] - 1)

    @property
    def n_k(self):
        return np.diff(self.row_ptr.astype(np.int64))


def encode(A, bs: int = 32) -> Encoded:
    r = _CsrRef(A)
    nb = (A.n + bs - 1) // bs
    c_rp = np.zeros(nb + 1, dtype=np.int32)
    L = lib()
    tot = L.or_encode_structure(r.ref(), bs, _p(c_rp), None)
    c_col = np.empty(max(tot, 1), dtype=np.int32)
    L.or_encode_structure(r.ref(), bs, _p(c_rp), _p(c_col))
    c_val = np.empty(max(tot, 1))
    L.or_encode_values(r.ref(), bs, _p(c_rp), _p(c_col), _p(c_val))
    K = np.empty(nb)
    rn = np.empty(A.n)
    S = np.empty(nb)
    cn = np.empty(nb)
    L.or_encode_bound(r.ref(), bs, _p(c_rp), _p(c_val), _p(K), _p(rn), _p(S), _p(cn))
    return Encoded(bs, c_rp, c_col[:tot], c_val[:tot], K, rn, S, cn)


def philox4x32_10(ctr, key):
    c = np.ascontiguousarray(ctr, dtype=np.uint32)
    k = np.ascontiguousarray(key, dtype=np.uint32)
    o = np.empty(4, dtype=np.uint32)
    lib().or_philox4x32_10(_p(c), _p(k), _p(o))
    return o


def burst_table() -> np.ndarray:
    t = np.empty(65, dtype=np.uint64)
    lib().or_burst_table(_p(t))
    return t


def rate_chunk(lam: float) -> int:
    return int(lib().or_rate_chunk(lam))


def poisson_table(mu: float, cap: int = 1024) -> np.ndarray:
    t = np.zeros(cap, dtype=np.uint64)
    k = lib().or_poisson_table(mu, _p(t), cap)
    return t[:k].copy()


def rate_plan(A, enc: "Encoded", inj: Inject, max_rounds: int = 4, check: bool = True):
    """The explicit fault list a rate-mode spec expands to (R13): arrays
    (round, target, index, mask) ordered by (round, op position)."""
    r = _CsrRef(A)
    s = inj._struct()
    L = lib()
    cnt = L.or_rate_plan(r.ref(), enc.bs, _p(enc.row_ptr), 1 if check else 0, C.byref(s),
                         max_rounds, None, None, None, None)
    m = max(cnt, 1)
    ro, ta = np.zeros(m, np.int32), np.zeros(m, np.int32)
    ix, mk = np.zeros(m, np.int64), np.zeros(m, np.uint64)
    L.or_rate_plan(r.ref(), enc.bs, _p(enc.row_ptr), 1 if check else 0, C.byref(s), max_rounds,
                   _p(ro), _p(ta), _p(ix), _p(mk))
    return ro[:cnt], ta[:cnt], ix[:cnt], mk[:cnt]


def fault_mask(inj: Inject, round_: int, target: int, index: int, ops: int) -> int:
    s = inj._struct()
    return int(lib().or_fault_mask(C.byref(s), round_, target, index, ops))


@dataclass
class SpmvResult:
    status: int
    y: np.ndarray
    y_pre: np.ndarray
    t1: np.ndarray
    t2: np.ndarray
    s: np.ndarray
    beta: float
    flags: list  # per round: sorted np.int32 array

    @property
    def flagged(self):
        return self.flags[0]

    def recomputed(self):
        """Blocks recomputed in each correction round r = 1..R (= flags[r-1])."""
        return self.flags[:-1]


def abft_spmv(A, enc: Encoded, x, inj: Inject | None = None, max_rounds: int = 4) -> SpmvResult:
    r = _CsrRef(A)
    x = np.ascontiguousarray(x, dtype=np.float64)
    nb = enc.nb
    y = np.empty(A.n)
    y_pre = np.empty(A.n)
    t1 = np.empty(nb)
    t2 = np.empty(nb)
    s = np.empty(nb)
    beta = C.c_double(0.0)
    fc = np.zeros(max_rounds + 1, dtype=np.int32)
    fl = np.zeros((max_rounds + 1) * max(nb, 1), dtype=np.int32)
    ist = inj._struct() if inj is not None else None
    st = lib().or_abft_spmv(r.ref(), enc.bs, _p(enc.row_ptr), _p(enc.col), _p(enc.val),
                            _p(enc.K), _p(x), C.byref(ist) if ist is not None else None,
                            max_rounds, _p(y), _p(y_pre), _p(t1), _p(t2), _p(s),
                            C.byref(beta), _p(fc), _p(fl))
    flags = [fl[q * nb: q * nb + fc[q]].copy() for q in range(max_rounds + 1)]
    return SpmvResult(st, y, y_pre, t1, t2, s, beta.value, flags)


@dataclass
class DenseEncoded:
    """Dense-check checksum (related work [30, 31]; oracle/abft_oracle.h)."""
    c: np.ndarray   # [n] column sums, PW over each column in row order (R23)
    k35: float      # [35]'s bound constant with m = N rows (R24)


def dense_encode(A) -> DenseEncoded:
    r = _CsrRef(A)
    c = np.empty(A.n)
    k = C.c_double(0.0)
    lib().or_dense_encode(r.ref(), _p(c), C.byref(k))
    return DenseEncoded(c, k.value)


@dataclass
class DenseResult:
    status: int
    y: np.ndarray          # after the last round
    y_pre: np.ndarray      # after round 0 (faults included)
    t1: float
    t2: float
    beta: float
    tau: float
    flag_rounds: np.ndarray  # [max_rounds+1] 1 where round r's check failed


def dense_spmv(A, enc: DenseEncoded, x, bound35: bool = False, inj: "Inject | None" = None,
               max_rounds: int = 4) -> DenseResult:
    """Dense check + complete recomputation."""
    r = _CsrRef(A)
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.empty(A.n)
    y_pre = np.empty(A.n)
    out = np.zeros(4)
    fr = np.zeros(max_rounds + 1, dtype=np.int32)
    ist = inj._struct() if inj is not None else None
    st = lib().or_dense_spmv(r.ref(), _p(enc.c), enc.k35, int(bound35), _p(x),
                             C.byref(ist) if ist is not None else None, max_rounds, _p(y),
                             _p(y_pre), _p(out), _p(fr))
    return DenseResult(st, y, y_pre, out[0], out[1], out[2], out[3], fr)


@dataclass
class PcgResult:
    status: int
    x: np.ndarray
    res_hist: np.ndarray
    iters: int
    spmv_calls: int
    flagged_blocks: int
    recomputed_blocks: int
    uncorrected_calls: int


def pcg(A, enc: Encoded, b, x0, diag=None, tol=1e-6, max_iter=0, inj: Inject | None = None,
        max_rounds=4, check=True, literal_stop=False) -> PcgResult:
    """or_pcg; literal_stop: stop when r^T r < tol (P:296 read literally)."""
    r = _CsrRef(A)
    b = np.ascontiguousarray(b, dtype=np.float64)
    x = np.array(x0, dtype=np.float64, copy=True)
    mi = max_iter if max_iter > 0 else 10 * A.n
    hist = np.zeros(mi + 1)
    stats = np.zeros(5, dtype=np.int64)
    d = None if diag is None else np.ascontiguousarray(diag, dtype=np.float64)
    ist = inj._struct() if inj is not None else None
    st = lib().or_pcg(r.ref(), enc.bs, _p(enc.row_ptr), _p(enc.col), _p(enc.val), _p(enc.K),
                      _p(b), _p(x), _p(d), tol, mi, C.byref(ist) if ist is not None else None,
                      max_rounds, (1 if check else 0) | (0x100 if literal_stop else 0),
                      _p(hist), _p(stats))
    it = int(stats[0])
    return PcgResult(st, x, hist[: it + 1].copy(), it, int(stats[1]), int(stats[2]),
                     int(stats[3]), int(stats[4]))


def pcg_cr(A, denc: DenseEncoded, b, x0, diag=None, tol=1e-6, max_iter=0,
           inj: "Inject | None" = None, ckpt_every: int = 20) -> "CrResult":
    """Checkpoint-rollback PCG baseline (abft_oracle.h or_pcg_cr).
    stats: iters, spmv_calls, rollbacks, executed, 0."""
    r = _CsrRef(A)
    n = A.n
    x = np.array(x0, dtype=np.float64, copy=True)
    b = np.ascontiguousarray(b, dtype=np.float64)
    mi = max_iter if max_iter > 0 else 10 * n
    hist = np.zeros(mi + 1)
    st = np.zeros(5, dtype=np.int64)
    dg = None if diag is None else np.ascontiguousarray(diag, dtype=np.float64)
    ist = inj._struct() if inj is not None else None
    status = lib().or_pcg_cr(r.ref(), _p(denc.c), _p(b), _p(x), _p(dg), tol, mi,
                             C.byref(ist) if ist is not None else None, ckpt_every, _p(hist),
                             _p(st))
    return CrResult(status, x, hist[: st[0] + 1], int(st[0]), int(st[1]), int(st[2]), int(st[3]))


@dataclass
class CrResult:
    status: int
    x: np.ndarray
    res_hist: np.ndarray
    iters: int        # iterations of the returned solution
    spmv_calls: int
    rollbacks: int
    executed: int     # executed iterations (re-executions count)


def dot_ranks(a, b, ranges) -> float:
    """Global dot product of the distributed PCG (R28): PW over the
    ranks (in rank order, padded with absent slots) of each rank's PW over
    its own rows.  One range [(0, n)] is the single-GPU PW dot (R2)."""
    prod = np.asarray(a, dtype=np.float64) * np.asarray(b, dtype=np.float64)
    return pw(np.array([pw(prod[r0:r1]) for r0, r1 in ranges], dtype=np.float64))


def pcg_ranks(A, b, x0, ranges, diag=None, tol=1e-6, max_iter=0) -> PcgResult:
    """Fault-free Jacobi-PCG (Saad Alg. 9.1, the paper's [19]) with
    every global reduction computed as `dot_ranks` over the row partition
    `ranges` -- the oracle of the distributed PCG.  Steps and
    rounding follow or_pcg line by line; without faults the protected SpMV's
    y is the plain SpMV (corrections recompute identical bits), so q = A p is
    `spmv`.  Status 0 / -5 (ENOCONV) / -7 (EBREAKDOWN) as or_pcg."""
    n = A.n
    b = np.ascontiguousarray(b, dtype=np.float64)
    x = np.array(x0, dtype=np.float64, copy=True)
    mi = max_iter if max_iter > 0 else 10 * n
    if diag is None:
        d = np.zeros(n)  # diag(A), a missing diagonal -> 0 (R21)
        rows = np.repeat(np.arange(n), np.diff(np.asarray(A.row_ptr, dtype=np.int64)))
        on = np.asarray(A.col) == rows
        d[rows[on]] = np.asarray(A.val)[on]
    else:
        d = np.asarray(diag, dtype=np.float64)
    calls = 1
    q = spmv(A, x)
    r = b - q
    z = r / d
    p = z.copy()
    rho = dot_ranks(r, z, ranges)
    thr = tol * np.sqrt(dot_ranks(b, b, ranges))
    res = np.sqrt(dot_ranks(r, r, ranges))
    hist = [res]
    it, status = 0, 0
    while not (res <= thr) and it < mi:
        if res != res:
            status = -7
            break
        q = spmv(A, p)
        calls += 1
        pq = dot_ranks(p, q, ranges)
        if not (pq > 0.0):
            status = -7
            break
        alpha = rho / pq
        x = x + alpha * p
        r = r - alpha * q
        z = r / d
        rho_new = dot_ranks(r, z, ranges)
        res = np.sqrt(dot_ranks(r, r, ranges))
        it += 1
        hist.append(res)
        beta = rho_new / rho
        rho = rho_new
        p = z + beta * p
    if status == 0 and not (res <= thr):
        status = -5
    return PcgResult(status, x, np.array(hist), it, calls, 0, 0, 0)


def pcg_cg1_ranks(A, b, x0, ranges, diag=None, tol=1e-6, max_iter=0) -> PcgResult:
    """Single-reduction Jacobi-PCG (Chronopoulos & Gear 1989, preconditioned
    form, R29 -- beyond the paper, which uses the
    textbook PCG of P:294-300).  The recurrence s = A p replaces the second
    reduction: per iteration the three dots (r, u), (r, r), (w, u) with
    u = M^-1 r, w = A u are one reduction.  Fault free; dots by `dot_ranks`.
        r0 = b - A x0, u0 = r0 / d, gamma0 = (r0, u0), res0 = ||r0||
        w0 = A u0, delta0 = (w0, u0), alpha0 = gamma0 / delta0, beta0 = 0,
        p = u0, s = w0
        j = 1, 2, ...: p = u + beta p; s = w + beta s; x = x + alpha p;
          r = r - alpha s; u = r / d; gamma' = (r, u); res = ||r||;
          w = A u; delta = (w, u); stop if res <= tol ||b||;
          beta = gamma' / gamma; alpha = gamma' / (delta - beta gamma' / alpha)
    In exact arithmetic the iterates are those of `pcg_ranks`; one SpMV more
    (w0).  Status 0 / -5 / -7 as or_pcg."""
    n = A.n
    b = np.ascontiguousarray(b, dtype=np.float64)
    x = np.array(x0, dtype=np.float64, copy=True)
    mi = max_iter if max_iter > 0 else 10 * n
    if diag is None:
        d = np.zeros(n)  # diag(A), a missing diagonal -> 0 (R21)
        rows = np.repeat(np.arange(n), np.diff(np.asarray(A.row_ptr, dtype=np.int64)))
        on = np.asarray(A.col) == rows
        d[rows[on]] = np.asarray(A.val)[on]
    else:
        d = np.asarray(diag, dtype=np.float64)
    r = b - spmv(A, x)
    u = r / d
    gamma = dot_ranks(r, u, ranges)
    thr = tol * np.sqrt(dot_ranks(b, b, ranges))
    res = np.sqrt(dot_ranks(r, r, ranges))
    hist, it, calls = [res], 0, 1
    if res <= thr:
        return PcgResult(0, x, np.array(hist), 0, calls, 0, 0, 0)
    w = spmv(A, u)
    calls += 1
    delta = dot_ranks(w, u, ranges)
    if not (delta > 0.0):
        return PcgResult(-7, x, np.array(hist), 0, calls, 0, 0, 0)
    alpha, beta = gamma / delta, 0.0
    p, s = u.copy(), w.copy()
    status = -5
    while it < mi:
        p = u + beta * p
        s = w + beta * s
        x = x + alpha * p
        r = r - alpha * s
        u = r / d
        g_new = dot_ranks(r, u, ranges)
        rr = dot_ranks(r, r, ranges)
        w = spmv(A, u)
        calls += 1
        delta = dot_ranks(w, u, ranges)
        it += 1
        res = np.sqrt(rr)
        hist.append(res)
        if res <= thr:
            status = 0
            break
        if res != res:
            status = -7
            break
        if it >= mi:
            break
        beta = g_new / gamma
        den = delta - beta * g_new / alpha
        if not (den > 0.0):
            status = -7
            break
        alpha = g_new / den
        gamma = g_new
    return PcgResult(status, x, np.array(hist), it, calls, 0, 0, 0)
