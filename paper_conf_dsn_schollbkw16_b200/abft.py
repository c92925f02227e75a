"""Thin Python binding of libabft.so (include/abft.h): argument marshalling
only.  Every step of the path runs in the library's CUDA kernels; there is no
CPU fallback -- if libabft.so is missing or no CUDA device is present, every
call raises.

PyTorch provides device memory and the current stream (plumbing only).
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

import numpy as np

from . import _build

_LIB = None

OK, EINVAL, ECUDA, ENOMEM, ENOTSUP, ENOCONV, EUNCORRECTED, EBREAKDOWN, ENCCL = (
    0, -1, -2, -3, -4, -5, -6, -7, -8)
NOCHECK, CHECK, AUTOCORRECT, DEBUG_CHECKSUMS, DEFER_FINISH = 0, 1, 2, 4, 8
DENSE_BOUND35 = 16  # abft_spmv_dense: tau = K35 ||x|| ([35]) instead of ||x|| ([30])
INJ_NONE, INJ_LIST, INJ_RATE, INJ_RESIDENT = 0, 1, 2, 3
PCG_LITERAL_STOP = 0x100

SYMBOLS = [
    "abft_encode", "abft_spmv", "abft_correct", "abft_flags", "abft_beta",
    "abft_checksum_matrix", "abft_debug_checksums", "abft_spmv_host", "abft_pcg",
    "abft_destroy", "abft_memcpy", "abft_status_string", "abft_last_cuda_error",
    "abft_burst_table", "abft_version", "abft_info", "abft_beta_partial", "abft_finish",
    "abft_dense_encode", "abft_spmv_dense", "abft_dense_result", "abft_dense_checksum",
    "abft_spmv_host_pipelined", "abft_host_alloc", "abft_host_free",
    "abft_pcg_dist_begin", "abft_pcg_dist_local", "abft_pcg_dist_combine",
    "abft_pcg_dist_status", "abft_poisson_table", "abft_rate_chunk", "abft_health",
    "abft_dist_unique_id", "abft_dist_create", "abft_dist_destroy", "abft_dist_encode",
    "abft_dist_needs", "abft_dist_set_send", "abft_dist_operand", "abft_dist_spmv",
    "abft_dist_begin", "abft_dist_buffers", "abft_dist_partial", "abft_dist_end", "abft_dist_pcg",
    "abft_halo_plan", "abft_inject_prepare", "abft_inject_list", "abft_inject_clear_masks",
]
PCG_PHASE_INIT, PCG_PHASE_DOT, PCG_PHASE_UPDATE, PCG_PHASE_P = 0, 1, 2, 3
PCG_PHASE_CG1_UPDATE, PCG_PHASE_CG1_DOT = 4, 5  # single-reduction variant
ENCODE_C_CSR = 1
CFMT_NAMES = {0: "csr-f64", 1: "int8+u16", 2: "int16+u16", 3: "f32+u16", 4: "f64+u16",
              5: "int8+pos", 6: "int16+pos", 7: "f32+pos", 8: "f64+pos"}


class AbftError(RuntimeError):
    def __init__(self, status, where):
        self.status = status
        msg = lib().abft_status_string(status).decode()
        if status == ECUDA:
            msg += ": " + lib().abft_last_cuda_error().decode()
        super().__init__(f"{where}: {msg} ({status})")


class _Csr(C.Structure):
    _fields_ = [("n", C.c_int64), ("nnz", C.c_int64), ("row_ptr", C.c_void_p),
                ("col_idx", C.c_void_p), ("val", C.c_void_p), ("n_cols", C.c_int64),
                ("x_offset", C.c_int64)]


class _Inj(C.Structure):
    _fields_ = [("mode", C.c_uint32), ("seed", C.c_uint64), ("call", C.c_uint64),
                ("lambda_", C.c_double), ("targets", C.c_uint32), ("n_list", C.c_int64),
                ("list_round", C.c_void_p), ("list_target", C.c_void_p),
                ("list_index", C.c_void_p), ("list_mask", C.c_void_p)]


class Info(C.Structure):
    _fields_ = [("n", C.c_int64), ("nnz", C.c_int64), ("nb", C.c_int64), ("nnz_c", C.c_int64),
                ("block_size", C.c_int32), ("c_format", C.c_int32), ("c_bytes", C.c_int64),
                ("groups", C.c_int64), ("general_groups", C.c_int64), ("lean", C.c_int32),
                ("max_rounds", C.c_int32), ("irr_groups", C.c_int64), ("lean_short", C.c_int32),
                ("lean_runs", C.c_int32), ("stream", C.c_int32), ("stream_g", C.c_int32),
                ("stream_stages", C.c_int32), ("col_perm", C.c_int32),
                ("pos_exc_rows", C.c_int64), ("stream_plain_bytes", C.c_int64),
                ("stream_check_bytes", C.c_int64), ("hub_chunks", C.c_int64)]

    def as_dict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_}
        d["c_format_name"] = CFMT_NAMES.get(self.c_format, "?")
        return d


class PcgStats(C.Structure):
    _fields_ = [("iters", C.c_int64), ("spmv_calls", C.c_int64), ("flagged_blocks", C.c_int64),
                ("recomputed_blocks", C.c_int64), ("uncorrected_calls", C.c_int64),
                ("converged", C.c_int32), ("final_residual", C.c_double)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


def lib_path() -> str:
    # ABFT_LIB: alternative build of the same library (tuning experiments)
    return os.environ.get("ABFT_LIB", _build.LIB)


def lib():
    """Load libabft.so (raises if it has not been built -- no fallback)."""
    global _LIB
    if _LIB is None:
        path = lib_path()
        if not os.path.exists(path):
            raise RuntimeError(f"libabft.so not built at {path}; run __graft_entry__.build()")
        L = C.CDLL(path)
        P, i32, i64, u32, d = C.c_void_p, C.c_int32, C.c_int64, C.c_uint32, C.c_double
        st = C.c_int
        L.abft_encode.restype = st
        L.abft_encode.argtypes = [P, i32, i32, u32, P, C.POINTER(P)]
        L.abft_spmv.restype = st
        L.abft_spmv.argtypes = [P, P, P, P, P, u32, P]
        L.abft_correct.restype = st
        L.abft_correct.argtypes = [P, P, P, i32, P, P]
        L.abft_flags.restype = st
        L.abft_flags.argtypes = [P, i32, C.POINTER(P), C.POINTER(P)]
        L.abft_beta.restype = st
        L.abft_beta.argtypes = [P, P, C.POINTER(P)]
        L.abft_checksum_matrix.restype = st
        L.abft_checksum_matrix.argtypes = [P, C.POINTER(P), C.POINTER(P), C.POINTER(P),
                                           C.POINTER(P), C.POINTER(i64), C.POINTER(i64)]
        L.abft_debug_checksums.restype = st
        L.abft_debug_checksums.argtypes = [P, C.POINTER(P), C.POINTER(P)]
        L.abft_spmv_host.restype = st
        L.abft_spmv_host.argtypes = [P, P, P, P, u32, P]
        L.abft_pcg.restype = st
        L.abft_pcg.argtypes = [P, P, P, P, d, i64, P, i32, P, C.POINTER(PcgStats), P]
        L.abft_pcg_dist_begin.restype = st
        L.abft_pcg_dist_begin.argtypes = [P, P, P, P, P, P, d, i64, i32, P, P]
        L.abft_pcg_dist_local.restype = st
        L.abft_pcg_dist_local.argtypes = [P, i32, i64, P, P]
        L.abft_pcg_dist_combine.restype = st
        L.abft_pcg_dist_combine.argtypes = [P, i32, i64, P, i32, P]
        L.abft_pcg_dist_status.restype = st
        L.abft_pcg_dist_status.argtypes = [P, C.POINTER(i32), C.POINTER(PcgStats), P]
        L.abft_destroy.restype = st
        L.abft_destroy.argtypes = [P]
        L.abft_memcpy.restype = st
        L.abft_memcpy.argtypes = [P, P, i64, P]
        L.abft_status_string.restype = C.c_char_p
        L.abft_status_string.argtypes = [st]
        L.abft_last_cuda_error.restype = C.c_char_p
        L.abft_burst_table.argtypes = [P]
        L.abft_poisson_table.restype = i32
        L.abft_poisson_table.argtypes = [d, P, i32]
        L.abft_rate_chunk.restype = i64
        L.abft_rate_chunk.argtypes = [d]
        L.abft_version.restype = C.c_char_p
        L.abft_info.restype = st
        L.abft_info.argtypes = [P, C.POINTER(Info)]
        L.abft_beta_partial.restype = st
        L.abft_beta_partial.argtypes = [P, P, P]
        L.abft_host_alloc.restype = st
        L.abft_host_alloc.argtypes = [i64, C.POINTER(P)]
        L.abft_host_free.restype = st
        L.abft_host_free.argtypes = [P]
        L.abft_spmv_host_pipelined.restype = st
        L.abft_spmv_host_pipelined.argtypes = [P, P, P, i32, P, u32, P]
        L.abft_dense_encode.restype = st
        L.abft_dense_encode.argtypes = [P, P]
        L.abft_spmv_dense.restype = st
        L.abft_spmv_dense.argtypes = [P, P, P, P, u32, P]
        L.abft_dense_result.restype = st
        L.abft_dense_result.argtypes = [P, P, P, P, P]
        L.abft_dense_checksum.restype = st
        L.abft_dense_checksum.argtypes = [P, C.POINTER(P)]
        L.abft_finish.restype = st
        L.abft_health.restype = st
        L.abft_health.argtypes = [P, P, C.POINTER(i32)]
        PI64 = C.POINTER(i64)
        L.abft_dist_unique_id.restype = st
        L.abft_dist_unique_id.argtypes = [P]
        L.abft_dist_create.restype = st
        L.abft_dist_create.argtypes = [i32, i32, P, P, C.POINTER(P)]
        L.abft_dist_destroy.restype = st
        L.abft_dist_destroy.argtypes = [P]
        L.abft_dist_encode.restype = st
        L.abft_dist_encode.argtypes = [P, P, i32, i32, u32, P, C.POINTER(P)]
        L.abft_dist_needs.restype = st
        L.abft_dist_needs.argtypes = [P, i32, PI64, P]
        L.abft_dist_set_send.restype = st
        L.abft_dist_set_send.argtypes = [P, i32, P, i64]
        L.abft_dist_operand.restype = st
        L.abft_dist_operand.argtypes = [P, C.POINTER(P), PI64, PI64]
        L.abft_dist_spmv.restype = st
        L.abft_dist_spmv.argtypes = [P, P, P, P, u32, P]
        L.abft_dist_begin.restype = st
        L.abft_dist_begin.argtypes = [P, P, P]
        L.abft_dist_buffers.restype = st
        L.abft_dist_buffers.argtypes = [P, i32, C.POINTER(P), PI64, C.POINTER(P), PI64]
        L.abft_dist_partial.restype = st
        L.abft_dist_partial.argtypes = [P, C.POINTER(P)]
        L.abft_dist_end.restype = st
        L.abft_dist_end.argtypes = [P, P, P, P, u32, P]
        L.abft_dist_pcg.restype = st
        L.abft_dist_pcg.argtypes = [P, P, P, P, d, i64, P, i32, i32, P, C.POINTER(PcgStats), P]
        L.abft_inject_prepare.restype = st
        L.abft_inject_prepare.argtypes = [P, P, u32, P]
        L.abft_inject_list.restype = st
        L.abft_inject_list.argtypes = [P, C.POINTER(P), C.POINTER(P), C.POINTER(P),
                                       C.POINTER(i32), C.POINTER(i32)]
        L.abft_inject_clear_masks.restype = st
        L.abft_inject_clear_masks.argtypes = [P, P]
        L.abft_halo_plan.restype = st
        L.abft_halo_plan.argtypes = [i32, i32, P, P, i64, P, PI64, PI64, P, P, P, i64]
        L.abft_finish.argtypes = [P, P, P, P, i32, i32, P, P]
        _LIB = L
    return _LIB


def _check(status, where):
    if status != OK:
        raise AbftError(status, where)


def _stream(stream=None):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return C.c_void_p(s.cuda_stream)


def _ptr(t):
    return None if t is None else C.c_void_p(t.data_ptr())


def _vec(t, min_len, what, optional=False):
    """Device pointer of a float64 tensor the library reads or writes:
    the C ABI only sees raw pointers, so dtype, device, contiguity and length
    are checked here (ValueError instead of an out-of-bounds access)."""
    if t is None:
        if optional:
            return None
        raise ValueError(f"{what}: tensor required")
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda or t.dtype != torch.float64:
        raise ValueError(f"{what}: expected a CUDA float64 tensor")
    if not t.is_contiguous():
        raise ValueError(f"{what}: tensor must be contiguous")
    if t.numel() < min_len:
        raise ValueError(f"{what}: {t.numel()} elements, need >= {min_len}")
    return C.c_void_p(t.data_ptr())


def burst_table() -> np.ndarray:
    t = np.zeros(65, dtype=np.uint64)
    lib().abft_burst_table(t.ctypes.data_as(C.c_void_p))
    return t


def poisson_table(mu: float, cap: int = 1024) -> np.ndarray:
    t = np.zeros(cap, dtype=np.uint64)
    k = lib().abft_poisson_table(mu, t.ctypes.data_as(C.c_void_p), cap)
    return t[:k].copy()


def rate_chunk(lam: float) -> int:
    return int(lib().abft_rate_chunk(lam))


class Inject:
    """Fault injection spec (abft_inject_t).  LIST plans are FaultPlan objects
    from `inputs`; RATE mode uses the device-side Philox injector."""

    def __init__(self, mode=INJ_NONE, seed=0, call=0, lam=0.0, targets=0b111, plan=None):
        self.mode, self.seed, self.call, self.lam, self.targets, self.plan = (
            mode, seed, call, lam, targets, plan)

    @staticmethod
    def from_plan(plan):
        return Inject(mode=INJ_LIST, plan=plan)

    @staticmethod
    def rate(seed, lam, targets=0b111, call=0):
        return Inject(mode=INJ_RATE, seed=seed, call=call, lam=lam, targets=targets)

    @staticmethod
    def resident():
        """The device fault list the handle's last injecting call built."""
        return Inject(mode=INJ_RESIDENT)

    def struct(self):
        s = _Inj()
        s.mode, s.seed, s.call, s.lambda_, s.targets = (self.mode, self.seed, self.call,
                                                        self.lam, self.targets)
        s.n_list = 0
        if self.mode == INJ_LIST and self.plan is not None and len(self.plan):
            self._keep = (np.ascontiguousarray(self.plan.round, np.int32),
                          np.ascontiguousarray(self.plan.target, np.int32),
                          np.ascontiguousarray(self.plan.index, np.int64),
                          np.ascontiguousarray(self.plan.mask, np.uint64))
            s.n_list = len(self.plan)
            (s.list_round, s.list_target, s.list_index, s.list_mask) = [
                a.ctypes.data for a in self._keep]
        return s


@dataclass
class CsrDevice:
    """CSR matrix resident on the device (torch tensors).  A row-block shard
    has n rows over n_cols local columns, its own rows' x entries starting at
    x_offset (include/abft.h abft_csr_t)."""
    n: int
    row_ptr: object
    col: object
    val: object
    n_cols: int = 0
    x_offset: int = 0

    @property
    def nnz(self):
        return int(self.col.numel())

    @staticmethod
    def from_host(A, device="cuda"):
        import torch
        return CsrDevice(A.n, torch.from_numpy(np.ascontiguousarray(A.row_ptr)).to(device),
                         torch.from_numpy(np.ascontiguousarray(A.col)).to(device),
                         torch.from_numpy(np.ascontiguousarray(A.val)).to(device))


class Handle:
    """abft_handle_t: owns C, K and scratch; keeps A alive (the library
    re-reads it in correction and PCG)."""

    def __init__(self, A: CsrDevice, block_size: int = 32, max_rounds: int = 4, stream=None,
                 c_csr: bool = False, _raw=None):
        self.A = A
        self.n = A.n
        self.n_cols = A.n_cols if A.n_cols > 0 else A.n
        self.block_size = block_size
        self.nb = (A.n + block_size - 1) // block_size
        self.max_rounds = max_rounds if max_rounds > 0 else 4
        if _raw is not None:  # a handle the library built (abft_dist_encode)
            self._h = _raw
            return
        csr = _Csr(A.n, A.nnz, A.row_ptr.data_ptr(), A.col.data_ptr() if A.nnz else 0,
                   A.val.data_ptr() if A.nnz else 0, A.n_cols, A.x_offset)
        h = C.c_void_p()
        _check(lib().abft_encode(C.byref(csr), block_size, max_rounds,
                                 ENCODE_C_CSR if c_csr else 0, _stream(stream), C.byref(h)),
               "abft_encode")
        self._h = h

    def inject_prepare(self, inject: Inject, mode=CHECK, stream=None):
        inj = inject.struct()
        _check(lib().abft_inject_prepare(self._h, C.byref(inj), mode, _stream(stream)),
               "abft_inject_prepare")

    def inject_clear_masks(self, stream=None):
        """Zero the resident list's masks (harness control: same lookups, no faults)."""
        _check(lib().abft_inject_clear_masks(self._h, _stream(stream)), "abft_inject_clear_masks")

    def inject_list(self, stream=None):
        """The resident device fault list as host arrays (keys, masks):
        decoded (round, target, index, mask)."""
        k, m, nd = C.c_void_p(), C.c_void_p(), C.c_void_p()
        nh, cap = C.c_int32(), C.c_int32()
        _check(lib().abft_inject_list(self._h, C.byref(k), C.byref(m), C.byref(nd), C.byref(nh),
                                      C.byref(cap)), "abft_inject_list")
        n = nh.value
        if nd.value:
            n = min(int(self._d2h(nd, 1, np.int32, stream)[0]), cap.value)
        keys = self._d2h(k, n, np.uint64, stream)
        masks = self._d2h(m, n, np.uint64, stream)
        return (keys >> np.uint64(58)).astype(np.int32), ((keys >> np.uint64(56)) & np.uint64(3)).astype(
            np.int32), (keys & np.uint64((1 << 56) - 1)).astype(np.int64), masks

    def health(self, stream=None) -> int:
        """1 if a grid barrier timed out since the last call (abft_health)."""
        e = C.c_int32(0)
        _check(lib().abft_health(self._h, _stream(stream), C.byref(e)), "abft_health")
        return e.value

    def info(self) -> dict:
        inf = Info()
        _check(lib().abft_info(self._h, C.byref(inf)), "abft_info")
        return inf.as_dict()

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            lib().abft_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- hot path --------------------------------------------------------
    def spmv(self, x, y=None, x_norm=None, inject: Inject | None = None, mode=CHECK, stream=None):
        import torch
        if y is None:
            y = torch.empty(self.n, dtype=torch.float64, device=x.device)
        px, py = _vec(x, self.n_cols, "x"), _vec(y, self.n, "y")
        pn = _vec(x_norm, 1, "x_norm", optional=True)
        inj = inject.struct() if inject is not None else None
        _check(lib().abft_spmv(self._h, px, py, pn,
                               C.byref(inj) if inj is not None else None, mode, _stream(stream)),
               "abft_spmv")
        return y

    def beta_partial(self, out, stream=None):
        """Enqueue this shard's PW sum of x_i^2 (after a DEFER_FINISH spmv)
        into the device f64 tensor `out` (one element)."""
        _check(lib().abft_beta_partial(self._h, _vec(out, 1, "out"), _stream(stream)),
               "abft_beta_partial")
        return out

    def finish(self, x, y, parts, rounds=None, inject: Inject | None = None, stream=None):
        """Steps 4-5 with beta = sqrt(PW(parts)) (parts: device f64 tensor of
        the per-rank partials in rank order)."""
        inj = inject.struct() if inject is not None else None
        r = self.max_rounds if rounds is None else rounds
        _check(lib().abft_finish(self._h, _vec(x, self.n_cols, "x"), _vec(y, self.n, "y"),
                                 _vec(parts, 1, "parts"), int(parts.numel()), r,
                                 C.byref(inj) if inj is not None else None, _stream(stream)),
               "abft_finish")
        return y

    def correct(self, x, y, max_rounds=0, inject: Inject | None = None, stream=None):
        inj = inject.struct() if inject is not None else None
        _check(lib().abft_correct(self._h, _vec(x, self.n_cols, "x"), _vec(y, self.n, "y"),
                                  max_rounds,
                                  C.byref(inj) if inj is not None else None, _stream(stream)),
               "abft_correct")
        return y

    def spmv_host(self, x_host: np.ndarray, y_host: np.ndarray, mode=CHECK | AUTOCORRECT,
                  stream=None) -> int:
        nf = C.c_int32(0)
        _check(lib().abft_spmv_host(self._h, x_host.ctypes.data_as(C.c_void_p),
                                    y_host.ctypes.data_as(C.c_void_p), C.byref(nf), mode,
                                    _stream(stream)), "abft_spmv_host")
        return nf.value

    def spmv_host_pipelined(self, x_hosts, y_hosts, mode=CHECK | AUTOCORRECT,
                            stream=None) -> np.ndarray:
        """len(x_hosts) products with host numpy buffers, copies overlapped
        across steps (include/abft.h); returns the round-0 flag counts."""
        k = len(x_hosts)
        xs = (C.c_void_p * k)(*[a.ctypes.data for a in x_hosts])
        ys = (C.c_void_p * k)(*[a.ctypes.data for a in y_hosts])
        nf = np.zeros(k, dtype=np.int32)
        _check(lib().abft_spmv_host_pipelined(self._h, xs, ys, k, nf.ctypes.data_as(C.c_void_p),
                                              mode, _stream(stream)), "abft_spmv_host_pipelined")
        return nf

    # -- results (device-resident; copied out on request) ----------------
    def _d2h(self, ptr, count, dtype, stream=None):
        out = np.empty(count, dtype=dtype)
        if count:
            _check(lib().abft_memcpy(out.ctypes.data_as(C.c_void_p), ptr, out.nbytes,
                                     _stream(stream)), "abft_memcpy")
        return out

    def flags(self, round_: int = 0, stream=None) -> np.ndarray:
        """Sorted flagged-block indices of round `round_` (copied to host)."""
        f, nf = C.c_void_p(), C.c_void_p()
        _check(lib().abft_flags(self._h, round_, C.byref(f), C.byref(nf)), "abft_flags")
        cnt = int(self._d2h(nf, 1, np.int32, stream)[0])
        return np.sort(self._d2h(f, cnt, np.int32, stream))

    def all_flags(self, stream=None):
        return [self.flags(r, stream) for r in range(self.max_rounds + 1)]

    def flag_count_ptr(self, round_: int = 0) -> int:
        f, nf = C.c_void_p(), C.c_void_p()
        _check(lib().abft_flags(self._h, round_, C.byref(f), C.byref(nf)), "abft_flags")
        return nf.value

    def beta(self, stream=None) -> float:
        b = C.c_void_p()
        _check(lib().abft_beta(self._h, _stream(stream), C.byref(b)), "abft_beta")
        return float(self._d2h(b, 1, np.float64, stream)[0])

    def checksum_matrix(self, stream=None):
        rp, col, val, K = C.c_void_p(), C.c_void_p(), C.c_void_p(), C.c_void_p()
        nnz_c, nb = C.c_int64(), C.c_int64()
        _check(lib().abft_checksum_matrix(self._h, C.byref(rp), C.byref(col), C.byref(val),
                                          C.byref(K), C.byref(nnz_c), C.byref(nb)),
               "abft_checksum_matrix")
        return (self._d2h(rp, nb.value + 1, np.int32, stream),
                self._d2h(col, nnz_c.value, np.int32, stream),
                self._d2h(val, nnz_c.value, np.float64, stream),
                self._d2h(K, nb.value, np.float64, stream))

    def debug_checksums(self, stream=None):
        t1, t2 = C.c_void_p(), C.c_void_p()
        _check(lib().abft_debug_checksums(self._h, C.byref(t1), C.byref(t2)),
               "abft_debug_checksums")
        return (self._d2h(t1, self.nb, np.float64, stream),
                self._d2h(t2, self.nb, np.float64, stream))

    # -- related-work baseline: dense check + complete recomputation -------
    def dense_encode(self, stream=None):
        """Build c = 1^T A and K35 for the dense check (include/abft.h)."""
        _check(lib().abft_dense_encode(self._h, _stream(stream)), "abft_dense_encode")
        return self

    def spmv_dense(self, x, y=None, inject: Inject | None = None, correct=True, bound35=False,
                   stream=None):
        import torch
        if y is None:
            y = torch.empty(self.n, dtype=torch.float64, device=x.device)
        inj = inject.struct() if inject is not None else None
        mode = (AUTOCORRECT if correct else 0) | (DENSE_BOUND35 if bound35 else 0)
        _check(lib().abft_spmv_dense(self._h, _vec(x, self.n_cols, "x"), _vec(y, self.n, "y"),
                                     C.byref(inj) if inj is not None else None, mode,
                                     _stream(stream)), "abft_spmv_dense")
        return y

    def dense_result(self, stream=None) -> dict:
        out = np.zeros(4)
        fr = np.zeros(self.max_rounds + 1, dtype=np.int32)
        k = C.c_double(0.0)
        _check(lib().abft_dense_result(self._h, out.ctypes.data_as(C.c_void_p),
                                       fr.ctypes.data_as(C.c_void_p), C.byref(k),
                                       _stream(stream)), "abft_dense_result")
        return {"t1": out[0], "t2": out[1], "beta": out[2], "tau": out[3], "flag_rounds": fr,
                "k35": k.value}

    def dense_checksum(self, stream=None) -> np.ndarray:
        c = C.c_void_p()
        _check(lib().abft_dense_checksum(self._h, C.byref(c)), "abft_dense_checksum")
        return self._d2h(c, self.n, np.float64, stream)

    # -- PCG ----------------------------------------------------------------
    def pcg(self, b, x, diag=None, tol=1e-6, max_iter=0, inject: Inject | None = None,
            check=True, res_hist=None, stream=None, literal_stop=False):
        # check: True = the method's protected SpMV, False = unprotected,
        # "checkpoint" = dense-check checkpoint-rollback baseline (
        # needs dense_encode(); stats: flagged_blocks = rollbacks,
        # recomputed_blocks = discarded iterations).  literal_stop: stop when
        # r^T r < tol (P:296 read literally) instead of ||r|| <= tol ||b||.
        st = PcgStats()
        inj = inject.struct() if inject is not None else None
        mode = (2 if check == "checkpoint" else (1 if check else 0)) | (
            PCG_LITERAL_STOP if literal_stop else 0)
        mi = max_iter if max_iter > 0 else 10 * self.n
        status = lib().abft_pcg(self._h, _vec(b, self.n, "b"), _vec(x, self.n, "x"),
                                _vec(diag, self.n, "diag", optional=True), tol, max_iter,
                                C.byref(inj) if inj is not None else None, mode,
                                _vec(res_hist, mi + 1, "res_hist", optional=True), C.byref(st),
                                _stream(stream))
        if status not in (OK, ENOCONV, EBREAKDOWN):
            _check(status, "abft_pcg")
        return status, st.as_dict()

    # -- distributed PCG steps (abft_pcg_dist_*; parallel.DistPcg drives them)
    def pcg_dist_begin(self, b, x, pext, q, diag=None, tol=1e-6, max_iter=1, check=True,
                       res_hist=None, stream=None):
        # pext / q: tensors or raw device pointers (the library-owned operand)
        rp = lambda t: C.c_void_p(t) if isinstance(t, int) else _ptr(t)  # noqa: E731
        _check(lib().abft_pcg_dist_begin(self._h, _ptr(b), _ptr(x), rp(pext), rp(q),
                                         _ptr(diag), tol, max_iter, 1 if check else 0,
                                         _ptr(res_hist), _stream(stream)), "abft_pcg_dist_begin")

    def pcg_dist_local(self, phase, it, send=None, stream=None):
        _check(lib().abft_pcg_dist_local(self._h, phase, it, _ptr(send), _stream(stream)),
               "abft_pcg_dist_local")

    def pcg_dist_combine(self, phase, it, recv, world, stream=None):
        _check(lib().abft_pcg_dist_combine(self._h, phase, it, _ptr(recv), world,
                                           _stream(stream)), "abft_pcg_dist_combine")

    def pcg_dist_status(self, stream=None):
        st, state = PcgStats(), C.c_int32(0)
        _check(lib().abft_pcg_dist_status(self._h, C.byref(state), C.byref(st),
                                          _stream(stream)), "abft_pcg_dist_status")
        return state.value, st.as_dict()


# ---------------------------------------------------------------------------
# Multi-GPU row-block shards (include/abft.h "Multi-GPU"): the halo plan, the
# pack, the NCCL exchange and the distributed PCG run in the library.
# ---------------------------------------------------------------------------
def dist_unique_id() -> bytes:
    buf = (C.c_char * 128)()
    _check(lib().abft_dist_unique_id(buf), "abft_dist_unique_id")
    return bytes(buf)


def halo_plan(rank: int, world: int, ranges, col):
    """Host-only local column order of a shard (abft_halo_plan): returns
    (local_col, n_below, n_above, recv_start[world], recv_count[world], halo)."""
    rg = np.ascontiguousarray(ranges, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    nb, na = C.c_int64(), C.c_int64()
    rs = np.zeros(world, np.int64)
    rc = np.zeros(world, np.int64)
    local = np.zeros(max(col.size, 1), np.int32)
    _check(lib().abft_halo_plan(rank, world, rg.ctypes.data, col.ctypes.data, col.size,
                                local.ctypes.data, C.byref(nb), C.byref(na), rs.ctypes.data,
                                rc.ctypes.data, None, 0), "abft_halo_plan")
    halo = np.zeros(max(nb.value + na.value, 1), np.int64)
    _check(lib().abft_halo_plan(rank, world, rg.ctypes.data, col.ctypes.data, col.size,
                                local.ctypes.data, C.byref(nb), C.byref(na), rs.ctypes.data,
                                rc.ctypes.data, halo.ctypes.data, halo.size), "abft_halo_plan")
    return local[:col.size], nb.value, na.value, rs, rc, halo[:nb.value + na.value]


class Dist:
    """abft_dist_t: this rank's place in the row partition and (nccl_id given)
    an NCCL communicator over the ranks."""

    def __init__(self, rank: int, world: int, ranges, nccl_id: bytes | None = None):
        self.rank, self.world = rank, world
        self.ranges = np.ascontiguousarray(ranges, dtype=np.int64)
        assert self.ranges.size == world + 1
        d = C.c_void_p()
        idbuf = None
        if nccl_id is not None:
            idbuf = (C.c_char * 128).from_buffer_copy(nccl_id)
        _check(lib().abft_dist_create(rank, world, self.ranges.ctypes.data, idbuf, C.byref(d)),
               "abft_dist_create")
        self._d = d
        self.nccl = nccl_id is not None

    @property
    def row0(self):
        return int(self.ranges[self.rank])

    @property
    def row1(self):
        return int(self.ranges[self.rank + 1])

    def encode(self, rows: "CsrDevice", block_size: int = 32, max_rounds: int = 4,
               c_csr: bool = False, stream=None) -> "DistHandle":
        """rows: this rank's rows, GLOBAL column indices (device CSR)."""
        csr = _Csr(rows.n, rows.nnz, rows.row_ptr.data_ptr(),
                   rows.col.data_ptr() if rows.nnz else 0,
                   rows.val.data_ptr() if rows.nnz else 0, 0, 0)
        h = C.c_void_p()
        _check(lib().abft_dist_encode(self._d, C.byref(csr), block_size, max_rounds,
                                      ENCODE_C_CSR if c_csr else 0, _stream(stream), C.byref(h)),
               "abft_dist_encode")
        return DistHandle(self, rows, block_size, max_rounds, h)

    def close(self):
        if getattr(self, "_d", None) and self._d.value:
            lib().abft_dist_destroy(self._d)
            self._d = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class DistHandle(Handle):
    """A shard handle from abft_dist_encode.  Device pointers of the
    library-owned operand / exchange buffers are plain ints."""

    def __init__(self, dist: Dist, rows, block_size, max_rounds, raw):
        super().__init__(rows, block_size, max_rounds, _raw=raw)
        self.dist = dist  # the communicator outlives the handle
        x, nc, off = C.c_void_p(), C.c_int64(), C.c_int64()
        _check(lib().abft_dist_operand(self._h, C.byref(x), C.byref(nc), C.byref(off)),
               "abft_dist_operand")
        self.x_ext_ptr, self.n_cols, self.own_offset = x.value, nc.value, off.value

    def own_ptr(self) -> int:
        return self.x_ext_ptr + 8 * self.own_offset

    def needs(self, peer: int) -> np.ndarray:
        c = C.c_int64()
        _check(lib().abft_dist_needs(self._h, peer, C.byref(c), None), "abft_dist_needs")
        out = np.zeros(max(c.value, 1), np.int64)
        _check(lib().abft_dist_needs(self._h, peer, C.byref(c), out.ctypes.data), "abft_dist_needs")
        return out[:c.value]

    def set_send(self, peer: int, idx) -> None:
        idx = np.ascontiguousarray(idx, dtype=np.int64)
        _check(lib().abft_dist_set_send(self._h, peer, idx.ctypes.data if idx.size else None,
                                        idx.size), "abft_dist_set_send")

    def buffers(self, peer: int):
        """(send ptr, send count, recv ptr, recv count) for `peer` (device)."""
        sp, sc, rp, rc = C.c_void_p(), C.c_int64(), C.c_void_p(), C.c_int64()
        _check(lib().abft_dist_buffers(self._h, peer, C.byref(sp), C.byref(sc), C.byref(rp),
                                       C.byref(rc)), "abft_dist_buffers")
        return sp.value, sc.value, rp.value, rc.value

    def partial_ptr(self) -> int:
        p = C.c_void_p()
        _check(lib().abft_dist_partial(self._h, C.byref(p)), "abft_dist_partial")
        return p.value

    def begin(self, x_own=None, stream=None):
        _check(lib().abft_dist_begin(self._h, _vec(x_own, self.n, "x_own", optional=True),
                                     _stream(stream)), "abft_dist_begin")

    def end(self, y, parts, inject: Inject | None = None, mode=CHECK | AUTOCORRECT, stream=None):
        inj = inject.struct() if inject is not None else None
        _check(lib().abft_dist_end(self._h, _vec(y, self.n, "y"),
                                   _vec(parts, self.dist.world, "parts"),
                                   C.byref(inj) if inj is not None else None, mode,
                                   _stream(stream)), "abft_dist_end")
        return y

    def dist_spmv(self, x_own, y, inject: Inject | None = None, mode=CHECK | AUTOCORRECT,
                  stream=None):
        inj = inject.struct() if inject is not None else None
        _check(lib().abft_dist_spmv(self._h, _vec(x_own, self.n, "x_own", optional=True),
                                    _vec(y, self.n, "y"),
                                    C.byref(inj) if inj is not None else None, mode,
                                    _stream(stream)), "abft_dist_spmv")
        return y

    def dist_pcg(self, b, x, diag=None, tol=1e-6, max_iter=0, inject: Inject | None = None,
                 check=True, res_hist=None, stream=None, variant="pcg"):
        st = PcgStats()
        inj = inject.struct() if inject is not None else None
        status = lib().abft_dist_pcg(self._h, _vec(b, self.n, "b"), _vec(x, self.n, "x"),
                                     _vec(diag, self.n, "diag", optional=True), tol, max_iter,
                                     C.byref(inj) if inj is not None else None, 1 if check else 0,
                                     1 if variant == "cg1" else 0,
                                     _vec(res_hist, 1, "res_hist", optional=True), C.byref(st),
                                     _stream(stream))
        if status not in (OK, ENOCONV, EBREAKDOWN):
            _check(status, "abft_dist_pcg")
        return status, st.as_dict()


class PinnedArray:
    """Page-locked host float64 array from the library's runtime
    (abft_host_alloc), for the host-buffer calls; .a is the numpy view."""

    def __init__(self, n: int):
        p = C.c_void_p()
        _check(lib().abft_host_alloc(8 * max(int(n), 1), C.byref(p)), "abft_host_alloc")
        self._p = p
        buf = (C.c_double * max(int(n), 1)).from_address(p.value)
        self.a = np.ctypeslib.as_array(buf)[: int(n)]

    def __del__(self):
        try:
            if self._p:
                lib().abft_host_free(self._p)
                self._p = None
        except Exception:
            pass


def encode(A, block_size: int = 32, max_rounds: int = 4, stream=None,
           c_csr: bool = False) -> Handle:
    """Encode a CSR matrix (host `inputs.CSR` or a `CsrDevice`).  c_csr forces
    the paper's plain CSR checksum matrix instead of the compact form."""
    if not isinstance(A, CsrDevice):
        A = CsrDevice.from_host(A)
    return Handle(A, block_size, max_rounds, stream, c_csr)
