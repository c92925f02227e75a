"""CPU-side checks of the C-ABI library: it builds for sm_100a, loads without
a GPU, exports every symbol include/abft.h declares, and its host-side
helpers agree with the oracle's independent implementations."""
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "abft.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(abft_[a-z_0-9]+)\s*\(", src)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_dsn_schollbkw16_b200 import _build, abft
    _build.build()
    return abft.lib()


def test_header_declares_the_boundary():
    names = declared_functions()
    for required in ["abft_encode", "abft_spmv", "abft_correct", "abft_pcg", "abft_flags",
                     "abft_destroy"]:
        assert required in names


def test_exports_every_declared_symbol(L):
    from paper_conf_dsn_schollbkw16_b200 import _build
    out = subprocess.run(["nm", "-D", "--defined-only", _build.LIB], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\bT (abft_\w+)", out))
    missing = [n for n in declared_functions() if n not in exported]
    assert not missing, missing
    for n in declared_functions():
        assert hasattr(L, n)


def test_binding_symbol_list_matches_header():
    from paper_conf_dsn_schollbkw16_b200 import abft
    assert sorted(abft.SYMBOLS) == declared_functions()


def test_sm100a_code_present():
    from paper_conf_dsn_schollbkw16_b200 import _build
    out = subprocess.run(["cuobjdump", "--list-elf", _build.LIB], capture_output=True, text=True)
    assert "sm_100a" in out.stdout


def test_status_strings(L):
    from paper_conf_dsn_schollbkw16_b200 import abft
    assert L.abft_status_string(0) == b"ok"
    assert b"unsupported" in L.abft_status_string(abft.ENOTSUP)
    assert L.abft_version().startswith(b"abft-b200")


def test_burst_table_matches_oracle(L, O):
    # The device injector's table (host-computed in libabft) and the oracle's
    # (computed independently in C) must be identical (R12).
    from paper_conf_dsn_schollbkw16_b200 import abft
    assert np.array_equal(abft.burst_table(), O.burst_table())


def test_fault_tables_match_oracle(L, O):
    # The Poisson CDF tables and the chunk rule of rate mode (R13)
    # are written separately in the library and in the oracle; both follow
    # the reading's definition, so the tables must agree entry for entry.
    from paper_conf_dsn_schollbkw16_b200 import abft
    for mu in (0.0, 1e-9, 1e-4, 0.01, 0.3, 1.0, 2.5, 4.0, 7.9):
        assert np.array_equal(abft.poisson_table(mu, 32), O.poisson_table(mu, 32)), mu
        assert np.array_equal(abft.poisson_table(mu, 1024), O.poisson_table(mu, 1024)), mu
    for lam in (0.0, 1e-12, 1e-8, 2.4e-7, 1e-6, 1e-4, 0.01, 0.5, 1.0):
        assert abft.rate_chunk(lam) == O.rate_chunk(lam), lam


def test_encode_rejects_bad_args_without_gpu(L):
    import ctypes as C
    from paper_conf_dsn_schollbkw16_b200 import abft
    h = C.c_void_p()
    assert L.abft_encode(None, 32, 4, 0, None, C.byref(h)) == abft.EINVAL
    csr = abft._Csr(0, 0, 0, 0, 0)
    assert L.abft_encode(C.byref(csr), 32, 4, 0, None, C.byref(h)) == abft.EINVAL
    csr = abft._Csr(10, 0, 8, 0, 0)
    assert L.abft_encode(C.byref(csr), 3, 4, 0, None, C.byref(h)) == abft.EINVAL
    assert L.abft_encode(C.byref(csr), 2048, 4, 0, None, C.byref(h)) == abft.ENOTSUP
    assert L.abft_spmv(None, None, None, None, None, 1, None) == abft.EINVAL


def test_pcg_dist_rejects_bad_args_without_gpu(L):
    # include/abft.h: a NULL handle (or a handle without _begin) is EINVAL;
    # nothing touches the device before the checks
    from paper_conf_dsn_schollbkw16_b200 import abft
    L_ = abft.lib()
    assert L_.abft_pcg_dist_begin(None, None, None, None, None, None, 1e-6, 10, 1, None,
                                  None) == abft.EINVAL
    for phase in (abft.PCG_PHASE_INIT, abft.PCG_PHASE_CG1_DOT, 9):
        assert L_.abft_pcg_dist_local(None, phase, 0, None, None) == abft.EINVAL
        assert L_.abft_pcg_dist_combine(None, phase, 0, None, 2, None) == abft.EINVAL
    assert L_.abft_pcg_dist_status(None, None, None, None) == abft.EINVAL
