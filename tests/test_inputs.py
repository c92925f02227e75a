"""Checks of the seeded input generators (no method arithmetic lives there)."""
import numpy as np
import scipy.sparse as sp

from paper_conf_dsn_schollbkw16_b200 import inputs as G


def _lap1d(n, d):
    return sp.diags([-np.ones(n - 1), d * np.ones(n), -np.ones(n - 1)], [-1, 0, 1])


def _as_scipy(A):
    return sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(A.n, A.n))


def test_lap2d_matches_kron():
    nx, ny = 7, 5
    A = G.laplacian_2d_5pt(nx, ny)
    I = sp.identity
    T = sp.kron(I(ny), _lap1d(nx, 0)) + sp.kron(_lap1d(ny, 0), I(nx)) + 4 * I(nx * ny)
    assert abs(_as_scipy(A) - T).max() == 0
    assert A.nnz == 5 * nx * ny - 2 * nx - 2 * ny


def test_lap3d_matches_kron():
    n = 6
    A = G.laplacian_3d_7pt(n)
    I = sp.identity
    L = _lap1d(n, 0)
    T = (sp.kron(I(n * n), L) + sp.kron(sp.kron(I(n), L), I(n)) + sp.kron(L, I(n * n))
         + 6 * I(n ** 3))
    assert abs(_as_scipy(A) - T).max() == 0


def test_27pt_structure():
    n = 5
    A = G.stencil_3d_27pt(n)
    assert A.nnz == (3 * n - 2) ** 3
    D = A.to_dense()
    assert np.array_equal(D, D.T)
    assert np.all(np.diag(D) == 26)
    assert A.row_lengths().max() == 27 and A.row_lengths().min() == 8


def test_columns_sorted_unique():
    for A in [G.laplacian_2d_5pt(9), G.laplacian_3d_7pt(5), G.stencil_3d_27pt(4),
              G.rmat(9, 8, 1), G.random_csr(40, 0.2, 1)]:
        for i in range(A.n):
            c = A.col[A.row_ptr[i]:A.row_ptr[i + 1]]
            assert np.all(np.diff(c) > 0)


def test_config_sizes():
    # exact nnz of configs[0] and configs[1]
    assert G.laplacian_2d_5pt(64).nnz == 20224
    assert G.laplacian_3d_7pt(32).nnz == 7 * 32 ** 3 - 6 * 32 ** 2


def test_splitmix64_reference():
    # splitmix64 with state 0: first outputs (Vigna's reference implementation)
    z = G.splitmix64(0, 2)
    assert int(z[0]) == 0xE220A8397B1DCDAF
    assert int(z[1]) == 0x6E789E6AA1B965F4


def test_uniform_vector_range():
    x = G.uniform_vector(100000, 42)
    assert x.min() >= -1 and x.max() < 1 and abs(x.mean()) < 0.01
    assert np.array_equal(x, G.uniform_vector(100000, 42))


def test_rmat_power_law():
    A = G.rmat(12, 16, 7)
    lens = A.row_lengths()
    assert A.nnz > 0.8 * 16 * 4096
    assert lens.max() > 20 * lens.mean()  # heavy tail
    assert (lens == 0).mean() > 0.2


def test_burst_mask():
    assert G.burst_mask(0, 1) == 1
    assert G.burst_mask(62, 5) == (1 << 62) | (1 << 63)
    assert G.burst_mask(10, 3) == 0b111 << 10
