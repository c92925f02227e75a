"""Seeded synthetic input generators shared by the CUDA path and the oracle.

This module holds NONE of the method's arithmetic (no checksums, no bounds, no
products, no sums of matrix entries): it only builds the matrices, vectors and
explicit fault plans both sides consume, so that parity tests compare the two
implementations on identical inputs (task rule: "only the seeded input
generators serve both, from a module of their own").

Workload recipes (DESIGN.md §"Input recipe"):

* Dirichlet Laplacians in natural ordering (x fastest, then y, then z), columns
  ascending within each row: 2-D 5-point (diag 4, off -1), 3-D 7-point
  (diag 6, off -1), 3-D 27-point (diag 26, off -1).  These are the synthetic
  analogues of the SPD SuiteSparse matrices of PAPER.md Table I.
* R-MAT (Graph500 Kronecker, a,b,c,d = .57,.19,.19,.05), duplicates removed,
  seeded vertex permutation, values ~ U[-1,1) -- the irregular power-law case
  of BASELINE.json configs[2].
* Vectors: x ~ U[-1,1) from splitmix64(seed): ((u >> 11) * 2^-53) * 2 - 1.
* Explicit fault plans (§IV-A): a burst of bit flips whose
  start bit is uniform in 0..63 and whose length is round(N(3, var 2)),
  clipped to >= 1 and truncated at bit 63.
"""
from __future__ import annotations

import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np

__all__ = [
    "CSR",
    "laplacian_2d_5pt",
    "laplacian_3d_7pt",
    "stencil_3d_27pt",
    "stencil_for_config",
    "stencil_rows",
    "rmat",
    "random_csr",
    "splitmix64",
    "uniform_vector",
    "burst_mask",
    "FaultPlan",
    "single_fault_plan",
    "TARGET_Y",
    "TARGET_T1",
    "TARGET_T2",
]

TARGET_Y, TARGET_T1, TARGET_T2 = 0, 1, 2

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


class CSR:
    """Square CSR matrix: row_ptr int32[n+1], col int32[nnz] (ascending per
    row, no duplicates), val float64[nnz]."""

    __slots__ = ("n", "row_ptr", "col", "val", "name")

    def __init__(self, row_ptr, col, val, name=""):
        self.row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int32)
        self.col = np.ascontiguousarray(col, dtype=np.int32)
        self.val = np.ascontiguousarray(val, dtype=np.float64)
        self.n = int(self.row_ptr.shape[0] - 1)
        self.name = name

    @property
    def nnz(self) -> int:
        return int(self.col.shape[0])

    def row_lengths(self) -> np.ndarray:
        return np.diff(self.row_ptr.astype(np.int64))

    def to_dense(self) -> np.ndarray:
        d = np.zeros((self.n, self.n))
        rows = np.repeat(np.arange(self.n), self.row_lengths())
        d[rows, self.col] = self.val
        return d

    def __repr__(self):
        return f"CSR({self.name!r}, n={self.n}, nnz={self.nnz})"


def _stencil(shape, offsets, diag, off, name, z_range=None):
    """Generic constant-coefficient stencil on a (nz, ny, nx) grid, natural
    ordering, Dirichlet boundary (neighbours outside the grid are dropped).
    z_range = (z0, z1) generates only the rows of planes z0..z1-1 (a row-block
    shard), with GLOBAL column indices."""
    nz, ny, nx = shape
    if nz * ny * nx >= 2**31:
        raise ValueError("grid too large for int32 indices")
    z0, z1 = z_range if z_range is not None else (0, nz)
    n = (z1 - z0) * ny * nx
    idx = np.arange(z0 * ny * nx, z1 * ny * nx, dtype=np.int64)
    x = idx % nx
    y = (idx // nx) % ny
    z = idx // (nx * ny)
    lin = [dz * nx * ny + dy * nx + dx for dz, dy, dx in offsets]
    order = np.argsort(lin, kind="stable")
    offsets = [offsets[o] for o in order]
    lin = [lin[o] for o in order]
    valids = []
    counts = np.zeros(n, dtype=np.int64)
    for dz, dy, dx in offsets:
        v = np.ones(n, dtype=bool)
        if dx:
            v &= (x + dx >= 0) & (x + dx < nx)
        if dy:
            v &= (y + dy >= 0) & (y + dy < ny)
        if dz:
            v &= (z + dz >= 0) & (z + dz < nz)
        valids.append(v)
        counts += v
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    nnz = int(row_ptr[-1])
    if nnz >= 2**31:
        raise ValueError("nnz too large for int32 row_ptr")
    col = np.empty(nnz, dtype=np.int32)
    val = np.empty(nnz, dtype=np.float64)
    pos = row_ptr[:-1].copy()
    base = z0 * ny * nx
    for (dz, dy, dx), l, v in zip(offsets, lin, valids):
        rows = idx[v]
        p = pos[rows - base]
        col[p] = (rows + l).astype(np.int32)
        val[p] = diag if (dz, dy, dx) == (0, 0, 0) else off
        pos[rows - base] += 1
        del rows, p
    return CSR(row_ptr.astype(np.int32), col, val, name)


def laplacian_2d_5pt(nx: int, ny: int | None = None) -> CSR:
    """2-D 5-point Dirichlet Laplacian (diag 4, off -1); BASELINE configs[0]
    uses 64x64."""
    ny = nx if ny is None else ny
    offs = [(0, 0, 0), (0, 0, -1), (0, 0, 1), (0, -1, 0), (0, 1, 0)]
    return _stencil((1, ny, nx), offs, 4.0, -1.0, f"lap2d5_{nx}x{ny}")


def laplacian_3d_7pt(n: int, ny: int | None = None, nz: int | None = None) -> CSR:
    """3-D 7-point Dirichlet Laplacian (diag 6, off -1); configs[1] = 128^3,
    configs[4] (PCG) = 192^3."""
    ny = n if ny is None else ny
    nz = n if nz is None else nz
    offs = [(0, 0, 0), (0, 0, -1), (0, 0, 1), (0, -1, 0), (0, 1, 0), (-1, 0, 0), (1, 0, 0)]
    return _stencil((nz, ny, n), offs, 6.0, -1.0, f"lap3d7_{n}x{ny}x{nz}")


def stencil_3d_27pt(n: int, ny: int | None = None, nz: int | None = None) -> CSR:
    """3-D 27-point stencil (diag 26, off -1, HPCG style); configs[3] = 256^3."""
    ny = n if ny is None else ny
    nz = n if nz is None else nz
    offs = [(dz, dy, dx) for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]
    return _stencil((nz, ny, n), offs, 26.0, -1.0, f"st3d27_{n}x{ny}x{nz}")


_OFFS = {
    "5pt": [(0, 0, 0), (0, 0, -1), (0, 0, 1), (0, -1, 0), (0, 1, 0)],
    "7pt": [(0, 0, 0), (0, 0, -1), (0, 0, 1), (0, -1, 0), (0, 1, 0), (-1, 0, 0), (1, 0, 0)],
    "27pt": [(dz, dy, dx) for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1)],
}
_DIAG = {"5pt": 4.0, "7pt": 6.0, "27pt": 26.0}


def stencil_rows(kind: str, nx: int, ny: int, nz: int, z0: int, z1: int) -> CSR:
    """Rows of planes z0..z1-1 of the (nz, ny, nx) `kind` stencil, global
    column indices (the row-block shard a rank owns)."""
    return _stencil((nz, ny, nx), list(_OFFS[kind]), _DIAG[kind], -1.0,
                    f"{kind}_{nx}x{ny}x{nz}[z{z0}:{z1}]", z_range=(z0, z1))


def stencil_for_config(kind: str, n: int) -> CSR:
    return {"5pt": lambda: laplacian_2d_5pt(n), "7pt": lambda: laplacian_3d_7pt(n),
            "27pt": lambda: stencil_3d_27pt(n)}[kind]()


def splitmix64(seed: int, count: int, start: int = 0) -> np.ndarray:
    """The splitmix64 sequence: state_i = seed + (i+1)*golden (mod 2^64), then
    the standard two-multiply finaliser."""
    with np.errstate(over="ignore"):
        i = np.arange(start + 1, start + count + 1, dtype=np.uint64)
        z = np.uint64(seed) + i * _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def uniform_vector(n: int, seed: int, start: int = 0) -> np.ndarray:
    """x_i ~ U[-1, 1): ((u >> 11) * 2^-53) * 2 - 1, exact in binary64.
    `start` gives entries start .. start+n-1 of the same sequence (a shard)."""
    u = splitmix64(seed, n, start)
    return (u >> np.uint64(11)).astype(np.float64) * (2.0 ** -53) * 2.0 - 1.0


def rmat(scale: int, edge_factor: int = 16, seed: int = 1, permute: bool = True,
         abcd=(0.57, 0.19, 0.19, 0.05)) -> CSR:
    """Graph500-style R-MAT with 2^scale vertices and edge_factor*2^scale
    generated edges.  Duplicate edges are removed, self loops kept, an
    optional seeded random vertex permutation is applied, values ~ U[-1,1).
    Columns are ascending within each row."""
    n = 1 << scale
    m = edge_factor * n
    rng = np.random.Generator(np.random.PCG64(seed))
    a, b, c, _ = abcd
    src = np.zeros(m, dtype=np.int64)
    dst = np.zeros(m, dtype=np.int64)
    # edges in fixed chunks, each with its own spawned stream (the result does
    # not depend on the thread count); numpy releases the GIL in the loops
    chunk = 1 << 22
    nch = (m + chunk - 1) // chunk
    seqs = np.random.SeedSequence(seed).spawn(nch)

    def fill(q):
        lo, hi = q * chunk, min(m, (q + 1) * chunk)
        g = np.random.Generator(np.random.PCG64(seqs[q]))
        s_, d_ = src[lo:hi], dst[lo:hi]
        for level in range(scale):
            r = g.random(hi - lo)
            bit_s = r >= a + b
            bit_d = ((r >= a) & (r < a + b)) | (r >= a + b + c)
            s_ |= bit_s.astype(np.int64) << level
            d_ |= bit_d.astype(np.int64) << level

    with ThreadPoolExecutor(max_workers=min(nch, os.cpu_count() or 1)) as ex:
        list(ex.map(fill, range(nch)))
    if permute:
        perm = rng.permutation(n).astype(np.int64)
        src = perm[src]
        dst = perm[dst]
    key = src * n + dst
    del src, dst
    key.sort()  # == np.unique (sorted, first occurrence kept), ~50x faster on large inputs
    keep = np.empty(key.shape[0], dtype=bool)
    keep[:1] = True
    np.not_equal(key[1:], key[:-1], out=keep[1:])
    key = key[keep]
    del keep
    rows = key // n
    cols = key - rows * n
    counts = np.bincount(rows, minlength=n)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    val = uniform_vector(int(key.shape[0]), seed + 0x5151)
    return CSR(row_ptr.astype(np.int32), cols.astype(np.int32), val,
               f"rmat{scale}_ef{edge_factor}{'_perm' if permute else ''}")


def random_csr(n: int, density: float, seed: int, integer: bool = False,
               empty_rows: float = 0.0, max_int: int = 8) -> CSR:
    """Small random square CSR for parity tests.  `integer` draws small
    integer values (exact sums, used for the eq. (2) invariant pins);
    `empty_rows` forces that fraction of rows to be empty."""
    rng = np.random.Generator(np.random.PCG64(seed))
    mask = rng.random((n, n)) < density
    if empty_rows > 0:
        mask[rng.random(n) < empty_rows, :] = False
    rows, cols = np.nonzero(mask)
    if integer:
        vals = rng.integers(-max_int, max_int + 1, size=rows.shape[0]).astype(np.float64)
    else:
        vals = rng.uniform(-1.0, 1.0, size=rows.shape[0])
    counts = np.bincount(rows, minlength=n)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    return CSR(row_ptr.astype(np.int32), cols.astype(np.int32), vals, f"rand{n}_{density}")


def hub_csr(n: int, seed: int, hub_lens=(1500, 4100), mid_frac: float = 0.08,
            mid_len=(33, 400), short_len=(0, 12)) -> CSR:
    """Random square CSR with every row-length class of the fused kernels:
    short rows (<= 32 entries), medium rows (33..1024) and hub rows (> 1024
    entries, split into chunks), placed at fixed rows; values ~ U[-1,1)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    lens = rng.integers(short_len[0], short_len[1] + 1, size=n)
    mid = rng.random(n) < mid_frac
    lens[mid] = rng.integers(mid_len[0], mid_len[1] + 1, size=int(mid.sum()))
    for t, L in enumerate(hub_lens):
        lens[(37 + t * (n // 2 + 5)) % n] = min(L, n)
    cols = [np.sort(rng.choice(n, size=int(L), replace=False)) for L in lens]
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(lens, out=row_ptr[1:])
    col = np.concatenate(cols).astype(np.int32) if n else np.zeros(0, np.int32)
    val = rng.uniform(-1.0, 1.0, size=col.shape[0])
    return CSR(row_ptr.astype(np.int32), col, val, f"hub{n}")


def burst_mask(start_bit: int, length: int) -> int:
    """XOR mask of a burst of `length` flipped bits starting at `start_bit`,
    truncated at bit 63 (no wrap) -- SURVEY.md §8(c) Q12 reading of P:196."""
    length = max(1, int(length))
    hi = min(start_bit + length - 1, 63)
    mask = 0
    for b in range(start_bit, hi + 1):
        mask |= 1 << b
    return mask


class FaultPlan:
    """Explicit fault list: entry e XORs `mask[e]` into the value produced for
    element `index[e]` of `target[e]` (0 = y row, 1 = t1 block, 2 = t2 block)
    in correction round `round[e]` (0 = the main pass).  `call` (optional):
    entry e only applies to the `call[e]`-th SpMV of a solve (PCG); None =
    every call."""

    def __init__(self, round_, target, index, mask, call=None):
        self.round = np.ascontiguousarray(round_, dtype=np.int32)
        self.target = np.ascontiguousarray(target, dtype=np.int32)
        self.index = np.ascontiguousarray(index, dtype=np.int64)
        self.mask = np.ascontiguousarray(mask, dtype=np.uint64)
        self.call = None if call is None else np.ascontiguousarray(call, dtype=np.int64)

    def __len__(self):
        return int(self.index.shape[0])

    @staticmethod
    def empty():
        return FaultPlan([], [], [], [])

    def concat(self, other: "FaultPlan") -> "FaultPlan":
        if (self.call is None) != (other.call is None):
            raise ValueError("concat of a per-call plan with an all-calls plan")
        return FaultPlan(np.concatenate([self.round, other.round]),
                         np.concatenate([self.target, other.target]),
                         np.concatenate([self.index, other.index]),
                         np.concatenate([self.mask, other.mask]),
                         None if self.call is None else np.concatenate([self.call, other.call]))


def single_fault_plan(n_elems: int, seed: int, target: int = TARGET_Y,
                      fault_free_value=None, sigma: float | None = None,
                      max_tries: int = 1000) -> FaultPlan:
    """One burst on a uniformly chosen element.  With `sigma` and
    the fault-free values, the burst is resampled until the corrupted value
    is sigma-significant; NaN/Inf count as significant."""
    rng = np.random.Generator(np.random.PCG64(seed))
    elem = int(rng.integers(0, n_elems))
    for _ in range(max_tries):
        start = int(rng.integers(0, 64))
        length = max(1, int(np.rint(rng.normal(3.0, np.sqrt(2.0)))))
        mask = burst_mask(start, length)
        if sigma is None or fault_free_value is None:
            break
        v = float(fault_free_value[elem])
        bits = np.array([v]).view(np.uint64)[0] ^ np.uint64(mask)
        verr = float(np.array([bits], dtype=np.uint64).view(np.float64)[0])
        if not np.isfinite(verr) or abs(verr) > abs(v) * (1 + sigma) or abs(verr) < abs(v) * (1 - sigma):
            break
    return FaultPlan([0], [target], [elem], [mask])
