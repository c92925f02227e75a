"""Pins for the CPU oracle (oracle/abft_oracle.c) against what PAPER.md and
the mathematics fix -- never against the oracle itself or the CUDA path.

Each test names the passage / property it pins.  These run without a GPU.
"""
import json
import math
import os
from fractions import Fraction

import numpy as np
import pytest

from paper_conf_dsn_schollbkw16_b200 import inputs as G

GOLD = os.path.join(os.path.dirname(__file__), "golden")
EPS = 2.0 ** -53
U = 2.0 ** -53  # unit roundoff


def csr_from_dense(D):
    D = np.asarray(D, dtype=np.float64)
    rows, cols = np.nonzero(D)
    counts = np.bincount(rows, minlength=D.shape[0])
    rp = np.concatenate([[0], np.cumsum(counts)])
    return G.CSR(rp, cols, D[rows, cols])


def exact_sum(vals):
    return sum((Fraction(float(v)) for v in vals), Fraction(0))


# --------------------------------------------------------------------------
# R2: canonical pairwise summation -- pinned by hand-computed
# cases whose result differs under every other grouping.
# --------------------------------------------------------------------------
class TestPairwise:
    def test_tree_grouping_power_of_two(self, O):
        # ((1 + u) + (u + u)) = 1 + 2u exactly; a left fold gives 1.0
        assert O.pw([1.0, U, U, U]) == 1.0 + 2 * U

    def test_absent_padding_three(self, O):
        # n = 3 -> (v0 + v1) + v2 = (1 + u) + u = 1.0 ; v0 + (v1 + v2) = 1 + 2u
        assert O.pw([1.0, U, U]) == 1.0

    def test_five_elements(self, O):
        # ((v0+v1)+(v2+v3)) + v4 with v4 alone in the right subtree
        # ((1 + u) + (u + u)) + (-1) = (1 + 2u) - 1 = 2u; a left fold gives 0
        assert O.pw([1.0, U, U, U, -1.0]) == 2 * U

    def test_empty_and_signed_zero(self, O):
        assert O.pw([]) == 0.0 and math.copysign(1, O.pw([])) == 1.0
        assert math.copysign(1, O.pw([-0.0])) == -1.0
        assert math.copysign(1, O.pw([-0.0, -0.0, -0.0])) == -1.0

    def test_slots_absent_differs_from_compacted(self, O):
        # slots [1, absent, u, u]: 1 + (u + u) = 1 + 2u; the compacted list
        # [1, u, u] gives 1.0 -- absent slots keep their tree position.
        v = np.array([1.0, 123.0, U, U])
        assert O.pw(v, [1, 0, 1, 1]) == 1.0 + 2 * U
        assert O.pw(v, [0, 0, 0, 0]) == 0.0

    def test_integers_exact(self, O):
        rng = np.random.default_rng(0)
        for n in [1, 2, 3, 7, 31, 32, 33, 1000]:
            v = rng.integers(-1000, 1000, n).astype(float)
            assert O.pw(v) == float(sum(int(a) for a in v))

    def test_error_bound(self, O):
        # |PW - exact| <= gamma_{ceil(log2 n)} * sum|v|  (Higham, Thm 4.1 / pairwise)
        rng = np.random.default_rng(1)
        for n in [10, 100, 1000, 4097]:
            v = rng.standard_normal(n) * 10.0 ** rng.integers(-5, 5, n)
            d = math.ceil(math.log2(n))
            g = d * U / (1 - d * U)
            err = abs(Fraction(O.pw(v)) - exact_sum(v))
            assert float(err) <= g * float(np.abs(v).sum())


# --------------------------------------------------------------------------
# SpMV: brute force against dense products on tiny inputs.
# --------------------------------------------------------------------------
class TestSpmv:
    def test_integer_exact(self, O):
        for seed in range(5):
            A = G.random_csr(37, 0.2, seed, integer=True, empty_rows=0.1)
            x = np.random.default_rng(seed).integers(-9, 10, 37).astype(float)
            y = O.spmv(A, x)
            assert np.array_equal(y, A.to_dense().astype(np.int64) @ x.astype(np.int64))

    def test_float_within_bound(self, O):
        A = G.random_csr(50, 0.3, 3)
        x = G.uniform_vector(50, 42)
        y = O.spmv(A, x)
        D = A.to_dense()
        for i in range(50):
            prods = [Fraction(float(D[i, j])) * Fraction(float(x[j])) for j in range(50) if D[i, j] != 0]
            n = max(len(prods), 1)
            g = (math.ceil(math.log2(n)) + 1) * U / (1 - 8 * U) if n > 1 else U
            bound = g * sum(abs(float(p)) for p in prods)
            assert abs(float(Fraction(y[i]) - sum(prods, Fraction(0)))) <= bound + 1e-300

    def test_empty_row_is_plus_zero(self, O):
        A = csr_from_dense([[0, 0], [1, 2]])
        y = O.spmv(A, np.array([-1.0, 1.0]))
        assert y[0] == 0.0 and math.copysign(1, y[0]) == 1.0 and y[1] == 1.0


# --------------------------------------------------------------------------
# Encoding
# --------------------------------------------------------------------------
def brute_structure(A, bs):
    D = A.to_dense() != 0
    # structural: use the CSR pattern, not numerical nonzeros
    P = np.zeros((A.n, A.n), dtype=bool)
    rows = np.repeat(np.arange(A.n), A.row_lengths())
    P[rows, A.col] = True
    del D
    nb = (A.n + bs - 1) // bs
    return [sorted(set(np.nonzero(P[k * bs:(k + 1) * bs].any(axis=0))[0].tolist())) for k in range(nb)]


class TestEncode:
    @pytest.mark.parametrize("n,bs", [(20, 5), (37, 4), (33, 32), (64, 1), (65, 8), (10, 10), (10, 64)])
    def test_structure_fig2_rule(self, O, n, bs):
        # Fig. 2 rule: a column appears in row k of C iff it holds >= 1
        # element of A_k.  Brute force with Python sets.
        A = G.random_csr(n, 0.15, n * 7 + bs, empty_rows=0.1)
        enc = O.encode(A, bs)
        exp = brute_structure(A, bs)
        assert enc.nb == len(exp)
        for k, cols in enumerate(exp):
            assert enc.col[enc.row_ptr[k]:enc.row_ptr[k + 1]].tolist() == cols
        assert np.array_equal(enc.n_k, [len(c) for c in exp])

    def test_explicit_zero_is_structural(self, O):
        # R5 (Q2): a stored 0.0 still counts as an element of A_k.
        A = G.CSR([0, 2, 3], [0, 1, 1], [1.0, 0.0, 2.0])
        enc = O.encode(A, 2)
        assert enc.col.tolist() == [0, 1] and enc.val.tolist() == [1.0, 2.0]

    @pytest.mark.parametrize("bs", [1, 2, 3, 8, 32])
    def test_values_integer_column_sums(self, O, bs):
        # c_k = w_k^T A_k with w = ones: dense column sums.
        A = G.random_csr(45, 0.2, bs, integer=True)
        enc = O.encode(A, bs)
        D = A.to_dense()
        for k in range(enc.nb):
            cs = D[k * bs:(k + 1) * bs].sum(axis=0)
            cols = enc.col[enc.row_ptr[k]:enc.row_ptr[k + 1]]
            assert np.array_equal(enc.val[enc.row_ptr[k]:enc.row_ptr[k + 1]], cs[cols])

    def test_bs1_c_equals_a(self, O):
        # "For block size 1, the checksum matrix C is equal to A."
        A = G.random_csr(40, 0.2, 11)
        enc = O.encode(A, 1)
        assert np.array_equal(enc.row_ptr, A.row_ptr)
        assert np.array_equal(enc.col, A.col)
        assert np.array_equal(enc.val, A.val)

    def test_laplacian_checksum_values(self, O):
        # Column sums of a 5-pt / 7-pt / 27-pt Laplacian row block are small
        # integers (diag + neighbours).  With the grid's x extent a multiple of
        # b_s = 32 (as in every BASELINE config) a block is a piece of one
        # x-line, so the sums are {-1,2,3} / {-1,4,5} / {-3,-2,-1,24,25}.
        for A, allowed in [(G.laplacian_2d_5pt(64, 8), {-1.0, 2.0, 3.0}),
                           (G.laplacian_3d_7pt(32, 4, 4), {-1.0, 4.0, 5.0}),
                           (G.stencil_3d_27pt(32, 4, 4), {-3.0, -2.0, -1.0, 24.0, 25.0})]:
            enc = O.encode(A, 32)
            assert set(np.unique(enc.val).tolist()) <= allowed
            D = A.to_dense()
            for k in range(enc.nb):
                cs = D[32 * k:32 * (k + 1)].sum(axis=0)
                cols = enc.col[enc.row_ptr[k]:enc.row_ptr[k + 1]]
                assert np.array_equal(enc.val[enc.row_ptr[k]:enc.row_ptr[k + 1]], cs[cols])

    def test_bound_bs1_closed_form(self, O):
        # b_s = 1: c_k = a_k, so tau_k = ((n_k + 0) ||a_k|| + n_k ||a_k||) eps beta
        #        = 2 n_k ||a_k|| eps beta  (P:158 with b_s = 1, C = A from P:248).
        # Rows with Pythagorean norms make the closed form exact.
        A = csr_from_dense([[3, 4, 0, 0], [0, 0, 5, 12], [8, 0, 15, 0], [0, 0, 0, 7]])
        enc = O.encode(A, 1)
        norms = [5.0, 13.0, 17.0, 7.0]
        nk = [2, 2, 2, 1]
        assert enc.K.tolist() == [2 * n * r * EPS for n, r in zip(nk, norms)]

    def test_bound_bsN_reduces_to_dense_bound(self, O):
        # b_s = N with every column non-empty: one block; P:158 becomes the
        # dense bound of [35] with m = N rows and n columns:
        #   ((n + 2m - 2) sum_i ||a_i|| + n ||c||) eps_M.
        A = csr_from_dense([[3, 4, 0], [0, 0, 5], [0, 0, 0]])  # col sums (3,4,5), ||c|| = 5*sqrt2
        enc = O.encode(A, 3)
        m, n = 3, 3
        sum_norms = 5.0 + 5.0 + 0.0
        c = math.sqrt(50.0)
        assert enc.K.shape == (1,)
        assert enc.K[0] == ((n + 2 * m - 2) * sum_norms + n * c) * EPS

    def test_bound_coefficient_uses_nk_not_n(self, O):
        # the sparse bound uses the number of NON-EMPTY columns n_k of
        # A_k, not N.  Block 0 touches 2 of 6 columns; b_s = 2.
        D = np.zeros((6, 6))
        D[0, 0] = 3
        D[0, 1] = 4
        D[1, 1] = 5
        D[1, 0] = 12  # ||a_0|| = 5, ||a_1|| = 13; c_0 = (15, 9)
        D[2:, 2:] = np.eye(4)
        A = csr_from_dense(D)
        enc = O.encode(A, 2)
        c0 = math.sqrt(15.0 ** 2 + 9.0 ** 2)
        assert enc.n_k.tolist() == [2, 2, 2]
        assert enc.K[0] == ((2 + 2 * 2 - 2) * 18.0 + 2 * c0) * EPS

    def test_c_value_is_pw_over_row_slots(self, O):
        # R4*: c_kj = PW over the b_s row slots of block k, with ABSENT slots
        # where a row lacks column j.  Column 0 of a 4-row block holds
        # (1, absent, 1e16, -1e16): PW = 1 + (1e16 + -1e16) = 1.0; a left fold
        # over the present rows gives (1 + 1e16) - 1e16 = 0.0.  Column 1 holds
        # (1, 1e16, -1e16, 1): PW = (1 + 1e16) + (-1e16 + 1) = 1e16 - 1e16 = 0,
        # a left fold gives ((1 + 1e16) - 1e16) + 1 = 1.0.
        D = np.zeros((4, 4))
        D[:, 0] = [1.0, 0.0, 1e16, -1e16]
        D[:, 1] = [1.0, 1e16, -1e16, 1.0]
        D[1, 2] = 1.0  # keeps row 1 non-empty
        A = csr_from_dense(D)
        enc = O.encode(A, 4)
        assert enc.col.tolist() == [0, 1, 2]
        assert enc.val.tolist() == [1.0, 0.0, 1.0]

    def test_block_norm_sum_is_pw_over_row_slots(self, O):
        # R7: S_k = PW over the b_s slots of ||a_i||.  diag(1, 2^53, 1, 1) with
        # b_s = 4: S = (1 + 2^53) + (1 + 1) = 2^53 + 2 (1 + 2^53 rounds to
        # 2^53, ties to even); a left fold gives 2^53.  ||c|| = sqrt((1 +
        # 2^106) + (1 + 1)) = 2^53, n_k = 4, m = n_k + 2 b_s - 2 = 10:
        # K = fl(fl(10 (2^53 + 2)) + 4 2^53) 2^-53 = (14 2^53 + 16) 2^-53
        # = 14 + 2^-49 (10 (2^53 + 2) = 10 2^53 + 20 rounds to + 16 at ulp 16);
        # with the left-fold S it would be exactly 14.
        A = csr_from_dense(np.diag([1.0, 2.0 ** 53, 1.0, 1.0]))
        enc = O.encode(A, 4)
        assert enc.S[0] == 2.0 ** 53 + 2
        assert enc.c_norm[0] == 2.0 ** 53
        assert enc.K[0] == 14.0 + 2.0 ** -49

    def test_ragged_last_block(self, O):
        # R3 (Q3): the last block holds only the existing rows; b_s stays literal.
        A = G.laplacian_2d_5pt(5)  # N = 25, b_s = 8 -> last block has 1 row
        enc = O.encode(A, 8)
        assert enc.nb == 4
        r = 24
        nk = enc.n_k[3]
        rn = math.sqrt(16 + 1 + 1)
        c = enc.val[enc.row_ptr[3]:enc.row_ptr[4]]
        assert c.tolist() == [-1.0, -1.0, 4.0]
        assert enc.K[3] == ((nk + 2 * 8 - 2) * rn + nk * math.sqrt(18.0)) * EPS
        del r


# --------------------------------------------------------------------------
# Detection, correction
# --------------------------------------------------------------------------
class TestWorkedExample:
    def test_golden_6x6(self, O):
        g = json.load(open(os.path.join(GOLD, "worked_example_6x6.json")))
        A = csr_from_dense(g["A_dense"])
        bs = g["block_size"]
        x = np.array(g["x"], dtype=float)
        enc = O.encode(A, bs)
        Cd = np.zeros((enc.nb, A.n))
        for k in range(enc.nb):
            for q in range(enc.row_ptr[k], enc.row_ptr[k + 1]):
                Cd[k, enc.col[q]] = enc.val[q]
        assert Cd.tolist() == g["C_dense"]
        assert enc.n_k.tolist() == g["n_k"]
        ok = O.abft_spmv(A, enc, x)
        assert ok.y.tolist() == g["y_fault_free"]
        assert ok.t1.tolist() == g["t1"] and ok.t2.tolist() == g["t2_fault_free"]
        assert ok.flagged.size == 0
        plan = G.FaultPlan([0], [G.TARGET_Y], [g["fault"]["element_1based"] - 1], [g["fault"]["mask"]])
        r = O.abft_spmv(A, enc, x, O.Inject.from_plan(plan), max_rounds=1)
        assert r.y_pre.tolist() == g["y_faulty"]
        assert (r.t1 - g["t1"]).tolist() == [0, 0, 0]
        assert (np.array(g["t1"]) - np.array(g["t2_faulty"])).tolist() == g["syndrome_faulty"]
        assert (r.flagged + 1).tolist() == g["flagged_blocks_1based"]
        rows = [i + 1 for k in r.flagged for i in range(k * bs, (k + 1) * bs)]
        assert rows == g["recomputed_rows_1based"]
        assert r.y.tolist() == g["y_fault_free"] and r.status == 0
        assert r.flags[1].size == 0


class TestDetection:
    def test_invariant_eq2_integers(self, O):
        # eq. (2): with integer A, x and all partial sums < 2^53 the
        # invariant holds exactly: t1 == t2, s == 0, for every b_s.
        for bs in [1, 2, 5, 32]:
            A = G.random_csr(70, 0.1, bs, integer=True, empty_rows=0.05)
            x = np.random.default_rng(bs).integers(-50, 50, 70).astype(float)
            enc = O.encode(A, bs)
            r = O.abft_spmv(A, enc, x)
            assert np.array_equal(r.t1, r.t2) and np.all(r.s == 0.0)
            assert r.flagged.size == 0

    @pytest.mark.parametrize("mat", ["lap2d", "lap3d", "st27", "rand", "rmat"])
    def test_no_false_positives(self, O, mat):
        # tau is an upper bound on rounding differences:
        # error-free runs flag nothing.
        A = {"lap2d": lambda: G.laplacian_2d_5pt(64), "lap3d": lambda: G.laplacian_3d_7pt(12),
             "st27": lambda: G.stencil_3d_27pt(10), "rand": lambda: G.random_csr(300, 0.05, 5),
             "rmat": lambda: G.rmat(10, 8, 3)}[mat]()
        enc = O.encode(A, 32)
        for seed in range(3):
            x = G.uniform_vector(A.n, 100 + seed)
            r = O.abft_spmv(A, enc, x)
            assert r.flagged.size == 0
            tau = enc.K * r.beta
            assert np.all(np.abs(r.s) <= tau)

    def test_beta_is_two_norm(self, O):
        x = G.uniform_vector(1000, 9)
        A = G.laplacian_2d_5pt(10)
        x = x[:A.n]
        r = O.abft_spmv(A, O.encode(A, 32), x)
        exact = float(exact_sum([Fraction(v) * Fraction(v) for v in x]))
        assert abs(r.beta - math.sqrt(exact)) <= 1e-15 * r.beta

    def test_large_faults_localized(self, O):
        # A fault with |delta| >= 2 tau_k must be flagged and localized to its
        # own block only; correction restores y exactly.
        A = G.laplacian_3d_7pt(10)
        enc = O.encode(A, 32)
        x = G.uniform_vector(A.n, 7)
        clean = O.spmv(A, x)
        base = O.abft_spmv(A, enc, x)
        hit = 0
        for seed in range(300):
            plan = G.single_fault_plan(A.n, seed)
            r = O.abft_spmv(A, enc, x, O.Inject.from_plan(plan), max_rounds=2)
            i = int(plan.index[0])
            k = i // 32
            delta = abs(r.y_pre[i] - clean[i]) if np.isfinite(r.y_pre[i]) else np.inf
            tau = enc.K[k] * base.beta
            if delta >= 2 * tau:
                hit += 1
                assert r.flagged.tolist() == [k]
            else:
                assert set(r.flagged.tolist()) <= {k}
            assert r.status == 0
            if r.flagged.size:  # detected -> the recomputation restores y exactly
                assert r.y.view(np.uint64).tolist() == clean.view(np.uint64).tolist()
            else:  # undetected -> only element i differs, by less than 2 tau
                d = np.nonzero(r.y != clean)[0]
                assert d.tolist() in ([], [i]) and delta < 2 * tau
        assert hit > 200

    def test_checksum_target_faults(self, O):
        # P:196 "Bit flips were also injected into operations that perform
        # error detection": a big fault in t1_k or t2_k flags block k; the
        # recomputation then clears it.
        A = G.laplacian_2d_5pt(32)
        enc = O.encode(A, 32)
        x = G.uniform_vector(A.n, 3)
        for tgt in (G.TARGET_T1, G.TARGET_T2):
            plan = G.FaultPlan([0], [tgt], [5], [1 << 62])
            r = O.abft_spmv(A, enc, x, O.Inject.from_plan(plan), max_rounds=1)
            assert r.flagged.tolist() == [5] and r.flags[1].size == 0 and r.status == 0

    def test_uncorrectable_reports(self, O):
        # A fault re-injected in every round is never cleared -> -6 (R11').
        A = G.laplacian_2d_5pt(16)
        enc = O.encode(A, 32)
        x = G.uniform_vector(A.n, 3)
        plan = G.FaultPlan([0, 1, 2], [0, 0, 0], [40, 40, 40], [1 << 60] * 3)
        r = O.abft_spmv(A, enc, x, O.Inject.from_plan(plan), max_rounds=2)
        assert r.status == -6 and r.flags[2].tolist() == [1]

    def test_nan_flags(self, O):
        # R5' (Q5): flag iff NOT(|s| <= tau) also flags NaN syndromes.
        A = G.laplacian_2d_5pt(8)
        enc = O.encode(A, 32)
        x = G.uniform_vector(A.n, 1)
        plan = G.FaultPlan([0], [0], [3], [0x7FF8000000000000])  # exponent -> NaN/Inf
        r = O.abft_spmv(A, enc, x, O.Inject.from_plan(plan), max_rounds=0)
        assert r.flagged.tolist() == [0]

    def test_zero_x_and_empty_blocks(self, O):
        # x = 0 -> beta = 0, tau = 0; s = 0 exactly so nothing is flagged.
        # An all-empty block has tau_k = 0 and s_k = 0 -> not flagged.
        A = G.random_csr(96, 0.1, 2)
        A2 = G.CSR(np.concatenate([A.row_ptr[:33], np.full(32, A.row_ptr[32]),
                                   A.row_ptr[65:] - (A.row_ptr[64] - A.row_ptr[32])]),
                   np.concatenate([A.col[:A.row_ptr[32]], A.col[A.row_ptr[64]:]]),
                   np.concatenate([A.val[:A.row_ptr[32]], A.val[A.row_ptr[64]:]]))
        enc = O.encode(A2, 32)
        assert enc.n_k[1] == 0 and enc.K[1] == 0.0
        r = O.abft_spmv(A2, enc, np.zeros(96))
        assert r.beta == 0.0 and r.flagged.size == 0
        r = O.abft_spmv(A2, enc, G.uniform_vector(96, 5))
        assert r.flagged.size == 0 and r.t1[1] == 0.0 and r.t2[1] == 0.0


# --------------------------------------------------------------------------
# Fault model
# --------------------------------------------------------------------------
class TestFaultModel:
    def test_philox_known_answers(self, O):
        # Random123 published known-answer vectors for philox4x32-10.
        kat = [([0, 0, 0, 0], [0, 0], [0x6627e8d5, 0xe169c58d, 0xbc57ac4c, 0x9b00dbd8]),
               ([0xffffffff] * 4, [0xffffffff] * 2, [0x408f276d, 0x41c83b0e, 0xa20bc7c6, 0x6d5451fd]),
               ([0x243f6a88, 0x85a308d3, 0x13198a2e, 0x03707344], [0xa4093822, 0x299f31d0],
                [0xd16cfe09, 0x94fdcceb, 0x5001e420, 0x24126ea1])]
        for c, k, o in kat:
            assert O.philox4x32_10(c, k).tolist() == o

    def test_burst_table_distribution(self, O):
        # burst length ~ Normal(mean 3, variance 2), read as
        # L = max(1, round(3 + sqrt2 Z)).  Compare the table's pmf with a
        # Monte-Carlo draw from numpy's normal generator.
        T = O.burst_table().astype(np.float64)
        assert T[0] == 0 and T[64] == 2 ** 32 and np.all(np.diff(T) >= 0)
        pmf = np.diff(T) / 2 ** 32  # P(L = l), l = 1..64
        z = np.random.default_rng(0).normal(3.0, math.sqrt(2.0), 2_000_000)
        L = np.maximum(1, np.rint(z)).astype(int)
        emp = np.bincount(L, minlength=65)[1:65] / L.size
        assert np.max(np.abs(emp - pmf)) < 2e-3
        mean = float((np.arange(1, 65) * pmf).sum())
        assert abs(mean - L.mean()) < 5e-3

    def test_poisson_table_vs_scipy(self, O):
        # R13: K ~ Poisson(mu) by inversion of T[k] = floor(2^32 P(K <= k))
        from scipy.stats import poisson
        assert O.poisson_table(0.0).tolist() == [2 ** 32]
        for mu in [1e-6, 0.5, 3.0, 31.9]:
            T = O.poisson_table(mu).astype(np.float64)
            assert T[-1] == 2 ** 32 and np.all(np.diff(T) >= 0)
            ks = np.arange(len(T) - 1)
            assert np.max(np.abs(T[:-1] / 2 ** 32 - poisson.cdf(ks, mu))) < 1e-9

    def test_rate_chunk(self, O):
        assert O.rate_chunk(0.0) == 2 ** 24 and O.rate_chunk(1e-8) == 2 ** 24
        for lam in [1e-6, 1e-4, 1e-2, 0.5]:
            ch = O.rate_chunk(lam)
            assert lam * ch <= 4 and (ch == 1 or lam * ch * 2 > 4)

    def _lap(self, O):
        A = G.laplacian_3d_7pt(12)
        return A, O.encode(A, 32)

    def test_rate_plan_is_poisson_process(self, O):
        # error events form a Poisson process over the arithmetic ops
        # (exponential gaps, mean 1/lambda): the count per call is
        # Poisson(lambda * ops), positions are uniform over the ops.
        A, enc = self._lap(O)
        ops_y, ops_t1, ops_t2 = 2 * A.nnz, 2 * int(enc.col.size), A.n
        ops = ops_y + ops_t1 + ops_t2
        lam = 20.0 / ops
        counts, tg = [], []
        for call in range(400):
            ro, ta, ix, mk = O.rate_plan(A, enc, O.Inject.rate(seed=3, lam=lam, call=call), 0)
            counts.append(len(ro))
            tg.extend(ta.tolist())
        counts = np.array(counts)
        assert abs(counts.mean() - 20.0) < 5 * math.sqrt(20.0 / 400)
        assert 0.7 < counts.var() / counts.mean() < 1.3  # Poisson dispersion
        tg = np.array(tg)
        for t, o in [(0, ops_y), (1, ops_t1), (2, ops_t2)]:
            p = o / ops
            assert abs((tg == t).mean() - p) < 5 * math.sqrt(p * (1 - p) / tg.size)

    def test_rate_plan_elements_weighted_by_ops(self, O):
        # a row with more entries (more ops) receives proportionally more events
        A, enc = self._lap(O)
        lam = 200.0 / (2 * A.nnz)
        idx = []
        for call in range(100):
            ro, ta, ix, mk = O.rate_plan(A, enc, O.Inject.rate(seed=5, lam=lam, call=call, targets=1), 0)
            assert np.all(ta == 0)
            idx.extend(ix.tolist())
        lens = A.row_lengths()
        hits = np.bincount(np.array(idx), minlength=A.n)
        for L in (4, 7):  # corner rows (4 entries) vs interior rows (7)
            sel = lens == L
            rate = hits[sel].sum() / sel.sum()
            expect = len(idx) * 2 * L / (2 * A.nnz)
            assert abs(rate - expect) < 0.15 * expect

    def test_rate_plan_masks_and_rounds(self, O):
        A, enc = self._lap(O)
        ro, ta, ix, mk = O.rate_plan(A, enc, O.Inject.rate(seed=1, lam=1e-3, call=2), 3)
        assert set(np.unique(ro).tolist()) <= {0, 1, 2, 3} and len(ro) > 100
        key = ro.astype(np.int64) * 4 + ta
        assert np.all(np.diff(key) >= 0)  # ordered by round, then op position
        for m in mk.tolist():
            lo = (m & -m).bit_length() - 1
            run = m >> lo
            assert m != 0 and run & (run + 1) == 0
        ro0, *_ = O.rate_plan(A, enc, O.Inject.rate(seed=1, lam=1e-3, call=2), 3, check=False)
        assert np.all(ro0 == 0)
        assert len(O.rate_plan(A, enc, O.Inject.rate(seed=1, lam=0.0), 3)[0]) == 0


# --------------------------------------------------------------------------
# PCG against SciPy's CG (an independent library routine)
# --------------------------------------------------------------------------
class TestPcg:
    def test_matches_scipy_cg(self, O):
        import scipy.sparse as sp
        import scipy.sparse.linalg as spla
        A = G.laplacian_3d_7pt(10)
        enc = O.encode(A, 32)
        xs = G.uniform_vector(A.n, 43)
        b = O.spmv(A, xs)
        x0 = G.uniform_vector(A.n, 44)
        r = O.pcg(A, enc, b, x0, tol=1e-6)
        assert r.status == 0
        S = sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(A.n, A.n))
        d = S.diagonal()
        M = spla.LinearOperator(S.shape, matvec=lambda v: v / d)
        xs_hist = []
        xsc, info = spla.cg(S, b, x0=x0.copy(), rtol=1e-6, atol=0.0, M=M,
                            callback=lambda xk: xs_hist.append(xk.copy()), maxiter=10 * A.n)
        assert info == 0
        assert r.iters == len(xs_hist)
        # residual histories agree (true residual of SciPy's iterates vs the
        # oracle's recursive residual) to well within 1e-10 * ||b||
        bn = np.linalg.norm(b)
        true_res = [np.linalg.norm(b - S @ xk) for xk in xs_hist]
        assert np.max(np.abs(np.array(true_res) - r.res_hist[1:])) < 1e-10 * bn
        assert np.linalg.norm(r.x - xsc) <= 1e-9 * np.linalg.norm(xsc)
        assert np.linalg.norm(r.x - xs) <= 1e-4 * np.linalg.norm(xs)

    def test_constant_diagonal_equals_cg(self, O):
        # Jacobi with a constant diagonal is plain CG up to scaling: the
        # iteration count equals SciPy's unpreconditioned CG.
        import scipy.sparse as sp
        import scipy.sparse.linalg as spla
        A = G.laplacian_2d_5pt(24)
        enc = O.encode(A, 32)
        b = O.spmv(A, G.uniform_vector(A.n, 1))
        x0 = np.zeros(A.n)
        r = O.pcg(A, enc, b, x0, tol=1e-8)
        S = sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(A.n, A.n))
        cnt = []
        spla.cg(S, b, x0=x0.copy(), rtol=1e-8, atol=0.0, callback=lambda xk: cnt.append(1))
        assert r.status == 0 and r.iters == len(cnt)

    def test_literal_stop_matches_scipy_atol(self, O):
        # P:296 read literally (R16*): stop when r^T r < eps, i.e. ||r|| <
        # sqrt(eps) -- SciPy's CG with rtol = 0, atol = sqrt(eps) stops at
        # the same iteration; the relative rule (R16) stops elsewhere here.
        import scipy.sparse as sp
        import scipy.sparse.linalg as spla
        A = G.laplacian_3d_7pt(10)
        enc = O.encode(A, 32)
        b = 40.0 * O.spmv(A, G.uniform_vector(A.n, 43))
        x0 = G.uniform_vector(A.n, 44)
        eps = 1e-6
        r = O.pcg(A, enc, b, x0, tol=eps, literal_stop=True)
        rel = O.pcg(A, enc, b, x0, tol=eps)
        assert r.status == 0 and r.iters != rel.iters
        assert r.res_hist[-1] ** 2 < eps * (1 + 1e-9) and r.res_hist[-2] ** 2 >= eps * (1 - 1e-9)
        S = sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(A.n, A.n))
        d = S.diagonal()
        M = spla.LinearOperator(S.shape, matvec=lambda v: v / d)
        cnt = []
        spla.cg(S, b, x0=x0.copy(), rtol=0.0, atol=np.sqrt(eps), M=M,
                callback=lambda xk: cnt.append(1), maxiter=10 * A.n)
        assert r.iters == len(cnt)

    def test_faulty_pcg_still_converges(self, O):
        # With faults in the protected SpMV at a high rate the solver still
        # converges because flagged blocks are recomputed.
        A = G.laplacian_3d_7pt(8)
        enc = O.encode(A, 32)
        xs = G.uniform_vector(A.n, 43)
        b = O.spmv(A, xs)
        x0 = G.uniform_vector(A.n, 44)
        clean = O.pcg(A, enc, b, x0, tol=1e-6)
        r = O.pcg(A, enc, b, x0, tol=1e-6, inj=O.Inject.rate(seed=9, lam=1e-4))
        assert r.status == 0 and r.flagged_blocks > 0 and r.recomputed_blocks >= r.flagged_blocks
        assert abs(r.iters - clean.iters) <= 3
        assert r.uncorrected_calls == 0

    def test_corrected_fault_leaves_pcg_bits_unchanged(self, O):
        # P:76 step 5: a fault the method flags is corrected by
        # recomputing its block, which restores y bit for bit, so a protected
        # PCG with one large fault in call 5 (a per-call list) has the
        # fault-free residual history and solution; the unprotected solve
        # with the same fault does not.
        A = G.laplacian_3d_7pt(8)
        enc = O.encode(A, 32)
        b = O.spmv(A, G.uniform_vector(A.n, 43))
        x0 = G.uniform_vector(A.n, 44)
        ref = O.pcg(A, enc, b, x0, tol=1e-6)
        plan = G.FaultPlan([0, 0], [0, 1], [100, 9],
                           [np.uint64(1) << np.uint64(61), np.uint64(1) << np.uint64(60)],
                           call=[5, 11])
        r = O.pcg(A, enc, b, x0, tol=1e-6, inj=O.Inject.from_plan(plan))
        assert r.status == 0 and r.flagged_blocks == 2 and r.uncorrected_calls == 0
        assert np.array_equal(r.res_hist.view(np.uint64), ref.res_hist.view(np.uint64))
        assert np.array_equal(r.x.view(np.uint64), ref.x.view(np.uint64))
        u = O.pcg(A, enc, b, x0, tol=1e-6, inj=O.Inject.from_plan(plan), check=False)
        assert not np.array_equal(u.res_hist[:8], ref.res_hist[:8])

    def test_unprotected_faulty_pcg_differs(self, O):
        A = G.laplacian_3d_7pt(8)
        enc = O.encode(A, 32)
        b = O.spmv(A, G.uniform_vector(A.n, 43))
        x0 = G.uniform_vector(A.n, 44)
        clean = O.pcg(A, enc, b, x0, tol=1e-6)
        r = O.pcg(A, enc, b, x0, tol=1e-6, inj=O.Inject.rate(seed=9, lam=1e-4), check=False)
        assert not np.array_equal(r.res_hist[: min(len(r.res_hist), len(clean.res_hist))],
                                  clean.res_hist[: min(len(r.res_hist), len(clean.res_hist))])


# --------------------------------------------------------------------------
# Related-work baseline: dense check [30, 31] with complete
# recomputation [31] (DESIGN.md
# R23-R25).  Pinned against column sums, eq. (1)'s invariant, the closed
# form of [35], the method's own encode at b_s = N, and fault behaviour.
# --------------------------------------------------------------------------
class TestDenseCheck:
    def test_c_is_column_sums_integer(self, O):
        A = G.random_csr(200, 0.05, 31, integer=True, empty_rows=0.1)
        D = np.zeros((A.n, A.n))
        for i in range(A.n):
            for q in range(A.row_ptr[i], A.row_ptr[i + 1]):
                D[i, A.col[q]] = A.val[q]
        e = O.dense_encode(A)
        assert np.array_equal(e.c, D.sum(axis=0))  # w = 1: c = 1^T A

    def test_c_laplacian_values(self, O):
        # 7-pt Dirichlet Laplacian (6 / -1): column sums are 6 - #neighbours
        e = O.dense_encode(G.laplacian_3d_7pt(6))
        assert set(np.unique(e.c).tolist()) == {0.0, 1.0, 2.0, 3.0}

    def test_c_pairwise_in_row_order(self, O):
        # column 0 holds (1, 1e16, -1e16, 1) in rows 0..3: PW gives
        # (1 + 1e16) + (-1e16 + 1) = 0; a left fold would give 1 (R23)
        D = np.array([[1.0, 1], [1e16, 0], [-1e16, 0], [1.0, 0]])
        D = np.pad(D, ((0, 0), (0, 2)))
        D[0, 1] = 1.0
        A = csr_from_dense(D)
        assert O.dense_encode(A).c[0] == 0.0

    def test_k35_closed_form(self, O):
        # A = diag(3, 4): sum ||a_i|| = 7, c = (3, 4), ||c|| = 5, n = m = 2:
        # ((2 + 2*2 - 2) * 7 + 2 * 5) * 2^-53 = 38 * 2^-53
        e = O.dense_encode(csr_from_dense(np.diag([3.0, 4.0])))
        assert e.k35 == 38.0 * EPS

    def test_k35_equals_method_bound_at_bs_n(self, O):
        # b_s = N: the method's bound reduces to [35];
        # integer stencil with every column present, N a power of two
        A = G.laplacian_2d_5pt(16)
        enc = O.encode(A, A.n)
        assert enc.nb == 1
        assert O.dense_encode(A).k35 == enc.K[0]

    def test_invariant_integer(self, O):
        # eq. (1)-(2): c^T x == w^T (A x) exactly for integer A and x
        A = G.random_csr(300, 0.04, 32, integer=True)
        x = np.random.default_rng(3).integers(-5, 6, A.n).astype(np.float64)
        r = O.dense_spmv(A, O.dense_encode(A), x)
        assert r.t1 == r.t2 and r.flag_rounds.sum() == 0

    @pytest.mark.parametrize("bound35", [False, True])
    def test_no_false_positive(self, O, bound35):
        for A in (G.laplacian_3d_7pt(10), G.random_csr(500, 0.02, 33), G.rmat(9, 8, 2)):
            e = O.dense_encode(A)
            for seed in range(3):
                x = G.uniform_vector(A.n, seed)
                r = O.dense_spmv(A, e, x, bound35=bound35)
                assert r.status == 0 and r.flag_rounds.sum() == 0
                assert np.array_equal(r.y, O.spmv(A, x))
                assert r.tau == (e.k35 * r.beta if bound35 else r.beta)  # P:262 / [35]

    @staticmethod
    def scale_mask(v, f=2.0 ** 20):
        """XOR mask that turns v into v * f (an exponent-field burst)."""
        return int(np.float64(v * f).view(np.uint64) ^ np.float64(v).view(np.uint64))

    def test_fault_flagged_and_recomputed(self, O):
        A = G.laplacian_3d_7pt(8)
        e = O.dense_encode(A)
        x = G.uniform_vector(A.n, 5)
        y = O.spmv(A, x)
        inj = O.Inject.from_plan(G.FaultPlan([0], [0], [77], [self.scale_mask(y[77])]))
        r = O.dense_spmv(A, e, x, inj=inj)
        assert r.status == 0 and r.flag_rounds.tolist() == [1, 0, 0, 0, 0]
        assert r.y_pre[77] == y[77] * 2.0 ** 20
        assert np.array_equal(r.y, y)  # complete recomputation

    def test_faults_every_round_exhaust(self, O):
        A = G.laplacian_2d_5pt(8)
        e = O.dense_encode(A)
        x = G.uniform_vector(A.n, 6)
        y = O.spmv(A, x)
        m = self.scale_mask(y[3])
        r0 = O.dense_spmv(A, e, x)
        mt1 = self.scale_mask(r0.t1)
        inj = O.Inject.from_plan(G.FaultPlan([0, 1, 2], [0, 1, 0], [3, 0, 3], [m, mt1, m]))
        r = O.dense_spmv(A, e, x, inj=inj, max_rounds=2)
        assert r.status == -6 and r.flag_rounds.tolist() == [1, 1, 1]

    def test_small_fault_below_norm_bound_missed(self, O):
        # the norm-based bound tau = ||x|| misses a fault the sparse
        # bound catches: the coverage gap of Fig. 7
        A = G.laplacian_3d_7pt(8)
        x = G.uniform_vector(A.n, 7)
        e = O.dense_encode(A)
        beta = math.sqrt(float(np.sum(x * x)))
        y = O.spmv(A, x)
        i = 100
        delta_target = 1e-3 * beta
        mask = np.float64(y[i] + delta_target).view(np.uint64) ^ np.float64(y[i]).view(np.uint64)
        inj = O.Inject.from_plan(G.FaultPlan([0], [0], [i], [int(mask)]))
        assert O.dense_spmv(A, e, x, inj=inj).flag_rounds[0] == 0
        enc = O.encode(A, 32)
        ref = O.abft_spmv(A, enc, x, inj)
        assert ref.flags[0].tolist() == [i // 32]


# --------------------------------------------------------------------------
# Related-work baseline: checkpoint-rollback PCG with dense
# checks (R26-R27).  Pinned: without faults it IS the
# plain Jacobi-PCG (itself pinned to SciPy above), bit for bit; under faults
# its bookkeeping obeys the rollback identities.  The rollback trajectory
# under random faults has no external reference (parity partially pinned).
# --------------------------------------------------------------------------
class TestPcgCheckpoint:
    def test_fault_free_equals_plain_pcg(self, O):
        A = G.laplacian_3d_7pt(10)
        enc = O.encode(A, 32)
        den = O.dense_encode(A)
        b = O.spmv(A, G.uniform_vector(A.n, 43))
        x0 = G.uniform_vector(A.n, 44)
        ref = O.pcg(A, enc, b, x0, tol=1e-6, check=False)
        r = O.pcg_cr(A, den, b, x0, tol=1e-6)
        assert r.status == 0 and r.rollbacks == 0
        assert r.iters == ref.iters == r.executed and r.spmv_calls == ref.iters + 1
        assert np.array_equal(r.res_hist, ref.res_hist) and np.array_equal(r.x, ref.x)

    def test_rollback_bookkeeping(self, O):
        A = G.laplacian_3d_7pt(8)
        den = O.dense_encode(A)
        xs = G.uniform_vector(A.n, 43)
        b = O.spmv(A, xs)
        x0 = G.uniform_vector(A.n, 44)
        r = O.pcg_cr(A, den, b, x0, tol=1e-6, inj=O.Inject.rate(seed=9, lam=1e-4, targets=1))
        assert r.rollbacks > 0
        # every executed iteration either advanced or was rolled back; each
        # rollback discards at most ckpt_every - 1 advanced iterations
        assert r.executed >= r.iters + r.rollbacks
        assert r.executed <= r.iters + r.rollbacks * 20
        assert r.spmv_calls >= r.executed + 1
        if r.status == 0:  # converged: the recursive residual met the test
            assert r.res_hist[-1] <= 1e-6 * np.linalg.norm(b)

    def test_detected_fault_rolls_back_to_fault_free_bits(self, O):
        # after a detection the solver restores the last sample and
        # re-executes from it.  A single fault in call 24 of the solve (the
        # SpMV of iteration 24; |delta| far above ||p||) is detected, the
        # state sampled after iteration 20 is restored, and iterations 21..24
        # run again: 4 more executed iterations and SpMV calls than the
        # fault-free solve.  The re-execution repeats the fault-free
        # operations exactly, so the returned x and residual history are the
        # fault-free run's bit for bit.
        A = G.laplacian_3d_7pt(8)
        den = O.dense_encode(A)
        b = O.spmv(A, G.uniform_vector(A.n, 43))
        x0 = G.uniform_vector(A.n, 44)
        ref = O.pcg_cr(A, den, b, x0, tol=1e-6)
        assert ref.rollbacks == 0 and ref.iters > 24
        plan = G.FaultPlan([0], [0], [77], [np.uint64(1) << np.uint64(62)], call=[24])
        r = O.pcg_cr(A, den, b, x0, tol=1e-6, inj=O.Inject.from_plan(plan))
        assert r.status == 0 and r.rollbacks == 1
        assert r.executed == ref.executed + 4 and r.spmv_calls == ref.spmv_calls + 4
        assert r.iters == ref.iters
        assert np.array_equal(r.res_hist.view(np.uint64), ref.res_hist.view(np.uint64))
        assert np.array_equal(r.x.view(np.uint64), ref.x.view(np.uint64))

    def test_sample_every_iteration_loses_nothing(self, O):
        # ckpt_every = 1: a rollback restores the state of the iteration it
        # interrupted, so executed = iters + rollbacks exactly
        A = G.laplacian_3d_7pt(8)
        den = O.dense_encode(A)
        b = O.spmv(A, G.uniform_vector(A.n, 43))
        x0 = G.uniform_vector(A.n, 44)
        r = O.pcg_cr(A, den, b, x0, tol=1e-6, ckpt_every=1,
                     inj=O.Inject.rate(seed=9, lam=1e-4, targets=1))
        assert r.rollbacks > 0 and r.executed == r.iters + r.rollbacks


# --------------------------------------------------------------------------
# Distributed PCG oracle (R28): dots partitioned by
# rank.  Pinned to the C oracle's PCG (independent code) and to SciPy's CG.
# --------------------------------------------------------------------------
class TestPcgRanks:
    def _problem(self, O, A):
        b = O.spmv(A, G.uniform_vector(A.n, 43))
        return b, G.uniform_vector(A.n, 44)

    def test_one_rank_is_single_gpu_pcg(self, O):
        A = G.laplacian_3d_7pt(10)
        b, x0 = self._problem(O, A)
        ref = O.pcg(A, O.encode(A, 32), b, x0, tol=1e-6, check=False)
        r = O.pcg_ranks(A, b, x0, [(0, A.n)], tol=1e-6)
        assert r.status == ref.status == 0 and r.iters == ref.iters
        assert np.array_equal(r.res_hist.view(np.uint64), ref.res_hist.view(np.uint64))
        assert np.array_equal(r.x.view(np.uint64), ref.x.view(np.uint64))

    @pytest.mark.parametrize("world", [2, 4])
    def test_power_of_two_ranks_are_bit_identical(self, O, world):
        # PW is padding independent (R2): equal power-of-two row ranges are
        # aligned subtrees, so rank partials + a tree over ranks = global PW.
        A = G.laplacian_3d_7pt(16)  # 4096 rows
        b, x0 = self._problem(O, A)
        ref = O.pcg(A, O.encode(A, 32), b, x0, tol=1e-6, check=False)
        ranges = [(r * A.n // world, (r + 1) * A.n // world) for r in range(world)]
        r = O.pcg_ranks(A, b, x0, ranges, tol=1e-6)
        assert r.iters == ref.iters
        assert np.array_equal(r.res_hist.view(np.uint64), ref.res_hist.view(np.uint64))
        assert np.array_equal(r.x.view(np.uint64), ref.x.view(np.uint64))

    def test_uneven_ranks_match_scipy(self, O):
        # 3 ranks of 12^3 / 3-plane-aligned rows: the summation order differs
        # from one GPU, the iterates still follow CG (SciPy) to rounding.
        import scipy.sparse as sp
        import scipy.sparse.linalg as spla
        A = G.laplacian_3d_7pt(12)
        b, x0 = self._problem(O, A)
        ranges = [(0, 576), (576, 1152), (1152, A.n)]
        r = O.pcg_ranks(A, b, x0, ranges, tol=1e-6)
        assert r.status == 0
        S = sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(A.n, A.n))
        d = S.diagonal()
        M = spla.LinearOperator(S.shape, matvec=lambda v: v / d)
        hist = []
        xsc, info = spla.cg(S, b, x0=x0.copy(), rtol=1e-6, atol=0.0, M=M,
                            callback=lambda xk: hist.append(np.linalg.norm(b - S @ xk)))
        assert info == 0 and r.iters == len(hist)
        assert np.max(np.abs(np.array(hist) - r.res_hist[1:])) < 1e-10 * np.linalg.norm(b)
        assert np.linalg.norm(r.x - xsc) <= 1e-9 * np.linalg.norm(xsc)

    def test_dot_ranks_special_cases(self, O):
        v = G.uniform_vector(1000, 5)
        w = G.uniform_vector(1000, 6)
        assert O.dot_ranks(v, w, [(0, 1000)]) == O.pw(v * w)
        # exact small-integer sums: any order gives the exact result
        a = np.arange(1, 101, dtype=np.float64)
        assert O.dot_ranks(a, np.ones(100), [(0, 7), (7, 50), (50, 100)]) == 5050.0
        assert O.dot_ranks(a, a, [(0, 0), (0, 100)]) == float(np.sum(a * a))


class TestPcgSingleReduction:
    """Chronopoulos-Gear PCG (R29): same Krylov iterates as PCG in exact
    arithmetic.  Pins: SciPy's CG (independent), finite termination on a
    diagonal matrix, and agreement with the textbook oracle to rounding."""

    def test_matches_scipy_cg(self, O):
        import scipy.sparse as sp
        import scipy.sparse.linalg as spla
        A = G.laplacian_3d_7pt(12)
        b = O.spmv(A, G.uniform_vector(A.n, 43))
        x0 = G.uniform_vector(A.n, 44)
        r = O.pcg_cg1_ranks(A, b, x0, [(0, A.n)], tol=1e-6)
        assert r.status == 0
        S = sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(A.n, A.n))
        d = S.diagonal()
        M = spla.LinearOperator(S.shape, matvec=lambda v: v / d)
        hist = []
        xsc, info = spla.cg(S, b, x0=x0.copy(), rtol=1e-6, atol=0.0, M=M,
                            callback=lambda xk: hist.append(np.linalg.norm(b - S @ xk)))
        assert info == 0 and r.iters == len(hist)
        assert r.spmv_calls == r.iters + 2
        assert np.max(np.abs(np.array(hist) - r.res_hist[1:])) < 1e-9 * np.linalg.norm(b)
        assert np.linalg.norm(r.x - xsc) <= 1e-8 * np.linalg.norm(xsc)

    def test_diagonal_matrix_one_iteration(self, O):
        # M^-1 A = I: the first step solves exactly (alpha = 1, x = x0 + u0)
        n = 64
        vals = 2.0 ** np.arange(-3, 3, dtype=np.float64).repeat(11)[:n]
        A = G.CSR(np.arange(n + 1, dtype=np.int32), np.arange(n, dtype=np.int32), vals)
        xs = G.uniform_vector(n, 3)
        b = vals * xs
        r = O.pcg_cg1_ranks(A, b, np.zeros(n), [(0, 32), (32, 64)], tol=1e-12)
        assert r.status == 0 and r.iters == 1
        assert np.array_equal(r.x, xs)

    def test_close_to_textbook_pcg(self, O):
        A = G.stencil_3d_27pt(10, 10, 12)
        b = O.spmv(A, G.uniform_vector(A.n, 43))
        x0 = G.uniform_vector(A.n, 44)
        ranges = [(0, 400), (400, A.n)]
        ref = O.pcg_ranks(A, b, x0, ranges, tol=1e-8)
        r = O.pcg_cg1_ranks(A, b, x0, ranges, tol=1e-8)
        assert r.status == ref.status == 0 and abs(r.iters - ref.iters) <= 1
        k = min(r.iters, ref.iters)
        assert np.max(np.abs(r.res_hist[:k] - ref.res_hist[:k])) < 1e-10 * np.linalg.norm(b)
        assert np.linalg.norm(r.x - ref.x) <= 1e-8 * np.linalg.norm(ref.x)
