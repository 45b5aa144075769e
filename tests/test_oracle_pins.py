"""Pins of the CPU oracle (oracle/bandlu_oracle.c) against things other than
itself (task ③): reference LAPACK bitwise (scipy/OpenBLAS), dense GEPP brute
force, an exact-rational golden of the paper's Fig. 2 shape, closed forms,
special cases and invariants.  CPU only.

Each pin is chosen so that a plausible oracle bug fails at least one test:
 * wrong pivot tie rule / index      -> scipy bitwise, ties test, dense GEPP
 * dropped fill zeroing / swap range -> scipy bitwise with NaN fill rows
 * wrong sign / transposed operand   -> closed form, dense GEPP, backward error
 * division instead of reciprocal    -> scipy bitwise (27% of quotients differ)
 * missing FMA / extra contraction   -> scipy bitwise (up to 7e-10 rel diffs)
"""
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
from tests.bandref import (band_factors_to_dense, band_to_dense, backward_error, dense_gepp,
                           same_bits)

L = pytest.importorskip("scipy.linalg.lapack")

# shapes of SURVEY Appendix A probe 4 (trf) -- all on LAPACK's dgbtf2 path (Q20)
TRF_SHAPES = [  # (m, n, kl, ku)
    (40, 40, 2, 3), (30, 30, 1, 1), (20, 20, 0, 0), (90, 90, 40, 64), (60, 60, 10, 7),
    (50, 50, 3, 0), (50, 50, 0, 3), (64, 64, 32, 32), (64, 64, 2, 2), (48, 48, 2, 32),
    (40, 40, 1, 1), (33, 33, 32, 0), (30, 20, 2, 3), (20, 30, 3, 2), (1, 1, 0, 0),
    (1, 5, 2, 1), (5, 1, 2, 1), (9, 9, 2, 3), (256, 256, 1, 1), (512, 512, 10, 10),
    (130, 70, 5, 9), (70, 130, 9, 5), (3, 40, 7, 2), (40, 3, 7, 2),
]
TRS_SHAPES = [  # (n, kl, ku, nrhs)
    (30, 2, 3, 1), (25, 1, 1, 2), (20, 3, 0, 1), (20, 0, 2, 3), (60, 10, 7, 1),
    (64, 2, 32, 16), (64, 32, 32, 2), (80, 10, 10, 1), (50, 1, 1, 5), (40, 0, 5, 2),
    (40, 5, 0, 2), (1, 0, 0, 1), (2, 1, 1, 1), (512, 10, 10, 1), (1024, 2, 32, 3),
]


def _scipy_trf(ab_c: np.ndarray, m, n, kl, ku):
    lu, piv, info = L.dgbtrf(ab_c.T.copy(order="F"), kl, ku, m=m, n=n)
    return lu.T, piv + 1, info


@pytest.mark.parametrize("m,n,kl,ku", TRF_SHAPES)
def test_trf_bitwise_vs_reference_lapack(m, n, kl, ku):
    """P2: oracle == reference LAPACK dgbtrf (dgbtf2 path) bitwise, incl. the
    NaN pattern of fill rows and corners (fill ignored on input, corners never
    written, Q5/Q6)."""
    A = I.gen_band(m, n, kl, ku, count=4, first=7)
    A0 = A.copy()
    ipiv, info = oracle.dgbtrf(A, m, n, kl, ku)
    for b in range(4):
        lu, piv, inf = _scipy_trf(A0[b], m, n, kl, ku)
        assert np.all(same_bits(lu, A[b]))
        assert np.array_equal(piv, ipiv[b])
        assert inf == info[b]


@pytest.mark.parametrize("n,kl,ku,nrhs", TRS_SHAPES)
def test_trs_bitwise_vs_reference_lapack(n, kl, ku, nrhs):
    A = I.gen_band(n, n, kl, ku, count=3)
    B = I.gen_rhs(n, nrhs, ldb=n + 3, count=3)  # padded ldb: rows >= n are NaN sentinels
    ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
    B0 = B.copy()
    oracle.dgbtrs(A, ipiv, B, n, kl, ku)
    for b in range(3):
        x, inf = L.dgbtrs(A[b].T.copy(order="F"), kl, ku, B0[b].T.copy(order="F"), ipiv[b] - 1)
        assert inf == 0
        assert np.all(same_bits(x.T, B[b]))
        assert np.all(np.isnan(B[b][:, n:]))  # ldb padding untouched


@pytest.mark.parametrize("n,kl,ku,nrhs", [(30, 2, 3, 2), (64, 10, 7, 1), (100, 1, 1, 4)])
def test_gbsv_bitwise_vs_reference_lapack(n, kl, ku, nrhs):
    A = I.gen_band(n, n, kl, ku, count=3)
    B = I.gen_rhs(n, nrhs, count=3)
    A0, B0 = A.copy(), B.copy()
    ipiv, info = oracle.dgbsv(A, B, n, kl, ku)
    for b in range(3):
        lu, piv, x, inf = L.dgbsv(kl, ku, A0[b].T.copy(order="F"), B0[b].T.copy(order="F"))
        assert inf == info[b] == 0
        assert np.array_equal(piv + 1, ipiv[b])
        assert np.all(same_bits(lu.T, A[b]))
        assert np.all(same_bits(x.T, B[b]))


@pytest.mark.parametrize("m,n,kl,ku", [(12, 12, 2, 3), (25, 25, 4, 1), (30, 30, 1, 1),
                                       (20, 14, 3, 2), (14, 20, 2, 4), (16, 16, 0, 3),
                                       (16, 16, 3, 0), (35, 35, 6, 6)])
def test_trf_vs_dense_gepp_bruteforce(m, n, kl, ku):
    """P1: band LU == dense textbook GEPP on the expanded matrix: same pivots,
    dense U has bandwidth <= kv and equals band U, band L column j after the
    later interchanges equals dense L column j."""
    A = I.gen_band(m, n, kl, ku, count=3, first=100)
    A0 = A.copy()
    ipiv, info, gap = oracle.dgbtrf(A, m, n, kl, ku, return_gap=True)
    for b in range(3):
        assert gap[b] > 1e-9  # tie-free input, pivots are unique
        D = band_to_dense(A0[b], m, n, kl, ku)
        LU, dpiv, dinfo = dense_gepp(D)
        assert np.array_equal(dpiv, ipiv[b]) and dinfo == info[b]
        mn = min(m, n)
        Ud = np.triu(LU[:mn, :])
        # U bandwidth <= kl + ku
        for i in range(mn):
            assert np.all(Ud[i, i + kl + ku + 1:] == 0)
        Lb, Ub = band_factors_to_dense(A[b], ipiv[b], m, n, kl, ku)
        Ld = np.tril(LU[:, :mn], -1) + np.eye(m, mn)
        scale = max(1.0, np.abs(Ud).max())
        assert np.abs(Ub - Ud).max() <= 1e-13 * scale
        assert np.abs(Lb - Ld).max() <= 1e-13
        # and P A = L U reconstructs the input
        P = np.eye(m)
        for j in range(mn):
            p = ipiv[b][j] - 1
            P[[j, p], :] = P[[p, j], :]
        assert np.abs(P @ D - Lb @ Ub).max() <= 1e-13 * max(1.0, np.abs(D).max())


def test_fig2_shape_exact_golden():
    """Golden: exact-rational band LU of a 9x9 (kl=2, ku=3) matrix (the shape of
    the paper's Fig. 2) -- pivots exact, factors and solution within
    a few ulps of the exact rationals."""
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "fig2_9x9_kl2_ku3.json")))
    n, kl, ku = g["n"], g["kl"], g["ku"]
    kv = kl + ku
    ldab = 2 * kl + ku + 1
    Ad = np.array([[float(Fraction(v)) for v in row] for row in g["A_dense"]])
    ab = np.full((1, n, ldab), np.nan)
    for j in range(n):
        for i in range(max(0, j - ku), min(n, j + kl + 1)):
            ab[0, j, kv + i - j] = Ad[i, j]
    B = np.array([float(Fraction(v)) for v in g["b"]]).reshape(1, 1, n)
    ipiv, info = oracle.dgbsv(ab, B, n, kl, ku)
    assert info[0] == 0
    assert list(ipiv[0]) == g["ipiv"]
    for key, val in g["lu_band"].items():
        r, c = map(int, key.split(","))
        exact = float(Fraction(val))
        assert abs(ab[0, c, r] - exact) <= 1e-13 * max(1.0, abs(exact)), (r, c)
    x = np.array([float(Fraction(v)) for v in g["x"]])
    assert np.abs(B[0, 0] - x).max() <= 1e-12 * max(1.0, np.abs(x).max())


@pytest.mark.parametrize("n", [1, 2, 3, 17, 64, 200])
def test_closed_form_tridiagonal(n):
    """P4: tridiag(-1, 2, -1): no interchanges, u_ii = (i+1)/i, l_i = -i/(i+1),
    superdiagonal -1, fill row 0; b = 1 -> x_i = i (n+1-i) / 2 (1-based i)."""
    kl = ku = 1
    ab = np.full((1, n, 4), np.nan)
    ab[0, :, 1] = -1.0  # superdiagonal
    ab[0, :, 2] = 2.0   # diagonal
    ab[0, :, 3] = -1.0  # subdiagonal
    ab[0, 0, 1] = np.nan       # corner
    ab[0, n - 1, 3] = np.nan   # corner
    B = np.ones((1, 1, n))
    ipiv, info = oracle.dgbsv(ab, B, n, kl, ku)
    i = np.arange(1, n + 1)
    assert info[0] == 0 and np.array_equal(ipiv[0], i)
    assert np.abs(ab[0, :, 2] - (i + 1) / i).max() <= 1e-14  # a few ulps; a structural bug is O(1)
    if n > 1:
        assert np.abs(ab[0, :n - 1, 3] - (-i[:-1] / (i[:-1] + 1))).max() <= 1e-14
        assert np.all(ab[0, 1:, 1] == -1.0)
        assert np.all(ab[0, 2:, 0] == 0.0)  # fill row: zero, no fill occurred
    assert np.isnan(ab[0, 0, 0]) and np.isnan(ab[0, 0, 1]) and np.isnan(ab[0, n - 1, 3])
    x = i * (n + 1 - i) / 2.0
    assert np.abs(B[0, 0] - x).max() <= 1e-14 * x.max() * max(1, n / 16)


def test_diagonal_case():
    """P5: kl = ku = 0 (ldab = 1): identity pivots, factors untouched, x = b/d
    bitwise, info = first zero diagonal."""
    n = 50
    d = I.gen_band(n, n, 0, 0, count=1)[:, :, :]
    B = I.gen_rhs(n, 2, count=1)
    d0, B0 = d.copy(), B.copy()
    ipiv, info = oracle.dgbsv(d, B, n, 0, 0)
    assert info[0] == 0 and np.array_equal(ipiv[0], np.arange(1, n + 1))
    assert np.array_equal(d, d0)
    assert np.array_equal(B[0], B0[0] / d0[0, :, 0][None, :])
    d2 = d0.copy()
    d2[0, 7, 0] = 0.0
    d2[0, 30, 0] = 0.0
    ipiv, info = oracle.dgbtrf(d2, n, n, 0, 0)
    assert info[0] == 8


@pytest.mark.parametrize("n,kl,ku", [(200, 10, 10), (300, 1, 1), (150, 2, 32), (100, 32, 32)])
def test_diagonally_dominant_no_pivoting(n, kl, ku):
    """P6: column diagonally dominant => GEPP never interchanges: identity ipiv
    and all fill rows zero."""
    A = I.gen_band(n, n, kl, ku, count=2)
    kv = kl + ku
    for b in range(2):
        for j in range(n):
            col = A[b, j, kl:kv + kl + 1]
            s = np.nansum(np.abs(col)) - abs(col[ku])
            A[b, j, kv] = s + 1.0
    ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
    assert np.all(info == 0)
    assert np.array_equal(ipiv, np.tile(np.arange(1, n + 1), (2, 1)))
    for b in range(2):
        for j in range(n):
            for r in range(kl):
                if j - kv + r >= 0:
                    assert A[b, j, r] == 0.0


@pytest.mark.parametrize("kl,ku", [(2, 3), (3, 0), (0, 2), (1, 1), (10, 10)])
@pytest.mark.parametrize("z", [1, 2, 20, 39, 40])
def test_planted_zero_column_info(kl, ku, z):
    """P7: a zero column z (1-based) of A gives info = z and ipiv[z-1] = z; with
    two zero columns, info = the first.  The factorization still completes."""
    n = 40
    A = I.gen_band(n, n, kl, ku, count=1)
    kv = kl + ku
    A[0, z - 1, kl:kv + kl + 1] = np.where(np.isnan(A[0, z - 1, kl:kv + kl + 1]), np.nan, 0.0)
    A2 = A.copy()
    ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
    assert info[0] == z and ipiv[0, z - 1] == z
    if z < n:
        A2[0, n - 1, kl:kv + kl + 1] = np.where(np.isnan(A2[0, n - 1, kl:kv + kl + 1]), np.nan, 0.0)
        ipiv2, info2 = oracle.dgbtrf(A2, n, n, kl, ku)
        assert info2[0] == z


@pytest.mark.parametrize("m,n,kl,ku", [(60, 60, 3, 2), (64, 64, 10, 7), (30, 45, 4, 4), (45, 30, 4, 4)])
def test_invariants_and_sentinels(m, n, kl, ku):
    """P8: ipiv[j] in [j+1, min(m, j+1+kl)]; info in {0} U [1, min(m,n)];
    input fill values ignored; corner and padding rows never written."""
    ldab = 2 * kl + ku + 1 + 3
    A = I.gen_band(m, n, kl, ku, ldab=ldab, count=3)
    Ab = A.copy()
    Ab[:, :, :kl] = 12345.0  # different fill-row input: must not matter
    ipiv, info = oracle.dgbtrf(A, m, n, kl, ku)
    ipiv_b, info_b = oracle.dgbtrf(Ab, m, n, kl, ku)
    j = np.arange(min(m, n))
    assert np.all(ipiv >= j + 1) and np.all(ipiv <= np.minimum(m, j + 1 + kl))
    assert np.array_equal(ipiv, ipiv_b) and np.array_equal(info, info_b)
    outm = I.band_output_mask(m, n, kl, ku, ldab)
    assert np.all(same_bits(A[:, outm], Ab[:, outm]))
    # padding rows still NaN; corners below/above the matrix still NaN
    # (for m < n LAPACK's SET_FILLIN also zeroes fill rows of rows >= m -- see DESIGN.md)
    assert np.all(np.isnan(A[:, :, 2 * kl + ku + 1:]))
    kv = kl + ku
    for c in range(n):
        for r in range(2 * kl + ku + 1):
            i = c - kv + r
            if i < 0 or (i >= m and r >= kl):
                assert np.all(np.isnan(A[:, c, r])), (c, r)


@pytest.mark.parametrize("n,kl,ku,nrhs", [(64, 2, 2, 1), (256, 1, 1, 1), (512, 10, 10, 1),
                                           (300, 2, 32, 16), (400, 32, 32, 1), (512, 2, 3, 1),
                                           (512, 10, 7, 1)])
def test_backward_error(n, kl, ku, nrhs):
    """P9: scaled backward error ||Ax-b||_1/(||A||_1 ||x||_1 n eps) <= 10 (north_star)."""
    A = I.gen_band(n, n, kl, ku, count=2)
    B = I.gen_rhs(n, nrhs, count=2)
    A0, B0 = A.copy(), B.copy()
    ipiv, info = oracle.dgbsv(A, B, n, kl, ku)
    for b in range(2):
        D = band_to_dense(A0[b], n, n, kl, ku)
        eta = backward_error(D, B[b].T, B0[b].T)
        assert eta <= 10.0, eta


def test_gbsv_singular_leaves_b_untouched():
    """P10 / Q11: info > 0 => B bitwise unchanged (LAPACK DGBSV)."""
    n, kl, ku = 30, 2, 3
    A = I.gen_band(n, n, kl, ku, count=2)
    A[1, 5, kl:] = np.where(np.isnan(A[1, 5, kl:]), np.nan, 0.0)
    B = I.gen_rhs(n, 2, count=2)
    B0 = B.copy()
    ipiv, info = oracle.dgbsv(A, B, n, kl, ku)
    assert info[0] == 0 and info[1] == 6
    assert np.array_equal(B[1], B0[1])
    assert not np.array_equal(B[0], B0[0])


def test_pivot_tie_first_index():
    """Q2: |candidates| tie -> first index (no interchange)."""
    ab = np.array([[[np.nan, 1.0, -1.0]]])  # n=1? use n=2 below
    n, kl, ku = 2, 1, 0
    ab = np.full((1, n, 2 * kl + ku + 1), np.nan)
    ab[0, 0, 1] = 1.0   # A(0,0)
    ab[0, 0, 2] = -1.0  # A(1,0)
    ab[0, 1, 1] = 3.0   # A(1,1)
    ipiv, info = oracle.dgbtrf(ab, n, n, kl, ku)
    assert list(ipiv[0]) == [1, 2]
    assert ab[0, 0, 2] == -1.0 and ab[0, 1, 1] == 3.0 - (-1.0) * 0.0


def test_quick_returns():
    A = np.zeros((2, 0, 3))
    ipiv, info = oracle.dgbtrf(A, 0, 0, 1, 0)
    assert np.all(info == 0)
    A = I.gen_band(5, 5, 1, 1, count=1)
    A0 = A.copy()
    ipiv, info = oracle.dgbtrf(A, 0, 5, 1, 1)
    assert np.all(same_bits(A, A0))


def test_generator_is_counter_based():
    """Any shard regenerates identically; values independent of ldab padding."""
    a = I.gen_band(64, 64, 2, 2, count=10)
    b = I.gen_band(64, 64, 2, 2, count=4, first=3)
    c = I.gen_band(64, 64, 2, 2, ldab=11, count=10)
    assert np.array_equal(a[3:7], b, equal_nan=True)
    assert np.array_equal(a, c[:, :, :7], equal_nan=True)
    v = a[~np.isnan(a)]
    assert v.min() >= -1.0 and v.max() < 1.0 and abs(v.mean()) < 0.05
    assert I.shard_range(10000, 3, 8) == (3750, 5000)


def test_alg_bytes_match_survey_table():
    assert sum(I.alg_bytes(64, 64, 2, 2, 1)) == 11012
    assert sum(I.alg_bytes(256, 256, 1, 1, 1)) == 28596
    assert sum(I.alg_bytes(512, 512, 10, 10, 1)) == 347140
    assert sum(I.alg_bytes(1024, 1024, 2, 32, 16)) == 1149452
    assert I.nominal_flops(512, 10, 10, 1) == (106035, 30702)


# ---------------------------------------------------------------- trans = 'T'
@pytest.mark.parametrize("n,kl,ku,nrhs", [(30, 2, 3, 2), (64, 10, 10, 1), (50, 1, 1, 3), (40, 5, 0, 2),
                                           (40, 0, 5, 2), (128, 2, 32, 4), (1, 0, 0, 1), (2, 1, 1, 1)])
def test_trs_transposed_vs_reference_lapack_and_residual(n, kl, ku, nrhs):
    """f2: dgbtrs('T') solves A^T X = B.  OpenBLAS reorders the dot products,
    so the pin is (a) normwise agreement with reference LAPACK to 1e-12 and
    (b) the scaled backward error of A^T x = b <= 10."""
    A = I.gen_band(n, n, kl, ku, count=3)
    A0 = A.copy()
    B = I.gen_rhs(n, nrhs, ldb=n + 2, count=3)
    B0 = B.copy()
    ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
    oracle.dgbtrs(A, ipiv, B, n, kl, ku, trans="T")
    for b in range(3):
        x, inf = L.dgbtrs(A[b].T.copy(order="F"), kl, ku, B0[b].T.copy(order="F"), ipiv[b] - 1, trans=1)
        X = B[b][:, :n]
        assert np.abs(x.T[:, :n] - X).max() <= 1e-12 * max(1.0, np.abs(X).max())
        assert np.all(np.isnan(B[b][:, n:]))
        D = band_to_dense(A0[b], n, n, kl, ku)
        assert backward_error(D.T, X.T, B0[b][:, :n].T) <= 10.0


def test_trs_transposed_special_cases():
    # diagonal: x = b / d bitwise
    n = 20
    d = I.gen_band(n, n, 0, 0, count=1)
    B = I.gen_rhs(n, 2, count=1)
    B0 = B.copy()
    ipiv, info = oracle.dgbtrf(d, n, n, 0, 0)
    oracle.dgbtrs(d, ipiv, B, n, 0, 0, trans="T")
    assert np.array_equal(B[0], B0[0] / d[0, :, 0][None, :])
    # symmetric tridiag(-1, 2, -1): A^T = A, so 'T' and 'N' solutions agree to rounding
    n = 50
    ab = np.full((1, n, 4), np.nan)
    ab[0, :, 1] = -1.0; ab[0, :, 2] = 2.0; ab[0, :, 3] = -1.0
    ipiv, info = oracle.dgbtrf(ab, n, n, 1, 1)
    Bn = np.ones((1, 1, n)); Bt = np.ones((1, 1, n))
    oracle.dgbtrs(ab, ipiv, Bn, n, 1, 1, trans="N")
    oracle.dgbtrs(ab, ipiv, Bt, n, 1, 1, trans="T")
    i = np.arange(1, n + 1)
    assert np.abs(Bt[0, 0] - i * (n + 1 - i) / 2).max() <= 1e-11
    assert np.abs(Bt - Bn).max() <= 1e-11
