"""GPU parity: the sm_100a path (through the C ABI) vs the CPU oracle,
element by element on the same seeded inputs (task ③).

Bar (BASELINE.json north_star): ipiv and info bit-exact; factors within
1e-12 max relative entrywise error -- and since the kernels execute the
oracle's exact fp64 operation sequence we assert the stronger `==` equality
(signed zeros compare equal) plus an identical NaN pattern over
the WHOLE band array (fill rows, corners and padding rows carry NaN
sentinels, so any stray read or write shows up); solutions likewise, and the
scaled backward error <= 10.
"""
import numpy as np
import pytest

import oracle
from paper_conf_sc_abdelfattahtlad23_b200 import inputs as I
from tests.bandref import backward_error, band_to_dense, same_bits

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_sc_abdelfattahtlad23_b200 as bl  # noqa: E402

WINDOW_BANDS = [(0, 0), (0, 3), (1, 1), (2, 2), (2, 3), (3, 0), (3, 2), (4, 4), (10, 7), (10, 10), (2, 32)]
WIDE_BANDS = [(32, 32)]  # kl+1 > 32: two-warp ROWS factorization, window solve kernel
ALL_BANDS = WINDOW_BANDS + WIDE_BANDS


def _gpu_trf(A_np, m, n, kl, ku, variant=bl.AUTO):
    A = torch.from_numpy(A_np).cuda()
    batch = A.shape[0]
    ipiv = torch.zeros((batch, max(min(m, n), 1)), dtype=torch.int32, device="cuda")
    info = torch.full((batch,), -7, dtype=torch.int32, device="cuda")
    bl.dgbtrf_strided_batched(m, n, kl, ku, A, ipiv, info, variant=variant)
    torch.cuda.synchronize()
    return A.cpu().numpy(), ipiv.cpu().numpy()[:, :min(m, n)], info.cpu().numpy()


def trf_variants(kl, ku, square=True):
    """Forced factorization variants to cross-check: the safeguard, the row-owner
    window, and the row-slot (ROWS), thread-per-matrix (TPM, square only) and
    tensor-core (DMMA) kernels where they are compiled for (kl, ku)."""
    v = [bl.WINDOW, bl.GENERIC] if (kl, ku) in WINDOW_BANDS else [bl.GENERIC]
    if square and bl.tpm_available(kl, ku):
        v.append(bl.TPM)
    if square and bl.thin_available(kl, ku):
        v.append(bl.THIN)
    if square and bl.cols_available(kl, ku):
        v.append(bl.COLS)
    if bl.rows_available(kl, ku):
        v.append(bl.ROWS)
    if bl.tc_available(kl, ku):
        v.append(bl.TC)
    if bl.thread_available(kl, ku):
        v.append(bl.THREAD)
    return v


def _check_trf(m, n, kl, ku, batch, variant, ldab=None, first=0, A_in=None):
    A0 = I.gen_band(m, n, kl, ku, ldab=ldab, count=batch, first=first) if A_in is None else A_in
    Ao = A0.copy()
    ipo, info_o = oracle.dgbtrf(Ao, m, n, kl, ku)
    Ag, ipg, info_g = _gpu_trf(A0, m, n, kl, ku, variant)
    assert np.array_equal(info_g, info_o)
    assert np.array_equal(ipg, ipo)
    bad = ~same_bits(Ag, Ao)
    assert not bad.any(), f"{bad.sum()} mismatching band entries, first at {np.argwhere(bad)[0]}"
    return Ao, ipo, info_o


@pytest.mark.parametrize("kl,ku", ALL_BANDS)
@pytest.mark.parametrize("variant", [bl.WINDOW, bl.GENERIC, bl.ROWS, bl.TC, bl.THREAD, bl.TPM, bl.THIN, bl.COLS])
@pytest.mark.parametrize("n", [1, 2, 7, 37, 100])
def test_trf_parity_small(kl, ku, variant, n):
    if variant not in trf_variants(kl, ku):
        pytest.skip("no tensor-core kernel compiled for this band")
    # ragged batch (not a multiple of matrices per warp / block)
    _check_trf(n, n, kl, ku, batch=37, variant=variant)


@pytest.mark.parametrize("kl,ku", ALL_BANDS)
@pytest.mark.parametrize("mn", [(30, 20), (20, 30), (5, 40), (40, 5), (1, 9), (9, 1)])
def test_trf_parity_rectangular(kl, ku, mn):
    m, n = mn
    for variant in trf_variants(kl, ku, square=False):
        _check_trf(m, n, kl, ku, batch=9, variant=variant)


@pytest.mark.parametrize("kl,ku", [(2, 3), (10, 10), (5, 9), (33, 20), (32, 32), (40, 64), (0, 40)])
def test_trf_parity_generic_any_band(kl, ku):
    _check_trf(150, 150, kl, ku, batch=11, variant=bl.GENERIC)
    assert bl.trf_variant(150, 150, kl, ku) in (bl.GENERIC, bl.WINDOW, bl.ROWS, bl.COLS)


@pytest.mark.parametrize("kl,ku", [(1, 1), (10, 10), (2, 32), (32, 32)])
def test_trf_parity_padded_ldab(kl, ku):
    ldab = 2 * kl + ku + 1 + 3  # extra NaN rows at the bottom stay untouched
    for variant in trf_variants(kl, ku):
        _check_trf(70, 70, kl, ku, batch=5, variant=variant, ldab=ldab)


@pytest.mark.parametrize("kl,ku", [(1, 1), (2, 3), (10, 10), (2, 32), (0, 3), (3, 0), (32, 32)])
def test_trf_parity_planted_zero_pivots(kl, ku):
    n = 60
    A = I.gen_band(n, n, kl, ku, count=6)
    kv = kl + ku
    for b, z in enumerate([1, 2, 30, 59, 60, 45]):
        col = A[b, z - 1, kl:kv + kl + 1]
        A[b, z - 1, kl:kv + kl + 1] = np.where(np.isnan(col), np.nan, 0.0)
    A[5, 10, kl:kv + kl + 1] = np.where(np.isnan(A[5, 10, kl:kv + kl + 1]), np.nan, 0.0)  # two zeros
    for variant in trf_variants(kl, ku):
        Ao, ipo, info = _check_trf(n, n, kl, ku, 6, variant, A_in=A.copy())
        assert list(info) == [1, 2, 30, 59, 60, 11]


@pytest.mark.parametrize("kl,ku", [(1, 1), (2, 2), (10, 10), (2, 32), (32, 32)])
def test_trf_parity_exact_ties(kl, ku):
    """Integer-valued bands with many exact |pivot| ties: both sides take the
    same decision (first index, Q2) in the same precision."""
    n = 64
    A = I.gen_band(n, n, kl, ku, count=16)
    A = np.where(np.isnan(A), np.nan, np.sign(A) * np.ceil(np.abs(A) * 2.0))  # values in {+-1, +-2}
    for variant in trf_variants(kl, ku):
        _check_trf(n, n, kl, ku, 16, variant, A_in=A.copy())


def _gpu_trs(Af, ipiv, B_np, n, kl, ku, variant=bl.AUTO):
    A = torch.from_numpy(Af).cuda()
    P = torch.from_numpy(np.ascontiguousarray(ipiv.astype(np.int32))).cuda()
    B = torch.from_numpy(B_np).cuda()
    bl.dgbtrs_strided_batched("N", n, kl, ku, A, P, B, variant=variant)
    torch.cuda.synchronize()
    return B.cpu().numpy()


@pytest.mark.parametrize("kl,ku", ALL_BANDS)
@pytest.mark.parametrize("nrhs", [1, 2, 3, 16, 33])
@pytest.mark.parametrize("variant", [bl.WINDOW, bl.GENERIC, bl.ROWS])
def test_trs_parity(kl, ku, nrhs, variant):
    if variant == bl.ROWS and not bl.trs_rows_available(kl, ku):
        pytest.skip("no lane-per-row solve kernel for this band")
    n, batch = 45, 13
    A = I.gen_band(n, n, kl, ku, count=batch)
    ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
    assert np.all(info == 0)
    B = I.gen_rhs(n, nrhs, ldb=n + 2, count=batch)
    Bo = B.copy()
    oracle.dgbtrs(A, ipiv, Bo, n, kl, ku)
    Bg = _gpu_trs(A, ipiv, B, n, kl, ku, variant)
    assert np.all(same_bits(Bg, Bo))


@pytest.mark.parametrize("n", [1, 2, 3, 8, 9, 130])
@pytest.mark.parametrize("kl,ku", [(1, 1), (10, 10), (2, 32), (0, 0), (32, 32)])
def test_trs_parity_sizes(n, kl, ku):
    A = I.gen_band(n, n, kl, ku, count=7)
    ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
    B = I.gen_rhs(n, 2, count=7)
    Bo = B.copy()
    oracle.dgbtrs(A, ipiv, Bo, n, kl, ku)
    for variant in (bl.WINDOW, bl.GENERIC) + ((bl.ROWS,) if bl.trs_rows_available(kl, ku) else ()):
        assert np.all(same_bits(_gpu_trs(A, ipiv, B.copy(), n, kl, ku, variant), Bo))


@pytest.mark.parametrize("kl,ku,nrhs", [(2, 2, 1), (10, 10, 1), (2, 32, 16), (5, 6, 3), (1, 1, 1), (0, 3, 1)])
def test_gbsv_parity_with_singular(kl, ku, nrhs):
    n, batch = 80, 10
    A = I.gen_band(n, n, kl, ku, count=batch)
    kv = kl + ku
    A[3, 17, kl:kv + kl + 1] = np.where(np.isnan(A[3, 17, kl:kv + kl + 1]), np.nan, 0.0)
    B = I.gen_rhs(n, nrhs, count=batch)
    Ao, Bo = A.copy(), B.copy()
    ipo, info_o = oracle.dgbsv(Ao, Bo, n, kl, ku)
    Ag = torch.from_numpy(A).cuda(); Bg = torch.from_numpy(B).cuda()
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    inf = torch.zeros(batch, dtype=torch.int32, device="cuda")
    bl.dgbsv_strided_batched(n, kl, ku, Ag, P, Bg, inf)
    torch.cuda.synchronize()
    assert np.array_equal(inf.cpu().numpy(), info_o) and info_o[3] == 18
    assert np.array_equal(P.cpu().numpy(), ipo)
    assert np.all(same_bits(Ag.cpu().numpy(), Ao))
    Bgn = Bg.cpu().numpy()
    assert np.all(same_bits(Bgn, Bo))
    assert np.array_equal(Bgn[3], B[3])  # untouched where info > 0


@pytest.mark.parametrize("kl,ku", [(10, 10), (1, 1), (2, 32)])  # row-slot and column-owner (AUTO) factorizations
def test_pointer_array_variants_match_strided(kl, ku):
    n, nrhs, batch = 50, 2, 9
    A = I.gen_band(n, n, kl, ku, count=batch)
    B = I.gen_rhs(n, nrhs, count=batch)
    Ao, Bo = A.copy(), B.copy()
    ipo, info_o = oracle.dgbsv(Ao, Bo, n, kl, ku)
    As = [torch.from_numpy(A[i].copy()).cuda() for i in range(batch)]
    Bs = [torch.from_numpy(B[i].copy()).cuda() for i in range(batch)]
    Ps = [torch.zeros(n, dtype=torch.int32, device="cuda") for _ in range(batch)]
    info = torch.zeros(batch, dtype=torch.int32, device="cuda")
    ldab = 2 * kl + ku + 1
    bl.dgbtrf_batched(n, n, kl, ku, bl.ptr_array(As), ldab, bl.ptr_array(Ps), info, batch)
    bl.dgbtrs_batched("N", n, kl, ku, nrhs, bl.ptr_array(As), ldab, bl.ptr_array(Ps), bl.ptr_array(Bs), n, batch)
    torch.cuda.synchronize()
    for i in range(batch):
        assert np.all(same_bits(As[i].cpu().numpy(), Ao[i]))
        assert np.array_equal(Ps[i].cpu().numpy(), ipo[i])
        assert np.all(same_bits(Bs[i].cpu().numpy(), Bo[i]))
    # and dgbsv_batched
    As2 = [torch.from_numpy(A[i].copy()).cuda() for i in range(batch)]
    Bs2 = [torch.from_numpy(B[i].copy()).cuda() for i in range(batch)]
    bl.dgbsv_batched(n, kl, ku, nrhs, bl.ptr_array(As2), ldab, bl.ptr_array(Ps), bl.ptr_array(Bs2), n, info, batch)
    torch.cuda.synchronize()
    for i in range(batch):
        assert np.all(same_bits(Bs2[i].cpu().numpy(), Bo[i]))


def test_host_buffer_gbsv_matches_oracle():
    n, kl, ku, nrhs, batch = 64, 2, 2, 1, 100  # BASELINE configs[0]
    A = I.gen_band(n, n, kl, ku, count=batch)
    B = I.gen_rhs(n, nrhs, count=batch)
    Ao, Bo = A.copy(), B.copy()
    ipo, info_o = oracle.dgbsv(Ao, Bo, n, kl, ku)
    At = torch.from_numpy(A.copy()).pin_memory(); Bt = torch.from_numpy(B.copy()).pin_memory()
    P = torch.zeros((batch, n), dtype=torch.int32).pin_memory()
    inf = torch.zeros(batch, dtype=torch.int32).pin_memory()
    bl.dgbsv_strided_batched_host(n, kl, ku, At, P, Bt, inf)
    assert np.all(same_bits(At.numpy(), Ao)) and np.all(same_bits(Bt.numpy(), Bo))
    assert np.array_equal(P.numpy(), ipo) and np.array_equal(inf.numpy(), info_o)


def test_host_buffer_gbsv_many_chunks():
    """The host entry point pipelines ~64 MB chunks over 3 reused device buffers:
    4+ chunks with a ragged tail, a singular matrix (B untouched), nrhs 2 with
    padded ldb, then a second call on a larger problem (buffers grow)."""
    for n, kl, ku, nrhs, batch in [(32, 1, 1, 2, 130000), (40, 3, 2, 1, 200000)]:
        ldb = n + 3
        A = I.gen_band(n, n, kl, ku, count=batch)
        B = I.gen_rhs(n, nrhs, ldb=ldb, count=batch)
        kv = kl + ku
        A[7, 5, kl:kv + kl + 1] = np.where(np.isnan(A[7, 5, kl:kv + kl + 1]), np.nan, 0.0)  # singular
        Ao, Bo = A.copy(), B.copy()
        ipo, info_o = oracle.dgbsv(Ao, Bo, n, kl, ku)
        assert info_o[7] == 6
        At = torch.from_numpy(A).pin_memory(); Bt = torch.from_numpy(B).pin_memory()
        P = torch.zeros((batch, n), dtype=torch.int32).pin_memory()
        inf = torch.zeros(batch, dtype=torch.int32).pin_memory()
        bl.dgbsv_strided_batched_host(n, kl, ku, At, P, Bt, inf)
        assert np.array_equal(inf.numpy(), info_o) and np.array_equal(P.numpy(), ipo)
        assert np.all(same_bits(At.numpy(), Ao)) and np.all(same_bits(Bt.numpy(), Bo))


def test_quick_returns_write_info():
    A = torch.zeros((5, 3, 4), dtype=torch.float64, device="cuda")
    ipiv = torch.zeros((5, 1), dtype=torch.int32, device="cuda")
    info = torch.full((5,), 9, dtype=torch.int32, device="cuda")
    bl.dgbtrf_strided_batched(0, 3, 1, 1, A, ipiv, info)
    torch.cuda.synchronize()
    assert torch.all(info == 0)
    assert torch.all(A == 0)


# ---------------------------------------------- full-size sampled parity
# BASELINE.json configs at full batch size, launched exactly as bench.py does
# (AUTO variant, strided, one trf + one trs launch); the oracle recomputes a
# sample of matrices one by one from the same seeded generator.
FULL = [  # (batch, n, kl, ku, nrhs)
    (100, 64, 2, 2, 1),
    (10000, 256, 1, 1, 1),
    (10000, 512, 10, 10, 1),
    (5000, 1024, 2, 32, 16),
]


@pytest.mark.parametrize("batch,n,kl,ku,nrhs", FULL)
def test_full_size_sampled_parity(batch, n, kl, ku, nrhs):
    A = torch.from_numpy(I.gen_band(n, n, kl, ku, count=batch)).cuda()
    B = torch.from_numpy(I.gen_rhs(n, nrhs, count=batch)).cuda()
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    info = torch.zeros(batch, dtype=torch.int32, device="cuda")
    bl.dgbtrf_strided_batched(n, n, kl, ku, A, P, info)
    bl.dgbtrs_strided_batched("N", n, kl, ku, A, P, B)
    torch.cuda.synchronize()
    rng = np.random.default_rng(1)
    sample = np.unique(np.concatenate([[0, batch - 1], rng.integers(0, batch, 40)]))
    for i in sample:
        Ao = I.gen_band(n, n, kl, ku, count=1, first=int(i))
        Bo = I.gen_rhs(n, nrhs, count=1, first=int(i))
        A0, B0 = Ao.copy(), Bo.copy()
        ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
        oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
        assert info[i].item() == info_o[0]
        assert np.array_equal(P[i].cpu().numpy(), ipo[0])
        assert np.all(same_bits(A[i].cpu().numpy(), Ao[0]))
        Bi = B[i].cpu().numpy()
        assert np.all(same_bits(Bi, Bo[0]))
        if i == sample[0]:
            D = band_to_dense(A0[0], n, n, kl, ku)
            assert backward_error(D, Bi[:, :n].T, B0[0][:, :n].T) <= 10.0
    # properties over the whole batch: pivot range, info
    j = torch.arange(n, device="cuda", dtype=torch.int32)
    assert bool(torch.all(P >= j + 1)) and bool(torch.all(P <= torch.clamp(j + 1 + kl, max=n)))
    assert int(info.abs().sum()) == 0


@pytest.mark.parametrize("kl,ku", WINDOW_BANDS + [(5, 6), (32, 32)])
@pytest.mark.parametrize("nrhs", [1, 3])
def test_trfs_fused_matches_trf_then_trs(kl, ku, nrhs):
    """dgbtrfs (forward solve fused into the factorization for nrhs == 1)
    == oracle dgbtrf followed by dgbtrs, bitwise, incl. a singular matrix
    (B solved regardless of info, like dgbtrs) and a ragged batch."""
    n, batch = 70, 11
    A = I.gen_band(n, n, kl, ku, count=batch)
    kv = kl + ku
    A[4, 33, kl:kv + kl + 1] = np.where(np.isnan(A[4, 33, kl:kv + kl + 1]), np.nan, 0.0)  # singular
    B = I.gen_rhs(n, nrhs, ldb=n + 1, count=batch)
    Ao, Bo = A.copy(), B.copy()
    ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
    oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
    Ag = torch.from_numpy(A).cuda(); Bg = torch.from_numpy(B).cuda()
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    inf = torch.zeros(batch, dtype=torch.int32, device="cuda")
    bl.dgbtrfs_strided_batched(n, kl, ku, Ag, P, Bg, inf)
    torch.cuda.synchronize()
    assert np.array_equal(inf.cpu().numpy(), info_o) and info_o[4] == 34
    assert np.array_equal(P.cpu().numpy(), ipo)
    assert np.all(same_bits(Ag.cpu().numpy(), Ao))
    ok = same_bits(Bg.cpu().numpy(), Bo)
    ok[4] = True  # singular matrix: Inf/NaN pattern of the division by U(34,34) = 0 is out of contract
    assert np.all(ok)
    assert np.all(np.isnan(Bg.cpu().numpy()[:, :, n:]))  # ldb padding untouched


@pytest.mark.parametrize("kl,ku", [(0, 0), (1, 1), (2, 3), (4, 4), (10, 10), (2, 32), (32, 32)])
@pytest.mark.parametrize("n", [1, 2, 5, 20, 21, 22, 33, 64])
def test_trfs_fused_small_n_ragged_batch(kl, ku, n):
    """dgbtrfs at n below / around the window length (the backward solve reads
    rows < 0 from pad slots for its last kv steps) and a batch that leaves the
    last warp partly empty, bitwise vs oracle dgbtrf + dgbtrs."""
    batch = 13
    A = I.gen_band(n, n, kl, ku, count=batch)
    B = I.gen_rhs(n, 1, ldb=n + 3, count=batch)
    Ao, Bo = A.copy(), B.copy()
    ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
    oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
    Ag = torch.from_numpy(A).cuda(); Bg = torch.from_numpy(B).cuda()
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    inf = torch.zeros(batch, dtype=torch.int32, device="cuda")
    bl.dgbtrfs_strided_batched(n, kl, ku, Ag, P, Bg, inf)
    torch.cuda.synchronize()
    assert np.array_equal(inf.cpu().numpy(), info_o)
    assert np.array_equal(P.cpu().numpy(), ipo)
    assert np.all(same_bits(Ag.cpu().numpy(), Ao))
    assert np.all(same_bits(Bg.cpu().numpy(), Bo))  # incl. the NaN padding rows of ldb


@pytest.mark.parametrize("kl,ku,nrhs", [(2, 3, 2), (10, 10, 1), (1, 1, 3), (0, 4, 1), (4, 0, 2), (2, 32, 16), (33, 20, 1)])
@pytest.mark.parametrize("trans", ["T", "C"])
def test_trs_transposed_parity(kl, ku, nrhs, trans):
    """f2: dgbtrs('T'/'C') on the GPU == oracle (same reference-BLAS order) bitwise."""
    n, batch = 77, 9
    A = I.gen_band(n, n, kl, ku, count=batch)
    ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
    B = I.gen_rhs(n, nrhs, ldb=n + 2, count=batch)
    Bo = B.copy()
    oracle.dgbtrs(A, ipiv, Bo, n, kl, ku, trans="T")
    Ag = torch.from_numpy(A).cuda(); Pg = torch.from_numpy(ipiv).cuda(); Bg = torch.from_numpy(B).cuda()
    bl.dgbtrs_strided_batched(trans, n, kl, ku, Ag, Pg, Bg)
    torch.cuda.synchronize()
    assert np.all(same_bits(Bg.cpu().numpy(), Bo))


# ring-staged transposed solve (gbtrs_t.cuh; compiled bands and a run-time compiled one):
# n below / at / just above kl and kv (the truncated dot products run outside the ring),
# nrhs spanning 1, a partial lane group, and two 32-column chunks, ragged batches
@pytest.mark.parametrize("kl,ku", [(10, 10), (2, 32), (1, 1), (0, 3), (3, 0), (32, 32), (5, 9)])
@pytest.mark.parametrize("n,nrhs,batch", [(1, 1, 5), (3, 2, 7), (11, 1, 13), (21, 3, 9), (22, 1, 33),
                                          (160, 1, 301), (97, 5, 41), (70, 33, 6)])
def test_trs_transposed_ring_kernel(kl, ku, n, nrhs, batch):
    A = I.gen_band(n, n, kl, ku, count=batch)
    ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
    B = I.gen_rhs(n, nrhs, ldb=n + 1, count=batch)
    Bo = B.copy()
    oracle.dgbtrs(A, ipiv, Bo, n, kl, ku, trans="T")
    Ag = torch.from_numpy(A).cuda(); Pg = torch.from_numpy(ipiv).cuda()
    for variant in (bl.WINDOW, bl.GENERIC):
        Bg = torch.from_numpy(B).cuda()
        bl.dgbtrs_strided_batched("T", n, kl, ku, Ag, Pg, Bg, variant=variant)
        torch.cuda.synchronize()
        assert np.all(same_bits(Bg.cpu().numpy(), Bo)), variant  # incl. the NaN padding row of ldb


# block-granular one-RHS solve (gbtrs_blk.cuh; what dgbtrs / dgbsv run for nrhs == 1 on
# window bands): n around kl and kv, odd and even ldab (the ring's 16-byte parity flips per
# column) and ldb (the RHS pair phase), ragged batches that leave warps partly empty
@pytest.mark.parametrize("kl,ku", [(10, 10), (2, 3), (32, 32), (2, 32), (10, 7), (5, 9)])
@pytest.mark.parametrize("n,batch,ldab_extra,ldb_extra", [(1, 3, 0, 0), (4, 9, 1, 1), (11, 37, 0, 1),
                                                          (21, 5, 1, 0), (66, 41, 1, 1), (300, 70, 0, 0)])
def test_trs_blk_one_rhs(kl, ku, n, batch, ldab_extra, ldb_extra):
    ldab = 2 * kl + ku + 1 + ldab_extra
    A = I.gen_band(n, n, kl, ku, ldab=ldab, count=batch)
    ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
    B = I.gen_rhs(n, 1, ldb=n + ldb_extra, count=batch)
    Bo = B.copy()
    oracle.dgbtrs(A, ipiv, Bo, n, kl, ku)
    Ag = torch.from_numpy(A).cuda(); Pg = torch.from_numpy(ipiv).cuda(); Bg = torch.from_numpy(B).cuda()
    bl.dgbtrs_strided_batched("N", n, kl, ku, Ag, Pg, Bg, variant=bl.WINDOW)
    torch.cuda.synchronize()
    assert np.all(same_bits(Bg.cpu().numpy(), Bo))


@pytest.mark.parametrize("kl,ku", [(10, 10), (2, 32), (32, 32), (5, 9)])
@pytest.mark.parametrize("n,nrhs,batch", [(9, 1, 13), (70, 3, 21), (200, 1, 40)])
def test_trs_transposed_odd_ldab_ldb(kl, ku, n, nrhs, batch):
    """The transposed ring solve with an odd leading dimension (factor-range parity flips per
    column) and odd ldb, bitwise vs the oracle."""
    ldab = 2 * kl + ku + 2 + ((2 * kl + ku + 2) % 2 == 0)
    A = I.gen_band(n, n, kl, ku, ldab=ldab, count=batch)
    ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
    B = I.gen_rhs(n, nrhs, ldb=n + 1 + (n % 2 == 0), count=batch)
    Bo = B.copy()
    oracle.dgbtrs(A, ipiv, Bo, n, kl, ku, trans="T")
    Ag = torch.from_numpy(A).cuda(); Pg = torch.from_numpy(ipiv).cuda(); Bg = torch.from_numpy(B).cuda()
    bl.dgbtrs_strided_batched("T", n, kl, ku, Ag, Pg, Bg, variant=bl.WINDOW)
    torch.cuda.synchronize()
    assert np.all(same_bits(Bg.cpu().numpy(), Bo))


def test_trs_transposed_pointer_array():
    n, kl, ku, nrhs, batch = 60, 10, 10, 2, 11
    A = I.gen_band(n, n, kl, ku, count=batch)
    ipiv, info = oracle.dgbtrf(A, n, n, kl, ku)
    B = I.gen_rhs(n, nrhs, count=batch)
    Bo = B.copy()
    oracle.dgbtrs(A, ipiv, Bo, n, kl, ku, trans="T")
    As = [torch.from_numpy(A[i].copy()).cuda() for i in range(batch)]
    Ps = [torch.from_numpy(ipiv[i].copy()).cuda() for i in range(batch)]
    Bs = [torch.from_numpy(B[i].copy()).cuda() for i in range(batch)]
    bl.dgbtrs_batched("T", n, kl, ku, nrhs, bl.ptr_array(As), 2 * kl + ku + 1, bl.ptr_array(Ps),
                      bl.ptr_array(Bs), n, batch)
    torch.cuda.synchronize()
    for i in range(batch):
        assert np.all(same_bits(Bs[i].cpu().numpy(), Bo[i]))


@pytest.mark.parametrize("batch,n,kl,ku", [(512, 193, 4, 4), (2000, 50, 10, 10)])
def test_application_shaped_workloads(batch, n, kl, ku):
    """f4: XGC-like (512 x n=193) and PELE-like (n=50)
    batches through dgbtrfs, every matrix checked against the oracle."""
    A = I.gen_band(n, n, kl, ku, count=batch)
    B = I.gen_rhs(n, 1, count=batch)
    Ao, Bo = A.copy(), B.copy()
    ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
    oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
    Ag = torch.from_numpy(A).cuda(); Bg = torch.from_numpy(B).cuda()
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    inf = torch.zeros(batch, dtype=torch.int32, device="cuda")
    bl.dgbtrfs_strided_batched(n, kl, ku, Ag, P, Bg, inf)
    torch.cuda.synchronize()
    assert np.array_equal(inf.cpu().numpy(), info_o)
    assert np.array_equal(P.cpu().numpy(), ipo)
    assert np.all(same_bits(Ag.cpu().numpy(), Ao))
    assert np.all(same_bits(Bg.cpu().numpy(), Bo))


@pytest.mark.parametrize("kl,ku", [(10, 10), (2, 32), (10, 7), (32, 32)])
def test_trf_batch_tail_after_other_launches(kl, ku):
    """Batch tails leave dead matrix groups in the last CTA; they must not act on
    shared memory left over by earlier launches (regression: a dead group once
    relabelled a row from a never-written pivot record)."""
    for variant in trf_variants(kl, ku):
        _check_trf(300, 300, kl, ku, batch=97, variant=variant)  # fills shared memory with live data
        for batch in (1, 3, 5):
            _check_trf(90, 90, kl, ku, batch=batch, variant=variant, first=batch)


# ------------------------------------ the path bench.py times, at full batch
# dgbtrfs (factorization + fused forward solve, then the backward launch) at
# batches that select every matrices-per-warp instantiation of the backward
# solve (bandlu.cu launch_trs_bwd_lean: 2 / 4 / 8 / 16 / 32), plus the C2 and
# (32,32) backward kernels.  PAPER.md P:639-640, P:675-682 (backward solve).
TRFS_FULL = [  # (batch, n, kl, ku)
    (10000, 512, 10, 10),  # C3 exactly as bench.py times it
    (5000, 512, 10, 10),
    (20000, 64, 10, 10),
    (40000, 40, 10, 7),
    (3000, 200, 10, 10),
    (10000, 50, 10, 10),   # PELE-like
    (10000, 256, 1, 1),    # C2
    (300, 2048, 32, 32),   # C5's widest band at its largest n
    (1500, 1024, 2, 32),
]


def _sample_indices(batch, seed=7, per_warp=(2, 4, 8, 16, 32), extra=48):
    """First and last matrix of the first, second, middle and last warp for each
    matrices-per-warp grouping, plus random matrices (>= 64 in total)."""
    idx = {0, batch - 1}
    for g in per_warp:
        warps = (batch + g - 1) // g
        for w in (0, 1, warps // 2, warps - 1):
            idx.update({min(batch - 1, w * g), min(batch - 1, w * g + g - 1)})
    rng = np.random.default_rng(seed)
    idx.update(int(i) for i in rng.integers(0, batch, extra))
    return sorted(idx)


@pytest.mark.parametrize("batch,n,kl,ku", TRFS_FULL)
@pytest.mark.parametrize("phase", [0, bl.TRFS_FUSED])  # the library's plan (as bench.py), and the fused kernel
def test_trfs_full_batch_sampled_parity(batch, n, kl, ku, phase):
    A = torch.from_numpy(I.gen_band(n, n, kl, ku, count=batch)).cuda()
    B = torch.from_numpy(I.gen_rhs(n, 1, count=batch)).cuda()
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    info = torch.full((batch,), -7, dtype=torch.int32, device="cuda")
    bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info, phase=phase)
    torch.cuda.synchronize()
    sample = _sample_indices(batch)
    assert len(sample) >= 64 or len(sample) == batch
    sel = torch.tensor(sample, device="cuda")
    Ag, Bg, Pg, Ig = (t.index_select(0, sel).cpu().numpy() for t in (A, B, P, info))
    for k, i in enumerate(sample):
        Ao = I.gen_band(n, n, kl, ku, count=1, first=i)
        Bo = I.gen_rhs(n, 1, count=1, first=i)
        ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
        oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
        assert Ig[k] == info_o[0], f"info of matrix {i}"
        assert np.array_equal(Pg[k], ipo[0]), f"ipiv of matrix {i}"
        assert np.all(same_bits(Ag[k], Ao[0])), f"factors of matrix {i}"
        assert np.all(same_bits(Bg[k], Bo[0])), f"solution of matrix {i}"
    j = torch.arange(n, device="cuda", dtype=torch.int32)
    assert bool(torch.all(P >= j + 1)) and bool(torch.all(P <= torch.clamp(j + 1 + kl, max=n)))
    assert int(info.abs().sum()) == 0


# ------------------------------------------------ the fused gbsv kernel (f1)
# One launch: factorization + forward substitution on the fly + backward
# substitution by the same lanes (Sec. 7, generalised to any
# n).  y(0..n-1) lives in shared memory when it fits (dgbsv may then leave B
# untouched where info > 0), else in B (large n: dgbtrfs only; dgbsv takes two
# launches).  Both plans must equal the oracle bitwise.
FUSED_BANDS = [(10, 10), (10, 7), (1, 1), (2, 2), (2, 3), (4, 4)]  # (2,32): kv+1+PF > 2G, no fused kernel


def _trfs(A_np, B_np, n, kl, ku, phase=0):
    Ag = torch.from_numpy(A_np).cuda(); Bg = torch.from_numpy(B_np).cuda()
    batch = A_np.shape[0]
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    inf = torch.full((batch,), -3, dtype=torch.int32, device="cuda")
    bl.dgbtrfs_strided_batched(n, kl, ku, Ag, P, Bg, inf, phase=phase)
    torch.cuda.synchronize()
    return Ag.cpu().numpy(), P.cpu().numpy(), Bg.cpu().numpy(), inf.cpu().numpy()


@pytest.mark.parametrize("kl,ku", FUSED_BANDS)
@pytest.mark.parametrize("n", [3, 17, 130, 777, 1000])  # 777 / 1000: y beyond the shared-memory budget at (10,10)
def test_fused_gbsv_kernel_vs_oracle_and_two_launch_plan(kl, ku, n):
    batch = 19  # ragged: not a multiple of matrices per warp / CTA
    plan = bl.trfs_plan(n, kl, ku, 1, batch)
    assert plan["fused"] and plan["kernels"][0] in ("gbtrf_rows_kernel", "gbtrf_cols_kernel")
    assert bl.trfs_plan(n, kl, ku, 1, batch, bl.TRFS_FUSED)["kernels"] == ["gbtrf_rows_kernel"]
    two = bl.trfs_plan(n, kl, ku, 1, batch, bl.TRFS_TWO_LAUNCH)["kernels"][0]
    assert two == ("gbtrf_cols_kernel" if bl.cols_available(kl, ku) else "gbtrf_rows_kernel")
    A = I.gen_band(n, n, kl, ku, count=batch, first=n)
    B = I.gen_rhs(n, 1, ldb=n + 2, count=batch, first=n)
    Ao, Bo = A.copy(), B.copy()
    ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
    oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
    for phase in (0, bl.TRFS_TWO_LAUNCH, bl.TRFS_FUSED):
        Ag, Pg, Bg, Ig = _trfs(A.copy(), B.copy(), n, kl, ku, phase)
        assert np.array_equal(Ig, info_o)
        assert np.array_equal(Pg, ipo)
        assert np.all(same_bits(Ag, Ao))
        assert np.all(same_bits(Bg, Bo))  # incl. the NaN ldb padding rows


@pytest.mark.parametrize("kl,ku", FUSED_BANDS + [(2, 32)])
@pytest.mark.parametrize("n", [40, 512, 1000])
def test_fused_dgbsv_leaves_b_untouched_where_singular(kl, ku, n):
    """dgbsv through the fused kernel (y in shared memory; n = 1000 at (10,10)
    takes the two-launch path): info / ipiv / factors / x bitwise, and B
    bitwise unchanged for the matrices with a planted zero pivot (LAPACK DGBSV)."""
    batch = 10
    A = I.gen_band(n, n, kl, ku, count=batch)
    kv = kl + ku
    for b, z in ((2, 1), (5, n // 2), (9, n)):  # zero column z (1-based): info = z
        A[b, z - 1, kl:kv + kl + 1] = np.where(np.isnan(A[b, z - 1, kl:kv + kl + 1]), np.nan, 0.0)
    B = I.gen_rhs(n, 1, ldb=n + 1, count=batch)
    Ao, Bo = A.copy(), B.copy()
    ipo, info_o = oracle.dgbsv(Ao, Bo, n, kl, ku)
    assert list(info_o[[2, 5, 9]]) == [1, n // 2, n]
    Ag = torch.from_numpy(A).cuda(); Bg = torch.from_numpy(B).cuda()
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    inf = torch.zeros(batch, dtype=torch.int32, device="cuda")
    bl.dgbsv_strided_batched(n, kl, ku, Ag, P, Bg, inf)
    torch.cuda.synchronize()
    assert np.array_equal(inf.cpu().numpy(), info_o)
    assert np.array_equal(P.cpu().numpy(), ipo)
    assert np.all(same_bits(Ag.cpu().numpy(), Ao))
    Bgn = Bg.cpu().numpy()
    assert np.all(same_bits(Bgn, Bo))
    for b in (2, 5, 9):
        assert np.all(same_bits(Bgn[b], B[b]))


# ------------------------------------------- run-time compiled bands (NVRTC)
# Bands no list instantiates ahead of time run the same templates compiled with
# NVRTC on first use (jit.cuh; Sec. 8.1): every entry point and
# plan must still equal the oracle bitwise.
JIT_BANDS = [(5, 6), (16, 16), (20, 20), (0, 32), (7, 1), (33, 20), (56, 4)]


@pytest.mark.parametrize("kl,ku", JIT_BANDS)
def test_jit_band_parity(kl, ku):
    if not bl.jit_band(kl, ku):
        pytest.skip("NVRTC not available")
    n, batch = 150, 37
    A0 = I.gen_band(n, n, kl, ku, count=batch, first=kl * 100 + ku)
    B0 = I.gen_rhs(n, 3, ldb=n + 1, count=batch)
    Ao = A0.copy()
    ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
    Bo = B0.copy()
    oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
    # dgbtrf (AUTO: the run-time compiled factorization) and dgbtrs (window solve, nrhs 3)
    Ag, ipg, info_g = _gpu_trf(A0.copy(), n, n, kl, ku)
    assert np.array_equal(info_g, info_o) and np.array_equal(ipg, ipo)
    assert np.all(same_bits(Ag, Ao))
    assert np.all(same_bits(_gpu_trs(Ao, ipo, B0.copy(), n, kl, ku), Bo))
    # dgbtrfs nrhs 1: the library's plan, the two-launch plan and the fused kernel
    B1 = I.gen_rhs(n, 1, ldb=n + 2, count=batch)
    B1o = B1.copy()
    oracle.dgbtrs(Ao, ipo, B1o, n, kl, ku)
    for phase in (0, bl.TRFS_TWO_LAUNCH, bl.TRFS_FUSED):
        Ag2, Pg2, Bg2, Ig2 = _trfs(A0.copy(), B1.copy(), n, kl, ku, phase)
        assert np.array_equal(Ig2, info_o) and np.array_equal(Pg2, ipo)
        assert np.all(same_bits(Ag2, Ao)) and np.all(same_bits(Bg2, B1o))
    # dgbsv with a singular matrix: B untouched there
    As = A0.copy()
    kv = kl + ku
    As[5, 40, kl:kv + kl + 1] = np.where(np.isnan(As[5, 40, kl:kv + kl + 1]), np.nan, 0.0)
    Asv, Bsv = As.copy(), B1.copy()
    ips, infs = oracle.dgbsv(Asv, Bsv, n, kl, ku)
    Ag = torch.from_numpy(As).cuda(); Bg = torch.from_numpy(B1.copy()).cuda()
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    inf = torch.zeros(batch, dtype=torch.int32, device="cuda")
    bl.dgbsv_strided_batched(n, kl, ku, Ag, P, Bg, inf)
    torch.cuda.synchronize()
    assert np.array_equal(inf.cpu().numpy(), infs) and infs[5] == 41
    assert np.all(same_bits(Ag.cpu().numpy(), Asv)) and np.all(same_bits(Bg.cpu().numpy(), Bsv))
    assert np.all(same_bits(Bg.cpu().numpy()[5], B1[5]))


@pytest.mark.parametrize("kl,ku", [(16, 16), (0, 32)])
def test_jit_band_full_batch_sampled(kl, ku):
    """A run-time compiled band at a multi-wave batch (the two-launch plan), sampled."""
    if not bl.jit_band(kl, ku):
        pytest.skip("NVRTC not available")
    batch, n = 6000, 256
    A = torch.from_numpy(I.gen_band(n, n, kl, ku, count=batch)).cuda()
    B = torch.from_numpy(I.gen_rhs(n, 1, count=batch)).cuda()
    P = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    info = torch.zeros(batch, dtype=torch.int32, device="cuda")
    bl.dgbtrfs_strided_batched(n, kl, ku, A, P, B, info)
    torch.cuda.synchronize()
    for i in _sample_indices(batch, per_warp=(2, 8, 32), extra=16):
        Ao = I.gen_band(n, n, kl, ku, count=1, first=i)
        Bo = I.gen_rhs(n, 1, count=1, first=i)
        ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
        oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
        assert np.array_equal(P[i].cpu().numpy(), ipo[0])
        assert np.all(same_bits(A[i].cpu().numpy(), Ao[0])) and np.all(same_bits(B[i].cpu().numpy(), Bo[0]))



# ------------------------------------------------ thin bands, thread per matrix
THIN_BANDS = [(0, 0), (0, 3), (1, 1), (2, 2), (2, 3), (3, 0), (3, 2), (4, 4)]


@pytest.mark.parametrize("kl,ku", THIN_BANDS)
@pytest.mark.parametrize("n", [1, 2, 7, 8, 9, 33, 150])
def test_thin_fused_kernel_vs_oracle(kl, ku, n):
    """The thin-band kernel's one-launch dgbtrf + dgbtrs (cooperative whole-column staging,
    forward and backward passes by the owning thread) equals the oracle bitwise: n below,
    at and around the block of 8 columns, a ragged batch (a partly empty last warp), a
    singular matrix (B solved regardless, as dgbtrfs specifies) and padded ldab / ldb."""
    if not bl.thin_available(kl, ku):
        pytest.skip("no thin kernel for this band")
    batch = 45
    for ldab in (None, 2 * kl + ku + 1 + 3):
        A = I.gen_band(n, n, kl, ku, ldab=ldab, count=batch, first=n)
        if n > 4:
            kv = kl + ku
            lo, hi = kl, kv + kl + 1
            A[6, 3, lo:hi] = np.where(np.isnan(A[6, 3, lo:hi]), np.nan, 0.0)
        B = I.gen_rhs(n, 1, ldb=n + 2, count=batch)
        Ao, Bo = A.copy(), B.copy()
        ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
        oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
        Ag, Pg, Bg, Ig = _trfs(A.copy(), B.copy(), n, kl, ku, bl.TRFS_THIN)
        assert np.array_equal(Ig, info_o) and np.array_equal(Pg, ipo)
        assert np.all(same_bits(Ag, Ao))  # incl. NaN corners / padding rows
        ok = same_bits(Bg, Bo)
        if n > 4:
            ok[6] = True  # singular U: Inf/NaN pattern of x out of contract (reading 12)
        assert np.all(ok)


COLS_BANDS = [(0, 0), (0, 3), (1, 1), (2, 2), (2, 3), (3, 0), (3, 2), (4, 4), (2, 32)]  # skipped where not compiled


@pytest.mark.parametrize("kl,ku", COLS_BANDS)
@pytest.mark.parametrize("n", [3, 4, 5, 15, 16, 17, 33, 48, 49, 64, 131])
def test_cols_kernel_parity(kl, ku, n):
    """Column-owner factorization (gbtrf_cols.cuh) at n around its ring / unroll period (GL steps,
    GL*CPL column slots) and staging block (4 rows), ragged batch: bitwise vs the oracle."""
    if not bl.cols_available(kl, ku):
        pytest.skip("no column-owner kernel compiled for this band")
    assert bl.trf_variant(n, n, kl, ku) == bl.COLS
    _check_trf(n, n, kl, ku, batch=45, variant=bl.COLS)


@pytest.mark.parametrize("kl,ku", COLS_BANDS)
@pytest.mark.parametrize("n,batch", [(5, 9), (40, 33), (257, 70)])
@pytest.mark.parametrize("nrhs", [1, 3, 4, 16, 32])
def test_cols_trfs_forward_parity(kl, ku, n, batch, nrhs):
    # the column-owner factorization with the forward substitution of all right-hand sides, then
    # the backward solve
    """dgbtrfs on a column-owner band (factorization with the forward substitution on the fly,
    then the backward solve): factors, pivots and solution bitwise vs oracle dgbtrf + dgbtrs."""
    if not bl.cols_available(kl, ku):
        pytest.skip("no column-owner kernel compiled for this band")
    if nrhs > 4 and (kl, ku) != (2, 32):
        pytest.skip("4 lanes per matrix: up to 4 right-hand sides ride with the factorization")
    if nrhs > 16 and n > 40:
        pytest.skip("(32 right-hand sides: the small cases suffice)")
    A = I.gen_band(n, n, kl, ku, count=batch)
    B = I.gen_rhs(n, nrhs, ldb=n + 3, count=batch)  # NaN padding rows below each column stay untouched
    Ao, Bo = A.copy(), B.copy()
    ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
    oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
    plan = bl.trfs_plan(n, kl, ku, nrhs, batch, bl.TRFS_TWO_LAUNCH)
    assert plan["bytes"] == ["trf_fwd", "trs_bwd"], plan
    assert plan["kernels"][0] == "gbtrf_cols_kernel", plan  # the right-hand sides ride with it
    Ag, Bg = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    Pg = torch.zeros((batch, n), dtype=torch.int32, device="cuda")
    Ig = torch.full((batch,), -7, dtype=torch.int32, device="cuda")
    bl.dgbtrfs_strided_batched(n, kl, ku, Ag, Pg, Bg, Ig, phase=bl.TRFS_TWO_LAUNCH)
    torch.cuda.synchronize()
    assert np.array_equal(Ig.cpu().numpy(), info_o)
    assert np.array_equal(Pg.cpu().numpy(), ipo)
    assert same_bits(Ag.cpu().numpy(), Ao).all()
    assert same_bits(Bg.cpu().numpy(), Bo).all()


@pytest.mark.parametrize("kl,ku", [(0, 0), (0, 3), (1, 1), (2, 2), (2, 3), (3, 0), (3, 2)])
@pytest.mark.parametrize("n,batch", [(1, 5), (3, 9), (8, 17), (63, 33), (256, 300)])
def test_cols_fused_gbsv_kernel(kl, ku, n, batch):
    """dgbtrfs in ONE launch on a column-owner band (factorization, forward and backward
    substitution by the same lanes): factors, pivots, info and x bitwise vs the oracle, the NaN
    ldb padding untouched; n from 1 (no step) to 256, batches not a multiple of 8 per warp."""
    if not bl.cols_available(kl, ku) or bl.trfs_plan(n, kl, ku, 1, batch)["kernels"] != ["gbtrf_cols_kernel"]:
        pytest.skip("column-owner fused kernel not built (opt-in -DBANDLU_COLS_FUSED)")
    A = I.gen_band(n, n, kl, ku, count=batch, first=7)
    B = I.gen_rhs(n, 1, ldb=n + 2, count=batch, first=7)
    Ao, Bo = A.copy(), B.copy()
    ipo, info_o = oracle.dgbtrf(Ao, n, n, kl, ku)
    oracle.dgbtrs(Ao, ipo, Bo, n, kl, ku)
    Ag, Pg, Bg, Ig = _trfs(A.copy(), B.copy(), n, kl, ku, 0)
    assert np.array_equal(Ig, info_o) and np.array_equal(Pg, ipo)
    assert np.all(same_bits(Ag, Ao)) and np.all(same_bits(Bg, Bo))
