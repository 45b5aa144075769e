"""C-ABI boundary tests that need no GPU: the shared library loads, exports
every symbol include/bandlu.h declares, and rejects illegal arguments with
LAPACK-numbered codes before touching the device (no compute calls here)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "bandlu.h")


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sc_abdelfattahtlad23_b200 import _build, binding
    _build.build()  # nvcc cross-compiles sm_100a without a GPU
    return binding.load()


def declared_functions():
    txt = open(HDR).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"^\s*int\s+(\w+)\s*\(", txt, flags=re.M)))


def test_header_declares_the_boundary():
    names = declared_functions()
    for n in ("dgbtrf_batched", "dgbtrf_strided_batched", "dgbtrs_batched", "dgbtrs_strided_batched",
              "dgbsv_batched", "dgbsv_strided_batched", "dgbsv_strided_batched_host"):
        assert n in names


def test_library_exports_every_declared_symbol(lib):
    from paper_conf_sc_abdelfattahtlad23_b200 import binding
    for name in declared_functions():
        assert hasattr(lib, name), name
    assert set(declared_functions()) <= set(binding.EXPORTS)
    assert lib.bandlu_version() >= 1


NULL = ctypes.c_void_p(0)
FAKE = ctypes.c_void_p(0x1000)  # never dereferenced: every case below fails argument checking


def test_trf_argument_errors(lib):
    f = lib.dgbtrf_strided_batched
    # (m, n, kl, ku, dA, ldab, strideA, dipiv, strideP, dinfo, batch, stream)
    assert f(-1, 4, 1, 1, FAKE, 4, 16, FAKE, 4, FAKE, 1, NULL) == -1
    assert f(4, -1, 1, 1, FAKE, 4, 16, FAKE, 4, FAKE, 1, NULL) == -2
    assert f(4, 4, -1, 1, FAKE, 4, 16, FAKE, 4, FAKE, 1, NULL) == -3
    assert f(4, 4, 1, -1, FAKE, 4, 16, FAKE, 4, FAKE, 1, NULL) == -4
    assert f(4, 4, 1, 1, FAKE, 3, 16, FAKE, 4, FAKE, 1, NULL) == -6  # ldab < 2kl+ku+1
    assert f(4, 4, 1, 1, NULL, 4, 16, FAKE, 4, FAKE, 1, NULL) == -5
    assert f(4, 4, 1, 1, FAKE, 4, 15, FAKE, 4, FAKE, 1, NULL) == -7
    assert f(4, 4, 1, 1, FAKE, 4, 16, NULL, 4, FAKE, 1, NULL) == -8
    assert f(4, 4, 1, 1, FAKE, 4, 16, FAKE, 3, FAKE, 1, NULL) == -9
    assert f(4, 4, 1, 1, FAKE, 4, 16, FAKE, 4, NULL, 1, NULL) == -10
    assert f(4, 4, 1, 1, FAKE, 4, 16, FAKE, 4, FAKE, -1, NULL) == -11
    assert f(4, 4, 1, 1, NULL, 4, 16, NULL, 4, NULL, 0, NULL) == 0  # batch 0: quick return, no launch
    g = lib.dgbtrf_batched  # LAPACK numbering
    assert g(4, 4, 1, 1, FAKE, 3, FAKE, FAKE, 1, NULL) == -6
    assert g(4, 4, 1, 1, FAKE, 4, FAKE, NULL, 1, NULL) == -8
    assert g(4, 4, 1, 1, FAKE, 4, FAKE, FAKE, -2, NULL) == -9


def test_trs_argument_errors(lib):
    f = lib.dgbtrs_strided_batched
    # (trans, n, kl, ku, nrhs, dA, ldab, strideA, dipiv, strideP, dB, ldb, strideB, batch, stream)
    ok = dict(n=4, kl=1, ku=1, nrhs=1, ldab=4, sA=16, sP=4, ldb=4, sB=4)

    def call(trans=b"N", **kw):
        a = dict(ok, **kw)
        return f(trans, a["n"], a["kl"], a["ku"], a["nrhs"], FAKE, a["ldab"], a["sA"], FAKE, a["sP"], FAKE,
                 a["ldb"], a["sB"], kw.get("batch", 1), NULL)
    assert call(trans=b"X") == -1
    assert call(n=-1) == -2
    assert call(kl=-1) == -3
    assert call(ku=-1) == -4
    assert call(nrhs=-1) == -5
    assert call(ldab=3) == -7
    assert call(sA=15) == -8
    assert call(sP=3) == -10
    assert call(ldb=3) == -12
    assert call(sB=3) == -13
    assert call(batch=-1) == -14
    assert call(trans=b"T", batch=0) == 0  # transposed solve supported; batch 0 = quick return
    assert call(trans=b"c", n=-1) == -2
    g = lib.dgbtrs_batched  # (trans,n,kl,ku,nrhs,A,ldab,P,B,ldb,batch,stream): LAPACK numbering
    assert g(b"N", 4, 1, 1, 1, FAKE, 4, FAKE, FAKE, 3, 1, NULL) == -10
    assert g(b"N", 4, 1, 1, 1, FAKE, 4, NULL, FAKE, 4, 1, NULL) == -8


def test_gbsv_argument_errors(lib):
    g = lib.dgbsv_batched  # (n,kl,ku,nrhs,A,ldab,P,B,ldb,info,batch,stream) -- LAPACK DGBSV numbering
    assert g(-1, 1, 1, 1, FAKE, 4, FAKE, FAKE, 4, FAKE, 1, NULL) == -1
    assert g(4, -1, 1, 1, FAKE, 4, FAKE, FAKE, 4, FAKE, 1, NULL) == -2
    assert g(4, 1, -1, 1, FAKE, 4, FAKE, FAKE, 4, FAKE, 1, NULL) == -3
    assert g(4, 1, 1, -1, FAKE, 4, FAKE, FAKE, 4, FAKE, 1, NULL) == -4
    assert g(4, 1, 1, 1, FAKE, 3, FAKE, FAKE, 4, FAKE, 1, NULL) == -6
    assert g(4, 1, 1, 1, FAKE, 4, FAKE, FAKE, 3, FAKE, 1, NULL) == -9
    assert g(4, 1, 1, 1, FAKE, 4, FAKE, FAKE, 4, NULL, 1, NULL) == -10
    s = lib.dgbsv_strided_batched
    assert s(4, 1, 1, 1, FAKE, 4, 16, FAKE, 4, FAKE, 3, 4, FAKE, 1, NULL) == -11
    h = lib.dgbsv_strided_batched_host
    assert h(4, 1, 1, 1, FAKE, 4, 16, FAKE, 4, FAKE, 4, 4, NULL, 1, NULL) == -13


def test_variant_heuristic_is_shape_only(lib):
    from paper_conf_sc_abdelfattahtlad23_b200 import binding as b
    assert b.trf_variant(512, 512, 10, 10) == b.ROWS
    assert b.rows_available(10, 10) and b.rows_available(2, 32) and b.rows_available(1, 1)
    assert not b.rows_available(0, 3) and not b.rows_available(3, 0)
    assert not b.tc_available(10, 10) and not b.thread_available(1, 1)  # opt-in builds only (-DBANDLU_WITH_TC/THREAD)
    # thin lower bands, square: the column-owner kernel; rectangular: row-slot / window kernels
    assert b.trf_variant(256, 256, 1, 1) == b.COLS and b.trf_variant(512, 512, 2, 3) == b.COLS
    assert b.trf_variant(300, 256, 1, 1) == b.ROWS
    assert b.trf_variant(64, 64, 0, 3) == b.COLS and b.trf_variant(64, 60, 0, 3) == b.WINDOW
    assert b.cols_available(3, 2) and b.cols_available(2, 32) and not b.cols_available(10, 10)
    assert not b.cols_available(4, 4)  # opt-in (-DBANDLU_COLS_WIDE): measured slower
    assert b.trf_variant(100, 100, 32, 32) == b.ROWS  # kl+1 > 32 lanes: two-warp row-slot kernel
    # band not instantiated ahead of time: run-time compiled row-slot kernels (NVRTC), else the safeguard
    assert b.trf_variant(100, 100, 33, 20) == (b.ROWS if b.jit_band(33, 20) else b.GENERIC)
    assert b.trs_variant(100, 32, 32, 1) == b.WINDOW
    assert b.trf_variant(0, 5, 1, 1) == b.GENERIC
    assert b.trs_variant(1024, 2, 32, 16) == b.WINDOW
    assert b.trs_variant(512, 10, 10, 1) == b.WINDOW  # lane-per-row solve measured slower here
    assert b.trs_variant(256, 1, 1, 1) == b.ROWS  # nrhs = 1, kl+ku+1 <= 4: lane-per-row solve
    assert b.trs_variant(512, 10, 10, 2) == b.WINDOW
    assert b.trs_rows_available(1, 1) and not b.trs_rows_available(2, 32)


def test_product_package_does_not_import_oracle():
    """The product path must not route through the oracle (task ③)."""
    pkg = os.path.join(ROOT, "paper_conf_sc_abdelfattahtlad23_b200")
    for dirpath, _, files in os.walk(pkg):
        for fn in files:
            if fn.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, fn)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, fn
                assert "bandlu_oracle" not in txt and "liboracle" not in txt, fn


def test_trfs_plan_reports_the_launches(lib):
    """bandlu_trfs_plan (no launch): the fused gbsv kernel for nrhs == 1 on row-slot
    bands while the batch fits in one wave of it, else the forward-fused factorization
    + backward launch; trf + trs where no fused path exists."""
    from paper_conf_sc_abdelfattahtlad23_b200 import binding as b
    p = b.trfs_plan(512, 10, 10, 1, 1000)
    assert p == {"kernels": ["gbtrf_rows_kernel"], "bytes": ["gbsv"], "fused": True}
    p = b.trfs_plan(512, 10, 10, 1, 10000)  # C3: 2.8 waves -> two launches
    assert p["kernels"] == ["gbtrf_rows_kernel", "gbtrs_bwd_kernel"] and p["bytes"] == ["trf_fwd", "trs_bwd"]
    assert b.trfs_plan(512, 10, 10, 1, 10000, b.TRFS_FUSED)["fused"]
    assert not b.trfs_plan(512, 10, 10, 1, 10, b.TRFS_TWO_LAUNCH)["fused"]
    p = b.trfs_plan(2048, 32, 32, 1, 100)
    assert p["kernels"] == ["gbtrf_wide_kernel", "gbtrs_window_kernel"] and not p["fused"]
    p = b.trfs_plan(1024, 2, 32, 1, 100)  # kl+ku+1+PF > 2G: no fused kernel for (2,32)
    assert p["kernels"] == ["gbtrf_cols_kernel", "gbtrs_window_kernel"] and not p["fused"]
    # C2 (beyond one wave of the row-slot fused kernel): column-owner factorization + forward, then
    # the backward kernel; C1 (within one wave): the row-slot fused kernel, one launch
    p = b.trfs_plan(256, 1, 1, 1, 10000)
    assert p["kernels"] == ["gbtrf_cols_kernel", "gbtrs_rows_kernel"] and not p["fused"]
    assert b.trfs_plan(256, 1, 1, 4, 10000)["kernels"] == ["gbtrf_cols_kernel", "gbtrs_window_kernel"]
    assert b.trfs_plan(64, 2, 2, 1, 100)["kernels"] == ["gbtrf_rows_kernel"]
    assert b.trfs_plan(256, 1, 1, 1, 10000, b.TRFS_FUSED)["kernels"] == ["gbtrf_rows_kernel"]
    p = b.trfs_plan(512, 10, 10, 1, 1000, b.TRFS_TWO_LAUNCH)
    assert p["kernels"] == ["gbtrf_rows_kernel", "gbtrs_bwd_kernel"]
    p = b.trfs_plan(1024, 2, 32, 16, 5000)
    # C4: the 16 right-hand sides ride with the column-owner factorization, then the backward solve
    assert p["kernels"] == ["gbtrf_cols_kernel", "gbtrs_window_kernel"] and p["bytes"] == ["trf_fwd", "trs_bwd"]
    p = b.trfs_plan(1024, 2, 32, 33, 5000)  # more right-hand sides than lanes (32): trf + trs
    assert p["kernels"] == ["gbtrf_cols_kernel", "gbtrs_window_kernel"] and p["bytes"] == ["trf", "trs"]
    p = b.trfs_plan(100, 5, 9, 1, 10, b.TRFS_TWO_LAUNCH)  # (5,9): not instantiated ahead of time
    if b.jit_band(5, 9):  # run-time compiled (NVRTC) kernels
        assert p["kernels"][0] == "gbtrf_rows_kernel" and p["kernels"][1] in ("gbtrs_bwd_kernel", "gbtrs_window_kernel", "gbtrs_blk_kernel")
    else:
        assert p["kernels"] == ["gbtrf_generic_kernel", "gbtrs_generic_kernel"]
    assert b.trfs_plan(0, 1, 1, 1, 10)["kernels"] == []
    assert lib.bandlu_trfs_plan(-1, 1, 1, 1, 1, 0, None) < 0
    assert lib.bandlu_trfs_plan(8, 1, 1, 1, 1, b.TRFS_TWO_LAUNCH | b.TRFS_FUSED, None) < 0


def test_jit_bands_compile_without_gpu(lib):
    """Every kernel a run-time compiled band uses compiles with NVRTC for sm_100a from
    the sources embedded in the library (no GPU needed): row-slot bands (incl. fused
    solve), a wide band (kl + 1 > 32) and a band without a fused solve (kv + 9 > 2G)."""
    from paper_conf_sc_abdelfattahtlad23_b200 import binding as b
    if not b.jit_band(5, 6):
        pytest.skip("NVRTC not available")
    for kl, ku in [(5, 6), (16, 16), (0, 40), (33, 20), (56, 4)]:  # (56, 4): wide, 4-column blocks
        assert b.jit_band(kl, ku)
        assert b.jit_check(kl, ku) == "", (kl, ku)
    assert not b.jit_band(10, 10) and not b.jit_band(2, 32)  # instantiated ahead of time
