"""Thin ctypes binding over the C ABI in include/bandlu.h (argument
marshalling only -- every step of the hot path runs in libbandlu.so's sm_100a
kernels).  There is no CPU fallback: if the shared library is missing or a
call fails, a RuntimeError is raised.

Tensor conventions (SURVEY 8(b) "Python view"): a strided batch of band
matrices is a contiguous float64 CUDA tensor A[batch, n, ldab] (column-major
AB(ldab, n) per matrix), ipiv int32 [batch, min(m, n)], info int32 [batch],
B float64 [batch, nrhs, ldb].  Calls are enqueued on torch's current CUDA
stream (or `stream=`), asynchronously.
"""
from __future__ import annotations

import ctypes
import os

import torch

from . import _build

AUTO, GENERIC, WINDOW, TC, ROWS, THREAD, TPM, THIN, COLS = 0, 1, 2, 3, 4, 5, 6, 7, 8
ERR_UNSUPPORTED, ERR_CUDA = 1000, 2000

_lib = None


class BandLUError(RuntimeError):
    def __init__(self, fn: str, code: int):
        if code < 0:
            msg = f"{fn}: argument {-code} is illegal"
        elif code == ERR_UNSUPPORTED:
            msg = f"{fn}: unsupported (variant / trans)"
        elif code >= ERR_CUDA:
            msg = f"{fn}: CUDA error {code - ERR_CUDA}"
        else:
            msg = f"{fn}: error {code}"
        super().__init__(msg)
        self.code = code


def lib_path() -> str:
    return _build.LIB


def load(build_if_missing: bool = False):
    """Load libbandlu.so (raise if it is missing: no fallback path exists)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_build.LIB):
        if build_if_missing:
            _build.build()
        else:
            raise RuntimeError(f"CUDA extension {_build.LIB} not built; run __graft_entry__.build()")
    lib = ctypes.CDLL(_build.LIB)
    i, i64, p, ch = ctypes.c_int, ctypes.c_int64, ctypes.c_void_p, ctypes.c_char
    sig = {
        "dgbtrf_batched": [i, i, i, i, p, i, p, p, i, p],
        "dgbtrf_strided_batched": [i, i, i, i, p, i, i64, p, i64, p, i, p],
        "dgbtrf_strided_batched_ex": [i, i, i, i, p, i, i64, p, i64, p, i, p, i],
        "dgbtrs_batched": [ch, i, i, i, i, p, i, p, p, i, i, p],
        "dgbtrs_strided_batched": [ch, i, i, i, i, p, i, i64, p, i64, p, i, i64, i, p],
        "dgbtrs_strided_batched_ex": [ch, i, i, i, i, p, i, i64, p, i64, p, i, i64, i, p, i],
        "dgbsv_batched": [i, i, i, i, p, i, p, p, i, p, i, p],
        "dgbsv_strided_batched": [i, i, i, i, p, i, i64, p, i64, p, i, i64, p, i, p],
        "dgbsv_strided_batched_host": [i, i, i, i, p, i, i64, p, i64, p, i, i64, p, i, p],
        "dgbtrfs_strided_batched": [i, i, i, i, p, i, i64, p, i64, p, i, i64, p, i, p],
        "dgbtrfs_strided_batched_ex": [i, i, i, i, p, i, i64, p, i64, p, i, i64, p, i, p, i],
        "bandlu_trf_variant": [i, i, i, i],
        "bandlu_tc_available": [i, i],
        "bandlu_rows_available": [i, i],
        "bandlu_trs_rows_available": [i, i],
        "bandlu_thread_available": [i, i],
        "bandlu_tpm_available": [i, i],
        "bandlu_thin_available": [i, i],
        "bandlu_cols_available": [i, i],
        "bandlu_jit_band": [i, i],
        "bandlu_jit_check": [i, i, p, i],
        "bandlu_trs_variant": [i, i, i, i],
        "bandlu_trfs_plan": [i, i, i, i, i, i, p],
        "bandlu_version": [],
    }
    for name, args in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = ctypes.c_int
    _lib = lib
    return lib


# exported symbol list (checked by tests against include/bandlu.h)
EXPORTS = ("dgbtrf_batched", "dgbtrf_strided_batched", "dgbtrf_strided_batched_ex", "dgbtrs_batched",
           "dgbtrs_strided_batched", "dgbtrs_strided_batched_ex", "dgbsv_batched", "dgbsv_strided_batched",
           "dgbsv_strided_batched_host", "dgbtrfs_strided_batched", "dgbtrfs_strided_batched_ex", "bandlu_trf_variant", "bandlu_trs_variant", "bandlu_tc_available", "bandlu_rows_available", "bandlu_trs_rows_available", "bandlu_thread_available",
           "bandlu_tpm_available", "bandlu_thin_available", "bandlu_cols_available", "bandlu_jit_band", "bandlu_jit_check", "bandlu_trfs_plan", "bandlu_version")


def _stream(stream):
    if stream is None:
        return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, torch.cuda.Stream):
        return ctypes.c_void_p(stream.cuda_stream)
    return ctypes.c_void_p(int(stream))


def _ptr(t: torch.Tensor | None):
    return ctypes.c_void_p(t.data_ptr() if t is not None and t.numel() > 0 else 0)


def _chk(fn: str, code: int):
    if code != 0:
        raise BandLUError(fn, code)


def _dev(t: torch.Tensor, dtype, name: str, ndim: int):
    if not (t.is_cuda and t.dtype == dtype and t.dim() == ndim and t.is_contiguous()):
        raise TypeError(f"{name}: need a contiguous CUDA {dtype} tensor of rank {ndim}")


def _shapes(A: torch.Tensor, n: int, ipiv: torch.Tensor | None, npiv: int, B: torch.Tensor | None = None,
            info: torch.Tensor | None = None) -> None:
    """Every tensor must describe the same batch on the same device: A [batch, n, ldab],
    ipiv [batch, >= npiv], B [batch, nrhs, ldb], info [batch] (the library trusts the
    sizes it is given, so a mismatch here would be an out-of-bounds access there)."""
    batch = A.shape[0]
    if A.shape[1] != n:
        raise ValueError(f"A.shape[1] = {A.shape[1]} must be n = {n}")
    for t, nm in ((ipiv, "ipiv"), (B, "B"), (info, "info")):
        if t is None:
            continue
        if t.shape[0] != batch:
            raise ValueError(f"{nm}.shape[0] = {t.shape[0]} must equal the batch {batch}")
        if t.device != A.device:
            raise ValueError(f"{nm} is on {t.device}, A on {A.device}")
    if ipiv is not None and ipiv.shape[1] < max(1, npiv):
        raise ValueError(f"ipiv.shape[1] = {ipiv.shape[1]} < {max(1, npiv)}")


def dgbtrf_strided_batched(m: int, n: int, kl: int, ku: int, A: torch.Tensor, ipiv: torch.Tensor,
                           info: torch.Tensor, variant: int = AUTO, stream=None) -> None:
    """In place: A [batch, n, ldab] -> LU factors; ipiv [batch, >=min(m,n)]; info [batch]."""
    _dev(A, torch.float64, "A", 3); _dev(ipiv, torch.int32, "ipiv", 2); _dev(info, torch.int32, "info", 1)
    batch, n_, ldab = A.shape
    _shapes(A, n, ipiv, min(m, n), info=info)
    f = load().dgbtrf_strided_batched_ex
    _chk("dgbtrf_strided_batched", f(m, n, kl, ku, _ptr(A), ldab, n * ldab, _ptr(ipiv), ipiv.shape[1],
                                     _ptr(info), batch, _stream(stream), variant))


def dgbtrs_strided_batched(trans: str, n: int, kl: int, ku: int, A: torch.Tensor, ipiv: torch.Tensor,
                           B: torch.Tensor, variant: int = AUTO, stream=None) -> None:
    """In place: B [batch, nrhs, ldb] <- A^{-1} B using dgbtrf factors."""
    _dev(A, torch.float64, "A", 3); _dev(ipiv, torch.int32, "ipiv", 2); _dev(B, torch.float64, "B", 3)
    _shapes(A, n, ipiv, n, B=B)
    batch, _, ldab = A.shape
    _, nrhs, ldb = B.shape
    f = load().dgbtrs_strided_batched_ex
    _chk("dgbtrs_strided_batched", f(trans.encode()[:1], n, kl, ku, nrhs, _ptr(A), ldab, n * ldab, _ptr(ipiv),
                                     ipiv.shape[1], _ptr(B), ldb, nrhs * ldb, batch, _stream(stream), variant))


def dgbsv_strided_batched(n: int, kl: int, ku: int, A: torch.Tensor, ipiv: torch.Tensor, B: torch.Tensor,
                          info: torch.Tensor, stream=None) -> None:
    _dev(A, torch.float64, "A", 3); _dev(ipiv, torch.int32, "ipiv", 2); _dev(B, torch.float64, "B", 3)
    _dev(info, torch.int32, "info", 1)
    _shapes(A, n, ipiv, n, B=B, info=info)
    batch, _, ldab = A.shape
    _, nrhs, ldb = B.shape
    _chk("dgbsv_strided_batched", load().dgbsv_strided_batched(
        n, kl, ku, nrhs, _ptr(A), ldab, n * ldab, _ptr(ipiv), ipiv.shape[1], _ptr(B), ldb, nrhs * ldb,
        _ptr(info), batch, _stream(stream)))


def dgbtrfs_strided_batched(n: int, kl: int, ku: int, A: torch.Tensor, ipiv: torch.Tensor, B: torch.Tensor,
                            info: torch.Tensor, stream=None, phase: int = 0) -> None:
    """dgbtrf then dgbtrs('N') (B solved for every matrix); fused forward solve when nrhs == 1.
    phase 1 / 2 run only the factorization / only the solve launch (profiling)."""
    _dev(A, torch.float64, "A", 3); _dev(ipiv, torch.int32, "ipiv", 2); _dev(B, torch.float64, "B", 3)
    _dev(info, torch.int32, "info", 1)
    _shapes(A, n, ipiv, n, B=B, info=info)
    batch, _, ldab = A.shape
    _, nrhs, ldb = B.shape
    _chk("dgbtrfs_strided_batched", load().dgbtrfs_strided_batched_ex(
        n, kl, ku, nrhs, _ptr(A), ldab, n * ldab, _ptr(ipiv), ipiv.shape[1], _ptr(B), ldb, nrhs * ldb,
        _ptr(info), batch, _stream(stream), phase))


def ptr_array(ts) -> torch.Tensor:
    """Device array of device pointers for the pointer-array entry points."""
    ptrs = [t.data_ptr() for t in ts]
    dev = ts[0].device if len(ts) else torch.device("cuda")
    return torch.tensor(ptrs, dtype=torch.int64, device=dev)


def dgbtrf_batched(m: int, n: int, kl: int, ku: int, A_ptrs: torch.Tensor, ldab: int, ipiv_ptrs: torch.Tensor,
                   info: torch.Tensor, batch: int, stream=None) -> None:
    _chk("dgbtrf_batched", load().dgbtrf_batched(m, n, kl, ku, _ptr(A_ptrs), ldab, _ptr(ipiv_ptrs), _ptr(info),
                                                 batch, _stream(stream)))


def dgbtrs_batched(trans: str, n: int, kl: int, ku: int, nrhs: int, A_ptrs: torch.Tensor, ldab: int,
                   ipiv_ptrs: torch.Tensor, B_ptrs: torch.Tensor, ldb: int, batch: int, stream=None) -> None:
    _chk("dgbtrs_batched", load().dgbtrs_batched(trans.encode()[:1], n, kl, ku, nrhs, _ptr(A_ptrs), ldab,
                                                 _ptr(ipiv_ptrs), _ptr(B_ptrs), ldb, batch, _stream(stream)))


def dgbsv_batched(n: int, kl: int, ku: int, nrhs: int, A_ptrs: torch.Tensor, ldab: int, ipiv_ptrs: torch.Tensor,
                  B_ptrs: torch.Tensor, ldb: int, info: torch.Tensor, batch: int, stream=None) -> None:
    _chk("dgbsv_batched", load().dgbsv_batched(n, kl, ku, nrhs, _ptr(A_ptrs), ldab, _ptr(ipiv_ptrs), _ptr(B_ptrs),
                                               ldb, _ptr(info), batch, _stream(stream)))


def dgbsv_strided_batched_host(n: int, kl: int, ku: int, A: torch.Tensor, ipiv: torch.Tensor, B: torch.Tensor,
                               info: torch.Tensor, stream=None) -> None:
    """End-to-end: HOST tensors (pinned recommended) in and out; synchronous."""
    for t, d, nm in ((A, torch.float64, "A"), (ipiv, torch.int32, "ipiv"), (B, torch.float64, "B"),
                     (info, torch.int32, "info")):
        if t.is_cuda or t.dtype != d or not t.is_contiguous():
            raise TypeError(f"{nm}: need a contiguous host {d} tensor")
    _shapes(A, n, ipiv, n, B=B, info=info)
    batch, _, ldab = A.shape
    _, nrhs, ldb = B.shape
    _chk("dgbsv_strided_batched_host", load().dgbsv_strided_batched_host(
        n, kl, ku, nrhs, _ptr(A), ldab, n * ldab, _ptr(ipiv), ipiv.shape[1], _ptr(B), ldb, nrhs * ldb,
        _ptr(info), batch, _stream(stream)))


def raw_call(name: str, *args) -> int:
    """Call an ABI entry point with raw ctypes arguments; returns its code (tests)."""
    return getattr(load(), name)(*args)


def trf_variant(m: int, n: int, kl: int, ku: int) -> int:
    return load().bandlu_trf_variant(m, n, kl, ku)


def tc_available(kl: int, ku: int) -> bool:
    """True if the opt-in tensor-core factorization (variant TC) is compiled for (kl, ku)."""
    return bool(load().bandlu_tc_available(kl, ku))


def rows_available(kl: int, ku: int) -> bool:
    """True if a row-slot factorization kernel (variant ROWS) is compiled for (kl, ku)."""
    return bool(load().bandlu_rows_available(kl, ku))


def thread_available(kl: int, ku: int) -> bool:
    """True if a thread-per-matrix factorization kernel (variant THREAD) is compiled for (kl, ku)."""
    return bool(load().bandlu_thread_available(kl, ku))


def tpm_available(kl: int, ku: int) -> bool:
    """True if the thread-per-matrix shared-memory-window factorization (variant TPM) is compiled for (kl, ku)."""
    return bool(load().bandlu_tpm_available(kl, ku))


def thin_available(kl: int, ku: int) -> bool:
    """True if the thin-band thread-per-matrix kernel (variant THIN) is compiled for (kl, ku)."""
    return bool(load().bandlu_thin_available(kl, ku))


def jit_band(kl: int, ku: int) -> bool:
    """True if (kl, ku) is served by run-time compiled (NVRTC) kernels (include/bandlu.h)."""
    return bool(load().bandlu_jit_band(kl, ku))


def jit_check(kl: int, ku: int) -> str:
    """Compile (no GPU needed) every run-time kernel the band uses; "" on success, else the error."""
    buf = ctypes.create_string_buffer(8192)
    rc = load().bandlu_jit_check(kl, ku, buf, len(buf))
    return "" if rc == 0 else buf.value.decode(errors="replace") or "failed"


def cols_available(kl: int, ku: int) -> bool:
    """True if a column-owner factorization kernel (dgbtrf variant COLS) is compiled for (kl, ku)."""
    return bool(load().bandlu_cols_available(kl, ku))


def trs_rows_available(kl: int, ku: int) -> bool:
    """True if a lane-per-row solve kernel (dgbtrs variant ROWS) is compiled for (kl, ku)."""
    return bool(load().bandlu_trs_rows_available(kl, ku))


def trs_variant(n: int, kl: int, ku: int, nrhs: int) -> int:
    return load().bandlu_trs_variant(n, kl, ku, nrhs)


KERNEL_NAMES = {1: "gbtrf_rows_kernel", 2: "gbtrf_window_kernel", 3: "gbtrf_wide_kernel", 4: "gbtrf_thread_kernel",
                5: "gbtrf_generic_kernel", 6: "gbtrs_bwd_kernel", 7: "gbtrs_rows_kernel", 8: "gbtrs_window_kernel",
                9: "gbtrs_generic_kernel", 10: "gbtrf_thin_kernel", 11: "gbtrs_blk_kernel",
                12: "gbtrf_cols_kernel"}
BYTE_KINDS = {1: "trf", 2: "trf_fwd", 3: "trs_bwd", 4: "trs", 5: "gbsv"}
TRFS_TWO_LAUNCH, TRFS_FUSED, TRFS_THIN = 16, 32, 64


def trfs_plan(n: int, kl: int, ku: int, nrhs: int, batch: int, phase: int = 0) -> dict:
    """The launches one dgbtrfs_strided_batched call (phase flag 0 / TRFS_TWO_LAUNCH /
    TRFS_FUSED) makes for a shape and batch (bandlu_trfs_plan)."""
    kinds = (ctypes.c_int * 4)()
    k = load().bandlu_trfs_plan(n, kl, ku, nrhs, batch, phase, kinds)
    if k < 0:
        raise BandLUError("bandlu_trfs_plan", k)
    codes = list(kinds)[:k]
    return {"kernels": [KERNEL_NAMES[c >> 4] for c in codes], "bytes": [BYTE_KINDS[c & 15] for c in codes],
            "fused": k == 1 and (codes[0] & 15) == 5}
