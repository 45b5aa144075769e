"""CPU oracle for batched band LU (dgbtrf) + banded solve (dgbtrs 'N') + dgbsv.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product package ``paper_conf_sc_abdelfattahtlad23_b200`` never
imports it, and the two share no code ("Oracle").

The arithmetic lives in ``bandlu_oracle.c`` (plain C, LAPACK DGBTF2 / DGBTRS /
DTBSV / DGBSV written out step by step; Sec. 5.1, Sec. 6
P:625-640, Sec. 3).  This module only builds/loads that library and
marshals numpy arrays into it.

Array conventions (same as the product's Python view):
  A    float64 [batch, n, ldab]   (column-major AB(ldab, n) per matrix)
  ipiv int32   [batch, min(m, n)] (1-based, LAPACK)
  info int32   [batch]
  B    float64 [batch, nrhs, ldb] (column-major B(ldb, nrhs) per matrix)
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "bandlu_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

CFLAGS = ["-O2", "-mfma", "-ffp-contract=off", "-fopenmp", "-shared", "-fPIC", "-std=c11"]


def build(force: bool = False) -> str:
    """Compile bandlu_oracle.c -> liboracle.so (gcc)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        i, i64, p, d = ctypes.c_int, ctypes.c_int64, ctypes.c_void_p, ctypes.c_double
        lib.oracle_dgbtf2.argtypes = [i, i, i, i, p, i, p, p]
        lib.oracle_dgbtf2.restype = d
        lib.oracle_dgbtrs_n.argtypes = [i, i, i, i, p, i, p, p, i]
        lib.oracle_dgbtrs_n.restype = None
        lib.oracle_dgbsv.argtypes = [i, i, i, i, p, i, p, p, i, p]
        lib.oracle_dgbsv.restype = None
        lib.oracle_dgbtrf_batch.argtypes = [i, i, i, i, p, i, i64, p, i64, p, p, i, i]
        lib.oracle_dgbtrf_batch.restype = None
        lib.oracle_dgbtrs_n_batch.argtypes = [i, i, i, i, p, i, i64, p, i64, p, i, i64, i, i]
        lib.oracle_dgbtrs_n_batch.restype = None
        lib.oracle_dgbtrs_t_batch.argtypes = [i, i, i, i, p, i, i64, p, i64, p, i, i64, i, i]
        lib.oracle_dgbtrs_t_batch.restype = None
        lib.oracle_dgbsv_batch.argtypes = [i, i, i, i, p, i, i64, p, i64, p, i, i64, p, i, i]
        lib.oracle_dgbsv_batch.restype = None
        lib.oracle_max_threads.argtypes = []
        lib.oracle_max_threads.restype = i
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


def _check(a: np.ndarray, dtype, ndim: int, name: str):
    if not isinstance(a, np.ndarray) or a.dtype != dtype or a.ndim != ndim or not a.flags.c_contiguous:
        raise TypeError(f"{name}: need C-contiguous {np.dtype(dtype).name} array of rank {ndim}")


def max_threads() -> int:
    return _load().oracle_max_threads()


def dgbtrf(A: np.ndarray, m: int, n: int, kl: int, ku: int, nthreads: int = 0,
           return_gap: bool = False):
    """In-place batched dgbtf2 on A [batch, n, ldab].  Returns (ipiv, info[, min_gap])."""
    _check(A, np.float64, 3, "A")
    batch, n_, ldab = A.shape
    assert n_ == n and ldab >= 2 * kl + ku + 1
    mn = min(m, n)
    ipiv = np.zeros((batch, max(mn, 0)), dtype=np.int32)
    info = np.zeros(batch, dtype=np.int32)
    gap = np.zeros(batch, dtype=np.float64)
    _load().oracle_dgbtrf_batch(m, n, kl, ku, _ptr(A), ldab, n * ldab, _ptr(ipiv), max(mn, 0),
                                _ptr(info), _ptr(gap), batch, nthreads)
    return (ipiv, info, gap) if return_gap else (ipiv, info)


def dgbtrs(A: np.ndarray, ipiv: np.ndarray, B: np.ndarray, n: int, kl: int, ku: int,
           nthreads: int = 0, trans: str = "N") -> None:
    """In-place batched dgbtrs(trans) on B [batch, nrhs, ldb] given factors A and ipiv."""
    _check(A, np.float64, 3, "A"); _check(B, np.float64, 3, "B"); _check(ipiv, np.int32, 2, "ipiv")
    batch, _, ldab = A.shape
    _, nrhs, ldb = B.shape
    f = _load().oracle_dgbtrs_n_batch if trans.upper() == "N" else _load().oracle_dgbtrs_t_batch
    f(n, kl, ku, nrhs, _ptr(A), ldab, n * ldab, _ptr(ipiv), ipiv.shape[1], _ptr(B), ldb, nrhs * ldb, batch,
      nthreads)


def dgbsv(A: np.ndarray, B: np.ndarray, n: int, kl: int, ku: int, nthreads: int = 0):
    """In-place batched dgbsv.  Returns (ipiv, info); B untouched where info > 0."""
    _check(A, np.float64, 3, "A"); _check(B, np.float64, 3, "B")
    batch, _, ldab = A.shape
    _, nrhs, ldb = B.shape
    ipiv = np.zeros((batch, n), dtype=np.int32)
    info = np.zeros(batch, dtype=np.int32)
    _load().oracle_dgbsv_batch(n, kl, ku, nrhs, _ptr(A), ldab, n * ldab, _ptr(ipiv), n,
                               _ptr(B), ldb, nrhs * ldb, _ptr(info), batch, nthreads)
    return ipiv, info
