"""Seeded synthetic workload generator shared by tests, smoke() and bench.py.

This module holds NONE of the method's arithmetic: it only draws numbers.
Both the oracle side and the CUDA side receive its arrays as inputs, so it is
the one module they share.

Recipe (shaped like the paper's sweeps P:415-453, P:549-552,
"diagonally non-dominant" random bands):
  * every VALID band entry (matrix row i in [0, m), column c in [0, n),
    c - ku <= i <= c + kl) is i.i.d. U(-1, 1);
  * fill rows (band rows 0..kl-1), unreferenced corners and padding rows
    (ldab > 2kl+ku+1) hold a NaN sentinel, so any read of them poisons the
    result and any write to a corner/padding position is visible;
  * B is U(-1, 1) in rows [0, n); rows n..ldb-1 hold the NaN sentinel.
Values are a counter-based hash (splitmix64) of (seed, stream, global matrix
index, column, band row), so any shard or subset of the batch can be
regenerated independently of the others (multi-GPU sharding, sampled parity
at full size) and independently of ldab / ldb padding.
"""
from __future__ import annotations

import numpy as np

SEED = 20231112
_A_STREAM = 0x0A
_B_STREAM = 0x0B
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_GOLD = np.uint64(0x9E3779B97F4A7C15)


def _mix(x: np.ndarray) -> np.ndarray:
    x = x.astype(np.uint64, copy=True)
    x ^= x >> np.uint64(30)
    x *= _M1
    x ^= x >> np.uint64(27)
    x *= _M2
    x ^= x >> np.uint64(31)
    return x


def _uniform_pm1(seed: int, stream: int, mat_idx: np.ndarray, local: np.ndarray) -> np.ndarray:
    """U(-1,1) from (seed, stream, matrix index, local element counter)."""
    key = _mix(np.array([(seed & 0xFFFFFFFF) | (stream << 32)], dtype=np.uint64))[0]
    with np.errstate(over="ignore"):
        ctr = (mat_idx.astype(np.uint64) << np.uint64(32)) ^ local.astype(np.uint64)
        z = _mix(ctr * _GOLD + key)
    u = (z >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)
    return 2.0 * u - 1.0


def band_valid_mask(m: int, n: int, kl: int, ku: int, ldab: int) -> np.ndarray:
    """bool [n, ldab]: True where AB(r, c) holds an ORIGINAL band entry of A."""
    kv = kl + ku
    c = np.arange(n)[:, None]
    r = np.arange(ldab)[None, :]
    i = c - kv + r  # matrix row of AB(r, c)
    return (r >= kl) & (r <= kv + kl) & (i >= 0) & (i < m)


def band_output_mask(m: int, n: int, kl: int, ku: int, ldab: int) -> np.ndarray:
    """bool [n, ldab]: positions that hold a factor entry after dgbtrf
    (U with its kl extra superdiagonals in rows 0..kv, L in rows kv+1..kv+kl),
    i.e. rows r <= 2kl+ku with matrix row in [0, m)."""
    kv = kl + ku
    c = np.arange(n)[:, None]
    r = np.arange(ldab)[None, :]
    i = c - kv + r
    return (r <= kv + kl) & (i >= 0) & (i < m)


def gen_band(m: int, n: int, kl: int, ku: int, ldab: int | None = None, count: int = 1,
             first: int = 0, seed: int = SEED, sentinel: float = np.nan) -> np.ndarray:
    """float64 [count, n, ldab]: matrices first .. first+count-1 of the workload."""
    ldab = 2 * kl + ku + 1 if ldab is None else ldab
    ldmin = 2 * kl + ku + 1
    assert ldab >= ldmin
    out = np.full((count, n, ldab), sentinel, dtype=np.float64)
    mask = band_valid_mask(m, n, kl, ku, ldab)
    cc, rr = np.nonzero(mask)
    if cc.size == 0 or count == 0:
        return out
    local = cc.astype(np.uint64) * np.uint64(ldmin) + rr.astype(np.uint64)
    # chunk over matrices to bound temporary memory
    step = max(1, (1 << 24) // max(1, cc.size))
    for s in range(0, count, step):
        e = min(count, s + step)
        idx = np.arange(first + s, first + e, dtype=np.uint64)[:, None]
        vals = _uniform_pm1(seed, _A_STREAM, idx, local[None, :])
        out[s:e, cc, rr] = vals
    return out


def gen_rhs(n: int, nrhs: int, ldb: int | None = None, count: int = 1, first: int = 0,
            seed: int = SEED, sentinel: float = np.nan) -> np.ndarray:
    """float64 [count, nrhs, ldb]; rows >= n hold the sentinel."""
    ldb = max(1, n) if ldb is None else ldb
    out = np.full((count, nrhs, ldb), sentinel, dtype=np.float64)
    if n == 0 or nrhs == 0 or count == 0:
        return out
    local = (np.arange(nrhs, dtype=np.uint64)[:, None] * np.uint64(n)
             + np.arange(n, dtype=np.uint64)[None, :]).reshape(-1)
    step = max(1, (1 << 24) // max(1, local.size))
    for s in range(0, count, step):
        e = min(count, s + step)
        idx = np.arange(first + s, first + e, dtype=np.uint64)[:, None]
        vals = _uniform_pm1(seed, _B_STREAM, idx, local[None, :]).reshape(e - s, nrhs, n)
        out[s:e, :, :n] = vals
    return out


def shard_range(batch: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous shard [lo, hi) of rank r out of R."""
    return (batch * rank) // world, (batch * (rank + 1)) // world


# ---- accounting (bytes / flops per matrix; SURVEY 8(d) exact forms) ----

def alg_bytes(m: int, n: int, kl: int, ku: int, nrhs: int) -> tuple[int, int]:
    """(B_trf, B_trs) algorithmic HBM bytes per matrix."""
    kv = kl + ku
    R = sum(min(m - 1, j + kl) - max(0, j - ku) + 1 for j in range(n) if max(0, j - ku) <= min(m - 1, j + kl))
    W = sum(min(m - 1, j + kl) - max(0, j - kv) + 1 for j in range(n) if max(0, j - kv) <= min(m - 1, j + kl))
    mn = min(m, n)
    b_trf = 8 * R + 8 * W + 4 * mn + 4
    b_trs = 8 * W + 4 * n + 16 * n * nrhs
    return b_trf, b_trs


def alg_bytes_fused(n: int, kl: int, ku: int, nrhs: int) -> tuple[int, int]:
    """(factor+forward kernel, backward kernel) algorithmic HBM bytes per square
    matrix for the fused path (dgbtrfs, nrhs == 1): the factorization kernel
    moves B_trf plus B in / y out; the backward kernel reads the U entries
    (rows max(0, j-kv)..j of each column) and y, and writes x.  It never
    re-reads L or ipiv, so the sum is below B_trf + B_trs."""
    kv = kl + ku
    b_trf, _ = alg_bytes(n, n, kl, ku, nrhs)
    wu = sum(min(j, kv) + 1 for j in range(n))
    return b_trf + 16 * n * nrhs, 8 * wu + 16 * n * nrhs


def nominal_flops(n: int, kl: int, ku: int, nrhs: int) -> tuple[int, int]:
    """(trf, trs) nominal flops per square matrix."""
    kv = kl + ku
    trf = 0
    for j in range(n):
        km = min(kl, n - 1 - j)
        trf += km + 2 * km * min(ku, n - 1 - j)
    trs = nrhs * (sum(2 * min(kl, n - 1 - j) for j in range(n - 1))
                  + sum(1 + 2 * min(kv, j) for j in range(n)))
    return trf, trs
