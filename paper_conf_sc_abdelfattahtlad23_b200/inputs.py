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


# ---- the same generator on a torch device (bitwise equal to gen_band / gen_rhs) ----
# bench.py fills HBM-sized sweep batches on the GPU without a host round trip
# (torch int64 arithmetic wraps modulo 2^64; logical shifts are masked).

def _s64(u: int) -> int:
    return u - (1 << 64) if u >= (1 << 63) else u


def _mix_t(x):
    import torch

    def srl(v, s):
        return (v >> s) & ((1 << (64 - s)) - 1)
    x = x ^ srl(x, 30)
    x = x * _s64(int(_M1))
    x = x ^ srl(x, 27)
    x = x * _s64(int(_M2))
    x = x ^ srl(x, 31)
    return x


def _uniform_pm1_t(seed: int, stream: int, mat_idx, local):
    import torch
    key = _s64(int(_mix(np.array([(seed & 0xFFFFFFFF) | (stream << 32)], dtype=np.uint64))[0]))
    ctr = (mat_idx << 32) ^ local
    z = _mix_t(ctr * _s64(int(_GOLD)) + key)
    u = ((z >> 11) & ((1 << 53) - 1)).to(torch.float64) * (1.0 / 9007199254740992.0)
    return 2.0 * u - 1.0


def gen_band_torch(m: int, n: int, kl: int, ku: int, count: int, first: int = 0, device="cpu",
                   ldab: int | None = None, seed: int = SEED, sentinel: float = float("nan"), out=None):
    """torch float64 [count, n, ldab] on `device`, bitwise equal to gen_band(...)."""
    import torch
    ldab = 2 * kl + ku + 1 if ldab is None else ldab
    ldmin = 2 * kl + ku + 1
    if out is None:
        out = torch.empty((count, n, ldab), dtype=torch.float64, device=device)
    out.fill_(sentinel)
    mask = band_valid_mask(m, n, kl, ku, ldab)
    cc, rr = np.nonzero(mask)
    if cc.size == 0 or count == 0:
        return out
    flat = torch.from_numpy((cc * ldab + rr).astype(np.int64)).to(out.device)
    local = torch.from_numpy((cc.astype(np.int64) * ldmin + rr)).to(out.device)[None, :]
    view = out.view(count, n * ldab)
    step = max(1, (1 << 24) // cc.size)
    for s in range(0, count, step):
        e = min(count, s + step)
        idx = torch.arange(first + s, first + e, dtype=torch.int64, device=out.device)[:, None]
        view[s:e].index_copy_(1, flat, _uniform_pm1_t(seed, _A_STREAM, idx, local))
    return out


def gen_rhs_torch(n: int, nrhs: int, count: int, first: int = 0, device="cpu", ldb: int | None = None,
                  seed: int = SEED, sentinel: float = float("nan"), out=None):
    """torch float64 [count, nrhs, ldb] on `device`, bitwise equal to gen_rhs(...)."""
    import torch
    ldb = max(1, n) if ldb is None else ldb
    if out is None:
        out = torch.empty((count, nrhs, ldb), dtype=torch.float64, device=device)
    out.fill_(sentinel)
    if n == 0 or nrhs == 0 or count == 0:
        return out
    local = torch.arange(nrhs * n, dtype=torch.int64, device=out.device)[None, :]
    step = max(1, (1 << 24) // (nrhs * n))
    for s in range(0, count, step):
        e = min(count, s + step)
        idx = torch.arange(first + s, first + e, dtype=torch.int64, device=out.device)[:, None]
        out[s:e, :, :n] = _uniform_pm1_t(seed, _B_STREAM, idx, local).view(e - s, nrhs, n)
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


def alg_bytes_kind(n: int, kl: int, ku: int, nrhs: int, kind: str) -> int:
    """Algorithmic HBM bytes per square matrix that ONE launch of the given class must
    move (bandlu_trfs_plan byte classes): trf = B_trf; trf_fwd = B_trf + B in / y out;
    trs_bwd = U entries + y in / x out; trs = B_trs; gbsv (the fused single launch) =
    B_trf + B in / x out -- U is produced and consumed inside the kernel."""
    b_trf, b_trs = alg_bytes(n, n, kl, ku, nrhs)
    f_trf, f_bwd = alg_bytes_fused(n, kl, ku, nrhs)
    return {"trf": b_trf, "trf_fwd": f_trf, "trs_bwd": f_bwd, "trs": b_trs, "gbsv": b_trf + 16 * n * nrhs}[kind]


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
