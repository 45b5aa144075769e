"""Writes tests/golden/fig2_9x9_kl2_ku3.json -- an EXACT (rational arithmetic)
band LU + solve of a 9x9 integer matrix with kl = 2, ku = 3, the shape of the
paper's Figure 2 band-layout example (Sec. 3; the figure's
entries are garbled in the extracted text, only its shape survives).

Independent of oracle/ and of the CUDA path: plain Python Fractions, textbook
GEPP on the dense matrix with LAPACK's pivot rule (first max |.|), with the
band-storage conventions of LAPACK DGBTRF (U with kl extra superdiagonals,
L multipliers stored in the pivot column, later swaps NOT applied to L:
"swap to the right only").  Run:  python make_fig2_golden.py
"""
import json
import os
import random
from fractions import Fraction as F

N, KL, KU = 9, 2, 3


def build_matrix(seed):
    rnd = random.Random(seed)
    A = [[F(0)] * N for _ in range(N)]
    for i in range(N):
        for j in range(max(0, i - KL), min(N, i + KU + 1)):
            v = 0
            while v == 0:
                v = rnd.randint(-9, 9)
            A[i][j] = F(v)
    return A


def band_lu_exact(A):
    """GEPP restricted to the band exactly as DGBTF2 does it (rows swapped only
    from column j to the right), in exact arithmetic."""
    A = [row[:] for row in A]
    ipiv, gaps = [], []
    for j in range(N):
        cand = list(range(j, min(N, j + KL + 1)))
        mags = [abs(A[i][j]) for i in cand]
        best = max(mags)
        p = cand[mags.index(best)]
        srt = sorted(mags, reverse=True)
        if len(srt) > 1 and best != 0:
            gaps.append(float((srt[0] - srt[1]) / srt[0]))
        ipiv.append(p + 1)
        assert best != 0
        if p != j:
            for c in range(j, N):
                A[j][c], A[p][c] = A[p][c], A[j][c]
        for i in range(j + 1, min(N, j + KL + 1)):
            A[i][j] = A[i][j] / A[j][j]
            for c in range(j + 1, N):
                A[i][c] -= A[i][j] * A[j][c]
    return A, ipiv, min(gaps)


def solve_exact(A, b):
    n = len(A)
    M = [row[:] + [b[i]] for i, row in enumerate(A)]
    for j in range(n):
        p = max(range(j, n), key=lambda i: abs(M[i][j]))
        M[j], M[p] = M[p], M[j]
        for i in range(j + 1, n):
            f = M[i][j] / M[j][j]
            for c in range(j, n + 1):
                M[i][c] -= f * M[j][c]
    x = [F(0)] * n
    for i in reversed(range(n)):
        s = M[i][n] - sum(M[i][c] * x[c] for c in range(i + 1, n))
        x[i] = s / M[i][i]
    return x


def main():
    seed = 0
    while True:
        A = build_matrix(seed)
        LU, ipiv, gap = band_lu_exact(A)
        if gap > 1e-3 and len(set(ipiv)) > 3 and any(p != i + 1 for i, p in enumerate(ipiv)):
            break
        seed += 1
    kv = KL + KU
    # band representation of the factors: AB(kv + i - j, j)
    lu_band = {}
    for j in range(N):
        for i in range(max(0, j - kv), min(N, j + KL + 1)):
            lu_band[f"{kv + i - j},{j}"] = str(LU[i][j])
    b = [F(i + 1) for i in range(N)]
    x = solve_exact(A, b)
    out = {
        "citation": "PAPER.md Sec. 3 Fig. 2 (P:277-291): 9x9 band matrix, kl=2, ku=3, LAPACK band "
                    "storage with kl fill rows; values are exact rationals from make_fig2_golden.py",
        "n": N, "kl": KL, "ku": KU, "seed": seed,
        "A_dense": [[str(v) for v in row] for row in A],
        "ipiv": ipiv,
        "lu_band": lu_band,
        "b": [str(v) for v in b],
        "x": [str(v) for v in x],
        "min_pivot_gap": gap,
    }
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "fig2_9x9_kl2_ku3.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print("wrote", path, "seed", seed, "ipiv", ipiv)


if __name__ == "__main__":
    main()
