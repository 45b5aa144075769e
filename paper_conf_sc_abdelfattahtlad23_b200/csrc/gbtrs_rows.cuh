// gbtrs_rows.cuh -- sm_100a banded solve A x = b with dgbtrf factors for ONE
// right-hand side (trans = 'N'), one LANE PER RHS ROW.
//
// What it computes: LAPACK DGBTRS('N') exactly (Sec. 6),
// the oracle's operation sequence (bitwise-equal results):
//   forward (FWD): for j = 0..n-2: swap b(j) <-> b(ipiv[j]-1) (pivots applied
//     progressively); if b(j) != 0: b(j+i) = fma(L(j+i,j), -b(j),
//     b(j+i)), i = 1..min(kl, n-1-j);
//   backward (DTBSV 'U','N','N', bandwidth kv): for j = n-1..0:
//     if b(j) != 0: b(j) = b(j) / U(j,j) (true division, reading Q9), then
//     b(i) = fma(-b(j), U(i,j), b(i)), i = j-1 .. max(0, j-kv).
//
// Why: the window solve (gbtrs_window.cuh) gives each
// (matrix, RHS column) ONE lane, so at nrhs = 1 a batch of 10k matrices is
// ~1.2k warps whose 512-step serial chains (division -> FMA -> division)
// leave the SM schedulers idle (C3: IPC ~0.3, 0.31 ms for 0.93 GB).  Here a
// group of G = pow2 >= kv+1 lanes shares one matrix and lane t holds the RHS
// rows r == t (mod G) -- a window of kv+1 consecutive rows sits on kv+1
// distinct lanes with no data movement as it slides:
//  * step j: the lane holding row j (d = (j-t) mod G == 0) divides, the value
//    reaches the group by one shuffle, lanes with 1 <= d <= kv apply one FMA
//    each with U(j-d, j) = AB[kv-d][j] -- the column's kv+1 band entries are
//    contiguous, so a group's loads of one column are one coalesced request;
//  * factor entries are loaded P steps ahead into a register ring (loop
//    unrolled by P); each lane's next RHS row (r - G backward, r + G forward)
//    is loaded G steps before it enters the window;
//  * forward: the interchange of rows j and l = ipiv[j]-1 (l - j <= kl < G)
//    is two shuffles; rows that retire are stored, and at the end of the
//    forward pass the lanes hold rows n-G..n-1, which is exactly the backward
//    pass's starting window -- no reload.
// 32/G (matrix, RHS column) units per warp; no shared memory, 64-72 registers.  Measured:
// AUTO for kl+ku+1 <= 4 only: it issues one division per matrix-step,
// the window solve one per warp-step for up to 32 matrices.
#pragma once
#include "common.cuh"

namespace bandlu {

template <int KL_, int KU_>
struct TrsRows {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU;
    static constexpr int G = pow2_ceil(KV + 1 > 2 ? KV + 1 : 2);  // lanes per matrix
    static constexpr int GPW = 32 / G;                           // matrices per warp
#ifndef BANDLU_TRS_ROWS_P
#define BANDLU_TRS_ROWS_P 8
#endif
    static constexpr int P = BANDLU_TRS_ROWS_P;                  // factor prefetch distance (steps)
    static constexpr int WARPS = 4;                              // warps per CTA
    static_assert(KV + 1 <= 32, "one lane per window row");
};

template <int KL, int KU, bool FWD, class AP, class PP, class BP>
__global__ void __launch_bounds__(TrsRows<KL, KU>::WARPS * 32)
    gbtrs_rows_kernel(int n, int nrhs, AP A, int ldab, PP Pv, BP Bv, int ldb, const int *__restrict__ skip_info,
                      int batch) {
    using C = TrsRows<KL, KU>;
    constexpr int KV = C::KV, G = C::G, P = C::P;
    const int lane = (int)lane_id();
    const int g = lane / G, t = lane % G;
    // one group per (matrix, RHS column)
    const int64_t unit = ((int64_t)blockIdx.x * C::WARPS + (threadIdx.x >> 5)) * C::GPW + g;
    const int64_t mat = unit / nrhs;
    bool live = unit < (int64_t)batch * nrhs;
    if (live && skip_info != nullptr && skip_info[mat] != 0) live = false;
    if (__ballot_sync(0xffffffffu, live) == 0u) return;
    // Dead groups run the loop (their lanes take part in the group shuffles) but
    // load and store nothing.
    const double *__restrict__ ab = live ? A.get(mat) : nullptr;
    double *bv = live ? Bv.get(mat) + (unit % nrhs) * (int64_t)ldb : nullptr;

    double x = 0.0, nx = 0.0;  // this lane's current row value, its next row value

    // ------------------------------------------------------------ forward
    if constexpr (FWD && KL > 0) {
        const int *__restrict__ ipiv = live ? Pv.get(mat) : nullptr;
        // step j: lane holds row j + e, e = (t - j) mod G; factor entry L(j+e, j) = AB[KV+e][j]
        auto lload = [&](int jj) -> double {
            const int e = (t - jj) & (G - 1);
            const bool ok = live && jj < n - 1 && e >= 1 && e <= KL && jj + e < n;
            return ok ? __ldg(ab + (int64_t)jj * ldab + KV + e) : 0.0;
        };
        auto pload = [&](int jj) -> int { return (live && jj < n - 1) ? __ldg(ipiv + jj) : 0; };
        double lr[P];
        int pr[P];
#pragma unroll
        for (int s = 0; s < P; ++s) {
            lr[s] = lload(s);
            pr[s] = pload(s);
        }
        x = (live && t < n) ? bv[t] : 0.0;
        nx = (live && t + G < n) ? bv[t + G] : 0.0;
#pragma unroll 1
        for (int j0 = 0; j0 < n; j0 += P) {
#pragma unroll
            for (int s = 0; s < P; ++s) {
                const int j = j0 + s;
                if (j >= n) break;
                const double lc = lr[s];
                const int pj = pr[s] - 1;  // l (0-based); unused at j = n-1
                lr[s] = lload(j + P);
                pr[s] = pload(j + P);
                const int e = (t - j) & (G - 1);
                double y = x;
                if (j < n - 1) {
                    // interchange b(j) <-> b(l): l - j <= KL < G, distinct lanes unless l == j
                    const double vj = __shfl_sync(0xffffffffu, x, j & (G - 1), G);
                    y = __shfl_sync(0xffffffffu, x, pj & (G - 1), G);  // new b(j)
                    if (e == pj - j && e != 0) x = vj;
                    if (e == 0) x = y;
                    if (e >= 1 && e <= KL && y != 0.0) x = __fma_rn(lc, -y, x);
                }
                if (e == 0 && j + G < n) {  // row j retires (the last G rows stay for the backward pass)
                    if (live) bv[j] = y;
                    x = nx;
                    nx = (live && j + 2 * G < n) ? bv[j + 2 * G] : 0.0;
                }
            }
        }
        // lanes now hold rows n-G..n-1 (row r == t mod G); next rows r - G are stored
        const int r0 = (n - 1) - ((n - 1 - t) & (G - 1));
        nx = (live && r0 - G >= 0) ? bv[r0 - G] : 0.0;
    } else {
        const int r0 = (n - 1) - ((n - 1 - t) & (G - 1));  // largest row <= n-1 with r == t (mod G)
        x = (live && r0 >= 0) ? bv[r0] : 0.0;
        nx = (live && r0 - G >= 0) ? bv[r0 - G] : 0.0;
    }

    // ------------------------------------------------------------ backward
    // step j: lane holds row j - d, d = (j - t) mod G; factor entry U(j-d, j) = AB[KV-d][j]
    // incremental load address: next load step jl, its d and column offset
    int jl = n - 1, dl = (jl - t) & (G - 1);
    int64_t cix = (int64_t)jl * ldab;
    auto uload_next = [&]() -> double {
        const bool ok = live && jl >= dl;  // d <= KV and row jl - d >= 0 (covers jl < 0)
        const double v = (ok && dl <= KV) ? __ldg(ab + cix + (KV - dl)) : 0.0;
        --jl;
        dl = (dl - 1) & (G - 1);
        cix -= ldab;
        return v;
    };
    double ur[P];
#pragma unroll
    for (int s = 0; s < P; ++s) ur[s] = uload_next();
    int d = (n - 1 - t) & (G - 1);  // d of the current step
    // full blocks of P steps; steps j < 0 of the last block do nothing (no stores,
    // no loads: their lanes have d > j)
#pragma unroll 1
    for (int j0 = n - 1; j0 >= 0; j0 -= P) {
#pragma unroll
        for (int s = 0; s < P; ++s) {
            const int j = j0 - s;
            const double uc = ur[s];
            ur[s] = uload_next();
            // b(j) != 0 decides the update (DTBSV), also if the quotient underflows to 0
            const bool own = (d == 0) && j >= 0;
            const bool nz = own && x != 0.0;
            const unsigned nzm = __ballot_sync(0xffffffffu, nz);
            const double xo = ddiv_rn_if(nz, x, uc);
            const double xj = __shfl_sync(0xffffffffu, xo, j & (G - 1), G);
            if (d >= 1 && d <= KV && ((nzm >> (g * G + (j & (G - 1)))) & 1u)) x = __fma_rn(-xj, uc, x);
            if (own) {  // row j is final
                if (live) bv[j] = xj;
                x = nx;
                nx = (live && j - 2 * G >= 0) ? bv[j - 2 * G] : 0.0;
            }
            d = (d - 1) & (G - 1);
        }
    }
}

}  // namespace bandlu
