// gbtrs_window.cuh -- sm_100a fused banded solve A X = B with dgbtrf factors
// (trans = 'N'), compiled per (KL, KU).
//
// What it computes: LAPACK DGBTRS('N') exactly (Sec. 6):
//   forward: for j = 0..n-2: swap B(j) <-> B(ipiv[j]-1) (pivots applied
//     progressively), then B(j+i) = fma(L(j+i,j), -B(j), B(j+i)),
//     skipped when B(j) == 0 (DGER);
//   backward (DTBSV 'U','N','N', bandwidth kv): for j = n-1..0,
//     if B(j) != 0: B(j) = B(j) / U(j,j) (true division, Q9), then
//     B(i) = fma(-B(j), U(i,j), B(i)) for i = j-1 .. j-kv.
//
// B200 design (the paper's blocked fwd/bwd kernels, Sec. 6, Fig. 6,
// cache nb columns of L/U in registers and nb+kl / nb+kv RHS entries in smem;
// here the roles flip):
//  * One LANE per (matrix, RHS column): a group of R = pow2 >= nrhs (<= 32)
//    lanes shares one matrix, 32/R matrices per warp.  Each lane keeps its
//    sliding RHS window -- KL+1 entries forward, KV+1 backward -- in
//    registers (slot = row mod window, loop unrolled by the window length),
//    so the whole serial chain runs in registers.  The row interchange is a
//    predicated select over the KL window slots.
//  * Both passes run in ONE kernel; the factor columns and the incoming RHS
//    entries are staged into a per-warp smem ring by warp-cooperative,
//    coalesced cp.async (L part only in the forward pass, U part only in the
//    backward pass, so each factor entry is read from HBM once), NB columns
//    per stage, double buffered, one __syncwarp per stage.
#pragma once
#include "common.cuh"

namespace bandlu {

template <int KL_, int KU_>
struct TrsWin {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU;
    static constexpr int WF = KL + 1, WB = KV + 1;  // forward / backward window lengths
    static constexpr int NB = 4;                    // columns per stage
    static constexpr int SLOT = WB > KL ? WB : KL;  // factor doubles per staged column (max of passes)
    // per-matrix ring: 2 stages x NB x (SLOT factor + 32 max RHS) doubles + 2 x NB ipiv
    __host__ __device__ static constexpr size_t stage_dbl(int R) { return (size_t)NB * (SLOT + R) + NB / 2 + 1; }
    __host__ __device__ static constexpr size_t group_dbl(int R) { return (2 * stage_dbl(R)) | 1; }  // odd pitch: conflict-free
    static constexpr size_t smem_bytes(int R) {
        return (size_t)(32 / R) * group_dbl(R) * sizeof(double) + (32 / R) * 3 * sizeof(void *);
    }
};

// Stage layout for one group (doubles, from the group base):
//   stage st at st*stage_dbl: [fac: NB*SLOT][rhs: NB*R][piv: NB ints]
template <int KL, int KU, class AP, class PP, class BP>
__global__ void __launch_bounds__(32)
    gbtrs_window_kernel(int n, int nrhs, AP A, int ldab, PP P, BP B, int ldb, const int *__restrict__ skip_info,
                        int batch, int R /* pow2 lanes per matrix */, int chunks /* rhs chunks per matrix */) {
    using C = TrsWin<KL, KU>;
    constexpr int KV = C::KV, WF = C::WF, WB = C::WB, NB = C::NB, SLOT = C::SLOT;
    extern __shared__ __align__(16) double smem[];
    const int lane = (int)lane_id();
    const int gpw = 32 / R;
    const int g = lane / R, t = lane % R;
    const int64_t unit = (int64_t)blockIdx.x * gpw + g;  // (matrix, rhs chunk)
    const int64_t mat = unit / chunks;
    const int r0 = (int)(unit % chunks) * 32;
    const int rhs = r0 + t;
    bool live = unit < (int64_t)batch * chunks;
    if (live && skip_info != nullptr && skip_info[mat] != 0) live = false;
    const bool act = live && rhs < nrhs;  // lane solves (and stores) a column
    // Dead groups stay in the warp: staging is warp-cooperative.  They compute
    // on zero-filled data and never touch global memory.
    if (__ballot_sync(0xffffffffu, live) == 0u) return;
    const unsigned wmask = 0xffffffffu;
    const void *dummy = g_dummy;

    const size_t SD = C::stage_dbl(R), GD = C::group_dbl(R);
    double **gA = reinterpret_cast<double **>(smem + gpw * GD);
    int **gP = reinterpret_cast<int **>(gA + gpw);
    double **gB = reinterpret_cast<double **>(gP + gpw);
    if (t == 0) {
        gA[g] = live ? const_cast<double *>(A.get(mat)) : nullptr;
        gP[g] = live ? const_cast<int *>(P.get(mat)) : nullptr;
        gB[g] = live ? B.get(mat) + (int64_t)r0 * ldb : nullptr;
    }
    __syncwarp();
    double *gbase = smem + g * GD;
    double *bcol = act ? gB[g] + (int64_t)t * ldb : nullptr;  // this lane's RHS column

    // --------------------------------------------------------- forward
    // stage k: columns c in [k*NB, k*NB+NB): L part AB(KV+1+i, c), i < KL
    // (zero beyond row n-1), ipiv[c], and RHS rows c+KL+1 (zero beyond n-1).
    auto stage_fwd = [&](int k) {
        const int c0 = k * NB;
        const int st = k & 1;
        if constexpr (KL > 0) {
            const int EF = NB * KL;
            for (int e = lane; e < gpw * EF; e += 32) {
                const int gg = e / EF, rem = e - gg * EF, cc = rem / KL, i = rem - cc * KL;
                double *dstg = smem + gg * GD + st * SD;
                const double *a = gA[gg];
                const int c = c0 + cc;
                const bool ok = (a != nullptr) && (c + 1 + i < n);
                cp_async8(smem_u32(dstg + cc * SLOT + i), ok ? a + (int64_t)c * ldab + (KV + 1 + i) : dummy,
                          ok ? 8u : 0u);
            }
        }
        for (int e = lane; e < gpw * NB * R; e += 32) {
            const int gg = e / (NB * R), rem = e - gg * (NB * R), rr = rem / NB, cc = rem - rr * NB;
            double *dstg = smem + gg * GD + st * SD + NB * SLOT;
            const double *b = gB[gg];
            const int row = c0 + cc + KL + 1;
            const bool ok = (b != nullptr) && (row < n) && (r0 + rr < nrhs);
            cp_async8(smem_u32(dstg + rr * NB + cc), ok ? b + (int64_t)rr * ldb + row : dummy, ok ? 8u : 0u);
        }
        for (int e = lane; e < gpw * NB; e += 32) {
            const int gg = e / NB, cc = e - gg * NB;
            int *dstg = reinterpret_cast<int *>(smem + gg * GD + st * SD + NB * (SLOT + R));
            const int *p = gP[gg];
            const int c = c0 + cc;
            const bool ok = (p != nullptr) && (c < n);
            cp_async4(smem_u32(dstg + cc), ok ? (const void *)(p + c) : dummy, ok ? 4u : 0u);
        }
        cp_async_commit();
    };

    if constexpr (KL > 0) {
        double w[WF];
#pragma unroll
        for (int i = 0; i < WF; ++i) w[i] = (act && i < n) ? bcol[i] : 0.0;
        stage_fwd(0);
        for (int j0 = 0; j0 < n; j0 += WF) {
#pragma unroll
            for (int s = 0; s < WF; ++s) {
                const int j = j0 + s;
                if (j >= n) break;
                const int cc = j & (NB - 1);
                if (cc == 0) {
                    cp_async_wait<0>();
                    __syncwarp(wmask);
                    stage_fwd(j / NB + 1);
                }
                const double *sg = gbase + ((j / NB) & 1) * SD;
                const int *piv = reinterpret_cast<const int *>(sg + NB * (SLOT + R));
                // interchange B(j) <-> B(l), l in [j, j+KL] (LAPACK never reads ipiv[n-1])
                const int d = (j < n - 1) ? piv[cc] - 1 - j : 0;
                double y = w[s];
#pragma unroll
                for (int i = 1; i < WF; ++i) {
                    const bool p = (d == i);
                    const double wi = w[(s + i) % WF];
                    w[(s + i) % WF] = p ? w[s] : wi;
                    y = p ? wi : y;
                }
                if (act) bcol[j] = y;
                if (y != 0.0) {
                    const double *lc = sg + cc * SLOT;
#pragma unroll
                    for (int i = 1; i < WF; ++i) w[(s + i) % WF] = __fma_rn(lc[i - 1], -y, w[(s + i) % WF]);
                }
                w[s] = sg[NB * SLOT + t * NB + cc];  // RHS row j+KL+1 (0 beyond n)
            }
        }
        cp_async_wait<0>();
        __syncwarp(wmask);  // y visible to the backward staging of other lanes
    }

    // --------------------------------------------------------- backward
    // step k handles row j = n-1-k; stage k covers steps [k*NB, k*NB+NB):
    // U part AB(r, j), r = 0..KV (zero above row 0), RHS rows j-KV-1 (0 if < 0).
    auto stage_bwd = [&](int k) {
        const int st = k & 1;
        const int EU = NB * WB;
        for (int e = lane; e < gpw * EU; e += 32) {
            const int gg = e / EU, rem = e - gg * EU, cc = rem / WB, r = rem - cc * WB;
            double *dstg = smem + gg * GD + st * SD;
            const double *a = gA[gg];
            const int j = n - 1 - (k * NB + cc);
            const bool ok = (a != nullptr) && (j >= 0) && (j - KV + r >= 0);
            cp_async8(smem_u32(dstg + cc * SLOT + r), ok ? a + (int64_t)j * ldab + r : dummy, ok ? 8u : 0u);
        }
        for (int e = lane; e < gpw * NB * R; e += 32) {
            const int gg = e / (NB * R), rem = e - gg * (NB * R), rr = rem / NB, cc = rem - rr * NB;
            double *dstg = smem + gg * GD + st * SD + NB * SLOT;
            const double *b = gB[gg];
            const int row = n - 1 - (k * NB + cc) - KV - 1;
            const bool ok = (b != nullptr) && (row >= 0) && (r0 + rr < nrhs);
            cp_async8(smem_u32(dstg + rr * NB + cc), ok ? b + (int64_t)rr * ldb + row : dummy, ok ? 8u : 0u);
        }
        cp_async_commit();
    };

    double x[WB];
#pragma unroll
    for (int i = 0; i < WB; ++i) x[i] = (act && n - 1 - i >= 0) ? bcol[n - 1 - i] : 0.0;
    stage_bwd(0);
    for (int k0 = 0; k0 < n; k0 += WB) {
#pragma unroll
        for (int s = 0; s < WB; ++s) {
            const int k = k0 + s;
            if (k >= n) break;
            const int j = n - 1 - k;
            const int cc = k & (NB - 1);
            if (cc == 0) {
                cp_async_wait<0>();
                __syncwarp(wmask);
                stage_bwd(k / NB + 1);
            }
            const double *sg = gbase + ((k / NB) & 1) * SD;
            const double *uc = sg + cc * SLOT;  // uc[r] = AB(r, j)
            double xj = x[s];
            if (xj != 0.0) {
                xj = __ddiv_rn(xj, uc[KV]);
#pragma unroll
                for (int i = 1; i < WB; ++i) x[(s + i) % WB] = __fma_rn(-xj, uc[KV - i], x[(s + i) % WB]);
            }
            if (act) bcol[j] = xj;
            x[s] = sg[NB * SLOT + t * NB + cc];  // y(j-KV-1) (0 if < 0)
        }
    }
    cp_async_wait<0>();
}

}  // namespace bandlu
