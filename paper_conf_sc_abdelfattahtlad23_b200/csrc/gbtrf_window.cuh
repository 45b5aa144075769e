// gbtrf_window.cuh -- sm_100a sliding-window band LU with partial pivoting,
// register resident, compiled per (KL, KU).
//
// What it computes: LAPACK DGBTF2 exactly (Sec. 5.1 pseudo-code
// P:350-367, ju rule P:492-494, "swap to the right only" P:358/P:369-374),
// same fp64 operation sequence as the oracle => bitwise-equal factors, ipiv,
// info.
//
// B200 design (differs from the paper's smem sliding window, Sec. 5.3
// P:485-556, Fig. 4; this is the register-file variant the paper proposes as
// future work in Sec. 8.1, made practical by instantiating the
// (kl, ku) pairs that matter):
//  * A group of G = pow2 >= KL+1 lanes owns one matrix; 32/G matrices share a
//    warp (per-warp instruction cost is shared by all of them).
//  * Row-owner mapping: each of the KL+1 active lanes holds ONE row of the
//    active window -- the KV+1 = KL+KU+1 values at columns j..j+KV -- in
//    registers.  Columns map to register slots (col mod W) and the step loop
//    is unrolled W times, so no register ever moves when the window slides.
//  * Row interchanges are relabelings: a lane carries the logical position of
//    its row.  LAPACK swaps only columns j..ju; beyond ju both rows hold
//    structural zeros, so swapping whole rows is identical.
//  * IAMAX: exact first-max via three redux.sync over the 64-bit |x| key and
//    the logical position (ties -> smallest position, Q2).
//  * The pivot row (U row j) goes through a 16-byte-aligned smem record that
//    is the broadcast source for the rank-1 update (FP64 FMA in registers)
//    and the source of the U-row store to HBM.  Multipliers are stored by
//    their owning lanes.  Each step thus needs one __syncwarp.
//  * Input rows are gathered by cp.async (LDGSTS, L1-allocating, zero-fill
//    outside the matrix) into a 2-batch row ring in smem, NR rows ahead of
//    use; the lane freed by the pivot row reloads its registers from it.
//  * Every input element is read from HBM once and every output element is
//    written once; the fill rows (input) are never read.
#pragma once
#include "common.cuh"

namespace bandlu {

template <int KL_, int KU_>
struct TrfWin {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU, W = KV + 1;
    static constexpr int G = pow2_ceil(KL + 1);  // lanes per matrix
    static constexpr int GPW = 32 / G;           // matrices per warp
    static constexpr int WP = (W + 1) & ~1;      // even row pitch (doubles) -> 16 B aligned rows
    static constexpr int NR = W <= 24 ? 8 : 4;   // rows per staging batch (power of 2)
    static constexpr int RR = 2 * NR;            // ring rows (2 batches)
    static constexpr int GROUP_DBL = (RR + 2) * WP;  // ring + 2 pivot-row records
    static constexpr int STAGE_IT = (NR * W + G - 1) / G;
    static constexpr int WARPS = 4;
    static constexpr size_t smem_bytes() { return (size_t)WARPS * GPW * GROUP_DBL * sizeof(double); }
};

template <int KL, int KU, class AP, class PP>
__global__ void __launch_bounds__(TrfWin<KL, KU>::WARPS * 32)
    gbtrf_window_kernel(int m, int n, AP A, int ldab, PP P, int *__restrict__ info, int batch) {
    using C = TrfWin<KL, KU>;
    constexpr int KV = C::KV, W = C::W, G = C::G, WP = C::WP, NR = C::NR, RR = C::RR;
    extern __shared__ __align__(16) double smem[];

    const int lane = (int)lane_id(), wib = (int)(threadIdx.x >> 5);
    const int g = lane / G, t = lane % G;
    const int64_t mat = ((int64_t)blockIdx.x * C::WARPS + wib) * C::GPW + g;
    const bool live = mat < batch;
    const unsigned wmask = __ballot_sync(0xffffffffu, live);
    if (!live) return;
    const unsigned gmask = (G == 32) ? 0xffffffffu : (((1u << G) - 1u) << (g * G));

    double *__restrict__ ab = A.get(mat);
    int *__restrict__ ipiv = P.get(mat);
    if (m <= 0 || n <= 0) {
        if (t == 0) info[mat] = 0;
        return;
    }
    double *ring = smem + (size_t)(wib * C::GPW + g) * C::GROUP_DBL;
    double *rec = ring + RR * WP;

    // Stage input rows [qb, qb+NR) (row layout: ring[a][c] = A(q, q-KL+c)).
    auto stage = [&](int b) {
        const int qb = KL + 1 + b * NR;
        double *half = ring + (b & 1) * NR * WP;
#pragma unroll
        for (int k = 0; k < C::STAGE_IT; ++k) {
            const int e = t + k * G;
            if (e < NR * W) {
                const int a = e / W, c = e - a * W;
                const int q = qb + a, col = q - KL + c;
                const bool ok = (q < m) && (col < n);
                const double *src = ok ? ab + (int64_t)col * ldab + (KV + KL - c) : ab;
                cp_async8(smem_u32(half + a * WP + c), src, ok ? 8u : 0u);
            }
        }
        cp_async_commit();
    };

    // Window registers: v[c % W] = row value at column c, rows 0..KL first.
    double v[W];
    int pos = (t <= KL) ? t : 0x7fffffff;
#pragma unroll
    for (int c = 0; c < W; ++c) {
        const bool ok = (t <= KL) && (t < m) && (c < n) && (c <= t + KU);
        v[c] = ok ? ab[(int64_t)c * ldab + (KV + t - c)] : 0.0;
    }
    stage(0);

    int linfo = 0;
    const int mn = min(m, n);
    for (int j0 = 0; j0 < mn; j0 += W) {
#pragma unroll
        for (int s = 0; s < W; ++s) {
            const int j = j0 + s;
            if (j >= mn) break;
            const bool batch_start = (j & (NR - 1)) == 0;
            if (batch_start) cp_async_wait<0>();

            // ---- IAMAX over the candidates (logical rows j..min(j+KL, m-1))
            const double x = v[s];
            const bool cand = (t <= KL) && (pos < m);
            const uint64_t key = cand ? abs_key(x) : 0ull;
            const unsigned hi = (unsigned)(key >> 32), lo = (unsigned)key;
            const unsigned mhi = __reduce_max_sync(gmask, hi);
            const unsigned mlo = __reduce_max_sync(gmask, hi == mhi ? lo : 0u);
            const bool win = (hi == mhi) && (lo == mlo);
            const unsigned ppos = __reduce_min_sync(gmask, win ? (unsigned)pos : 0xffffffffu);
            const bool is_piv = ((unsigned)pos == ppos);
            const bool zp = (mhi | mlo) == 0u;  // exact zero pivot (all candidates are +-0)

            // ---- pivot row -> smem record (U row j: columns j..j+KV)
            double *rc = rec + (j & 1) * WP;
            if (is_piv) {
#pragma unroll
                for (int c = 0; c < W; c += 2) {
                    double2 d;
                    d.x = v[(s + c) % W];
                    d.y = (c + 1 < W) ? v[(s + c + 1) % W] : 0.0;
                    *reinterpret_cast<double2 *>(rc + c) = d;
                }
                ipiv[j] = (int)ppos + 1;
            }
            __syncwarp(wmask);
            if (batch_start) stage(j / NR + 1);

            if (zp && linfo == 0) linfo = j + 1;
            // interchange = relabel: the old row j takes the pivot row's place
            if (pos == j && !is_piv) pos = (int)ppos;

            // ---- SCAL: multiplier = x * RN(1/p) (DSCAL(ONE/pivot), Q7)
            double l = x;
            if (!zp) {
                const double r = __drcp_rn(rc[0]);
                l = __dmul_rn(x, r);
            }
            if (cand && !is_piv) ab[(int64_t)j * ldab + (KV + pos - j)] = l;

            // ---- RANK-1 update of the window (DGER, alpha = -1, FMA)
            if (!zp) {
#pragma unroll
                for (int c = 0; c < W; c += 2) {  // record padded to WP (even): rc[c+1] exists
                    const double2 u = *reinterpret_cast<const double2 *>(rc + c);
                    if (c >= 1) v[(s + c) % W] = __fma_rn(l, -u.x, v[(s + c) % W]);
                    if (c + 1 < W) v[(s + c + 1) % W] = __fma_rn(l, -u.y, v[(s + c + 1) % W]);
                }
            }

            // ---- U row j -> HBM: U(j, j+c) at AB(KV-c, j+c)
#pragma unroll
            for (int c0 = 0; c0 < W; c0 += G) {
                const int c = c0 + t;
                if (c < W && j + c < n) ab[(int64_t)(j + c) * ldab + (KV - c)] = rc[c];
            }

            // ---- slide: the pivot lane takes row j+KL+1; column j leaves all rows
            if (is_piv) {
                const int q = j + KL + 1;
                pos = q;
                const double *rr = ring + ((q - KL - 1) & (RR - 1)) * WP;
#pragma unroll
                for (int c = 0; c < W; c += 2) {
                    const double2 d = *reinterpret_cast<const double2 *>(rr + c);
                    v[(s + 1 + c) % W] = d.x;
                    if (c + 1 < W) v[(s + 2 + c) % W] = d.y;
                }
            } else {
                v[s] = 0.0;
            }
        }
    }
    cp_async_wait<0>();

    // LAPACK's SET_FILLIN also zeroes fill-row positions whose matrix row is
    // >= m when m < n (those rows are never pivot rows here).
    if (m < n) {
        for (int c = m + KU + 1 + t; c <= min(n - 1, m + KV - 1); c += G) {
#pragma unroll 1
            for (int r = 0; r < KL; ++r) {
                const int i = c - KV + r;
                const bool zeroed = (c >= KU + 1 && c <= min(KV, n) - 1 && r >= KV - c) || (c >= KV && c - KV < mn);
                if (i >= m && zeroed) ab[(int64_t)c * ldab + r] = 0.0;
            }
        }
    }
    if (t == 0) info[mat] = linfo;
}

}  // namespace bandlu
