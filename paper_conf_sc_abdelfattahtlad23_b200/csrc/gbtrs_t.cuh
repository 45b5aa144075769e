// gbtrs_t.cuh -- sm_100a banded solve A^T X = B with dgbtrf factors
// (trans = 'T'/'C'), compiled per (KL, KU).
//
// What it computes: LAPACK DGBTRS('T') exactly, in the oracle's order
// (oracle_dgbtrs_t; Sec. 6 P:625-640 gives the 'N' case, the
// transposed one is the LAPACK routine the paper's API mirrors):
//   pass 1, U^T z = b (DTBSV 'U','T','N', bandwidth kv): for j = 0..n-1:
//     temp = b(j); temp = fma(-U(i,j), z(i), temp) for i = max(0,j-kv) .. j-1
//     (farthest row first); z(j) = temp / U(j,j) (true division);
//   pass 2, L^T P^T x = z: for j = n-2..0: temp = 0; temp = fma(x(j+i),
//     L(j+i,j), temp) for i = 1..min(kl, n-1-j); x(j) = x(j) - temp; then
//     swap x(j) <-> x(ipiv[j]-1).
//
// B200 design (same machinery as gbtrs_window.cuh, roles of the passes
// swapped): one LANE per (matrix, RHS column), R = pow2 >= nrhs lanes per
// matrix; pass 1 keeps the last kv results in registers and reads U column j
// (rows 0..kv, contiguous) from a smem ring filled by 16-byte cp.async chunks
// split over the matrix's copy lanes; pass 2 keeps rows j..j+kl in registers,
// reads L column j (rows kv+1..kv+kl) and ipiv[j] from the ring, and the
// interchange is a predicated select over the window.  Row j+kl is final
// after step j (later swaps reach at most j-1+kl), so it is stored then.
//  * Steps run in blocks of UB with ONE cp.async group and one wait per block
//    and no barrier inside it: pass 1's dot product for step j+1 only needs
//    z(j) in its last FMA, so the compiler overlaps it with step j's FMA chain
//    and division (the order of every chain is unchanged).  Measured C3
//    (10,10), n = 512, 10^4 matrices: 0.616 ms vs 0.915 ms with a wait and
//    barrier per step, vs 3.46 ms for the thread-per-column generic kernel.
//  * Each lane copies the RHS rows of a block as 16-byte aligned pairs (not one
//    8-byte copy per row: at 16 RHS per matrix that was the LSU cost).
//  * The first kv steps of pass 1 and the last kl steps of pass 2 (the
//    truncated dot products) run straight from global memory, so the ring
//    loop has no per-element predicates.
#pragma once
#include "common.cuh"

#ifndef BANDLU_TRST_STEPS_NARROW
#define BANDLU_TRST_STEPS_NARROW 16  // column steps in flight, kl + ku + 1 <= 5
#endif
#ifndef BANDLU_TRST_STEPS_WIDE
#define BANDLU_TRST_STEPS_WIDE 8
#endif
#ifndef BANDLU_TRST_UB
#define BANDLU_TRST_UB 4  // steps per block when the window is longer than 8
#endif

namespace bandlu {

template <int KL_, int KU_>
struct TrsT {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU;
    static constexpr int STEPS = (KV + 1 <= 5) ? BANDLU_TRST_STEPS_NARROW : BANDLU_TRST_STEPS_WIDE;
    // blocks of UB steps share one cp.async group and one wait; NB blocks in flight
    static constexpr int UB1 = KV <= 8 ? (KV > 0 ? KV : 1) : BANDLU_TRST_UB;
    static constexpr int UB2 = KL <= 8 ? (KL > 0 ? KL : 1) : BANDLU_TRST_UB;
    static constexpr int NB1 = (STEPS + UB1 - 1) / UB1 < 2 ? 2 : (STEPS + UB1 - 1) / UB1;
    static constexpr int NB2 = (STEPS + UB2 - 1) / UB2 < 2 ? 2 : (STEPS + UB2 - 1) / UB2;
    static constexpr int NS1 = NB1 * UB1, NS2 = NB2 * UB2;  // ring slots per pass
    // pass-1 slot: [SP1: U rows 0..kv, 16-byte rounded]; pass-2 slot: [SP2: L rows][ipiv, pad].
    // RHS rows move per block: each lane copies the UB rows a block consumes as 16-byte aligned
    // pairs (UB + 2 doubles at most) into its area of the block's RHS buffer.
    static constexpr int SP1 = ((KV + 1 + 2) + 1) & ~1;
    static constexpr int SP2 = ((KL + 2) + 1) & ~1;
    static constexpr int SL1 = SP1, SL2 = SP2 + 2;
    static constexpr int RB1 = ((UB1 + 2) + 1) & ~1, RB2 = ((UB2 + 2) + 1) & ~1;
    __host__ __device__ static constexpr int p1_dbl(int R) { return NS1 * SL1 + NB1 * RB1 * R; }
    __host__ __device__ static constexpr int p2_dbl(int R) { return NS2 * SL2 + NB2 * RB2 * R; }
    __host__ __device__ static constexpr int ring_dbl(int R) { return p1_dbl(R) > p2_dbl(R) ? p1_dbl(R) : p2_dbl(R); }
    // pitch == 2 (mod 4) doubles: the groups' reads of one slot offset sit in different banks
    __host__ __device__ static constexpr int group_dbl(int R) { return ring_dbl(R) + (6 - ring_dbl(R) % 4) % 4; }
    static constexpr int PAD = 2;
    static size_t smem_bytes(int R, int gpw) { return (size_t)(PAD + gpw * group_dbl(R)) * 8; }
};

template <int KL, int KU, class AP, class PP, class BP>
__global__ void __launch_bounds__(32)
    gbtrs_t_kernel(int n, int nrhs, AP A, int ldab, PP P, BP B, int ldb, int batch,
                   int R /* pow2 lanes per matrix */, int chunks /* rhs chunks per matrix */,
                   int gpw /* matrices (groups) per warp, <= 32 / R */) {
    using C = TrsT<KL, KU>;
    constexpr int KV = C::KV, UB1 = C::UB1, UB2 = C::UB2, NB1 = C::NB1, NB2 = C::NB2, NS1 = C::NS1, NS2 = C::NS2;
    extern __shared__ __align__(16) double smem[];
    const int lane = (int)lane_id();
    const int g = lane / R, t = lane % R;
    const int64_t unit = (int64_t)blockIdx.x * gpw + g;  // (matrix, rhs chunk)
    const int64_t mat = unit / chunks;
    const int r0 = (int)(unit % chunks) * 32;
    const bool live = g < gpw && unit < (int64_t)batch * chunks;
    const bool act = live && (r0 + t < nrhs);  // lane solves (and stores) a column
    if (__ballot_sync(0xffffffffu, live) == 0u) return;

    const int GD = C::group_dbl(R);
    constexpr int SD1 = C::SL1, SD2 = C::SL2, RB1 = C::RB1, RB2 = C::RB2;
    double *gring = smem + C::PAD + (g < gpw ? g : 0) * GD;
    const double *ab = live ? A.get(mat) : nullptr;
    const int *ipiv = live ? P.get(mat) : nullptr;
    double *bcol = act ? B.get(mat) + (int64_t)(r0 + t) * ldb : nullptr;
    const void *dummy = g_dummy;
    const uint32_t gring_s = smem_u32(gring);
    // this lane's RHS rows qlo..qlo+cnt-1 (zero outside 0..n-1) -> dst as 16-byte aligned pairs
    // starting at row qlo - o, o = (qlo + ph) & 1
    const int ph = act ? (int)((reinterpret_cast<uintptr_t>(bcol) >> 3) & 1) : 0;
    auto issue_rows = [&](uint32_t dst, int qlo, int cnt) {
        if (g >= gpw) return;
        const int q0 = qlo - ((qlo + ph) & 1);
        for (int r = q0; r < qlo + cnt; r += 2, dst += 16) {
            if (act && r >= 0 && r + 1 < n) {
                cp_async16(dst, bcol + r, 16u);
            } else if (act && r >= 0 && r < n) {  // last row: its 8 bytes, zero-fill the rest
                cp_async16(dst, bcol + r, 8u);
            } else if (act && r == -1 && n > 0) {  // (row -1, row 0)
                st_shared_f64_if(true, dst, 0.0);
                cp_async8(dst + 8, bcol, 8u);
            } else {
                cp_async16(dst, dummy, 0u);
            }
        }
    };
    // parity of a factor range's first element: its offset inside the 16-byte aligned slot
    auto delta_of = [&](int64_t lo) { return live ? (int)((reinterpret_cast<uintptr_t>(ab + lo) >> 3) & 1) : 0; };

    // copy role: CPG lanes per group split the 16-byte chunks of a factor range
    const int CPG = 32 / gpw;
    const int cg = lane / CPG, cq = lane % CPG;
    const int64_t cunit = (int64_t)blockIdx.x * gpw + cg;
    const bool clive = cunit < (int64_t)batch * chunks;
    const double *cab = clive ? A.get(cunit / chunks) : nullptr;
    const int *cipiv = clive ? P.get(cunit / chunks) : nullptr;
    const uint32_t cring_s = smem_u32(smem + C::PAD + cg * GD);
    auto issue_fac = [&](uint32_t dst, int64_t lo, int cnt) {
        const uintptr_t a = reinterpret_cast<uintptr_t>(cab + lo);
        const uintptr_t a0 = a & ~(uintptr_t)15, a1 = (a + (uintptr_t)cnt * 8 + 15) & ~(uintptr_t)15;
        const int nch = (int)((a1 - a0) >> 4);
        for (int q = cq; q < nch; q += CPG) cp_async16(dst + q * 16, reinterpret_cast<const void *>(a0 + q * 16), 16u);
    };

    // ================================================= pass 1: U^T z = b
    const int np = n < KV ? n : KV;
    if (act) {  // rows j < kv: truncated dot products, straight from global
#pragma unroll 1
        for (int j = 0; j < np; ++j) {
            const double *col = ab + (int64_t)j * ldab + KV - j;  // col[i] = U(i, j)
            double temp = bcol[j];
#pragma unroll 1
            for (int i = 0; i < j; ++i) temp = __fma_rn(-col[i], bcol[i], temp);
            bcol[j] = __ddiv_rn(temp, col[j]);
        }
    }
    const int n1 = n - KV;  // steps k = 0..n1-1: column j = KV + k, U rows 0..KV (slot k % NS1)
    if (n1 > 0) {
        // block b: steps b*UB1 .. +UB1-1 and their rows b(KV + k) (RHS buffer b % NB1)
        const uint32_t rhs1 = gring_s + (uint32_t)((NS1 * SD1 + t * RB1) * 8);
        auto issue_blk = [&](int b) {  // the UB1 steps of block b, one cp.async group
            if (b * UB1 < n1) {
                if (clive) {
#pragma unroll 1
                    for (int s = 0; s < UB1; ++s) {
                        const int k = b * UB1 + s;
                        if (k >= n1) break;
                        issue_fac(cring_s + (uint32_t)((k % NS1) * SD1 * 8), (int64_t)(KV + k) * ldab, KV + 1);
                    }
                }
                issue_rows(rhs1 + (uint32_t)((b % NB1) * R * RB1 * 8), KV + b * UB1, UB1);
            }
            cp_async_commit();
        };
#pragma unroll 1
        for (int b = 0; b < NB1; ++b) issue_blk(b);
        const int d1 = delta_of(0) ^ (int)(((int64_t)ldab * KV) & 1);  // parity of column KV's start
        const int dstep = ldab & 1;                                     // parity flips per column if ldab odd
        constexpr int XS = KV + UB1;
        double x[XS];  // x[p] = z(k0 + p): the KV previous results, then this block's
#pragma unroll
        for (int p = 0; p < XS; ++p) x[p] = (p < KV && act) ? bcol[p] : 0.0;
#pragma unroll 1
        for (int b = 0, k0 = 0; k0 < n1; ++b, k0 += UB1) {
            cp_async_wait<NB1 - 1>();
            __syncwarp();
            // no barrier inside the block: step s+1's dot product overlaps step s's division
            const double *rin = gring + NS1 * SD1 + ((b % NB1) * R + t) * RB1 + ((KV + k0 + ph) & 1);
#pragma unroll
            for (int s = 0; s < UB1; ++s) {
                const int k = k0 + s, rs = k % NS1;
                const double *slot = gring + rs * SD1;
                const double *uc = slot + (d1 ^ ((k & 1) & dstep));  // uc[r] = AB(r, j) = U(j-KV+r, j)
                double temp = rin[s];                               // b(j)
#pragma unroll
                for (int i = 0; i < KV; ++i) temp = __fma_rn(-uc[i], x[s + i], temp);
                const double z = __ddiv_rn(temp, uc[KV]);  // steps past n1: stale slot, never stored
                x[s + KV] = z;
                if (act && k < n1) bcol[KV + k] = z;
            }
            __syncwarp();
            issue_blk(b + NB1);
#pragma unroll
            for (int p = 0; p < XS; ++p) x[p] = (p + UB1 < XS) ? x[p + UB1] : 0.0;
        }
        cp_async_wait<0>();
    }
    __threadfence_block();
    __syncwarp();

    // ========================================= pass 2: L^T P^T x = z
    if constexpr (KL > 0) {
        const int jb0 = n - 1 - KL;  // ring steps: j = jb0 .. 0 (full length-KL dot products)
        if (act) {                   // j = n-2 .. jb0+1: truncated, straight from global
#pragma unroll 1
            for (int j = n - 2; j > jb0 && j >= 0; --j) {
                const int lm = min(KL, n - 1 - j);
                const double *lc = ab + (int64_t)j * ldab + KV;  // lc[i] = L(j+i, j)
                double temp = 0.0;
#pragma unroll 1
                for (int i = 1; i <= lm; ++i) temp = __fma_rn(bcol[j + i], lc[i], temp);
                bcol[j] = __dsub_rn(bcol[j], temp);
                const int l = ipiv[j] - 1;
                if (l != j) {
                    const double tt = bcol[l];
                    bcol[l] = bcol[j];
                    bcol[j] = tt;
                }
            }
        }
        if (jb0 >= 0) {
            __threadfence_block();
            __syncwarp();
            // blocks of UB2 rows aligned to row 0: block bi covers rows bi*UB2 .. bi*UB2+UB2-1
            // (top block: rows > jb0 were done above); row j uses slot j % NS2
            // (RHS buffer bi % NB2 holds rows bi*UB2 .. +UB2-1: z(j) for j <= jb0)
            const uint32_t rhs2 = gring_s + (uint32_t)((NS2 * SD2 + t * RB2) * 8);
            auto issue_blk = [&](int bi) {
                if (bi >= 0) {
                    if (clive) {
#pragma unroll 1
                        for (int p = UB2 - 1; p >= 0; --p) {
                            const int j = bi * UB2 + p;
                            if (j > jb0) continue;
                            const uint32_t dst = cring_s + (uint32_t)((j % NS2) * SD2 * 8);
                            if (cq == 0) cp_async4(dst + C::SP2 * 8, cipiv + j, 4u);
                            issue_fac(dst, (int64_t)j * ldab + KV + 1, KL);
                        }
                    }
                    issue_rows(rhs2 + (uint32_t)((bi % NB2) * R * RB2 * 8), bi * UB2, UB2);
                }
                cp_async_commit();
            };
            const int btop = jb0 / UB2;
#pragma unroll 1
            for (int b = 0; b < NB2; ++b) issue_blk(btop - b);
            const int d2 = delta_of(KV + 1);  // parity of column 0's L rows; flips per column if ldab odd
            const int dstep = ldab & 1;
            constexpr int XS = UB2 + KL;
            double v[XS];  // v[p] = x(bi*UB2 + p)
#pragma unroll
            for (int p = 0; p < XS; ++p) {
                const int row = btop * UB2 + p;
                v[p] = (act && row > jb0 && row < n) ? bcol[row] : 0.0;
            }
#pragma unroll 1
            for (int bi = btop; bi >= 0; --bi) {
                cp_async_wait<NB2 - 1>();
                __syncwarp();
                const double *rin = gring + NS2 * SD2 + ((bi % NB2) * R + t) * RB2 + ((bi * UB2 + ph) & 1);
#pragma unroll
                for (int s = 0; s < UB2; ++s) {
                    const int pj = UB2 - 1 - s;  // row j = bi*UB2 + pj
                    const int j = bi * UB2 + pj;
                    const bool run = j <= jb0;   // top block: rows > jb0 were done above
                    const double *slot = gring + (j % NS2) * SD2;
                    const double *lc = slot + (d2 ^ ((j & 1) & dstep));  // lc[i-1] = L(j+i, j)
                    double temp = 0.0;
#pragma unroll
                    for (int i = 1; i <= KL; ++i) temp = __fma_rn(v[pj + i], lc[i - 1], temp);
                    const double xj = run ? __dsub_rn(rin[pj], temp) : v[pj];
                    const int d = run ? reinterpret_cast<const int *>(slot + C::SP2)[0] - 1 - j : 0;
                    double y = xj;  // interchange x(j) <-> x(j+d)
#pragma unroll
                    for (int i = 1; i <= KL; ++i) {
                        const bool p = (d == i);
                        const double vi = v[pj + i];
                        v[pj + i] = p ? xj : vi;
                        y = p ? vi : y;
                    }
                    v[pj] = y;
                    if (act && run) bcol[j + KL] = v[pj + KL];  // final: later swaps reach at most j-1+KL
                }
                __syncwarp();
                issue_blk(bi - NB2);
                if (bi > 0) {
#pragma unroll
                    for (int p = XS - 1; p >= UB2; --p) v[p] = v[p - UB2];
                }
            }
            cp_async_wait<0>();
            if (act) {
#pragma unroll
                for (int p = 0; p < KL; ++p) bcol[p] = v[p];  // rows 0..KL-1 (n >= KL+1 here)
            }
        }
    }
}

}  // namespace bandlu
