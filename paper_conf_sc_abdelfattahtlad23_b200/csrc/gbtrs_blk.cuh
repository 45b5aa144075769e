// gbtrs_blk.cuh -- sm_100a banded solve A X = B with dgbtrf factors
// (trans = 'N'), block-granular ring, compiled per (KL, KU).
//
// What it computes: LAPACK DGBTRS('N') exactly, in the oracle's order
// (oracle_dgbtrs_n; Sec. 6):
//   forward (kl > 0): for j = 0..n-2: swap b(j) <-> b(ipiv[j]-1) (pivots
//     applied progressively); if b(j) != 0: b(j+i) =
//     fma(L(j+i,j), -b(j), b(j+i)), i = 1..min(kl, n-1-j) (DGER);
//   backward (DTBSV 'U','N','N', bandwidth kv): for j = n-1..0:
//     if x(j) != 0: x(j) = x(j) / U(j,j) (true division); x(i) =
//     fma(-x(j), U(i,j), x(i)), i = j-1 .. max(0, j-kv).
//
// Same machinery as gbtrs_t.cuh (the transposed solve): one LANE per
// (matrix, RHS column), R = pow2 >= nrhs lanes per matrix; each pass keeps a
// sliding window of RHS rows in registers -- the current row, the K rows it
// updates (K = kl forward, kv backward) and the UB rows entering during the
// block -- and reads the factor column of each step from a smem ring filled
// by 16-byte cp.async chunks split over the matrix's copy lanes.  Steps run
// in blocks of UB with ONE cp.async group and one wait per block and no
// barrier inside it, so the scheduler overlaps the steps' loads and chains.
// Window rows outside the matrix (below row n-1 forward, above row 0
// backward) may pick up garbage from fill entries; they are never swapped in
// (pivots stay inside the matrix) and never stored.
#pragma once
#include "common.cuh"

#ifndef BANDLU_TRSB_STEPS_NARROW
#define BANDLU_TRSB_STEPS_NARROW 16  // column steps in flight, kl + ku + 1 <= 5
#endif
#ifndef BANDLU_TRSB_STEPS_WIDE
#define BANDLU_TRSB_STEPS_WIDE 8
#endif
#ifndef BANDLU_TRSB_UB
#define BANDLU_TRSB_UB 4  // steps per block when the window is longer than 8
#endif

namespace bandlu {

template <int KL_, int KU_>
struct TrsBlk {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU;
    static constexpr int STEPS = (KV + 1 <= 5) ? BANDLU_TRSB_STEPS_NARROW : BANDLU_TRSB_STEPS_WIDE;
    static constexpr int UBF = KL <= 8 ? (KL > 0 ? KL + 1 : 1) : BANDLU_TRSB_UB;  // forward steps per block
    static constexpr int UBB = KV <= 8 ? KV + 1 : BANDLU_TRSB_UB;                 // backward steps per block
    static constexpr int NBF = (STEPS + UBF - 1) / UBF < 2 ? 2 : (STEPS + UBF - 1) / UBF;
    static constexpr int NBB = (STEPS + UBB - 1) / UBB < 2 ? 2 : (STEPS + UBB - 1) / UBB;
    static constexpr int NSF = NBF * UBF, NSB = NBB * UBB;  // ring slots per pass
    // forward slot: [SPF: L rows kv+1..kv+kl, 16-byte rounded][ipiv, pad]; backward slot: [SPB: U rows
    // 0..kv].  RHS rows move per block: each lane copies the UB rows a block consumes as 16-byte
    // aligned pairs (UB + 2 doubles at most) into its area of the block's RHS buffer.
    static constexpr int SPF = ((KL + 2) + 1) & ~1;
    static constexpr int SPB = ((KV + 1 + 2) + 1) & ~1;
    static constexpr int SLF = SPF + 2, SLB = SPB;
    static constexpr int RBF = ((UBF + 2) + 1) & ~1, RBB = ((UBB + 2) + 1) & ~1;  // doubles per lane and block
    __host__ __device__ static constexpr int fwd_dbl(int R) { return NSF * SLF + NBF * RBF * R; }
    __host__ __device__ static constexpr int bwd_dbl(int R) { return NSB * SLB + NBB * RBB * R; }
    __host__ __device__ static constexpr int ring_dbl(int R) { return fwd_dbl(R) > bwd_dbl(R) ? fwd_dbl(R) : bwd_dbl(R); }
    // pitch == 2 (mod 4) doubles: the groups' reads of one slot offset sit in different banks
    __host__ __device__ static constexpr int group_dbl(int R) { return ring_dbl(R) + (6 - ring_dbl(R) % 4) % 4; }
    static constexpr int PAD = 2;
    static size_t smem_bytes(int R, int gpw) { return (size_t)(PAD + gpw * group_dbl(R)) * 8; }
};

#ifdef BANDLU_TRSB_MINB
#define BANDLU_TRSB_BOUNDS __launch_bounds__(32, BANDLU_TRSB_MINB)
#else
#define BANDLU_TRSB_BOUNDS __launch_bounds__(32)
#endif
template <int KL, int KU, class AP, class PP, class BP>
__global__ void BANDLU_TRSB_BOUNDS
    gbtrs_blk_kernel(int n, int nrhs, AP A, int ldab, PP P, BP B, int ldb, const int *__restrict__ skip_info,
                     int batch, int R /* pow2 lanes per matrix */, int chunks /* rhs chunks per matrix */,
                     int gpw /* matrices (groups) per warp, <= 32 / R */,
                     int fwd /* 0: forward substitution already applied (fused gbtrf) */) {
    using C = TrsBlk<KL, KU>;
    constexpr int KV = C::KV, UBF = C::UBF, UBB = C::UBB, NBF = C::NBF, NBB = C::NBB, NSF = C::NSF, NSB = C::NSB;
    extern __shared__ __align__(16) double smem[];
    const int lane = (int)lane_id();
    const int g = lane / R, t = lane % R;
    const int64_t unit = (int64_t)blockIdx.x * gpw + g;  // (matrix, rhs chunk)
    const int64_t mat = unit / chunks;
    const int r0 = (int)(unit % chunks) * 32;
    bool live = g < gpw && unit < (int64_t)batch * chunks;
    if (live && skip_info != nullptr && skip_info[mat] != 0) live = false;  // dgbsv: info > 0
    const bool act = live && (r0 + t < nrhs);  // lane solves (and stores) a column
    if (__ballot_sync(0xffffffffu, live) == 0u) return;

    const int GD = C::group_dbl(R);
    constexpr int SDF = C::SLF, SDB = C::SLB, RBF = C::RBF, RBB = C::RBB;
    double *gring = smem + C::PAD + (g < gpw ? g : 0) * GD;
    const double *ab = live ? A.get(mat) : nullptr;
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
    const int dstep = ldab & 1;  // the parity flips per column when ldab is odd

    // copy role: CPG lanes per group split the 16-byte chunks of a factor range
    const int CPG = 32 / gpw;
    const int cg = lane / CPG, cq = lane % CPG;
    const int64_t cunit = (int64_t)blockIdx.x * gpw + cg;
    const bool clive =
        cunit < (int64_t)batch * chunks && !(skip_info != nullptr && skip_info[cunit / chunks] != 0);
    const double *cab = clive ? A.get(cunit / chunks) : nullptr;
    const int *cipiv = clive ? P.get(cunit / chunks) : nullptr;
    const uint32_t cring_s = smem_u32(smem + C::PAD + cg * GD);
    auto issue_fac = [&](uint32_t dst, int64_t lo, int cnt) {
        const uintptr_t a = reinterpret_cast<uintptr_t>(cab + lo);
        const uintptr_t a0 = a & ~(uintptr_t)15, a1 = (a + (uintptr_t)cnt * 8 + 15) & ~(uintptr_t)15;
        const int nch = (int)((a1 - a0) >> 4);
        for (int q = cq; q < nch; q += CPG) cp_async16(dst + q * 16, reinterpret_cast<const void *>(a0 + q * 16), 16u);
    };

    // ============================================== forward: L y = P b
    if (KL > 0 && fwd) {
        // step j (slot j % NSF): L rows KV+1..KV+KL of column j, ipiv[j]; block b: entering rows
        // b*UBF+KL+1 .. +UBF-1 (RHS buffer b % NBF)
        const uint32_t rhs_f = gring_s + (uint32_t)((NSF * SDF + t * RBF) * 8);
        auto issue_blk = [&](int b) {
            if (b * UBF < n) {
#pragma unroll 1
                for (int s = 0; s < UBF; ++s) {
                    const int j = b * UBF + s;
                    if (j >= n) break;
                    const uint32_t dst = cring_s + (uint32_t)((j % NSF) * SDF * 8);
                    if (clive) {
                        if (cq == 0 && j < n - 1) cp_async4(dst + C::SPF * 8, cipiv + j, 4u);
                        issue_fac(dst, (int64_t)j * ldab + KV + 1, KL);
                    }
                }
                issue_rows(rhs_f + (uint32_t)((b % NBF) * R * RBF * 8), b * UBF + KL + 1, UBF);
            }
            cp_async_commit();
        };
#pragma unroll 1
        for (int b = 0; b < NBF; ++b) issue_blk(b);
        const int df = delta_of(KV + 1);
        constexpr int XS = KL + 1 + UBF;
        double v[XS];  // v[p] = b(j0 + p): row j0+s is step s's row, the KL below it, then the entering rows
#pragma unroll
        for (int p = 0; p < XS; ++p) v[p] = (p <= KL && act && p < n) ? bcol[p] : 0.0;
#pragma unroll 1
        for (int b = 0, j0 = 0; j0 < n; ++b, j0 += UBF) {
            cp_async_wait<NBF - 1>();
            __syncwarp();
            // this block's entering rows: row j0+KL+1+s at rin[s]
            const double *rin = gring + NSF * SDF + ((b % NBF) * R + t) * RBF + ((j0 + KL + 1 + ph) & 1);
#pragma unroll
            for (int s = 0; s < UBF; ++s) {
                const int j = j0 + s;
                const double *slot = gring + (j % NSF) * SDF;
                const double *lc = slot + (df ^ ((j & 1) & dstep));  // lc[i-1] = L(j+i, j)
                // interchange b(j) <-> b(j+d) (LAPACK never reads ipiv[n-1])
                const int d = (j < n - 1) ? reinterpret_cast<const int *>(slot + C::SPF)[0] - 1 - j : 0;
                double y = v[s];
#pragma unroll
                for (int i = 1; i <= KL; ++i) {
                    const bool p = (d == i);
                    const double vi = v[s + i];
                    v[s + i] = p ? v[s] : vi;
                    y = p ? vi : y;
                }
                if (act && j < n) bcol[j] = y;
                if (y != 0.0) {
#pragma unroll
                    for (int i = 1; i <= KL; ++i) v[s + i] = __fma_rn(lc[i - 1], -y, v[s + i]);
                }
                v[s + KL + 1] = rin[s];  // row j+KL+1 (0 beyond n-1)
            }
            __syncwarp();
            issue_blk(b + NBF);
#pragma unroll
            for (int p = 0; p < XS; ++p) v[p] = (p + UBF < XS) ? v[p + UBF] : 0.0;
        }
        cp_async_wait<0>();
        __threadfence_block();
        __syncwarp();
    }

    // ============================================== backward: U x = y
    {
        // step kk (slot kk % NSB): column j = n-1-kk, U rows 0..KV; block b: entering rows
        // n-2-KV-b*UBB down to n-1-KV-(b+1)*UBB (RHS buffer b % NBB)
        const uint32_t rhs_b = gring_s + (uint32_t)((NSB * SDB + t * RBB) * 8);
        auto issue_blk = [&](int b) {
            if (b * UBB < n) {
                if (clive) {
#pragma unroll 1
                    for (int s = 0; s < UBB; ++s) {
                        const int kk = b * UBB + s;
                        if (kk >= n) break;
                        // rows max(0, KV-j)..KV only (rows above 0 would feed dead window rows): the
                        // chunks go where the full column's would, so uc[] offsets do not change
                        const int j = n - 1 - kk, rlo = j < KV ? KV - j : 0;
                        const int d0 = (int)((reinterpret_cast<uintptr_t>(cab + (int64_t)j * ldab) >> 3) & 1);
                        issue_fac(cring_s + (uint32_t)(((kk % NSB) * SDB + ((d0 + rlo) & ~1)) * 8),
                                  (int64_t)j * ldab + rlo, KV + 1 - rlo);
                    }
                }
                issue_rows(rhs_b + (uint32_t)((b % NBB) * R * RBB * 8), n - 1 - KV - (b + 1) * UBB, UBB);
            }
            cp_async_commit();
        };
#pragma unroll 1
        for (int b = 0; b < NBB; ++b) issue_blk(b);
        const int db = delta_of((int64_t)(n - 1) * ldab);
        constexpr int XS = KV + 1 + UBB;
        double u[XS];  // u[p] = x(n-1-kk0-p): step s's row, the KV above it, then the entering rows
#pragma unroll
        for (int p = 0; p < XS; ++p) u[p] = (p <= KV && act && n - 1 - p >= 0) ? bcol[n - 1 - p] : 0.0;
#pragma unroll 1
        for (int b = 0, kk0 = 0; kk0 < n; ++b, kk0 += UBB) {
            cp_async_wait<NBB - 1>();
            __syncwarp();
            // this block's entering rows: row n-2-KV-kk0-s at rin[UBB-1-s]
            const int qlo = n - 1 - KV - kk0 - UBB;
            const double *rin = gring + NSB * SDB + ((b % NBB) * R + t) * RBB + ((qlo + ph) & 1);
#pragma unroll
            for (int s = 0; s < UBB; ++s) {
                const int kk = kk0 + s, j = n - 1 - kk;
                const double *slot = gring + (kk % NSB) * SDB;
                const double *uc = slot + (db ^ ((kk & 1) & dstep));  // uc[r] = AB(r, j) = U(j-KV+r, j)
                double xj = u[s];
                if (xj != 0.0) {
                    xj = __ddiv_rn(xj, uc[KV]);
#pragma unroll
                    for (int i = 1; i <= KV; ++i) u[s + i] = __fma_rn(-xj, uc[KV - i], u[s + i]);
                }
                if (act && j >= 0) bcol[j] = xj;
                u[s + KV + 1] = rin[UBB - 1 - s];  // row j-KV-1 (0 above row 0)
            }
            __syncwarp();
            issue_blk(b + NBB);
#pragma unroll
            for (int p = 0; p < XS; ++p) u[p] = (p + UBB < XS) ? u[p + UBB] : 0.0;
        }
        cp_async_wait<0>();
    }
}

}  // namespace bandlu
