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
//    so the whole serial chain runs in registers; the row interchange is a
//    predicated select over the window slots.
//  * Both passes run in ONE kernel.  For every column step the lanes of a
//    group copy exactly the part of the factor column that pass needs -- L
//    rows forward, U rows backward, rounded out to 16 B -- with 16-byte
//    cp.async chunks into an NS-deep per-group smem ring (so each factor
//    entry is read from HBM once); RHS entries and pivots ride along as
//    8/4-byte cp.async.  (One bulk/TMA copy per matrix-column was tried: its
//    uniform operands serialize 32 per-lane copies per step.)
#pragma once
#include "common.cuh"

namespace bandlu {

template <int KL_, int KU_>
struct TrsWin {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU;
    static constexpr int WF = KL + 1, WB = KV + 1;         // forward / backward window lengths
    static constexpr int NS = 8;                           // ring depth (column steps in flight)
    static constexpr int FMAX = (KL > WB ? KL : WB) + 2;   // factor doubles per slot (+16 B rounding)
    static constexpr int SP = (FMAX + 1) & ~1;             // even -> 16 B aligned slots
    // slot: [SP factor doubles][R rhs doubles][R ipiv ints], padded to an even number of doubles
    __host__ __device__ static constexpr int slot_dbl(int R) {
        return ((SP + R + (R + 1) / 2) + 1) & ~1;
    }
    // group pitch == 2 (mod 4) doubles: lanes of different groups reading the same
    // slot offset hit different banks (<= 2-way for 64-bit); keeps 16 B alignment
    __host__ __device__ static constexpr int group_dbl(int R) { return NS * slot_dbl(R) + (6 - (NS * slot_dbl(R)) % 4) % 4; }
    static constexpr int PAD = (KV + 3) & ~1;  // leading pad: backward reads up to KV doubles before a slot
    static size_t smem_bytes(int R, int gpw) { return (size_t)(PAD + gpw * group_dbl(R)) * 8; }
};

template <int KL, int KU, class AP, class PP, class BP>
__global__ void __launch_bounds__(32)
    gbtrs_window_kernel(int n, int nrhs, AP A, int ldab, PP P, BP B, int ldb, const int *__restrict__ skip_info,
                        int batch, int R /* pow2 lanes per matrix */, int chunks /* rhs chunks per matrix */,
                        int gpw /* matrices (groups) per warp, <= 32 / R */,
                        int fwd /* 0: forward substitution already applied (fused gbtrf) */) {
    using C = TrsWin<KL, KU>;
    constexpr int KV = C::KV, WF = C::WF, WB = C::WB, NS = C::NS, SP = C::SP;
    extern __shared__ __align__(16) double smem[];
    const int lane = (int)lane_id();
    const int g = lane / R, t = lane % R;
    const int64_t unit = (int64_t)blockIdx.x * gpw + g;  // (matrix, rhs chunk)
    const int64_t mat = unit / chunks;
    const int r0 = (int)(unit % chunks) * 32;
    bool live = g < gpw && unit < (int64_t)batch * chunks;
    if (live && skip_info != nullptr && skip_info[mat] != 0) live = false;
    const bool act = live && (r0 + t < nrhs);  // lane solves (and stores) a column
    if (__ballot_sync(0xffffffffu, live) == 0u) return;
    // Dead groups stay (warp-wide barriers); they copy nothing and store nothing.
    const bool leader = (t == 0);

    const int SD = C::slot_dbl(R), GD = C::group_dbl(R);
    double *gring = smem + C::PAD + (g < gpw ? g : 0) * GD;
    const uint32_t gring_s = smem_u32(gring);

    const double *ab = live ? A.get(mat) : nullptr;
    const int *ipiv = live ? P.get(mat) : nullptr;
    double *bcol = act ? B.get(mat) + (int64_t)(r0 + t) * ldb : nullptr;  // this lane's RHS column
    const void *dummy = g_dummy;
    auto slot_rhs_s = [&](int rs) { return gring_s + (uint32_t)((rs * SD + SP + t) * 8); };
    auto slot_piv_s = [&](int rs) { return gring_s + (uint32_t)((rs * SD + SP + R) * 8 + t * 4); };

    // Global step k: forward steps k < nf (column k), then backward steps
    // k = nf + kk, kk = 0..n-1 (column n-1-kk).  The factor range of a step:
    const int nf = (KL > 0 && fwd) ? n : 0;
    auto fac_range = [&](int k, int64_t &lo, int &cnt) {
        if (k < nf) {  // L rows KV+1 .. KV+lm of column k
            const int lm = min(KL, n - 1 - k);
            lo = (int64_t)k * ldab + KV + 1;
            cnt = lm > 0 ? lm : 0;
        } else {  // U rows max(0, KV-j) .. KV of column j
            const int j = n - 1 - (k - nf);
            const int r = max(0, KV - j);
            lo = (int64_t)j * ldab + r;
            cnt = KV + 1 - r;
        }
    };
    // 16-byte chunks of the factor range (rounded out).  The copy is split over
    // CPG = 32/gpw "copy lanes" per group (lane -> group lane/CPG, fixed), so a
    // warp issues ~nch/CPG chunk copies per lane per step whatever R is.
    const int CPG = 32 / gpw;
    const int cg = lane / CPG, cq = lane % CPG;  // copy group / copy lane within it
    const int64_t cunit = (int64_t)blockIdx.x * gpw + cg;
    const bool clive = cunit < (int64_t)batch * chunks &&
                       !(skip_info != nullptr && skip_info[cunit / chunks] != 0);
    const double *cab = clive ? A.get(cunit / chunks) : nullptr;
    const uint32_t cring_s = smem_u32(smem + C::PAD + cg * GD);
    auto issue_fac = [&](int k) {
        if (k >= nf + n || !clive) return;
        int64_t lo;
        int cnt;
        fac_range(k, lo, cnt);
        if (cnt <= 0) return;
        const uintptr_t a = reinterpret_cast<uintptr_t>(cab + lo);
        const uintptr_t a0 = a & ~(uintptr_t)15, a1 = (a + (uintptr_t)cnt * 8 + 15) & ~(uintptr_t)15;
        const int nch = (int)((a1 - a0) >> 4);
        const uint32_t dst = cring_s + (uint32_t)((k % NS) * SD * 8);
        for (int q = cq; q < nch; q += CPG) cp_async16(dst + q * 16, reinterpret_cast<const void *>(a0 + q * 16), 16u);
    };
    // first needed factor element of step k, inside its slot
    auto fac_ptr = [&](int k) -> const double * {
        int64_t lo;
        int cnt;
        fac_range(k, lo, cnt);
        const int delta = live ? (int)((reinterpret_cast<uintptr_t>(ab + lo) >> 3) & 1) : 0;
        return gring + (k % NS) * SD + delta;
    };
    const bool inwarp = g < gpw;  // lanes past the warp's groups own no ring: never copy
    auto issue_vec_fwd = [&](int k) {  // RHS row k+KL+1 and ipiv[k] for forward step k
        const int rs = k % NS;
        if (!inwarp) return;
        const int row = k + KL + 1;
        const bool okb = act && row < n;
        cp_async8(slot_rhs_s(rs), okb ? (const void *)(bcol + row) : dummy, okb ? 8u : 0u);
        const bool okp = live && k < n;
        cp_async4(slot_piv_s(rs), okp ? (const void *)(ipiv + k) : dummy, okp ? 4u : 0u);
        cp_async_commit();
    };
    auto issue_vec_bwd = [&](int kk) {  // backward step kk (row j = n-1-kk): RHS row j-KV-1
        const int rs = (nf + kk) % NS;
        if (!inwarp) return;
        const int row = n - 1 - kk - KV - 1;
        const bool okb = act && row >= 0 && kk < n;
        cp_async8(slot_rhs_s(rs), okb ? (const void *)(bcol + row) : dummy, okb ? 8u : 0u);
        cp_async_commit();
    };

    // ------------------------------------------------------------ forward
    // one cp.async group per step: its factor chunks + its RHS entry / pivot
    if (KL > 0 && nf > 0) {
#pragma unroll 1
        for (int k = 0; k < NS; ++k) {
            issue_fac(k);
            issue_vec_fwd(k);
        }
        double w[WF];
#pragma unroll
        for (int i = 0; i < WF; ++i) w[i] = (act && i < n) ? bcol[i] : 0.0;
#pragma unroll 1
        for (int j0 = 0; j0 < n; j0 += WF) {
#pragma unroll
            for (int s = 0; s < WF; ++s) {
                const int j = j0 + s;
                if (j >= n) break;
                const int rs = j % NS;
                cp_async_wait<NS - 1>();
                __syncwarp();  // chunks copied by the group's other lanes
                const double *lc = fac_ptr(j);  // lc[i-1] = L(j+i, j); rows >= n: dead slots
                // interchange B(j) <-> B(l), l in [j, j+KL] (LAPACK never reads ipiv[n-1])
                const int d = (j < n - 1) ? ld_shared_s32(slot_piv_s(rs)) - 1 - j : 0;
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
#pragma unroll
                    for (int i = 1; i < WF; ++i) w[(s + i) % WF] = __fma_rn(lc[i - 1], -y, w[(s + i) % WF]);
                }
                w[s] = ld_shared_f64(slot_rhs_s(rs));  // RHS row j+KL+1 (0 beyond n)
                __syncwarp();
                if (j + NS < n) {
                    issue_fac(j + NS);
                    issue_vec_fwd(j + NS);
                } else {
                    cp_async_commit();
                }
            }
        }
    }
    cp_async_wait<0>();
    __threadfence_block();
    __syncwarp();

    // ------------------------------------------------------------ backward
#pragma unroll 1
    for (int kk = 0; kk < NS; ++kk) {
        issue_fac(nf + kk);
        issue_vec_bwd(kk);
    }
    // Backward window: row j-i (i = 0..KV) of step kk = kk0+s sits in slot s+i;
    // the row entering at step kk (j-WB) goes to slot s+WB.  Blocks of UB steps
    // are unrolled and the window then shifts down by UB slots (keeps the
    // kernel small for wide bands; UB = WB for narrow ones = pure rotation).
    constexpr int UB = WB <= 12 ? WB : 4;
    constexpr int XS = WB + UB;
    double x[XS];
#pragma unroll
    for (int i = 0; i < XS; ++i) x[i] = (i < WB && act && n - 1 - i >= 0) ? bcol[n - 1 - i] : 0.0;
#pragma unroll 1
    for (int kk0 = 0; kk0 < n; kk0 += UB) {
#pragma unroll
        for (int s = 0; s < UB; ++s) {
            const int kk = kk0 + s;
            if (kk >= n) break;
            const int k = nf + kk, j = n - 1 - kk;
            const int rs = k % NS;
            cp_async_wait<NS - 1>();
            __syncwarp();
            const double *uc = fac_ptr(k) - max(0, KV - j);  // uc[r] = AB(r, j), r >= KV - j valid
            double xj = x[s];
            if (xj != 0.0) {
                xj = __ddiv_rn(xj, uc[KV]);
                // rows j-i < 0 (last KV steps) read the pad / neighbouring slot: they only
                // feed window slots of rows < 0, which are never stored (dead slots)
#pragma unroll
                for (int i = 1; i < WB; ++i) x[s + i] = __fma_rn(-xj, uc[KV - i], x[s + i]);
            }
            if (act) bcol[j] = xj;
            x[s + WB] = ld_shared_f64(slot_rhs_s(rs));  // y(j-KV-1) (0 if < 0)
            __syncwarp();
            issue_fac(k + NS);
            issue_vec_bwd(kk + NS);  // commits the step's group
        }
#pragma unroll
        for (int i = 0; i < XS; ++i) x[i] = (i + UB < XS) ? x[i + UB] : 0.0;
    }
    cp_async_wait<0>();
}

}  // namespace bandlu
