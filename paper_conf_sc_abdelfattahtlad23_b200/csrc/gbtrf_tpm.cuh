// gbtrf_tpm.cuh -- sm_100a band LU with partial pivoting, one THREAD per
// matrix: the matrix's active window lives in shared memory, panels of NB = 4
// columns are factored in registers, and the trailing rank-4 update touches
// every window element once per panel instead of once per column.
//
// What it computes: LAPACK DGBTF2 exactly (Sec. 5.1 pseudo-code
// P:350-367, ju rule P:492-494, right-only swaps P:358/P:369-374), the same
// fp64 operation sequence as the oracle => bitwise-equal factors, ipiv, info:
// every element receives its rank-1 FMAs in increasing column order --
// blocking changes when an FMA is issued, never its operands or its order.
// FWD: the forward substitution of DGBTRS('N') for one right-hand side rides
// along (the paper's augmented [A|B], Sec. 7).
//
// Why: the row-owner register kernels (gbtrf_rows.cuh)
// broadcast every pivot row through shared memory -- ~32 wavefronts and ~90
// warp instructions per matrix-column step at C3, latency-bound at 12 warps
// per SM.  Here a thread owns a matrix, so there is no broadcast, no
// cross-lane reduction (the pivot search is a sequential first-max scan,
// exactly IDAMAX's), and one warp instruction serves MPW matrices.  Shared
// memory holds the rows of the panel (KL+NB slots of WC = KV+NB columns,
// circular in the column index, lane-interleaved so that any per-lane slot
// choice is conflict-free); row interchanges relabel slots.
//
// Per panel (steps j0 .. j0+NB-1):
//  1. the NB rows entering the panel (labels j0+KL ..) take the slots of the
//     previous panel's pivot rows: their panel columns come from registers
//     prefetched one panel ahead, their trailing columns were copied by
//     cp.async at the end of the previous panel;
//  2. the panel columns of every slot are loaded to registers and factored:
//     per step IAMAX (first max, ties -> smallest logical row), relabel,
//     multipliers x * RN(1/p), rank-1 update of the remaining panel columns,
//     U row / L column / y stored straight from registers;
//  3. per trailing column pair: the NB U rows are finished in registers (the
//     pivot rows still owe the updates of the panel's earlier steps, applied
//     in step order) and stored, and every slot gets its NB FMAs in step order
//     (one shared-memory read and write per element per panel; the pivot
//     slots' multipliers are zeroed first, and their stale trailing values are
//     overwritten by the next panel's rows anyway).
#pragma once
#include "common.cuh"

namespace bandlu {

template <int KL_, int KU_, int MPW_>
struct TrfTpm {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU, MPW = MPW_;
    static constexpr int NB = 4;                   // panel width
    static constexpr int S = KL + NB;              // row slots (labels j0 .. j0+KL+NB-1)
    static constexpr int WC = (KV + NB + 1) & ~1;  // window columns (even: column pairs)
    static constexpr int WCP = WC / 2;             // column pairs, circular
    static constexpr int TP = (KV + 1) / 2;        // trailing pairs per panel
    static constexpr int NT = WC - NB;             // trailing columns copied per entering row
    static constexpr uint32_t PAIRB = MPW * 16, SLOTB = WCP * PAIRB;
    static_assert(WCP >= 2 + TP, "window");
    static_assert(MPW % 8 == 0 && MPW <= 32, "matrices per CTA: whole quarter-warps (bank groups)");
    // + a staging area: the panel columns of the NB rows entering the next panel;
    // + (FWD) the right-hand-side entry of every slot (the augmented column of [A|B])
    static constexpr uint32_t STGB = NB * 2 * PAIRB, BB = S * MPW * 8;
    static constexpr size_t cta_bytes() { return (size_t)S * SLOTB + STGB + BB; }
};

// One CTA = MPW threads (a partial warp for MPW < 32): every thread touches only
// its own lane-interleaved shared memory, so no warp synchronisation is needed.
template <int KL, int KU, int MPW, bool FWD, class AP, class PP, class BP>
__global__ void __launch_bounds__(MPW) gbtrf_tpm_kernel(int n, AP A, int ldab, PP P, int *__restrict__ info,
                                                     int batch, BP Bv) {
    using C = TrfTpm<KL, KU, MPW>;
    constexpr int KV = C::KV, NB = C::NB, S = C::S, WCP = C::WCP, TP = C::TP, NT = C::NT;
    constexpr uint32_t PAIRB = C::PAIRB, SLOTB = C::SLOTB;
    extern __shared__ __align__(16) double smem[];
    const int lane = (int)threadIdx.x;  // blockDim.x == MPW
    const int64_t mat = (int64_t)blockIdx.x * MPW + lane;
    const bool live = mat < batch;
    if (n <= 0) {
        if (live) info[mat] = 0;
        return;
    }
    double *__restrict__ ab = live ? A.get(mat) : g_dummy;
    int *__restrict__ ipiv = live ? P.get(mat) : nullptr;
    double *__restrict__ bv = (FWD && live) ? Bv.get(mat) : g_dummy;
    const int m = n;  // square (dgbtrfs / dgbsv); rectangular dgbtrf uses the row-slot kernel
    const int64_t ld1 = ldab - 1;  // band storage: A(q, c) at ab + KV + q + c * (ldab - 1)
    const uint32_t sbase = smem_u32(smem) + (uint32_t)lane * 16u;
    auto wrap = [](int p) { return p >= WCP ? p - WCP : p; };

    const uint32_t stg = sbase + S * SLOTB;                               // staging pairs
    const uint32_t bbase = smem_u32(smem) + S * SLOTB + C::STGB + lane * 8u;  // b of slot r: + r * MPW * 8
    // ---- prologue: rows 0 .. S-1 into slots 0 .. S-1, columns 0 .. WC-1 (zero outside the band)
    int lab[S];
#pragma unroll
    for (int r = 0; r < S; ++r) {
        lab[r] = r;
#pragma unroll
        for (int c = 0; c < C::WC; ++c) {
            const bool ok = live && r < m && c < n && c >= r - KL && c <= r + KU;
            cp_async8(sbase + r * SLOTB + (c >> 1) * PAIRB + (c & 1) * 8u, ok ? ab + KV + r + c * ld1 : g_dummy,
                      ok ? 8u : 0u);
        }
        if constexpr (FWD) {
            const bool okb = live && r < m;
            cp_async8(bbase + r * MPW * 8, okb ? bv + r : g_dummy, okb ? 8u : 0u);
        }
    }
    cp_async_commit();
    // panel columns of the rows entering the next panel (labels j1+KL+k), copied one
    // panel ahead into the staging area (pairs (k, 0..1) at stg + (2k + h) * PAIRB);
    // one cp.async group per call (possibly empty), so the group count stays uniform
    auto prefetch_next = [&](int j1) {
        const double *g = ab + KV + (j1 + KL) + j1 * ld1;  // A(j1+KL, j1)
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            const bool rowok = live && j1 + KL + k < m;
#pragma unroll
            for (int kk = 0; kk < NB; ++kk) {  // A(j1+KL+k, j1+kk): in the band iff kk >= k
                const bool ok = kk >= k && rowok && j1 + kk < n;
                if (j1 < n)
                    cp_async8(stg + (2 * k + (kk >> 1)) * PAIRB + (kk & 1) * 8u, ok ? g + k + kk * ld1 : g_dummy,
                              ok ? 8u : 0u);
            }
        }
        cp_async_commit();
    };
    prefetch_next(NB);
    uint32_t pslb[NB];  // shared address of the panel's pivot slots (label j0+k after the panel)
#pragma unroll
    for (int k = 0; k < NB; ++k) pslb[k] = sbase;
    int linfo = 0;

#pragma unroll 1
    for (int j0 = 0; j0 < n; j0 += NB) {
        const int pp0 = (j0 >> 1) % WCP;  // pair position of column j0
        const uint32_t po0 = pp0 * PAIRB, po1 = wrap(pp0 + 1) * PAIRB;
        cp_async_wait<1>();  // panel 0: the prologue rows; later: the entering rows' panel columns
        if (j0 > 0) {
            // ---- 1. entering rows: panel columns from the staging area; labels
#pragma unroll
            for (int k = 0; k < NB; ++k) {
                st_shared_v2_if(true, pslb[k] + po0, ld_shared_v2(stg + (2 * k) * PAIRB));
                st_shared_v2_if(true, pslb[k] + po1, ld_shared_v2(stg + (2 * k + 1) * PAIRB));
            }
#pragma unroll
            for (int r = 0; r < S; ++r) {
                const int d = lab[r] - (j0 - NB);  // 0..NB-1: the slot held the previous panel's pivot d
                if ((unsigned)d < (unsigned)NB) lab[r] += KL + NB;
            }
            prefetch_next(j0 + NB);
        }
        // ---- 2. panel columns of every slot -> registers, factored
        double pv[S][NB];
#pragma unroll
        for (int r = 0; r < S; ++r) {
            const double2 a = ld_shared_v2(sbase + r * SLOTB + po0), b = ld_shared_v2(sbase + r * SLOTB + po1);
            pv[r][0] = a.x;
            pv[r][1] = a.y;
            pv[r][2] = b.x;
            pv[r][3] = b.y;
        }
        int ipv[NB];
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            const int j = j0 + k;
            ipv[k] = 0;
            if (j >= n) break;
            // IAMAX over the candidates (logical rows j .. min(j+KL, m-1)): first max |x|,
            // ties to the smallest logical row
            int bs = 0, bl = 0x7fffffff;
            double bx = 0.0, bax = -1.0, bu[NB];
#pragma unroll
            for (int kk = 0; kk < NB; ++kk) bu[kk] = 0.0;
            bool cand[S];
#pragma unroll
            for (int r = 0; r < S; ++r) {
                const int L = lab[r];
                cand[r] = (unsigned)(L - j) <= (unsigned)KL && L < m;
                const double x = pv[r][k], ax = fabs(x);
                if (cand[r] && (ax > bax || (ax == bax && L < bl))) {
                    bs = r;
                    bl = L;
                    bx = x;
                    bax = ax;
#pragma unroll
                    for (int kk = k + 1; kk < NB; ++kk) bu[kk] = pv[r][kk];
                }
            }
            ipv[k] = bl + 1;
            const bool zp = (bx == 0.0);
            if (live && zp && linfo == 0) linfo = j + 1;
            // interchange = relabel: the pivot slot becomes logical row j, the slot that
            // held row j takes the pivot's old label
            pslb[k] = sbase + bs * SLOTB;
#pragma unroll
            for (int r = 0; r < S; ++r) lab[r] = (r == bs) ? j : ((lab[r] == j) ? bl : lab[r]);
            // SCAL (x * RN(1/p), Q7) -> L column j; rank-1 update of the remaining panel columns
            const double rinv = drcp_rn_nz(bx);
            double *colj = ab + KV + j * ld1;  // &AB(KV + i - j, j) = colj + i  (i = logical row)
#pragma unroll
            for (int r = 0; r < S; ++r) {
                const bool c = cand[r] && r != bs;
                const double x = pv[r][k];
                const double l = zp ? x : __dmul_rn(x, rinv);
                st_global_f64_if(live && c, colj + lab[r], l);
                const double lm = (c && !zp) ? l : 0.0;
                if (c) pv[r][k] = l;
#pragma unroll
                for (int kk = k + 1; kk < NB; ++kk) pv[r][kk] = __fma_rn(lm, -bu[kk], pv[r][kk]);
            }
            // U row j, panel part: U(j, j .. j0+NB-1)
            double *uj = ab + KV + j + j * ld1;  // &A(j, j); A(j, c) = uj + (c - j) * ld1
            st_global_f64_if(live, uj, bx);
#pragma unroll
            for (int kk = k + 1; kk < NB; ++kk) st_global_f64_if(live && j0 + kk < n, uj + (kk - k) * ld1, bu[kk]);
        }
        // ---- write back the panel columns: pivot slots keep their values (the
        // multipliers they had before they were chosen: read below), the other
        // slots get zeros -- these positions become the window's last columns next
        // panel, fill (structural zeros) for every row that stays.  Then the
        // pivot slots' multipliers are zeroed for the trailing update.
        const int jl = min(j0 + NB, n);  // steps done this panel: j0 .. jl-1
#pragma unroll
        for (int r = 0; r < S; ++r) {
            const bool piv = (unsigned)(lab[r] - j0) < (unsigned)(jl - j0);
            st_shared_v2_if(true, sbase + r * SLOTB + po0,
                            piv ? make_double2(pv[r][0], pv[r][1]) : make_double2(0.0, 0.0));
            st_shared_v2_if(true, sbase + r * SLOTB + po1,
                            piv ? make_double2(pv[r][2], pv[r][3]) : make_double2(0.0, 0.0));
#pragma unroll
            for (int k = 0; k < NB; ++k) pv[r][k] = piv ? 0.0 : pv[r][k];
        }
        // multipliers of the pivot rows from the panel's earlier steps: l(p_k, k')
        double lp[NB][NB];
#pragma unroll
        for (int k = 0; k < NB; ++k)
#pragma unroll
            for (int kk = 0; kk < NB; ++kk) lp[k][kk] = 0.0;
#pragma unroll
        for (int k = 1; k < NB; ++k) {
            if (j0 + k >= n) break;
#pragma unroll
            for (int kk = 0; kk < k; ++kk) lp[k][kk] = ld_shared_f64(pslb[k] + (kk < 2 ? po0 : po1) + (kk & 1) * 8u);
        }
        cp_async_wait<1>();  // the rows entering this panel: trailing columns (and b) landed
        if constexpr (FWD) {
            // ---- forward substitution of the panel (DGBTRS 'N' forward loop on the augmented
            // column): y_k = b of pivot row k after the panel's earlier steps, then every
            // other row's b gets its NB updates in step order (DGER skips y_k == 0)
            double y[NB];
#pragma unroll
            for (int k = 0; k < NB; ++k) {
                y[k] = 0.0;
                if (j0 + k < n) {
                    y[k] = ld_shared_f64(bbase + ((pslb[k] - sbase) / SLOTB) * (MPW * 8));
#pragma unroll
                    for (int kk = 0; kk < k; ++kk)
                        if (y[kk] != 0.0) y[k] = __fma_rn(lp[k][kk], -y[kk], y[k]);
                    st_global_f64_if(live, bv + j0 + k, y[k]);
                }
            }
#pragma unroll
            for (int r = 0; r < S; ++r) {
                double b = ld_shared_f64(bbase + r * MPW * 8);
#pragma unroll
                for (int k = 0; k < NB; ++k)
                    if (y[k] != 0.0) b = __fma_rn(pv[r][k], -y[k], b);
                st_shared_f64_if(true, bbase + r * MPW * 8, b);
            }
        }
        // ---- 3. trailing columns, pair by pair
        double *ucol = ab + KV + j0 + (j0 + NB) * ld1;  // &A(j0, j0+NB); A(j0+k, c) = ucol + k + (c-j0-NB)*ld1
#pragma unroll 1
        for (int i = 0; i < TP; ++i) {
            const uint32_t po = wrap(pp0 + 2 + i) * PAIRB;
            const int c0 = j0 + NB + 2 * i;  // columns c0, c0+1
            double2 u[NB];
#pragma unroll
            for (int k = 0; k < NB; ++k) u[k] = ld_shared_v2(pslb[k] + po);
            // finish the U rows: pivot row k still owes the updates of steps 0 .. k-1
#pragma unroll
            for (int k = 1; k < NB; ++k) {
#pragma unroll
                for (int kk = 0; kk < k; ++kk) {
                    u[k].x = __fma_rn(lp[k][kk], -u[kk].x, u[k].x);
                    u[k].y = __fma_rn(lp[k][kk], -u[kk].y, u[k].y);
                }
            }
            // U rows j0+k, columns c0, c0+1 (U bandwidth kv: c - (j0+k) <= KV)
#pragma unroll
            for (int k = 0; k < NB; ++k) {
                const bool rk = live && j0 + k < n;
                st_global_f64_if(rk && c0 < n && NB + 2 * i <= k + KV, ucol + k, u[k].x);
                st_global_f64_if(rk && c0 + 1 < n && NB + 2 * i + 1 <= k + KV, ucol + k + ld1, u[k].y);
            }
            ucol += 2 * ld1;
            // every slot: NB FMAs per element in step order
#pragma unroll
            for (int r = 0; r < S; ++r) {
                const uint32_t a_s = sbase + r * SLOTB + po;
                double2 a = ld_shared_v2(a_s);
#pragma unroll
                for (int k = 0; k < NB; ++k) {
                    a.x = __fma_rn(pv[r][k], -u[k].x, a.x);
                    a.y = __fma_rn(pv[r][k], -u[k].y, a.y);
                }
                st_shared_v2_if(true, a_s, a);
            }
        }
        // ---- 4. ipiv; the rows entering the next panel: trailing columns into this
        // panel's pivot slots (cp.async, zero outside the band)
        if (live) {
#pragma unroll
            for (int k = 0; k < NB; ++k)
                if (j0 + k < n) ipiv[j0 + k] = ipv[k];
        }
        if (j0 + NB < n) {
            const int j1 = j0 + NB;
            const int pp1 = wrap(pp0 + 2);
            // A(j1+KL+k, j1+NB+i) at g + k + i*ld1; in the band iff i <= KV - NB + k
            const double *g = ab + KV + (j1 + KL) + (j1 + NB) * ld1;
#pragma unroll
            for (int i = 0; i < NT; ++i) {
                const uint32_t dofs = wrap(pp1 + 2 + (i >> 1)) * PAIRB + (i & 1) * 8u;
                const bool colok = live && j1 + NB + i < n;
#pragma unroll
                for (int k = 0; k < NB; ++k) {
                    const bool ok = colok && i <= KV - NB + k && j1 + KL + k < m;
                    cp_async8(pslb[k] + dofs, ok ? g + k + i * ld1 : g_dummy, ok ? 8u : 0u);
                }
            }
            if constexpr (FWD) {
#pragma unroll
                for (int k = 0; k < NB; ++k) {
                    const bool okb = live && j1 + KL + k < m;
                    cp_async8(bbase + ((pslb[k] - sbase) / SLOTB) * (MPW * 8), okb ? bv + j1 + KL + k : g_dummy,
                              okb ? 8u : 0u);
                }
            }
        }
        cp_async_commit();
    }
    cp_async_wait<0>();
    if (live) info[mat] = linfo;
}

}  // namespace bandlu
