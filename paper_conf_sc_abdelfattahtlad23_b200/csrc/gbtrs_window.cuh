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
//    copies.  (One bulk/TMA copy per matrix-column was tried: its uniform
//    operands serialize 32 per-lane copies per step.)
//  * Right-hand sides move in 16-byte PAIRS of rows: a per-lane ring of row
//    pairs, each pair one 16-byte cp.async issued AHEAD pairs before use, and
//    results stored as 16-byte pairs (per-lane phase: pair = rows 2P-ph,
//    2P-ph+1 with ph = (address of the column / 8) & 1, so every pair is
//    16-byte aligned).  A per-lane 8-byte copy or store per row was the
//    kernel's largest shared-memory / L1 cost at nrhs = 16 (one wavefront per
//    lane).  The pivot index is copied once per matrix (group leader) and read
//    back as a broadcast.
#pragma once
#include "common.cuh"

#ifndef __CUDACC_RTC__
#include <type_traits>
#endif

#ifndef BANDLU_TRS_NS_NARROW
#define BANDLU_TRS_NS_NARROW 16
#endif

#ifndef BANDLU_TRS_NS_WIDE
#define BANDLU_TRS_NS_WIDE 4
#endif

namespace bandlu {

template <int KL_, int KU_>
struct TrsWin {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU;
    static constexpr int WF = KL + 1, WB = KV + 1;         // forward / backward window lengths
    // ring depth (column steps in flight): narrow bands need more steps to cover HBM latency
    static constexpr int NS = (WB <= 5) ? BANDLU_TRS_NS_NARROW : BANDLU_TRS_NS_WIDE;
    static constexpr int FMAX = (KL > WB ? KL : WB) + 2;   // factor doubles per slot (+16 B rounding)
    static constexpr int SP = (FMAX + 1) & ~1;             // even -> 16 B aligned slots
    // slot: [SP factor doubles][ipiv int, pad][R rhs doubles when rows move one per step]
    __host__ __device__ static constexpr int slot_dbl(int R, bool pairs) { return SP + 2 + (pairs ? 0 : (R + 1) & ~1); }
    static constexpr int AHEAD = (NS + 2) / 2;             // RHS pairs in flight (2*AHEAD-1 >= NS steps)
    static constexpr int RPN = pow2_ceil(AHEAD + 1);       // RHS pair ring depth (power of 2)
    // group: [NS slots][RPN pairs x R lanes x 2 doubles]; pitch == 2 (mod 4) doubles so that the
    // groups' broadcast reads of the same slot offset sit in different banks
    __host__ __device__ static constexpr int group_dbl(int R, bool pairs) {
        return NS * slot_dbl(R, pairs) + (pairs ? RPN * R * 2 : 0) +
               (6 - (NS * slot_dbl(R, pairs) + (pairs ? RPN * R * 2 : 0)) % 4) % 4;
    }
    static constexpr int PAD = (KV + 3) & ~1;  // leading pad: backward reads up to KV doubles before a slot
    static size_t smem_bytes(int R, int gpw, bool pairs) { return (size_t)(PAD + gpw * group_dbl(R, pairs)) * 8; }
};

// PAIRS: RHS rows staged / stored as 16-byte row pairs (nrhs >= 2); otherwise one
// 8-byte row per step (nrhs == 1: one lane per matrix, measured faster there).
// experiments: BANDLU_TRS_MAXREG (register cap) or BANDLU_TRS_MINB (resident CTAs); the default
// bound lets ptxas pick (C4: 128 registers; (32, 1) picked more and ran 2.83 vs 2.16 ms)
#if defined(BANDLU_TRS_MAXREG)
#define BANDLU_TRS_BOUNDS __maxnreg__(BANDLU_TRS_MAXREG)
#elif defined(BANDLU_TRS_MINB)
#define BANDLU_TRS_BOUNDS __launch_bounds__(32, BANDLU_TRS_MINB)
#else
#define BANDLU_TRS_BOUNDS __launch_bounds__(32)
#endif
template <int KL, int KU, bool PAIRS, class AP, class PP, class BP>
__global__ void BANDLU_TRS_BOUNDS
    gbtrs_window_kernel(int n, int nrhs, AP A, int ldab, PP P, BP B, int ldb, const int *__restrict__ skip_info,
                        int batch, int R /* pow2 lanes per matrix */, int chunks /* rhs chunks per matrix */,
                        int gpw /* matrices (groups) per warp, <= 32 / R */,
                        int fwd /* 0: forward substitution already applied (fused gbtrf) */) {
    using C = TrsWin<KL, KU>;
    constexpr int KV = C::KV, WF = C::WF, WB = C::WB, NS = C::NS, AHEAD = C::AHEAD, RPN = C::RPN;
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

    const int GD = C::group_dbl(R, PAIRS), SD = C::slot_dbl(R, PAIRS);
    double *gring = smem + C::PAD + (g < gpw ? g : 0) * GD;
    const uint32_t gring_s = smem_u32(gring);

    const double *ab = live ? A.get(mat) : nullptr;
    const int *ipiv = live ? P.get(mat) : nullptr;
    double *bcol = act ? B.get(mat) + (int64_t)(r0 + t) * ldb : nullptr;  // this lane's RHS column
    const void *dummy = g_dummy;
    auto slot_piv_s = [&](int rs) { return gring_s + (uint32_t)((rs * SD + C::SP) * 8); };

    // ---- RHS row pairs: pair P = rows 2P-ph, 2P-ph+1 (16-byte aligned in this lane's column)
    const int ph = act ? (int)((reinterpret_cast<uintptr_t>(bcol) >> 3) & 1) : 0;
    const uint32_t pring_s = gring_s + (uint32_t)(NS * SD * 8) + (uint32_t)(t * 16);
    auto pair_of = [&](int q) { return (q + ph) >> 1; };
    auto pair_s = [&](int P) { return pring_s + (uint32_t)((P & (RPN - 1)) * R * 16); };
    auto issue_pair = [&](int P) {  // no commit: rides in the current step's group
        if (g >= gpw) return;
        const int q0 = 2 * P - ph;  // rows q0, q0+1
        const uint32_t d = pair_s(P);
        if (act && q0 >= 0 && q0 + 1 < n) {
            cp_async16(d, bcol + q0, 16u);
        } else if (act && q0 >= 0 && q0 < n) {  // last row: its 8 bytes, zero-fill the rest
            cp_async16(d, bcol + q0, 8u);
        } else if (act && q0 == -1 && n > 0) {  // first pair with ph = 1: (zero, row 0)
            st_shared_f64_if(true, d, 0.0);
            cp_async8(d + 8, bcol, 8u);
        } else {
            cp_async16(d, dummy, 0u);
        }
    };
    auto read_row = [&](int q) { return ld_shared_f64(pair_s(pair_of(q)) + (uint32_t)(((q + ph) & 1) * 8)); };
    // one row per step (!PAIRS): row q -> this lane's entry of step slot rs
    auto slot_rhs_s = [&](int rs) { return gring_s + (uint32_t)((rs * SD + C::SP + 2 + t) * 8); };
    auto issue_row = [&](int rs, int q) {
        if (g >= gpw) return;
        const bool ok = act && q >= 0 && q < n;
        cp_async8(slot_rhs_s(rs), ok ? (const void *)(bcol + q) : dummy, ok ? 8u : 0u);
    };

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
    const int *cipiv = clive ? P.get(cunit / chunks) : nullptr;
    const uint32_t cring_s = smem_u32(smem + C::PAD + cg * GD);
    auto issue_fac = [&](int k) {
        if (k >= nf + n || !clive) return;
        int64_t lo;
        int cnt;
        fac_range(k, lo, cnt);
        if (k < nf && cq == 0 && k < n - 1)  // pivot of forward step k, once per matrix
            cp_async4(cring_s + (uint32_t)(((k % NS) * SD + C::SP) * 8), cipiv + k, 4u);
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

    // ------------------------------------------------------------ forward
    // one cp.async group per step: its factor chunks (+ pivot) and, at the start of
    // each RHS pair, the pair AHEAD pairs later
    if (KL > 0 && nf > 0) {
        const int q0 = KL + 1;  // first RHS row staged (rows 0..KL are read directly)
        if constexpr (PAIRS)
            for (int P = pair_of(q0); P <= pair_of(q0) + AHEAD; ++P) issue_pair(P);
#pragma unroll 1
        for (int k = 0; k < NS; ++k) {
            issue_fac(k);
            if constexpr (!PAIRS) issue_row(k, k + KL + 1);
            cp_async_commit();
        }
        double w[WF];
#pragma unroll
        for (int i = 0; i < WF; ++i) w[i] = (act && i < n) ? bcol[i] : 0.0;
        double ypend = 0.0;  // first row of the current output pair
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
                // result y_j: rows (j-1, j) leave as one 16-byte store
                if (!PAIRS) {
                    if (act) bcol[j] = y;
                } else if (act) {
                    if (((j + ph) & 1) == 0) {
                        if (j == n - 1) bcol[j] = y;
                        ypend = y;
                    } else if (j == 0) {
                        bcol[0] = y;
                    } else {
                        *reinterpret_cast<double2 *>(bcol + j - 1) = make_double2(ypend, y);
                    }
                }
                if (y != 0.0) {
#pragma unroll
                    for (int i = 1; i < WF; ++i) w[(s + i) % WF] = __fma_rn(lc[i - 1], -y, w[(s + i) % WF]);
                }
                const int q = j + KL + 1;  // RHS row entering the window
                if constexpr (PAIRS)
                    w[s] = read_row(q);  // (0 beyond n)
                else
                    w[s] = ld_shared_f64(slot_rhs_s(rs));
                __syncwarp();
                if constexpr (PAIRS) {
                    if (((q + ph) & 1) == 0 && q != q0) issue_pair(pair_of(q) + AHEAD);
                } else if (j + NS < n) {
                    issue_row((j + NS) % NS, j + NS + KL + 1);
                }
                issue_fac(j + NS);
                cp_async_commit();
            }
        }
    }
    cp_async_wait<0>();
    __threadfence_block();
    __syncwarp();

    // ------------------------------------------------------------ backward
    const int qb0 = n - 1 - WB;  // first RHS row staged (rows n-1 .. n-WB are read directly)
    if constexpr (PAIRS)
        for (int P = pair_of(qb0); P >= pair_of(qb0) - AHEAD; --P) issue_pair(P);
#pragma unroll 1
    for (int kk = 0; kk < NS; ++kk) {
        issue_fac(nf + kk);
        if constexpr (!PAIRS) issue_row((nf + kk) % NS, qb0 - kk);
        cp_async_commit();
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
    double xpend = 0.0;  // upper row of the current output pair
#pragma unroll 1
    for (int kk0 = 0; kk0 < n; kk0 += UB) {
#pragma unroll
        for (int s = 0; s < UB; ++s) {
            const int kk = kk0 + s;
            if (kk >= n) break;
            const int k = nf + kk, j = n - 1 - kk;
            cp_async_wait<NS - 1>();
            __syncwarp();
            const double *uc = fac_ptr(k) - max(0, KV - j);  // uc[r] = AB(r, j), r >= KV - j valid
            // U column as 16-byte pairs when its smem parity is the same on every lane (strided
            // batches with an even stride): half the load instructions
            const uint32_t ua = smem_u32(uc);
            const bool pe = __all_sync(0xffffffffu, ((ua >> 3) & 1u) == 0u);
            const bool po = !pe && __all_sync(0xffffffffu, ((ua >> 3) & 1u) == 1u);
            double xj = x[s];
            if (xj != 0.0) {
                xj = __ddiv_rn(xj, uc[KV]);
                // rows j-i < 0 (last KV steps) read the pad / neighbouring slot: they only
                // feed window slots of rows < 0, which are never stored (dead slots)
                auto pairs = [&](auto par) {  // element e = KV - i; pair (e0, e0+1) 16-byte aligned
#pragma unroll
                    for (int e0 = -decltype(par)::value; e0 < KV; e0 += 2) {
                        const double2 u2 = ld_shared_v2(ua + (uint32_t)(e0 * 8));
                        if (e0 >= 0) x[s + KV - e0] = __fma_rn(-xj, u2.x, x[s + KV - e0]);
                        if (e0 + 1 < KV) x[s + KV - e0 - 1] = __fma_rn(-xj, u2.y, x[s + KV - e0 - 1]);
                    }
                };
                if (pe) {
                    pairs(std::integral_constant<int, 0>{});
                } else if (po) {
                    pairs(std::integral_constant<int, 1>{});
                } else {
#pragma unroll
                    for (int i = 1; i < WB; ++i) x[s + i] = __fma_rn(-xj, uc[KV - i], x[s + i]);
                }
            }
            // result x_j: rows (j, j+1) leave as one 16-byte store
            if (!PAIRS) {
                if (act) bcol[j] = xj;
            } else if (act) {
                if (((j + ph) & 1) == 1) {
                    if (j == 0) bcol[0] = xj;
                    xpend = xj;
                } else if (j == n - 1) {
                    bcol[j] = xj;
                } else {
                    *reinterpret_cast<double2 *>(bcol + j) = make_double2(xj, xpend);
                }
            }
            const int q = j - WB;           // RHS row entering the window
            if constexpr (PAIRS)
                x[s + WB] = (q >= 0) ? read_row(q) : 0.0;
            else
                x[s + WB] = ld_shared_f64(slot_rhs_s(k % NS));  // (0 if q < 0)
            __syncwarp();
            if constexpr (PAIRS) {
                if (((q + ph) & 1) == 1 && q != qb0) issue_pair(pair_of(q) - AHEAD);
            } else if (kk + NS < n) {
                issue_row((k + NS) % NS, q - NS);
            }
            issue_fac(k + NS);
            cp_async_commit();
        }
#pragma unroll
        for (int i = 0; i < XS; ++i) x[i] = (i + UB < XS) ? x[i + UB] : 0.0;
    }
    cp_async_wait<0>();
}

}  // namespace bandlu
