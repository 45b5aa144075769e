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
//    active window -- the W = KL+KU+1 values at columns j..j+KV -- in
//    registers, column c in slot c mod W, slots paired into double2 so rows
//    move to/from shared memory with 128-bit accesses.  The column loop is
//    unrolled W times: sliding the window never moves a register.
//  * Row interchanges are relabelings: a lane carries the logical position of
//    its row.  LAPACK swaps only columns j..ju; beyond ju both rows hold
//    structural zeros, so swapping whole rows is identical.
//  * IAMAX: butterfly max of the high word of the |x| bit pattern + ballot;
//    exact slow path (low word, then smallest logical row) only when the
//    high words tie (zero pivots, exact ties) -- first-max semantics (Q2).
//  * The pivot row is broadcast to its group with width-G shuffles (the
//    shuffle path runs beside the shared-memory pipe, which the row staging
//    and the U store use); every lane then applies the rank-1 update with
//    FP64 FMAs in registers.  The pivot lane also drops its row (= U row j)
//    into a double-buffered smem record that the group stores to HBM one
//    step later.  Multipliers are stored by their owning lanes.
//  * Input rows are gathered one row per step by cp.async (LDGSTS,
//    L1-allocating, zero-fill outside the matrix) into a 16-row smem ring in
//    slot order, D = 8 rows ahead; the lane freed by the pivot row reloads
//    its registers from it with 128-bit loads.  Fill rows (input) are never
//    read; every input element is read from HBM once, every output element
//    written once.
#pragma once
#include "common.cuh"

// Tuning knobs (compile-time; overridable with -D for experiments)
#ifndef BANDLU_TRF_U
#define BANDLU_TRF_U 4
#endif
#ifndef BANDLU_TRF_MINB
#define BANDLU_TRF_MINB 3
#endif
#ifndef BANDLU_TRF_WARPS
#define BANDLU_TRF_WARPS 4
#endif
#ifndef BANDLU_TRF_D
#define BANDLU_TRF_D 8
#endif

namespace bandlu {

template <int KL_, int KU_>
struct TrfWin {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU, W = KV + 1;
    static constexpr int U = BANDLU_TRF_U;       // columns per unrolled block (window shift granularity)
    static constexpr int WS = W + U;             // register slots: column j0 + r in slot r during a block
    static constexpr int H = (WS + 1) / 2;       // double2 slot pairs
    static constexpr int WP = 2 * H + 2;         // record / ring-row pitch in doubles (16 B rows, +1 free slot)
    // lanes per matrix: pow2 >= KL+1; wide windows use >= 8 so that a warp's
    // smem rings (and so the resident warps per SM) stay within budget
    static constexpr int G = pow2_ceil(KL + 1) < (W > 24 ? 8 : 1) ? (W > 24 ? 8 : 1) : pow2_ceil(KL + 1);
    static constexpr int GPW = 32 / G;           // matrices per warp
    static constexpr int D = BANDLU_TRF_D;       // staging lead (rows)
    static constexpr int RR = 16;                // ring rows (power of 2, > D, multiple of U)
    static constexpr int GROUP_DBL = (RR + 2) * WP;  // ring + 2 pivot-row records (double buffered)
    static constexpr int SIT = (W + G - 1) / G;      // staged elements per lane per row
    static constexpr int WARPS = BANDLU_TRF_WARPS;
    // register budget: >= MINB CTAs per SM while the window fits
    static constexpr int MINB = W <= 24 ? BANDLU_TRF_MINB : 2;
    static constexpr size_t smem_bytes() { return (size_t)WARPS * GPW * GROUP_DBL * sizeof(double); }
};

// FWD: also apply the forward substitution of DGBTRS('N') to one right-hand
// side on the fly (Sec. 7: factorization of the augmented
// [A|B] "implicitly performs the forward triangular solve"): each lane carries
// its row's B entry, which moves with the row interchanges and receives the
// same rank-1 update (B(j+i) = fma(L(j+i,j), -y_j, B(j+i)), skipped when
// y_j == 0); the pivot lane stores y_j = B(j) when the row retires.  B then
// holds L^{-1} P B, exactly what dgbtrs's forward loop produces (m == n).
template <int KL, int KU, bool FWD, class AP, class PP, class BP>
__global__ void __launch_bounds__(TrfWin<KL, KU>::WARPS * 32, TrfWin<KL, KU>::MINB)
    gbtrf_window_kernel(int m, int n, AP A, int ldab, PP P, int *__restrict__ info, int batch, BP Bv) {
    using C = TrfWin<KL, KU>;
    constexpr int KV = C::KV, W = C::W, U = C::U, WS = C::WS, H = C::H, G = C::G, WP = C::WP, D = C::D,
                  RR = C::RR, SIT = C::SIT;
    static_assert(U % 2 == 0 && RR % U == 0, "block geometry");
    extern __shared__ __align__(16) double smem[];

    const int lane = (int)lane_id(), wib = (int)(threadIdx.x >> 5);
    const int g = lane / G, t = lane % G;
    const int64_t mat = ((int64_t)blockIdx.x * C::WARPS + wib) * C::GPW + g;
    const bool live = mat < batch;
    if (__ballot_sync(0xffffffffu, live) == 0u) return;
    // Dead groups (batch tail) stay in the warp for the warp-wide shuffles;
    // they have no candidates, never pivot and never touch global memory.

    double *__restrict__ ab = live ? A.get(mat) : nullptr;
    int *__restrict__ ipiv = live ? P.get(mat) : nullptr;
    double *__restrict__ bv = (FWD && live) ? Bv.get(mat) : nullptr;  // the right-hand side (FWD)
    if (m <= 0 || n <= 0) {
        if (live && t == 0) info[mat] = 0;
        return;
    }
    const int mloc = live ? m : 0;
    double *ring = smem + (size_t)(wib * C::GPW + g) * C::GROUP_DBL;
    const uint32_t ring_s = smem_u32(ring);
    const uint32_t rec_s = ring_s + RR * WP * 8;
    const double *safe = live ? ab : g_dummy;  // zero-fill copies never read it

    // Ring row of input row q (loaded at step j = q-KL-1, block offset o = j % U)
    // holds A(q, q-KL+c) at position o+1+c, zeros elsewhere, so one 128-bit
    // load per slot pair drops it into the window registers.  o is fixed per
    // ring row (RR % U == 0), so the zero positions are zeroed once here.
    for (int i = t; i < RR * WP; i += G) ring[i] = 0.0;
    __syncwarp();

    // ---- staging: lane t copies c = t + k*G (element at AB(KV+KL-c, q-KL+c))
    int soff[SIT];
#pragma unroll
    for (int k = 0; k < SIT; ++k) soff[k] = (t + k * G) * (ldab - 1) + (KV + KL);
    auto stage_row = [&](int q, const double *rowp) {
        const uint32_t dst = ring_s + (uint32_t)(((q & (RR - 1)) * WP + 1 + ((q - KL - 1) & (U - 1))) * 8);
#pragma unroll
        for (int k = 0; k < SIT; ++k) {
            const int c = t + k * G;
            if (c < W) {
                const bool ok = (q < mloc) && (q - KL + c < n);
                cp_async8(dst + c * 8, ok ? rowp + soff[k] : safe, ok ? 8u : 0u);
            }
        }
        if constexpr (FWD) {
            if (t == 0) {  // the row's right-hand side entry rides in the ring row's spare slot
                const bool okb = (q < mloc);
                const uint32_t dstb = ring_s + (uint32_t)(((q & (RR - 1)) * WP + 2 * H) * 8);
                cp_async8(dstb, okb ? (const void *)(bv + q) : (const void *)safe, okb ? 8u : 0u);
            }
        }
        cp_async_commit();
    };
#pragma unroll 1
    for (int d = 0; d < D; ++d) stage_row(KL + 1 + d, live ? ab + (int64_t)(1 + d) * ldab : g_dummy);
    const double *srow = live ? ab + (int64_t)(1 + D) * ldab : g_dummy;  // &A(q-KL, .) of the row staged next

    // ---- window registers (slot pairs): slot r = column j0 + r; rows 0..KL first
    double2 v2[H];
#define VS(k) (((k) & 1) ? v2[(k) >> 1].y : v2[(k) >> 1].x)
#pragma unroll
    for (int h = 0; h < H; ++h) {
        const int c0 = 2 * h, c1 = 2 * h + 1;
        const bool ok0 = live && (t <= KL) && (t < m) && (c0 < n) && (c0 <= t + KU);
        const bool ok1 = live && (t <= KL) && (t < m) && (c1 < n) && (c1 <= t + KU);
        v2[h].x = ok0 ? ab[(int64_t)c0 * ldab + (KV + t - c0)] : 0.0;
        v2[h].y = ok1 ? ab[(int64_t)c1 * ldab + (KV + t - c1)] : 0.0;
    }
    int pos = (live && t <= KL) ? t : 0x7fffffff;  // logical row held by this lane
    double bq = 0.0;                                 // FWD: this row's right-hand side entry
    if constexpr (FWD) bq = (live && t <= KL && t < m) ? bv[t] : 0.0;

    int linfo = 0;
    const int mn = min(m, n);
    double *colj = live ? ab + KV : nullptr;  // &AB(KV, j)
    int *ipj = ipiv;                           // &ipiv[j]
    const unsigned gbits = (G == 32) ? 0xffffffffu : ((1u << G) - 1u);
    const unsigned gbase = (unsigned)(g * G);
    int rb = 0;  // pivot-row record buffer of step j (double buffered)
#pragma unroll 1
    for (int j0 = 0; j0 < mn; j0 += U) {
#pragma unroll
        for (int s = 0; s < U; ++s) {  // column j = j0 + s sits in slot s
            const int j = j0 + s;
            if (j >= mn) break;
            cp_async_wait<D - 1>();  // row j+KL+1 landed (this lane's part)

            // ---- IAMAX over the candidates (logical rows j..min(j+KL, m-1))
            const double x = VS(s);
            const bool cand = (t <= KL) && (pos < mloc);
            const uint64_t key = cand ? abs_key(x) : 0ull;
            const unsigned hi = (unsigned)(key >> 32);
            unsigned mhi;
            if constexpr (C::GPW == 2) {  // two full-warp reductions beat a 4-round butterfly
                const unsigned m0 = __reduce_max_sync(0xffffffffu, g == 0 ? hi : 0u);
                const unsigned m1 = __reduce_max_sync(0xffffffffu, g == 1 ? hi : 0u);
                mhi = g == 0 ? m0 : m1;
            } else if constexpr (C::GPW == 1) {
                mhi = __reduce_max_sync(0xffffffffu, hi);
            } else {
                mhi = hi;
#pragma unroll
                for (int off = 1; off < G; off <<= 1) mhi = max(mhi, __shfl_xor_sync(0xffffffffu, mhi, off));
            }
            unsigned gb = (__ballot_sync(0xffffffffu, cand && hi == mhi) >> gbase) & gbits;
            if (__any_sync(0xffffffffu, live && __popc(gb) != 1)) {
                // exact tie-break: low word, then smallest logical row (first index)
                const unsigned lo = (unsigned)key;
                unsigned mlo = (cand && hi == mhi) ? lo : 0u;
#pragma unroll
                for (int off = 1; off < G; off <<= 1) mlo = max(mlo, __shfl_xor_sync(0xffffffffu, mlo, off));
                unsigned pp = (cand && hi == mhi && lo == mlo) ? (unsigned)pos : 0xffffffffu;
#pragma unroll
                for (int off = 1; off < G; off <<= 1) pp = min(pp, __shfl_xor_sync(0xffffffffu, pp, off));
                gb = (__ballot_sync(0xffffffffu, cand && (unsigned)pos == pp) >> gbase) & gbits;
            }
            const bool is_piv = (t == __ffs(gb) - 1);  // dead groups: gb = 0, nobody

            // ---- pivot row (U row j: slots s..s+KV) + its logical row -> smem record, 128-bit
            const uint32_t rcs = rec_s + (uint32_t)(rb * WP * 8);
            const double *rc = ring + RR * WP + rb * WP;
#pragma unroll
            for (int h = s / 2; h <= (s + KV) / 2; ++h) st_shared_v2_if(is_piv, rcs + h * 16, v2[h]);
            // spare pair after the slots: (B entry, logical row) of the pivot row
            st_shared_v2_if(is_piv, rcs + 2 * H * 8, make_double2(bq, __longlong_as_double((long long)pos)));
            __syncwarp();

            // ---- broadcast read: pivot value and pivot row (128-bit loads), its logical row
            double2 uu[KV / 2 + 2];
#pragma unroll
            for (int h = s / 2; h <= (s + KV) / 2; ++h) uu[h - s / 2] = *reinterpret_cast<const double2 *>(rc + 2 * h);
#define US(k) ((((k) & 1) ? uu[((k) >> 1) - s / 2].y : uu[((k) >> 1) - s / 2].x))
            const double2 yp = *reinterpret_cast<const double2 *>(rc + 2 * H);
            const int ppos = (int)__double_as_longlong(yp.y);
            const double p = US(s);
            const bool zp = (p == 0.0);  // exact zero pivot: all candidates are +-0
            if (is_piv) *ipj = ppos + 1;
            if (live && zp && linfo == 0) linfo = j + 1;
            if (live && pos == j && !is_piv) pos = ppos;  // interchange = relabel

            // ---- SCAL: multiplier = x * RN(1/p) (DSCAL(ONE/pivot), Q7)
            const double r = __drcp_rn(p);
            const double l = zp ? x : __dmul_rn(x, r);
            const double lu = zp ? 0.0 : l;  // zero pivot: no update
            if constexpr (FWD) {  // forward substitution on the fly (DGBTRS 'N' forward loop)
                const double y = yp.x;
                if (is_piv) bv[j] = y;
                if (y != 0.0) bq = __fma_rn(lu, -y, bq);
            }
            if (cand && !is_piv) colj[pos - j] = l;

            // ---- RANK-1 update of the window columns j+1..j+KV (DGER, alpha = -1, FMA)
#pragma unroll
            for (int k = s + 1; k <= s + KV; ++k) VS(k) = __fma_rn(lu, -US(k), VS(k));
#undef US

            // ---- U row j -> HBM: U(j, j+c) = record[s + c] at AB(KV-c, j+c)
#pragma unroll
            for (int k = 0; k < SIT; ++k) {
                const int c = t + k * G;
                if (live && c < W && j + c < n) colj[(int64_t)c * (ldab - 1)] = rc[s + c];
            }
            stage_row(j + KL + 1 + D, srow);

            // ---- slide: the pivot lane takes row j+KL+1 (ring row pre-positioned at slots s+1..s+W)
            if (is_piv) pos = j + KL + 1;
            const uint32_t rr = ring_s + (uint32_t)(((j + KL + 1) & (RR - 1)) * WP * 8);
#pragma unroll
            for (int h = (s + 1) / 2; h < H; ++h) ld_shared_v2_if(is_piv, rr + h * 16, v2[h]);  // tail zeros too
            if constexpr (FWD) ld_shared_f64_if(is_piv, rr + 2 * H * 8, bq);
            colj += ldab;
            srow += ldab;
            ++ipj;
            rb ^= 1;
        }
        // shift the window by U columns: slot r <- slot r+U (U even: whole pairs move)
#pragma unroll
        for (int h = 0; h < H; ++h) {
            if (h + U / 2 < H) {
                v2[h] = v2[h + U / 2];
            } else {
                v2[h].x = 0.0;
                v2[h].y = 0.0;
            }
        }
    }
    cp_async_wait<0>();
#undef VS
    if (!live) return;

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
