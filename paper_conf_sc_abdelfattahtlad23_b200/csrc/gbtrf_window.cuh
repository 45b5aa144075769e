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
//    registers.  Columns are processed in blocks of U = 4: during a block,
//    column j0+r sits in register slot r (slots paired into double2 so rows
//    move to/from shared memory with 128-bit accesses); after the block the
//    slots shift down by U (register moves), which keeps the unrolled code
//    small enough for the instruction cache.
//  * Row interchanges are relabelings: a lane carries the logical position of
//    its row.  LAPACK swaps only columns j..ju; beyond ju both rows hold
//    structural zeros, so swapping whole rows is identical.
//  * IAMAX: warp REDUX max of the high word of the |x| bit pattern + ballot;
//    exact slow path (low word, then smallest logical row) only when the
//    high words tie (zero pivots, exact ties) -- first-max semantics (Q2).
//  * The pivot lane drops its row (= U row j) and (B entry, logical row)
//    into an smem record; the group reads it back with 128-bit broadcast
//    loads and every lane applies the rank-1 update with FP64 FMAs in
//    registers.  Multipliers (band column j below the diagonal, contiguous)
//    are stored by their owning lanes each step.
//  * Global traffic moves in blocks of U rows: in band storage U consecutive
//    rows of one column are U contiguous doubles, so U lanes move one 32-byte
//    chunk.  Input rows j0+KL+1+D .. +U are gathered by cp.async (LDGSTS,
//    zero-fill outside the matrix) into an smem ring, D rows ahead; the lane
//    freed by a pivot row reloads its registers from the ring with 128-bit
//    loads.  The block's U pivot records are stored as U rows at block end.
//    Fill rows (input) are never read; every input element is read from HBM
//    once, every output element written once.
#pragma once
#include "common.cuh"

// Tuning knobs (compile-time; overridable with -D for experiments)
#ifndef BANDLU_TRF_D_NARROW
#define BANDLU_TRF_D_NARROW 8
#endif
#ifndef BANDLU_TRF_G_NARROW
#define BANDLU_TRF_G_NARROW 8
#endif
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
#define BANDLU_TRF_D 4  // staging lead in rows (multiple of U; 8 measured slower on C3)
#endif
#ifndef BANDLU_TRF_WP16
#define BANDLU_TRF_WP16 1
#endif

namespace bandlu {

template <int KL_, int KU_>
struct TrfWin {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU, W = KV + 1;
    static constexpr int U = BANDLU_TRF_U;       // columns per unrolled block (window shift granularity)
    static constexpr int WS = W + U;             // register slots: column j0 + r in slot r during a block
    static constexpr int H = (WS + 1) / 2;       // double2 slot pairs
    // Ring rows and pivot-row records are indexed by block slot (16-byte slot
    // pairs), then a spare pair at RP: (B entry) in ring rows, (B entry,
    // logical row) in records.  Pitch WP == 2 (mod 4) doubles.
    // Wide rows (>= 8-lane groups): WP == 4 (mod 16), so the U x U chunk
    // patterns of the block transfers (row offset bs, column offset bk ->
    // bs*WP + bk) hit 16 distinct 8-byte banks; short rows: WP == 2 (mod 4)
    // (smaller rings, measured better there).
    static constexpr int WP = (BANDLU_TRF_WP16 && pow2_ceil(KL + 1) >= 8) ? ((2 * H + 2 + 11) / 16) * 16 + 4
                                                                          : 2 * H + 2 + ((2 * H + 2) % 4 == 2 ? 0 : 2);
    static constexpr int RP = WP - 2;
    // lanes per matrix: pow2 >= KL+1; wide windows use >= 8 so that a warp's
    // smem rings (and so the resident warps per SM) stay within budget
    // (narrow bands: >= BANDLU_TRF_G_NARROW lanes, so that a batch spreads over more warps)
    static constexpr int GMIN = W > 24 ? 8 : (W <= 5 ? BANDLU_TRF_G_NARROW : 1);
    static constexpr int G = pow2_ceil(KL + 1) < GMIN ? GMIN : pow2_ceil(KL + 1);
    static constexpr int GPW = 32 / G;           // matrices per warp
    // staging lead (rows, multiple of U): narrow bands do little work per step, so the
    // HBM latency of a block's rows must be covered by more steps ahead
    static constexpr int D = (W <= 5) ? BANDLU_TRF_D_NARROW : BANDLU_TRF_D;
    static constexpr int DB = D / U;             // staging lead in blocks
    static constexpr int RR = pow2_ceil((DB + 1) * U);  // ring rows (power of 2, multiple of U)
    static constexpr int NREC = U;               // pivot-row records: this block's U rows
    static constexpr int GROUP_DBL = (RR + NREC) * WP;  // input-row ring + pivot-row records
    // Block transfers (U rows at a time): in band storage U consecutive rows of
    // one column are U contiguous doubles, so U lanes move one column chunk.
    static constexpr int BK = W + U - 1;         // columns touched by U consecutive rows
    static constexpr int BIT = (BK * U + G - 1) / G;  // block elements per lane
    // warps per CTA: up to BANDLU_TRF_WARPS while a CTA's rings fit ~76 KB (3 CTAs/SM)
    static constexpr int WARPS_FIT = (76 * 1024) / (GPW * GROUP_DBL * 8);
    static constexpr int WARPS = WARPS_FIT < 1 ? 1 : (WARPS_FIT < BANDLU_TRF_WARPS ? WARPS_FIT : BANDLU_TRF_WARPS);
    // register budget: >= MINB CTAs per SM while the window fits
    static constexpr int MINB = (W <= 24 ? BANDLU_TRF_MINB * 4 : 8) / WARPS;  // (12 or 8 resident warps)
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
    constexpr int KV = C::KV, W = C::W, U = C::U, WS = C::WS, H = C::H, G = C::G, WP = C::WP, RP = C::RP, D = C::D,
                  RR = C::RR, BK = C::BK, BIT = C::BIT;
    static_assert(U % 2 == 0 && RR % U == 0 && D % U == 0 && (U & (U - 1)) == 0, "block geometry");
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

    // Ring row of input row q (needed at step q-KL-1, block offset o = (q-KL-1) % U)
    // holds A(q, q-KL+c) at position o+1+c, zeros elsewhere, so one 128-bit
    // load per slot pair drops it into the window registers.  o is fixed per
    // ring row (RR % U == 0), so the zero positions are zeroed once here.
    for (int i = t; i < RR * WP; i += G) ring[i] = 0.0;
    __syncwarp();

    // ---- block element e = t + k*G of this lane: row offset bs = e % U, column
    // offset bk = e / U.  Rows qb..qb+U-1 (qb = first row of a block, qb-KL-1 a
    // multiple of U) span columns qb-KL .. qb-KL+BK-1; A(qb+bs, qb-KL+bk) sits at
    // AB(KV+KL+bs-bk, qb-KL+bk) and (c = bk-bs in 0..KV) at ring position 1+bk.
    // U rows of the previous block: record bs holds U row j0+bs at slots
    // bs..bs+KV; U(j0+bs, j0+bk) goes to AB(KV+bs-bk, j0+bk).  Both are U
    // contiguous doubles per column: U lanes, one 32-byte chunk.
    // element offset from &AB(0, first column): bk*(ldab-1) + bs
    const int bo0 = (t / U) * (ldab - 1) + (t % U), bstep = (G / U) * (ldab - 1);
    auto boff = [&](int k) -> int {
        if constexpr (G % U == 0) return bo0 + k * bstep;  // bs fixed per lane
        const int e = t + k * G;
        return (e / U) * (ldab - 1) + (e % U);
    };
    unsigned bmask = 0;  // bit k: element k lies inside the band row (0 <= bk-bs <= KV)
#pragma unroll
    for (int k = 0; k < BIT; ++k) {
        const int e = t + k * G, bs = e % U, bk = e / U;
        if (bk < BK && bk - bs >= 0 && bk - bs <= KV) bmask |= 1u << k;
    }
    // rows qb..qb+U-1 -> ring (cp.async, zero-fill outside the matrix);
    // colq = &AB(0, qb-KL).  One commit group per block.
    auto stage_block = [&](int qb, const double *colq) {
#pragma unroll
        for (int k = 0; k < BIT; ++k) {
            const int e = t + k * G, bs = e % U, bk = e / U;
            if (bmask >> k & 1u) {
                const int q = qb + bs;
                const bool ok = (q < mloc) && (qb - KL + bk < n);
                const uint32_t dst = ring_s + (uint32_t)(((q & (RR - 1)) * WP + 1 + bk) * 8);
                cp_async8(dst, ok ? colq + boff(k) + (KV + KL) : safe, ok ? 8u : 0u);
            }
        }
        if constexpr (FWD) {
#pragma unroll
            for (int i = t; i < U; i += G) {  // the row's right-hand side entry rides in the ring row's spare slot
                const int q = qb + i;
                const bool okb = (q < mloc);
                const uint32_t dstb = ring_s + (uint32_t)(((q & (RR - 1)) * WP + RP) * 8);
                cp_async8(dstb, okb ? (const void *)(bv + q) : (const void *)safe, okb ? 8u : 0u);
            }
        }
        cp_async_commit();
    };
#pragma unroll 1
    for (int d = 0; d < C::DB; ++d)
        stage_block(KL + 1 + d * U, live ? ab + (int64_t)(1 + d * U) * ldab : g_dummy);
    const double *scol = live ? ab + (int64_t)(1 + D) * ldab : g_dummy;  // &AB(0, qb-KL) of the block staged next

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
    double *colb = live ? ab : nullptr;       // &AB(0, j0)
    int *ipj = ipiv;                           // &ipiv[j]
    const unsigned gbits = (G == 32) ? 0xffffffffu : ((1u << G) - 1u);
    const unsigned gbase = (unsigned)(g * G);
#pragma unroll 1
    for (int j0 = 0; j0 < mn; j0 += U) {
        cp_async_wait<C::DB - 1>();  // rows j0+KL+1 .. j0+KL+U landed (this lane's part; the
                                     // __syncwarp below publishes them to the pivot lanes)
        stage_block(j0 + KL + 1 + D, scol);
        scol += (int64_t)U * ldab;
#pragma unroll
        for (int s = 0; s < U; ++s) {  // column j = j0 + s sits in slot s
            const int j = j0 + s;
            if (j >= mn) break;

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
            const uint32_t rcs = rec_s + (uint32_t)(s * WP * 8);
            const double *rc = reinterpret_cast<const double *>(ring) + (rcs - ring_s) / 8;
#pragma unroll
            for (int h = s / 2; h <= (s + KV) / 2; ++h) st_shared_v2_if(is_piv, rcs + h * 16, v2[h]);
            // spare pair after the slots: (B entry, logical row) of the pivot row
            st_shared_v2_if(is_piv, rcs + RP * 8, make_double2(bq, __longlong_as_double((long long)pos)));
            __syncwarp();

            // ---- broadcast read: pivot value and pivot row, its logical row
            double2 uu[KV / 2 + 2];
#pragma unroll
            for (int h = s / 2; h <= (s + KV) / 2; ++h) uu[h - s / 2] = *reinterpret_cast<const double2 *>(rc + 2 * h);
#define US(k) ((((k) & 1) ? uu[((k) >> 1) - s / 2].y : uu[((k) >> 1) - s / 2].x))
            const double2 yp = *reinterpret_cast<const double2 *>(rc + RP);
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

            // ---- slide: the pivot lane takes row j+KL+1 (ring row pre-positioned at slots s+1..s+W)
            if (is_piv) pos = j + KL + 1;
            const uint32_t rr = ring_s + (uint32_t)(((j + KL + 1) & (RR - 1)) * WP * 8);
#pragma unroll
            for (int h = (s + 1) / 2; h < H; ++h) ld_shared_v2_if(is_piv, rr + h * 16, v2[h]);  // tail zeros too
            if constexpr (FWD) ld_shared_f64_if(is_piv, rr + RP * 8, bq);
            colj += ldab;
            ++ipj;
        }
        // ---- U rows j0 .. j0+U-1 (this block's pivot rows) -> HBM, 32-byte column chunks
        __syncwarp();
#pragma unroll
        for (int k = 0; k < BIT; ++k) {
            const int e = t + k * G, bs = e % U, bk = e / U;
            if (live && (bmask >> k & 1u) && j0 + bs < mn && j0 + bk < n)
                colb[boff(k) + KV] = ld_shared_f64(rec_s + (uint32_t)((bs * WP + bk) * 8));
        }
        colb += (int64_t)U * ldab;
        __syncwarp();  // records are rewritten by the next block's pivot lanes
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
    __syncwarp();
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
