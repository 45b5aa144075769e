// gbtrf_rows.cuh -- sm_100a band LU with partial pivoting, R row slots per
// lane, the incoming rows of a block preloaded into free slots.
//
// What it computes: LAPACK DGBTF2 exactly (Sec. 5.1 pseudo-code
// P:350-367, ju rule P:492-494, right-only swaps P:358/P:369-374), the same
// fp64 operation sequence as the oracle => bitwise-equal factors, ipiv, info.
//
// Why a second register-window kernel: the row-owner
// window (gbtrf_window.cuh) is bounded by the shared-memory pipe -- per
// matrix-column step ~42 wavefronts: the pivot row written to a record by one
// lane, read back by the 16 lanes of the matrix with 128-bit loads, and the
// next band row loaded by the retiring pivot lane alone.  Measured on B200
// (tools/probes/lsu_probe4.cu): a broadcast LDS.64 costs one cycle per warp
// whatever the number of distinct addresses (<= 128 B), a 1-lane LDS.128 two.
// So this kernel
//  * packs more matrices into a warp: G lanes per matrix hold R rows each
//    (G*R >= KL+1+U slots; C3 (10,10): G = 8, R = 2 -> 4 matrices per warp,
//    one broadcast read serves all four);
//  * broadcasts the pivot row with 64-bit loads (one per column);
//  * loads a block's U incoming band rows at block start, all at once, into
//    the slots freed by the previous block's pivot rows (ballot + rank), so
//    no lane reloads its registers inside the column step.  A preloaded row
//    is not a pivot candidate until its step (pos <= j + KL); before that its
//    multiplier is forced to 0 (its column-j entry is a structural zero), so
//    it receives no update -- exactly DGBTF2, where that row is outside the
//    active window.
// Interchanges are relabelings (reading 10), IAMAX is first-max
// (exact 64-bit key compare, ties by smallest logical row; reading 2).
//
// Build-time experiment flags (DESIGN.md Sec. 6 records each measurement; none is on by default):
//   exact variants  BANDLU_ROWS_FASTCHAIN, _SHFL_P, _LOOKAHEAD, _REC64, _KEY64, _NOHOIST, _LDS64,
//                   _IPIV_STEP, _Y_BLOCK, _NBLK, _U, _MAXREG, _MINW -- bitwise equal, measured
//                   slower or equal;
//   timing-only     BANDLU_ABL_NOSTAGE, _NOOUT, _NOREC, _NOSHIFT, _NOSEARCH, _NORCP, _HALF --
//                   remove work to see what it costs; their RESULTS ARE WRONG (never in the library).
#pragma once
#include "backsolve_fused.cuh"
#include "common.cuh"
#ifndef __CUDACC_RTC__
#include <type_traits>
#endif

#ifndef BANDLU_ROWS_WARPS
#define BANDLU_ROWS_WARPS 4
#endif

namespace bandlu {

template <int KL_, int KU_, int G_, int R_>
struct TrfRows {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU, W = KV + 1;
    static constexpr int G = G_, R = R_, GPW = 32 / G;
#ifndef BANDLU_ROWS_U
#define BANDLU_ROWS_U 4
#endif
    static constexpr int U = BANDLU_ROWS_U;      // columns per block (preload / record granularity)
#ifndef BANDLU_ROWS_NBLK
#define BANDLU_ROWS_NBLK 1
#endif
    // blocks per register-window shift: with 2 the window holds NBLK*U extra columns and the
    // second block of a pair addresses its slots U further on, halving the shift moves
    static constexpr int NBLK = BANDLU_ROWS_NBLK;
    static constexpr int WS = W + NBLK * U, H = (WS + 1) / 2;
    static_assert(G * R >= KL + 1 + U, "slots: KL+1 active rows + U preloaded rows");
    static_assert(32 % G == 0, "group size");
    // ring row / record pitch (doubles), spare pair at RP: (B entry[, logical row])
    static constexpr int WP = (G >= 8) ? ((2 * H + 2 + 11) / 16) * 16 + 4 : 2 * H + 2 + ((2 * H + 2) % 4 == 2 ? 0 : 2);
    static constexpr int RP = WP - 2;
    static constexpr int D = U, DB = D / U;      // staging lead (rows / blocks)
    static constexpr int RR = pow2_ceil((DB + 1) * U);
    static constexpr int NREC = U;
    // group pitch == 2 (mod 16) doubles: the GPW groups of a warp read their
    // records at the same offsets, so their 64-bit broadcasts must sit in
    // distinct banks (a multiple of 128 B would make them a GPW-way conflict)
    static constexpr int GROUP_DBL = ((RR + NREC) * WP + 13) / 16 * 16 + 2;
    static constexpr int BK = W + U - 1;
    static constexpr int BIT = (BK * U + G - 1) / G;
    static_assert(BIT <= 32, "block element mask");
    static constexpr int WARPS_FIT = (72 * 1024) / (GPW * GROUP_DBL * 8);
    // wide windows (W > 24) run 8 warps/SM: 2 per scheduler, so each thread may use up to 255
    // registers (the register file is split per scheduler: 3 warps each would cap it at 168)
#ifndef BANDLU_ROWS_WIDE_WARPS
#define BANDLU_ROWS_WIDE_WARPS 2
#endif
#ifndef BANDLU_ROWS_WIDE_MINW
#define BANDLU_ROWS_WIDE_MINW 8
#endif
    static constexpr int WMAX = W > 24 ? BANDLU_ROWS_WIDE_WARPS : BANDLU_ROWS_WARPS;
    static constexpr int WARPS = WARPS_FIT < 1 ? 1 : (WARPS_FIT < WMAX ? WARPS_FIT : WMAX);
#ifndef BANDLU_ROWS_MINW
#define BANDLU_ROWS_MINW 12
#endif
    // resident warps per SM target (wide windows: 8, as the window kernel)
    static constexpr int MINB = ((W <= 24 ? BANDLU_ROWS_MINW : BANDLU_ROWS_WIDE_MINW) + WARPS - 1) / WARPS;
    static constexpr size_t smem_bytes() { return (size_t)WARPS * GPW * GROUP_DBL * sizeof(double); }
    // fused solve with y in shared memory: each group also holds y(0..n-1)
    __host__ __device__ static constexpr int ypad(int n) { return (n + 15) & ~15; }
    static constexpr size_t smem_bytes_y(int n) { return (size_t)WARPS * GPW * (GROUP_DBL + ypad(n)) * sizeof(double); }
};

// Kernel modes (template FL, bit flags):
//   FL_FWD: forward substitution of one right-hand side on the fly (y = L^-1 P b);
//   FL_BWD: then the backward substitution in the same kernel (backsolve_fused.cuh):
//           one launch computes dgbtrf + dgbtrs('N') = the fused gbsv kernel;
//   FL_YSM: y kept in shared memory (n doubles per matrix) instead of B;
//   FL_SKIPI: B written only where info == 0 (dgbsv; needs FL_YSM).
enum : int { FL_FWD = 1, FL_BWD = 2, FL_YSM = 4, FL_SKIPI = 8 };

// max of a 32-bit value over the G lanes of each group (all 32 lanes call)
template <int G>
__device__ __forceinline__ unsigned group_max_u32(unsigned v, int g) {
    if constexpr (G == 32) {
        return __reduce_max_sync(0xffffffffu, v);
    } else if constexpr (G == 16) {
        const unsigned m0 = __reduce_max_sync(0xffffffffu, g == 0 ? v : 0u);
        const unsigned m1 = __reduce_max_sync(0xffffffffu, g == 1 ? v : 0u);
        return g == 0 ? m0 : m1;
    } else {
#pragma unroll
        for (int off = 1; off < G; off <<= 1) v = max(v, __shfl_xor_sync(0xffffffffu, v, off));
        return v;
    }
}
template <int G>
__device__ __forceinline__ unsigned group_min_u32(unsigned v) {
#pragma unroll
    for (int off = 1; off < G; off <<= 1) v = min(v, __shfl_xor_sync(0xffffffffu, v, off));
    return v;
}

// BANDLU_ROWS_MAXREG (experiments): a register cap instead of the resident-CTA target
#ifdef BANDLU_ROWS_MAXREG
#define BANDLU_ROWS_BOUNDS(...) __maxnreg__(BANDLU_ROWS_MAXREG)
#else
#define BANDLU_ROWS_BOUNDS(...) __launch_bounds__(__VA_ARGS__::WARPS * 32, __VA_ARGS__::MINB)
#endif
template <int KL, int KU, int G, int R, int FL, class AP, class PP, class BP>
__global__ void BANDLU_ROWS_BOUNDS(TrfRows<KL, KU, G, R>)
    gbtrf_rows_kernel(int m, int n, AP A, int ldab, PP P, int *__restrict__ info, int batch, BP Bv) {
    using C = TrfRows<KL, KU, G, R>;
    constexpr bool FWD = FL & FL_FWD, BWD = FL & FL_BWD, YSM = FL & FL_YSM, SKIPI = FL & FL_SKIPI;
    static_assert(!BWD || FWD, "the fused backward solve needs the forward pass");
    static_assert(!YSM || BWD, "y in shared memory only with the fused backward solve");
    static_assert(!SKIPI || YSM, "dgbsv semantics (B untouched where info > 0) need y off B");
    constexpr int KV = C::KV, U = C::U, H = C::H, WP = C::WP, RP = C::RP, D = C::D, RR = C::RR, BK = C::BK,
                  BIT = C::BIT;
    constexpr int FREE = 0x7fffffff;
#ifdef BANDLU_ROWS_NOHOIST
    constexpr bool HOIST = false;
#else
    constexpr bool HOIST = C::W <= 24;
#endif
    extern __shared__ __align__(16) double smem[];

    const int lane = (int)lane_id(), wib = (int)(threadIdx.x >> 5);
    const int g = lane / G, t = lane % G;
    const int64_t mat = ((int64_t)blockIdx.x * C::WARPS + wib) * C::GPW + g;
    const bool live = mat < batch;
    if (__ballot_sync(0xffffffffu, live) == 0u) return;

    double *__restrict__ ab = live ? A.get(mat) : nullptr;
    int *__restrict__ ipiv = live ? P.get(mat) : nullptr;
    double *__restrict__ bv = (FWD && live) ? Bv.get(mat) : nullptr;
    if (m <= 0 || n <= 0) {
        if (live && t == 0) info[mat] = 0;
        return;
    }
    const int mloc = live ? m : 0;
    const int gpitch = C::GROUP_DBL + (YSM ? C::ypad(n) : 0);
    double *ring = smem + (size_t)(wib * C::GPW + g) * gpitch;
    const uint32_t ybuf_s = smem_u32(ring) + C::GROUP_DBL * 8;  // YSM: y(0..n-1)
    const uint32_t ring_s = smem_u32(ring);
    const uint32_t rec_s = ring_s + RR * WP * 8;
    const double *safe = live ? ab : g_dummy;

    // Ring row of input row q holds A(q, q-KL+c) at position o+1+c
    // (o = (q-KL-1) % U, fixed per ring row), zeros elsewhere.
    for (int i = t; i < RR * WP; i += G) ring[i] = 0.0;
    __syncwarp();

    // ---- block transfers: element e = t + k*G -> row offset bs = e % U, column offset bk = e / U
    const int bo0 = (t / U) * (ldab - 1) + (t % U), bstep = (G / U) * (ldab - 1);
    auto boff = [&](int k) -> int {
        if constexpr (G % U == 0) return bo0 + k * bstep;
        const int e = t + k * G;
        return (e / U) * (ldab - 1) + (e % U);
    };
    unsigned bmask = 0;
#pragma unroll
    for (int k = 0; k < BIT; ++k) {
        const int e = t + k * G, bs = e % U, bk = e / U;
        if (bk < BK && bk - bs >= 0 && bk - bs <= KV) bmask |= 1u << k;
    }
    // G % U == 0: lane t always moves row offset bs = t % U of the block, columns
    // bk = t / U + k * KS -- per-k offsets are immediates / one pointer stride
    constexpr int KS = G / U;
    const int64_t kstride = (int64_t)KS * (ldab - 1);
    auto stage_block = [&](int qb, const double *colq) {
#ifdef BANDLU_ABL_NOSTAGE
        if (qb >= 0) { cp_async_commit(); return; }
#endif
        if constexpr (G % U == 0) {
            const int q = qb + t % U, c0 = qb - KL + t / U;
            const bool rowok = q < mloc;
            const uint32_t dst0 = ring_s + (uint32_t)(((q & (RR - 1)) * WP + 1 + t / U) * 8);
            const double *src = colq + bo0 + (KV + KL);
#pragma unroll
            for (int k = 0; k < BIT; ++k) {
                if (bmask >> k & 1u) {
                    const bool ok = rowok && (c0 + k * KS < n);
                    cp_async8(dst0 + (uint32_t)(k * KS * 8), ok ? src + k * kstride : safe, ok ? 8u : 0u);
                }
            }
        } else {
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
        }
        if constexpr (FWD) {
#pragma unroll
            for (int i = t; i < U; i += G) {
                const int q = qb + i;
                const bool okb = (q < mloc);
                const uint32_t dstb = ring_s + (uint32_t)(((q & (RR - 1)) * WP + RP) * 8);
                cp_async8(dstb, okb ? (const void *)(bv + q) : (const void *)safe, okb ? 8u : 0u);
            }
        }
        cp_async_commit();
    };
#pragma unroll 1
    for (int d = 0; d < C::DB; ++d) stage_block(KL + 1 + d * U, live ? ab + (int64_t)(1 + d * U) * ldab : g_dummy);
    const double *scol = live ? ab + (int64_t)(1 + D) * ldab : g_dummy;

    // ---- window registers: slot r of row slot i = column j0 + r; rows 0..KL in slots i = ri*G + t
    double2 v[R][H];
    int pos[R];
    double bq[R];
#define VS(ri, k) (((k) & 1) ? v[ri][(k) >> 1].y : v[ri][(k) >> 1].x)
#pragma unroll
    for (int ri = 0; ri < R; ++ri) {
        const int i = ri * G + t;
        const bool row_ok = live && (i <= KL) && (i < m);
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int c0 = 2 * h, c1 = 2 * h + 1;
            const bool ok0 = row_ok && (c0 < n) && (c0 <= i + KU);
            const bool ok1 = row_ok && (c1 < n) && (c1 <= i + KU);
            v[ri][h].x = ok0 ? ab[(int64_t)c0 * ldab + (KV + i - c0)] : 0.0;
            v[ri][h].y = ok1 ? ab[(int64_t)c1 * ldab + (KV + i - c1)] : 0.0;
        }
        pos[ri] = (live && i <= KL) ? i : FREE;
        bq[ri] = 0.0;
        if constexpr (FWD) bq[ri] = row_ok ? bv[i] : 0.0;
    }

    int linfo = 0;
    const int mn = min(m, n);
    double *colj = live ? ab + KV : nullptr;  // &AB(KV, j)
    double *colb = live ? ab : nullptr;       // &AB(0, j0)
    int *ipj = ipiv;
    int pv[U];     // the block's pivots (1-based), stored once per block by lane 0 of the group
    double yv[U];  // FWD: the block's y(j), likewise
#pragma unroll
    for (int s = 0; s < U; ++s) {
        pv[s] = 0;
        yv[s] = 0.0;
    }
    const unsigned gbits = (G == 32) ? 0xffffffffu : ((1u << G) - 1u);
    const unsigned gbase = (unsigned)(g * G);
    const unsigned below = (1u << t) - 1u;
#ifdef BANDLU_ROWS_LOOKAHEAD
    constexpr bool LA = true;
#else
    constexpr bool LA = false;
#endif
    struct PivState {
        double x[R];
        bool cand[R];
        int pb, rb;
        unsigned gb;
    } ps;
    // IAMAX of step s (column j): first max |x| over the candidate rows, exact
    // (64-bit key, ties by smallest logical row; reading 2)
    auto search = [&](int s, int j, PivState &o) {
        uint64_t kb = 0;
        int pb = FREE, rb = 0;
        bool cb = false;
#pragma unroll
        for (int ri = 0; ri < R; ++ri) {
            o.x[ri] = VS(ri, s);
            o.cand[ri] = (pos[ri] <= j + KL) && (pos[ri] < mloc);
#ifndef BANDLU_ROWS_KEY64
            // |x| as integer words (no DADD |x| on the FP64 pipe in the search chain; C3 -0.3%)
            const uint64_t k = o.cand[ri] ? (((uint64_t)((unsigned)__double2hiint(o.x[ri]) & 0x7fffffffu) << 32) |
                                             (unsigned)__double2loint(o.x[ri]))
                                          : 0ull;
#else
            const uint64_t k = o.cand[ri] ? abs_key(o.x[ri]) : 0ull;
#endif
            const bool better = o.cand[ri] && (!cb || k > kb || (k == kb && pos[ri] < pb));
            if (better) {
                kb = k;
                pb = pos[ri];
                rb = ri;
                cb = true;
            }
        }
#ifdef BANDLU_ABL_NOSEARCH
        if (j >= 0) { o.pb = pb; o.rb = rb; o.gb = 1u; return; }
#endif
        const unsigned hi = (unsigned)(kb >> 32);
        const unsigned mhi = group_max_u32<G>(hi, g);
        unsigned gb = (__ballot_sync(0xffffffffu, cb && hi == mhi) >> gbase) & gbits;
        if (__any_sync(0xffffffffu, live && __popc(gb) != 1)) {
            // exact tie-break: low word, then smallest logical row (first index)
            const unsigned lo = (unsigned)kb;
            const unsigned mlo = group_max_u32<G>((cb && hi == mhi) ? lo : 0u, g);
            const unsigned pp = group_min_u32<G>((cb && hi == mhi && lo == mlo) ? (unsigned)pb : 0xffffffffu);
            gb = (__ballot_sync(0xffffffffu, cb && (unsigned)pb == pp) >> gbase) & gbits;
        }
        o.pb = pb;
        o.rb = rb;
        o.gb = gb;
    };
    // one block of U columns; its column j0+s sits in register slot OFF+s
    auto blk = [&](auto offc, int j0) {
        constexpr int OFF = decltype(offc)::value;
        cp_async_wait<C::DB - 1>();  // rows j0+KL+1 .. j0+KL+U landed (this lane's part)
        __syncwarp();
        // ---- preload rows j0+KL+1+o (o = 0..U-1) into the first U free slots of the group
        {
            int before = 0;
#pragma unroll
            for (int ri = 0; ri < R; ++ri) {
                const bool fr = (pos[ri] == FREE) || (pos[ri] >= mloc);
                const unsigned fb = (__ballot_sync(0xffffffffu, fr) >> gbase) & gbits;
                const int rank = before + __popc(fb & below);
                const bool take = fr && rank < U;
                const int q = j0 + KL + 1 + rank;
                const uint32_t rr = ring_s + (uint32_t)((q & (RR - 1)) * WP * 8);
#pragma unroll
                for (int h = 0; h < H - OFF / 2; ++h) ld_shared_v2_if(take, rr + h * 16, v[ri][h + OFF / 2]);
                if constexpr (FWD) ld_shared_f64_if(take, rr + RP * 8, bq[ri]);
                if (take) pos[ri] = q;
                before += __popc(fb);
            }
        }
        stage_block(j0 + KL + 1 + D, scol);
        scol += (int64_t)U * ldab;
#pragma unroll
        for (int s = 0; s < U; ++s) {  // column j = j0 + s sits in slot s
            const int j = j0 + s;
            if (j >= mn) break;

            // ---- IAMAX over the candidates (logical rows j..min(j+KL, m-1)); with LOOKAHEAD
            // the search of step s > 0 already ran inside step s-1, right after column j's update
            if (!LA || s == 0) search(s + OFF, j, ps);
            double x[R];
            bool cand[R];
#pragma unroll
            for (int ri = 0; ri < R; ++ri) {
                x[ri] = ps.x[ri];
                cand[ri] = ps.cand[ri];
            }
            const int pb = ps.pb, rb = ps.rb;
            const unsigned gb = ps.gb;
            const bool is_piv = (t == __ffs(gb) - 1);
#ifdef BANDLU_ROWS_FASTCHAIN
            // ---- (experiment, -DBANDLU_ROWS_FASTCHAIN) the step's dependency chain bypasses
            // the shared-memory record: every lane computes RN(1/x) of its own candidate
            // while the search runs, and the pivot lane's reciprocal, logical row and
            // column-(j+1) entry -- all the next pivot search depends on -- arrive by shuffle.
            // At 1,250 matrices per GPU the record write -> read -> RN(1/p) path held 15% of
            // the stall samples, yet removing it measured 0.2341 vs 0.2343 ms (and 0.968 vs
            // 0.960 ms at 10,000): the step time is its instruction count, not that chain.
            const int plane = (int)gbase + max(__ffs(gb) - 1, 0);
            double xs = x[0], u1s = VS(0, s + 1 + OFF);
#pragma unroll
            for (int ri = 1; ri < R; ++ri) {
                xs = (rb == ri) ? x[ri] : xs;
                u1s = (rb == ri) ? VS(ri, s + 1 + OFF) : u1s;
            }
            const double rinv = __shfl_sync(0xffffffffu, drcp_rn_nz(xs), plane);
            const double u1 = __shfl_sync(0xffffffffu, u1s, plane);
            const int ppos_f = __shfl_sync(0xffffffffu, pb, plane);
#endif

            // ---- pivot row (U row j: slots s..s+KV) + (B entry, logical row) -> record s
            const uint32_t rcs = rec_s + (uint32_t)(s * WP * 8);
#if defined(BANDLU_ROWS_REC64)
            // 64-bit record stores: one wavefront each for the GPW pivot lanes (a 128-bit store
            // from lanes in both half-warps takes two)
#pragma unroll
            for (int ri = 0; ri < R; ++ri) {
#pragma unroll
                for (int k = s; k <= s + KV; ++k) st_shared_f64_if(is_piv && rb == ri, rcs + k * 8, VS(ri, k + OFF));
            }
#elif !defined(BANDLU_ABL_NOREC)
#pragma unroll
            for (int ri = 0; ri < R; ++ri) {
#pragma unroll
                for (int h = s / 2; h <= (s + KV) / 2; ++h) {
#ifdef BANDLU_ABL_HALF
                    // (timing experiment, wrong results) half the record stores
                    if (h != s / 2 && (h & 1)) continue;
#endif
                    st_shared_v2_if(is_piv && rb == ri, rcs + h * 16, v[ri][h + OFF / 2]);
                }
            }
#else
            st_shared_v2_if(is_piv, rcs + (s / 2) * 16, v[0][s / 2 + OFF / 2]);
#endif
            {
                double bsel = bq[0];
#pragma unroll
                for (int ri = 1; ri < R; ++ri) bsel = (rb == ri) ? bq[ri] : bsel;
                st_shared_v2_if(is_piv, rcs + RP * 8, make_double2(bsel, __longlong_as_double((long long)pb)));
            }
            __syncwarp();

            // ---- broadcast read (64-bit: one cycle per warp for all groups)
            const double2 yp = ld_shared_v2(rcs + RP * 8);
            // the update's pivot-row reads issue before RN(1/p): their latency overlaps it (C3
            // factorization 0.926 -> 0.918 ms with KEY32; windows W <= 24 only: ~10 more registers)
            const int HLO = (s + 1) / 2;
            double2 u2h[KV / 2 + 2];
            if constexpr (HOIST) {
#pragma unroll
                for (int h = HLO; h <= (s + KV) / 2; ++h) u2h[h - HLO] = ld_shared_v2(rcs + h * 16);
            }
#ifdef BANDLU_ROWS_FASTCHAIN
            const int ppos = ppos_f;
            const bool zp = (rinv == 0.0);
#else
            const int ppos = (int)__double_as_longlong(yp.y);
#ifdef BANDLU_ROWS_SHFL_P
            // pivot value straight from the pivot lane (off the record write -> read chain)
            double xpv = x[0];
#pragma unroll
            for (int ri = 1; ri < R; ++ri) xpv = (rb == ri) ? x[ri] : xpv;
            const double p = __shfl_sync(0xffffffffu, xpv, (int)gbase + max(__ffs(gb) - 1, 0));
#else
            const double p = ld_volatile_shared_f64(rcs + s * 8);
#endif
            const bool zp = (p == 0.0);
#endif
#ifndef BANDLU_ROWS_IPIV_STEP
            pv[s] = ppos + 1;  // stored once per block (C3 factorization 0.979 -> 0.960 ms)
#else
            if (is_piv) *ipj = ppos + 1;
#endif
            if (live && zp && linfo == 0) linfo = j + 1;

            // ---- interchange = relabel; the pivot slot retires after this step
            bool pslot[R];
#pragma unroll
            for (int ri = 0; ri < R; ++ri) {
                pslot[ri] = is_piv && rb == ri;
                if (live && pos[ri] == j && !pslot[ri]) pos[ri] = ppos;  // dead groups: no record was written
            }

            // ---- SCAL: multiplier = x * RN(1/p) (DSCAL(ONE/pivot), Q7)
#ifndef BANDLU_ROWS_FASTCHAIN
#ifdef BANDLU_ABL_NORCP
            const double rinv = p;
#else
            const double rinv = __drcp_rn(p);
#endif
#endif
            double lu[R];
#pragma unroll
            for (int ri = 0; ri < R; ++ri) {
                const double l = zp ? x[ri] : __dmul_rn(x[ri], rinv);
                lu[ri] = (cand[ri] && !zp) ? l : 0.0;
#ifndef BANDLU_ABL_NOOUT
                if (cand[ri] && !pslot[ri]) colj[pos[ri] - j] = l;
#endif
            }
            if constexpr (FWD) {
                const double y = yp.x;
#ifdef BANDLU_ROWS_Y_BLOCK
                yv[s] = y;
#else
                if constexpr (YSM) st_shared_f64_if(is_piv, ybuf_s + (uint32_t)j * 8u, y);
                else if (is_piv) bv[j] = y;
#endif
                if (y != 0.0) {
#pragma unroll
                    for (int ri = 0; ri < R; ++ri) bq[ri] = __fma_rn(lu[ri], -y, bq[ri]);
                }
            }
            // ---- RANK-1 update of the window columns j+1..j+KV (DGER, alpha = -1, FMA)
#ifndef BANDLU_ROWS_LDS64
            // 128-bit broadcast reads of slot pairs (2h, 2h+1) covering s+1 .. s+KV: half the
            // load instructions of 64-bit reads for the same shared-memory wavefronts (C3
            // factorization 1.016 -> 0.981 ms)
            if (LA) {
#pragma unroll
                for (int ri = 0; ri < R; ++ri)
                    if (pslot[ri]) pos[ri] = FREE;
            }
#pragma unroll
            for (int h = (s + 1) / 2; h <= (s + KV) / 2; ++h) {
#if defined(BANDLU_ABL_HALF)
                // (timing experiment, wrong results) half the broadcast loads
                const double2 u2 = ld_shared_v2(rcs + ((h & 1) && h > (s + 1) / 2 ? h - 1 : h) * 16);
#else
                const double2 u2 = HOIST ? u2h[h - HLO] : ld_shared_v2(rcs + h * 16);
#endif
#ifdef BANDLU_ROWS_FASTCHAIN
                // column j+1 (slot s+1) uses the shuffled value (bitwise the record's)
                const double ua = (2 * h == s + 1) ? u1 : u2.x, ub = (2 * h + 1 == s + 1) ? u1 : u2.y;
#else
                const double ua = u2.x, ub = u2.y;
#endif
#pragma unroll
                for (int ri = 0; ri < R; ++ri) {
                    if (2 * h >= s + 1) VS(ri, 2 * h + OFF) = __fma_rn(lu[ri], -ua, VS(ri, 2 * h + OFF));
                    if (2 * h + 1 <= s + KV)
                        VS(ri, 2 * h + 1 + OFF) = __fma_rn(lu[ri], -ub, VS(ri, 2 * h + 1 + OFF));
                }
                // column j+1 (slot s+1) is final for step j+1: its pivot search overlaps the
                // rest of this update
                if (LA && h == (s + 1) / 2 && s + 1 < U && j + 1 < mn) search(s + 1 + OFF, j + 1, ps);
            }
#else
#pragma unroll
            for (int k = 1; k <= KV; ++k) {
                const double uk = ld_volatile_shared_f64(rcs + (s + k) * 8);
#pragma unroll
                for (int ri = 0; ri < R; ++ri) VS(ri, s + k + OFF) = __fma_rn(lu[ri], -uk, VS(ri, s + k + OFF));
            }
#endif
#pragma unroll
            for (int ri = 0; ri < R; ++ri)
                if (pslot[ri]) pos[ri] = FREE;
            colj += ldab;
            ++ipj;
        }
        // ---- U rows j0 .. j0+U-1 (the block's records) -> HBM, 32-byte column chunks
        __syncwarp();
#ifdef BANDLU_ABL_NOOUT
        if (j0 < 0) {
#else
        if constexpr (G % U == 0) {
#endif
            const bool rowok = live && j0 + t % U < mn;
            const int c0 = j0 + t / U;
            const uint32_t src0 = rec_s + (uint32_t)(((t % U) * WP + t / U) * 8);
            double *dst = colb + bo0 + KV;
#pragma unroll
            for (int k = 0; k < BIT; ++k) {
                if ((bmask >> k & 1u) && rowok && c0 + k * KS < n)
                    dst[k * kstride] = ld_shared_f64(src0 + (uint32_t)(k * KS * 8));
            }
        } else {
#pragma unroll
            for (int k = 0; k < BIT; ++k) {
                const int e = t + k * G, bs = e % U, bk = e / U;
                if (live && (bmask >> k & 1u) && j0 + bs < mn && j0 + bk < n)
                    colb[boff(k) + KV] = ld_shared_f64(rec_s + (uint32_t)((bs * WP + bk) * 8));
            }
        }
        colb += (int64_t)U * ldab;
#ifndef BANDLU_ROWS_IPIV_STEP
        if (live && t == 0) {
            int *ip = ipiv + j0;
            if (U == 4 && j0 + U <= mn && (reinterpret_cast<uintptr_t>(ip) & 15) == 0) {
                *reinterpret_cast<int4 *>(ip) = make_int4(pv[0], pv[1 % U], pv[2 % U], pv[3 % U]);
            } else {
#pragma unroll
                for (int s = 0; s < U; ++s)
                    if (j0 + s < mn) ip[s] = pv[s];
            }
        }
#endif
#ifdef BANDLU_ROWS_Y_BLOCK
        if constexpr (FWD) {
            if (live && t == 0) {
                double *yp4 = bv + j0;
                if (U == 4 && j0 + U <= mn && (reinterpret_cast<uintptr_t>(yp4) & 15) == 0) {
                    reinterpret_cast<double2 *>(yp4)[0] = make_double2(yv[0], yv[1 % U]);
                    reinterpret_cast<double2 *>(yp4)[1] = make_double2(yv[2 % U], yv[3 % U]);
                } else {
#pragma unroll
                    for (int s = 0; s < U; ++s)
                        if (j0 + s < mn) yp4[s] = yv[s];
                }
            }
        }
#endif
        __syncwarp();
    };
#pragma unroll 1
    for (int j0 = 0; j0 < mn; j0 += C::NBLK * U) {
        blk(std::integral_constant<int, 0>{}, j0);
        if constexpr (C::NBLK == 2) {
            if (j0 + U < mn) blk(std::integral_constant<int, U>{}, j0 + U);
        }
        // shift the window by NBLK*U columns: slot r <- slot r+NBLK*U
        constexpr int SH = C::NBLK * U;
#pragma unroll
        for (int ri = 0; ri < R; ++ri) {
#pragma unroll
            for (int k = 0; k < 2 * H; ++k) {
#ifdef BANDLU_ABL_NOSHIFT
                if (k + SH >= 2 * H) VS(ri, k) = 0.0;
#else
                VS(ri, k) = (k + SH < 2 * H) ? VS(ri, k + SH) : 0.0;
#endif
            }
        }
    }
    cp_async_wait<0>();
    __syncwarp();
#undef VS
    if constexpr (BWD) {  // fused gbsv: U x = y while the other resident matrices still factor
        const bool wr = live && (!SKIPI || linfo == 0);
        backsolve_group<KV, G, YSM>(n, ab, ldab, bv, ybuf_s, live, wr, t, (int)gbase);
    }
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
