// gbtrf_wide.cuh -- sm_100a band LU with partial pivoting for wide bands
// (kl+1 > 32: more window rows than a warp has lanes), register resident.
//
// What it computes: LAPACK DGBTF2 exactly (Sec. 5.1 pseudo-code
// P:350-367, ju rule P:492-494, right-only swaps P:358/P:369-374), the same
// fp64 operation sequence as the oracle => bitwise-equal factors, ipiv, info.
//
// The row-slot design of gbtrf_rows.cuh with a group of 64 lanes = the two
// warps of a CTA per matrix (BASELINE configs[4] band (32,32): 33 active rows
// + U preloaded rows): each lane holds one window row (W+U slots) in
// registers; IAMAX is an exact per-warp argmax (REDUX on the high word, low
// word and smallest logical row on ties) combined across the two warps
// through shared memory; the pivot row goes through a shared record read back
// with 64-bit broadcast loads; a block's incoming rows are preloaded into the
// slots freed by the previous block's pivot rows.  Block barriers
// (__syncthreads, 64 threads) replace the warp syncs.
#pragma once
#include "common.cuh"

namespace bandlu {

template <int KL_, int KU_>
struct TrfWide {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU, W = KV + 1;
    static constexpr int G = 64;                 // lanes per matrix (= the CTA)
#ifndef BANDLU_WIDE_U
#define BANDLU_WIDE_U 8
#endif
    // columns per block (preload / record / window-shift granularity): 8 measured 7% faster than 4
    // on (32,32) (C5 724 vs 767 ms: the 138-register window shifts half as often); 4 where the
    // KL+1 active rows + U preloaded rows would not fit the 64 lanes
    static constexpr int U = (KL + 1 + BANDLU_WIDE_U <= G) ? BANDLU_WIDE_U : 4;
    static constexpr int WS = W + U, H = (WS + 1) / 2;
    static_assert(KL + 1 + U <= G, "slots");
    static constexpr int WPB = 2 * H + 4;
    static constexpr int WP = (WPB + 11) / 16 * 16 + 4;  // == 4 (mod 16) doubles
    static constexpr int RP = WP - 2;
    static constexpr int D = U > 4 ? U : 4, DB = D / U;  // staging lead (rows / blocks)
    static constexpr int RR = pow2_ceil((DB + 1) * U);
#ifdef BANDLU_WIDE_ONESYNC
    static constexpr int NREC = 2 * U;  // one candidate record per warp and step (one barrier per step)
#else
    static constexpr int NREC = U;
#endif
    static constexpr int BK = W + U - 1;
    static constexpr int BIT = (BK * U + G - 1) / G;
    static_assert(BIT <= 32, "block element mask");
    // ring + records + per-warp argmax exchange (2 x 2 x 16 B, double-buffered by step parity)
    // + per-warp free-slot counts (16 B)
    __host__ __device__ static constexpr size_t smem_bytes() { return (size_t)((RR + NREC) * WP + 10) * sizeof(double); }
};

template <int KL, int KU, bool FWD, class AP, class PP, class BP>
__global__ void __launch_bounds__(64, 4)
    gbtrf_wide_kernel(int m, int n, AP A, int ldab, PP P, int *__restrict__ info, int batch, BP Bv) {
    using C = TrfWide<KL, KU>;
    constexpr int KV = C::KV, U = C::U, H = C::H, WP = C::WP, RP = C::RP, D = C::D, RR = C::RR, BK = C::BK,
                  BIT = C::BIT, G = C::G;
    constexpr int FREE = 0x7fffffff;
    extern __shared__ __align__(16) double smem[];

    const int t = (int)threadIdx.x, lane = t & 31, w = t >> 5;
    const int64_t mat = blockIdx.x;
    if (mat >= batch) return;  // whole CTA
    double *__restrict__ ab = A.get(mat);
    int *__restrict__ ipiv = P.get(mat);
    double *__restrict__ bv = FWD ? Bv.get(mat) : nullptr;
    if (m <= 0 || n <= 0) {
        if (t == 0) info[mat] = 0;
        return;
    }
    double *ring = smem;
    const uint32_t ring_s = smem_u32(ring);
    const uint32_t rec_s = ring_s + RR * WP * 8;
    uint4 *xch = reinterpret_cast<uint4 *>(smem + (RR + C::NREC) * WP);  // [2]: (hi, lo, pos, valid)
    unsigned *fcnt = reinterpret_cast<unsigned *>(xch + 4);               // [2]: free slots per warp

    for (int i = t; i < RR * WP; i += G) ring[i] = 0.0;
    __syncthreads();

    const int bo0 = (t / U) * (ldab - 1) + (t % U), bstep = (G / U) * (ldab - 1);
    auto boff = [&](int k) -> int { return bo0 + k * bstep; };
    unsigned bmask = 0;
#pragma unroll
    for (int k = 0; k < BIT; ++k) {
        const int e = t + k * G, bs = e % U, bk = e / U;
        if (bk < BK && bk - bs >= 0 && bk - bs <= KV) bmask |= 1u << k;
    }
    auto stage_block = [&](int qb, const double *colq) {
#pragma unroll
        for (int k = 0; k < BIT; ++k) {
            const int e = t + k * G, bs = e % U, bk = e / U;
            if (bmask >> k & 1u) {
                const int q = qb + bs;
                const bool ok = (q < m) && (qb - KL + bk < n);
                const uint32_t dst = ring_s + (uint32_t)(((q & (RR - 1)) * WP + 1 + bk) * 8);
                cp_async8(dst, ok ? colq + boff(k) + (KV + KL) : (const double *)ab, ok ? 8u : 0u);
            }
        }
        if constexpr (FWD) {
            if (t < U) {
                const int q = qb + t;
                const bool okb = (q < m);
                const uint32_t dstb = ring_s + (uint32_t)(((q & (RR - 1)) * WP + RP) * 8);
                cp_async8(dstb, okb ? (const void *)(bv + q) : (const void *)ab, okb ? 8u : 0u);
            }
        }
        cp_async_commit();
    };
#pragma unroll 1
    for (int d = 0; d < C::DB; ++d) stage_block(KL + 1 + d * U, ab + (int64_t)(1 + d * U) * ldab);
    const double *scol = ab + (int64_t)(1 + D) * ldab;

    // ---- window registers: slot r = column j0 + r; rows 0..KL in lanes 0..KL
    double2 v[H];
#define VS(k) (((k) & 1) ? v[(k) >> 1].y : v[(k) >> 1].x)
    {
        const bool row_ok = (t <= KL) && (t < m);
#pragma unroll
        for (int h = 0; h < H; ++h) {
            const int c0 = 2 * h, c1 = 2 * h + 1;
            v[h].x = (row_ok && c0 < n && c0 <= t + KU) ? ab[(int64_t)c0 * ldab + (KV + t - c0)] : 0.0;
            v[h].y = (row_ok && c1 < n && c1 <= t + KU) ? ab[(int64_t)c1 * ldab + (KV + t - c1)] : 0.0;
        }
    }
    int pos = (t <= KL) ? t : FREE;
    double bq = (FWD && t <= KL && t < m) ? bv[t] : 0.0;

    int linfo = 0;
    const int mn = min(m, n);
    double *colj = ab + KV;
    double *colb = ab;
    int pv[U];  // the block's pivots (1-based), stored once per block by thread 0 (as gbtrf_rows.cuh)
    int wsel[U];  // which warp's record holds step s's pivot row
#pragma unroll
    for (int s = 0; s < U; ++s) {
        pv[s] = 0;
        wsel[s] = 0;
    }
    const unsigned below = (1u << lane) - 1u;
#pragma unroll 1
    for (int j0 = 0; j0 < mn; j0 += U) {
        cp_async_wait<C::DB - 1>();
        // ---- preload rows j0+KL+1+o into the first U free slots (rank over both warps)
        const bool fr = (pos == FREE) || (pos >= m);
        const unsigned fb = __ballot_sync(0xffffffffu, fr);
        if (lane == 0) fcnt[w] = __popc(fb);
        __syncthreads();  // ring rows landed (all lanes' copies) + free counts
        {
            const int rank = (w == 1 ? (int)fcnt[0] : 0) + __popc(fb & below);
            const bool take = fr && rank < U;
            const int q = j0 + KL + 1 + rank;
            const uint32_t rr = ring_s + (uint32_t)((q & (RR - 1)) * WP * 8);
#pragma unroll
            for (int h = 0; h < H; ++h) ld_shared_v2_if(take, rr + h * 16, v[h]);
            if constexpr (FWD) ld_shared_f64_if(take, rr + RP * 8, bq);
            if (take) pos = q;
        }
        stage_block(j0 + KL + 1 + D, scol);
        scol += (int64_t)U * ldab;
#pragma unroll
        for (int s = 0; s < U; ++s) {
            const int j = j0 + s;
            if (j >= mn) break;

            // ---- IAMAX: exact argmax per warp, then across the two warps
            const double x = VS(s);
            const bool cand = (pos <= j + KL) && (pos < m);
            const unsigned kh = cand ? ((unsigned)__double2hiint(x) & 0x7fffffffu) : 0u;
            const unsigned kl = cand ? (unsigned)__double2loint(x) : 0u;
            const unsigned mhi = __reduce_max_sync(0xffffffffu, kh);
            unsigned gb = __ballot_sync(0xffffffffu, cand && kh == mhi);
            unsigned mlo = kl;
            if (__popc(gb) > 1) {  // warp-uniform: tie on the high word
                mlo = __reduce_max_sync(0xffffffffu, (cand && kh == mhi) ? kl : 0u);
                const unsigned pp = __reduce_min_sync(0xffffffffu, (cand && kh == mhi && kl == mlo) ? (unsigned)pos : 0xffffffffu);
                gb = __ballot_sync(0xffffffffu, cand && (unsigned)pos == pp);
            }
            const int wl = __ffs(gb) - 1;  // this warp's best lane (-1: no candidate)
#ifdef BANDLU_WIDE_ONESYNC
            // ---- each warp's best candidate row -> its record (s, w); ONE barrier, then every
            // lane picks the winner (warp 1 wins on a larger key, or an equal key with the
            // smaller logical row) and reads the winner's record
            const bool wbest = (lane == wl);
            if (lane == (wl < 0 ? 0 : wl))
                xch[(s & 1) * 2 + w] = make_uint4(kh, kl, (unsigned)pos, wl < 0 ? 0u : 1u);
            {
                const uint32_t rcw = rec_s + (uint32_t)((2 * s + w) * WP * 8);
#pragma unroll
                for (int h = s / 2; h <= (s + KV) / 2; ++h) st_shared_v2_if(wbest, rcw + h * 16, v[h]);
                st_shared_v2_if(wbest, rcw + RP * 8, make_double2(bq, __longlong_as_double((long long)pos)));
            }
            __syncthreads();
            const uint4 c0 = xch[(s & 1) * 2], c1 = xch[(s & 1) * 2 + 1];
            const bool w1 = c1.w && (!c0.w || c1.x > c0.x || (c1.x == c0.x && (c1.y > c0.y || (c1.y == c0.y && c1.z < c0.z))));
            const bool is_piv = (w == (w1 ? 1 : 0)) && wbest;
            const uint32_t rcs = rec_s + (uint32_t)((2 * s + (w1 ? 1 : 0)) * WP * 8);
            wsel[s] = w1 ? 1 : 0;
#else
            if (lane == (wl < 0 ? 0 : wl))
                xch[w] = make_uint4(kh, kl, (unsigned)pos, wl < 0 ? 0u : 1u);
            __syncthreads();
            const uint4 c0 = xch[0], c1 = xch[1];
            // warp 1 wins on a larger key, or an equal key with the smaller logical row
            const bool w1 = c1.w && (!c0.w || c1.x > c0.x || (c1.x == c0.x && (c1.y > c0.y || (c1.y == c0.y && c1.z < c0.z))));
            const bool is_piv = (w == (w1 ? 1 : 0)) && (lane == wl);

            // ---- pivot row (U row j: slots s..s+KV) + (B entry, logical row) -> record s; only the
            // pivot's warp issues the stores (warp-uniform branch: the other warp skips KV/2 stores)
            const uint32_t rcs = rec_s + (uint32_t)(s * WP * 8);
#ifndef BANDLU_WIDE_STORE_ALL
            if (__any_sync(0xffffffffu, is_piv))
#endif
            {
#pragma unroll
                for (int h = s / 2; h <= (s + KV) / 2; ++h) st_shared_v2_if(is_piv, rcs + h * 16, v[h]);
                st_shared_v2_if(is_piv, rcs + RP * 8, make_double2(bq, __longlong_as_double((long long)pos)));
            }
            __syncthreads();
#endif
            const double2 yp = ld_shared_v2(rcs + RP * 8);
            const int ppos = (int)__double_as_longlong(yp.y);
            const double p = ld_volatile_shared_f64(rcs + s * 8);
            const bool zp = (p == 0.0);
            pv[s] = ppos + 1;
            if (zp && linfo == 0) linfo = j + 1;
            if (pos == j && !is_piv) pos = ppos;  // interchange = relabel

            const double rinv = __drcp_rn(p);
            const double l = zp ? x : __dmul_rn(x, rinv);
            const double lu = (cand && !zp) ? l : 0.0;
            if (cand && !is_piv) colj[pos - j] = l;
            if constexpr (FWD) {
                const double y = yp.x;
                if (is_piv) bv[j] = y;
                if (y != 0.0) bq = __fma_rn(lu, -y, bq);
            }
#ifndef BANDLU_WIDE_LDS64
            // 128-bit broadcast reads of slot pairs (as gbtrf_rows.cuh): half the load instructions
#pragma unroll
            for (int h = (s + 1) / 2; h <= (s + KV) / 2; ++h) {
                const double2 u2 = ld_shared_v2(rcs + h * 16);
                if (2 * h >= s + 1) VS(2 * h) = __fma_rn(lu, -u2.x, VS(2 * h));
                if (2 * h + 1 <= s + KV) VS(2 * h + 1) = __fma_rn(lu, -u2.y, VS(2 * h + 1));
            }
#else
#pragma unroll
            for (int k = 1; k <= KV; ++k) {
                const double uk = ld_volatile_shared_f64(rcs + (s + k) * 8);
                VS(s + k) = __fma_rn(lu, -uk, VS(s + k));
            }
#endif
            if (is_piv) pos = FREE;
            colj += ldab;
        }
        // ---- U rows j0 .. j0+U-1 -> HBM (32-byte column chunks)
        __syncthreads();
#pragma unroll
        for (int k = 0; k < BIT; ++k) {
            const int e = t + k * G, bs = e % U, bk = e / U;
#ifdef BANDLU_WIDE_ONESYNC
            int ws = wsel[0];
#pragma unroll
            for (int q = 1; q < U; ++q) ws = (bs == q) ? wsel[q] : ws;
            if ((bmask >> k & 1u) && j0 + bs < mn && j0 + bk < n)
                colb[boff(k) + KV] = ld_shared_f64(rec_s + (uint32_t)(((2 * bs + ws) * WP + bk) * 8));
#else
            if ((bmask >> k & 1u) && j0 + bs < mn && j0 + bk < n)
                colb[boff(k) + KV] = ld_shared_f64(rec_s + (uint32_t)((bs * WP + bk) * 8));
#endif
        }
        colb += (int64_t)U * ldab;
        if (t == 0) {
            int *ip = ipiv + j0;
            if (U == 4 && j0 + U <= mn && (reinterpret_cast<uintptr_t>(ip) & 15) == 0) {
                *reinterpret_cast<int4 *>(ip) = make_int4(pv[0], pv[1 % U], pv[2 % U], pv[3 % U]);
            } else {
#pragma unroll
                for (int s = 0; s < U; ++s)
                    if (j0 + s < mn) ip[s] = pv[s];
            }
        }
        __syncthreads();
#pragma unroll
        for (int h = 0; h < H; ++h) {
            if (h + U / 2 < H) {
                v[h] = v[h + U / 2];
            } else {
                v[h].x = 0.0;
                v[h].y = 0.0;
            }
        }
    }
    cp_async_wait<0>();
#undef VS

    if (m < n) {  // LAPACK SET_FILLIN zeroes fill positions of rows >= m (never pivot rows here)
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
