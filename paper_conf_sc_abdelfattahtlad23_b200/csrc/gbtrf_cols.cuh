// gbtrf_cols.cuh -- sm_100a band LU with partial pivoting for thin lower bands
// (kl <= 4): the lanes of a group own COLUMNS of the sliding window.
//
// What it computes: LAPACK DGBTF2 exactly (Sec. 5.1 pseudo-code
// P:350-367, ju rule P:492-494, right-only swaps P:358/P:369-374), the same
// fp64 operation sequence as the oracle => bitwise-equal factors, ipiv, info;
// with FL_FWD also the forward substitution of nrhs <= GL right-hand sides (DGBTRS
// 'N' first loop) on the fly: lane t carries right-hand side t as one
// more column slot, so y never round-trips through HBM before the backward solve.
//
// Why ("gbtrf_cols"): the row-slot kernel gives every lane a
// row of the window (kl+ku+1 doubles) and broadcasts the pivot row each step;
// for kl <= 4 most of a group's lanes hold incoming rows, the window costs
// 2(kl+ku+5) registers per lane and each step is ~1,000 cycles of latency.
// Here a group of GL lanes holds the window column-wise: lane t keeps CPL
// column slots, each with the kl+1 active rows of its column (positions
// 0..kl = logical rows j..j+kl), so a step is
//   * IAMAX over column j by its owner lane (kl+1 registers, first max),
//   * RN(1/pivot), the kl multipliers by the owner and one shuffle each,
//   * per column slot: u = a[p], the interchange by selects (rows j <-> j+p,
//     columns j..j+kv, "right only"), kl FMAs, U(j, c) = u to a staging row,
// and the window moves by renaming positions (row j retires, row j+kl+1
// enters as position kl from a shared-memory staging block).  Column c lives
// in ring slot c mod (GL*CPL); the owner of column j is lane j mod GL.
// Input rows arrive as 32-byte column chunks (4 rows x 1 column, cp.async, two
// blocks ahead); U rows leave the same way, one 4-row block at a time; the
// multipliers are stored by the owner lane.
#pragma once
#include "backsolve_fused.cuh"
#include "common.cuh"

namespace bandlu {

template <int KL_, int KU_, int GL_, int CPL_>
struct TrfCols {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU, W = KV + 1;
    static constexpr int GL = GL_, CPL = CPL_, NR = GL * CPL, GPW = 32 / GL;
    static_assert(NR >= W, "column ring covers the window");
    static_assert(GL >= 4 && GL % 4 == 0 && 32 % GL == 0, "group size");
    static constexpr int UB = 4;                  // rows per staging / output block
    static constexpr int BK = KV + UB;            // columns per block (cc = c - j0b)
    static constexpr int BKP = ((BK + 1) / 2) * 2;  // row pitch (doubles), 16-byte rows
    static constexpr int NSB = 4;                 // staging ring (pow2): two blocks ahead
    static constexpr int BIT = (BK * UB + GL - 1) / GL;
    // per group: NSB staging blocks + one output block (UB x BKP each) + NSB x UB x GL entries of
    // the right-hand sides (FL_FWD: lane t carries right-hand side t, nrhs <= GL)
    // (the right-hand-side staging only with FL_FWD)
    __host__ __device__ static constexpr int group_dbl(bool fwd) { return (NSB + 1) * UB * BKP + (fwd ? NSB * UB * GL : 0); }
    static constexpr int GROUP_DBL = group_dbl(true);
    static constexpr int WARPS = 4;
    static constexpr size_t smem_bytes(bool fwd = true) { return (size_t)WARPS * GPW * group_dbl(fwd) * sizeof(double); }
    static constexpr int minb_smem(bool fwd) { return (int)((227 * 1024) / smem_bytes(fwd)); }
    // resident CTAs per SM, shared memory permitting: 4 (128 registers) for the small windows;
    // C4's (2,32) (16 lanes x 3 slots, 120-136 registers since the UB-step passes) measured best at
    // 3 for the factorization alone (1.10 ms; 1.18 at 4) and 2-3 with the 16 right-hand sides
#ifndef BANDLU_COLS_MINB
#define BANDLU_COLS_MINB(fwd) (CPL * (KL + 1) >= 9 ? ((fwd) && GL >= 16 ? 2 : 3) : 4)
#endif
    static constexpr int minb(bool fwd) {
        return minb_smem(true) < BANDLU_COLS_MINB(fwd) ? (minb_smem(true) < 1 ? 1 : minb_smem(true)) : BANDLU_COLS_MINB(fwd);
    }
    static constexpr int MINB = minb(false);
};

// |x| as a 64-bit integer key from the two words (integer ops only; the 64-bit
// mask form compiles to DADD |x| on the FP64 pipe)
__device__ __forceinline__ uint64_t abs_key_w(double x) {
    const unsigned hi = (unsigned)__double2hiint(x) & 0x7fffffffu, lo = (unsigned)__double2loint(x);
    return ((uint64_t)hi << 32) | lo;
}

template <int KL, int KU, int GL, int CPL, int FL, class AP, class PP, class BP>
__global__ void __launch_bounds__(TrfCols<KL, KU, GL, CPL>::WARPS * 32, TrfCols<KL, KU, GL, CPL>::minb((FL & 1) != 0))
    gbtrf_cols_kernel(int n, AP A, int ldab, PP P, int *__restrict__ info, int batch, BP Bv, int nrhs, int ldb) {
    using C = TrfCols<KL, KU, GL, CPL>;
    constexpr bool FWD = FL & 1, BWD = FL & 2;  // FL_FWD, FL_BWD (gbtrf_rows.cuh)
    static_assert(!BWD || (FWD && FusedSolveAny<KL + KU, GL>::ok), "fused backward solve");
    constexpr int KV = C::KV, NR = C::NR, UB = C::UB, BK = C::BK, BKP = C::BKP, NSB = C::NSB, BIT = C::BIT;
    static_assert((NSB & (NSB - 1)) == 0, "staging ring");
    extern __shared__ __align__(16) double smem[];

    const int lane = (int)lane_id(), wib = (int)(threadIdx.x >> 5);
    const int g = lane / GL, t = lane % GL;
    const int gbase = g * GL;
    const int64_t mat = ((int64_t)blockIdx.x * C::WARPS + wib) * C::GPW + g;
    const bool live = mat < batch;
    if (__ballot_sync(0xffffffffu, live) == 0u) return;
    double *__restrict__ ab = live ? A.get(mat) : g_dummy;
    int *__restrict__ ipiv = live ? P.get(mat) : nullptr;
    // FWD: lane t owns right-hand side t (t < nrhs <= GL), B(:, t) = bcol[0 .. n-1]
    const bool rown = FWD && live && t < nrhs;
    double *__restrict__ bcol = rown ? Bv.get(mat) + (int64_t)t * ldb : g_dummy;
    // loop control uses n (the same for every group of the warp); memory predicates use nl
    // (0 for dead groups, so they run the same instruction stream without touching memory)
    const int nl = live ? n : 0;

    double *grp = smem + (size_t)(wib * C::GPW + g) * C::GROUP_DBL;
    const uint32_t stage_s = smem_u32(grp);                              // NSB x [UB][BKP]
    const uint32_t out_s = stage_s + NSB * UB * BKP * 8;                 // [UB][BKP]
    const uint32_t bst_s = out_s + UB * BKP * 8;                         // NSB x [UB][GL] RHS entries

    // ---- block transfers: lane t moves row offset so = t % UB, columns cc = t / UB + i * GL / UB
    const int so = t % UB, cc0 = t / UB;
    const int64_t xstride = (int64_t)(GL / UB) * (ldab - 1);
    // staging of block b (rows q0 = 4b+KL .. +3, entering at steps 4b .. 4b+3):
    // element (o, cc) = A(q0+o, 4b+cc) = AB(KV+q0+o-c, c), in band iff 0 <= cc-o <= KV
    auto stage_block = [&](int b) {
        const int j0b = b * UB;
        const double *src = ab + (int64_t)j0b * ldab + (int64_t)cc0 * (ldab - 1) + (KV + KL + so);
        const uint32_t dst0 = stage_s + (uint32_t)((((b & (NSB - 1)) * UB + so) * BKP + cc0) * 8);
        const bool rowok = (j0b + KL + so) < nl;
#pragma unroll
        for (int i = 0; i < BIT; ++i) {
            const int cc = cc0 + i * (GL / UB);
            // cc >= BK would land in the next staging row (pitch BKP = BK): no copy at all (a
            // zero-fill there raced with the real copy of that element)
            if (i * (GL / UB) < BK && cc < BK) {
                const bool ok = rowok && (cc - so >= 0) && (cc - so <= KV) && (j0b + cc < nl);
                cp_async8(dst0 + (uint32_t)(i * (GL / UB) * 8), ok ? (const void *)(src + i * xstride) : (const void *)g_dummy,
                          ok ? 8u : 0u);
            }
        }
        if constexpr (FWD) {  // rows q0 .. q0+3 of this lane's right-hand side (zeros past n / unowned)
            // (16-byte pairs with the entries held in registers for the block measured slower: C4
            // factorization + forward 1.99 vs 1.92 ms)
#pragma unroll
            for (int o = 0; o < UB; ++o) {
                const int q = j0b + KL + o;
                const bool ok = rown && q < nl;
                cp_async8(bst_s + (uint32_t)((((b & (NSB - 1)) * UB + o) * GL + t) * 8),
                          ok ? (const void *)(bcol + q) : (const void *)g_dummy, ok ? 8u : 0u);
            }
        }
        cp_async_commit();
    };
    // output block b: U(4b+o, 4b+cc) = AB(KV+o-cc, 4b+cc)
    auto flush_block = [&](int b) {
        __syncwarp();
        const int j0b = b * UB;
        double *dst = ab + (int64_t)j0b * ldab + (int64_t)cc0 * (ldab - 1) + (KV + so);
        const uint32_t src0 = out_s + (uint32_t)((so * BKP + cc0) * 8);
        const bool rowok = (j0b + so) < nl;
#pragma unroll
        for (int i = 0; i < BIT; ++i) {
            const int cc = cc0 + i * (GL / UB);
            if (i * (GL / UB) < BK) {
                const bool ok = rowok && cc < BK && (cc - so >= 0) && (cc - so <= KV) && (j0b + cc < nl);
                // (cc >= BK would read past the output block -- past the group's shared memory for
                // the last group of a CTA: predicated off, like the store)
                double x = 0.0;
                ld_shared_f64_if(cc < BK, src0 + (uint32_t)(i * (GL / UB) * 8), x);
                st_global_f64_if(ok, dst + i * xstride, x);
            }
        }
        __syncwarp();
    };

    // ---- window registers: a[k][r] = A(j+r, c_k) for the column c_k of slot k
    double a[CPL][KL + 1];
    double bc[KL + 1];  // FWD: entries j..j+KL of this lane's right-hand side
    double yv[UB];      // FWD: y(j0b .. j0b+3) of this lane's right-hand side, stored per block
#pragma unroll
    for (int o = 0; o < UB; ++o) yv[o] = 0.0;
    const bool a16y = ((reinterpret_cast<uintptr_t>(bcol) & 15) == 0);
#pragma unroll
    for (int k = 0; k < CPL; ++k) {
        const int c = k * GL + t;
#pragma unroll
        for (int r = 0; r <= KL; ++r) {
            const bool ok = (r < KL) && c < nl && r < nl && (r - c <= KL) && (c - r <= KU);
            a[k][r] = ok ? ab[(int64_t)c * ldab + (KV + r - c)] : 0.0;
        }
    }
#pragma unroll
    for (int r = 0; r <= KL; ++r) bc[r] = (rown && r < KL && r < nl) ? bcol[r] : 0.0;

    stage_block(0);
    stage_block(1);
    int linfo = 0;
    int pv[UB];
#pragma unroll
    for (int o = 0; o < UB; ++o) pv[o] = 0;
    double *lcol = ab + KV;  // &AB(KV, j): the multipliers of column j follow

    // ---- the entries of row j+KL (position KL at step j), read from the staging block one step
    // ahead so that the shared-memory latency is off the step's chain.  sn = the step's offset in
    // its ring turn (j0 = j - sn); the column of slot k at that step:
    double inc[CPL], incb = 0.0;
    auto fetch_incoming = [&](int j, int sn, int j0) {
        const int o = j % UB, b = j / UB;
        const uint32_t srow = stage_s + (uint32_t)((((b & (NSB - 1)) * UB + o) * BKP - (j - o)) * 8);
#pragma unroll
        for (int k = 0; k < CPL; ++k) {
            const int c = (k == 0 && t < sn) ? j0 + NR + t : j0 + k * GL + t;  // slot 0 of lanes < sn: next turn
            const bool ok = (c - j <= KV) && (j + KL < nl) && (c < nl);
            double x = 0.0;
            ld_shared_f64_if(ok, srow + (uint32_t)(c * 8), x);
            inc[k] = x;
        }
        if constexpr (FWD) {
            double x = 0.0;
            ld_shared_f64_if(rown, bst_s + (uint32_t)((((b & (NSB - 1)) * UB + o) * GL + t) * 8), x);
            incb = x;
        }
    };
    cp_async_wait<1>();  // block 0 landed
    __syncwarp();
    fetch_incoming(0, 0, 0);

#pragma unroll 1
    for (int j0 = 0; j0 < n; j0 += GL) {
        // [r2b] the GL steps of a ring turn run as GL/UB passes of an UB-step unrolled body: only the
        // step's position in its staging block (o) indexes registers; the owner lane (s) is a
        // run-time value (C4, GL = 16: code 4x smaller -- the instruction-cache misses were 12.6% of
        // the stall samples -- and 120-136 instead of 168-210 registers)
#ifdef BANDLU_COLS_FULL_UNROLL
#define BANDLU_COLS_SB_STEP GL
#else
#define BANDLU_COLS_SB_STEP UB
#endif
#pragma unroll 1
        for (int sb = 0; sb < GL && j0 + sb < n; sb += BANDLU_COLS_SB_STEP) {
#pragma unroll
        for (int so_ = 0; so_ < BANDLU_COLS_SB_STEP; ++so_) {
            const int s = sb + so_;
            const int j = j0 + s, o = so_ % UB, b = j / UB;
            if (j >= n) break;
            if (o == 0) stage_block(b + 2);
            // ---- row j+KL enters as position KL (zero outside its band / beyond n)
#pragma unroll
            for (int k = 0; k < CPL; ++k) a[k][KL] = inc[k];
#ifndef BANDLU_ABL_NOBIN
            if constexpr (FWD) bc[KL] = incb;
#endif

            // ---- owner of column j (lane s, slot 0): IAMAX (first max |x|, exact keys), RN(1/pivot)
#ifdef BANDLU_COLS_SPEC
            double rc[KL + 1];
#pragma unroll
            for (int r = 0; r <= KL; ++r) rc[r] = drcp_rn_nz(a[0][r]);
#endif
            int p = 0;
            {
                uint64_t kb = abs_key_w(a[0][0]);
#pragma unroll
                for (int r = 1; r <= KL; ++r) {
                    const uint64_t kr = abs_key_w(a[0][r]);
                    const bool better = (j + r < n) && kr > kb;
                    kb = better ? kr : kb;
                    p = better ? r : p;
                }
            }
            const bool own = (t == s);
            double piv = a[0][0];
#pragma unroll
            for (int r = 1; r <= KL; ++r) piv = (p == r) ? a[0][r] : piv;
            const bool zpl = (piv == 0.0);
#ifdef BANDLU_COLS_SPEC
            double rinv = rc[0];
#pragma unroll
            for (int r = 1; r <= KL; ++r) rinv = (p == r) ? rc[r] : rinv;
#else
            // (the slow-path CALL of RN(1/x) serialises speculative reciprocals: one, after the search)
            const double rinv = drcp_rn_nz(own ? piv : 1.0);
#endif
            // multipliers (DSCAL(ONE/pivot): x * RN(1/pivot), Q7) -> L(j+r, j); update factors
            double e[KL + 1];
#pragma unroll
            for (int r = 1; r <= KL; ++r) {
                const double xr = (p == r) ? a[0][0] : a[0][r];
                const double l = zpl ? xr : __dmul_rn(xr, rinv);
                st_global_f64_if(own && j + r < nl, lcol + r, l);
                e[r] = (zpl || j + r >= n) ? 0.0 : l;
            }
            const int pz = __shfl_sync(0xffffffffu, p | ((int)zpl << 4), gbase + s);
            p = pz & 15;
            const bool zp = (pz >> 4) != 0;
#pragma unroll
            for (int r = 1; r <= KL; ++r) e[r] = __shfl_sync(0xffffffffu, e[r], gbase + s);
            pv[o] = j + p + 1;
            if (zp && linfo == 0) linfo = j + 1;
            lcol += ldab;

            // ---- interchange + rank-1 update of every column slot (DGER, alpha = -1, FMA)
            const uint32_t orow = out_s + (uint32_t)((o * BKP - (j - o)) * 8);
#pragma unroll
            for (int k = 0; k < CPL; ++k) {
                const int c = (k == 0 && t < s) ? j0 + NR + t : j0 + k * GL + t;
                double u = a[k][0];
#pragma unroll
                for (int r = 1; r <= KL; ++r) u = (p == r) ? a[k][r] : u;
                // U(j, c) for the window columns c = j .. j+KV
                st_shared_f64_if((c >= j) && (c - j <= KV), orow + (uint32_t)(c * 8), u);
                double v[KL + 1];
#pragma unroll
                for (int r = 1; r <= KL; ++r) v[r] = __fma_rn(e[r], -u, (p == r) ? a[k][0] : a[k][r]);
#pragma unroll
                for (int r = 1; r <= KL; ++r) a[k][r - 1] = v[r];
                if (k == 0 && own) {  // column j retires; the slot starts column j + NR (zero rows)
#pragma unroll
                    for (int r = 0; r < KL; ++r) a[0][r] = 0.0;
                }
            }
            if constexpr (FWD) {  // the right-hand side columns: same interchange, DGER zero skip (per column)
                double y = bc[0];
#pragma unroll
                for (int r = 1; r <= KL; ++r) y = (p == r) ? bc[r] : y;
#ifdef BANDLU_COLS_YSTEP
                st_global_f64_if(rown && j < nl, bcol + j, y);
#else
                yv[o] = y;  // stored per 4-row block (a store per step cost 17% at C2)
#endif
                double v[KL + 1];
#pragma unroll
                for (int r = 1; r <= KL; ++r) {
                    v[r] = (p == r) ? bc[0] : bc[r];
                    fma_rn_if(y != 0.0, e[r], -y, v[r]);
                }
#pragma unroll
                for (int r = 1; r <= KL; ++r) bc[r - 1] = v[r];
            }
            // ---- block end: U rows and pivots of the 4 steps
            if (o == UB - 1 || j + 1 == n) {
                flush_block(b);
#ifndef BANDLU_COLS_YSTEP
                if constexpr (FWD) {
                    double *yd = bcol + (j - o);
                    if (o == UB - 1 && a16y) {  // predicated-off lanes move nothing
                        if (rown) {
                            reinterpret_cast<double2 *>(yd)[0] = make_double2(yv[0], yv[1 % UB]);
                            reinterpret_cast<double2 *>(yd)[1] = make_double2(yv[2 % UB], yv[3 % UB]);
                        }
                    } else {
#pragma unroll
                        for (int q = 0; q < UB; ++q) st_global_f64_if(rown && q <= o, yd + q, yv[q]);
                    }
                }
#endif
                if (live && t == 0) {
                    int *ip = ipiv + (j - o);
                    if (o == UB - 1 && (reinterpret_cast<uintptr_t>(ip) & 15) == 0) {
                        *reinterpret_cast<int4 *>(ip) = make_int4(pv[0], pv[1 % UB], pv[2 % UB], pv[3 % UB]);
                    } else {
#pragma unroll
                        for (int q = 0; q < UB; ++q)
                            if (q <= o) ip[q] = pv[q];
                    }
                }
            }
            // ---- next step's incoming entries (its block landed: wait for it at this block's end)
            if (j + 1 < n) {
                if (o == UB - 1) {
                    cp_async_wait<1>();
                    __syncwarp();
                }
                const bool turn = (s + 1 == GL);  // the next ring turn (slots rotate below)
                fetch_incoming(j + 1, turn ? 0 : s + 1, turn ? j0 + GL : j0);
            }
        }
        }
#undef BANDLU_COLS_SB_STEP
        // ---- ring turn: slot k <- slot k+1, the retired slot 0 (columns j0+NR+t) goes last
#pragma unroll
        for (int r = 0; r <= KL; ++r) {
            const double x0 = a[0][r];
#pragma unroll
            for (int k = 0; k + 1 < CPL; ++k) a[k][r] = a[k + 1][r];
            a[CPL - 1][r] = x0;
        }
    }
    cp_async_wait<0>();
    if constexpr (BWD) {  // [r2b] the fused gbsv kernel: U x = y by the same lanes (one right-hand side,
        // y(j) left in B(:,0) by lane 0, the U rows flushed above; backsolve_fused.cuh)
        __syncwarp();
        backsolve_group<KV, GL, false, FusedSolveAny<KV, GL>::PF>(n, ab, ldab, live ? Bv.get(mat) : g_dummy, 0u,
                                                                  live, live, t, gbase);
    }
    if (live && t == 0) info[mat] = (n > 0) ? linfo : 0;
}

}  // namespace bandlu
