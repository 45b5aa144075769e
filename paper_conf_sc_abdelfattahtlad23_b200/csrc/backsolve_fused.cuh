// backsolve_fused.cuh -- the backward substitution U x = y run by the lanes of
// a factorization kernel right after they factored their matrix: the fused
// gbsv kernel (Sec. 7 P:688-697 fuses factorization
// and solve into one kernel; the forward substitution already rides inside the
// factorization, see gbtrf_rows.cuh FWD).  One launch per dgbsv / dgbtrfs call
// instead of two, and the backward pass of a matrix overlaps the factorization
// of the other matrices resident on the SM.
//
// What it computes: DTBSV('U','N','N') with bandwidth kv for one right-hand
// side, exactly the oracle's order (reading Q9):
//   for j = n-1 .. 0:  if y(j) != 0:  x(j) = y(j) / U(j,j)   (true division)
//                                      y(i) = fma(-x(j), U(i,j), y(i)),
//                                      i = j-1 .. max(0, j-kv)
// Every y(i) receives its updates in decreasing j, as in the column loop.
//
// Mapping: the G lanes of a matrix group own the right-hand-side rows
// i == t (mod G).  At step j lane t holds two of them: yA = row j - e (the
// near one, distance e = (j - t) mod G) and yB = row j - e - G.  The lane with
// e == 0 owns the pivot row: it divides, one shuffle broadcasts x(j), the
// lanes whose rows are within kv of j apply one FMA each, and the owner then
// shifts yA <- yB.  Its next row (j - 2G) is read into a staging ring and
// merged into yB PF steps later (kv + 1 + PF <= 2G, so before that row enters
// the window): no instruction of the following steps waits for that load.
// The loop is unrolled by G steps over a G-aligned range (steps above n-1 are
// empty), so every lane role of a step -- owner, merging lane, ring slot -- is
// a compile-time constant.  U(i, j) = AB(kv - (j - i), j): a column's U entries
// are contiguous in band storage, so lane t's two prefetch loads per step
// (distances e and e + G) are two coalesced segments over the group, issued PF
// steps ahead into a register ring.
#pragma once
#include "common.cuh"

#ifndef BANDLU_FUSED_PF
#define BANDLU_FUSED_PF 8
#endif

namespace bandlu {

template <int KV, int G>
struct FusedSolve {
    static constexpr int PF = BANDLU_FUSED_PF;
    // two rows per lane suffice and the staging ring has PF steps before a row is used
    static constexpr bool ok = (KV + 1 + PF <= 2 * G) && (G % PF == 0 || PF % G == 0) && G >= 2;
};
// [r2b] the largest prefetch distance PF <= BANDLU_FUSED_PF (a power of two) that still satisfies
// the constraints: small groups (the column-owner kernel's 4 lanes) with a shorter lead
template <int KV, int G>
struct FusedSolveAny {
    static constexpr int pf(int x) {
        return x < 1 ? 0 : ((KV + 1 + x <= 2 * G) && (G % x == 0 || x % G == 0)) ? x : pf(x / 2);
    }
    static constexpr int PF = pf(BANDLU_FUSED_PF);
    static constexpr bool ok = PF > 0 && G >= 2;
};

// YSM: y(i) read from shared memory at ybuf_s + 8 i (else from bx[i], where the
// forward pass left it).  wr: this group stores x into bx (false for dead
// groups and, for dgbsv, where info > 0).  All 32 lanes of the warp call.
template <int KV, int G, bool YSM, int PF_ = FusedSolve<KV, G>::PF>
__device__ __forceinline__ void backsolve_group(int n, const double *ab, int ldab, double *bx, uint32_t ybuf_s,
                                                bool live, bool wr, int t, int gbase) {
    constexpr int PF = PF_;
    static_assert((KV + 1 + PF <= 2 * G) && (G % PF == 0 || PF % G == 0) && G >= 2,
                  "fused backward solve: needs kv + 1 + PF <= 2G");
    constexpr unsigned FULL = 0xffffffffu;
    constexpr int NR = PF > G ? PF : G;  // ring period (unroll)
    auto yload = [&](bool p, int r, double &v) {  // predicated: v unchanged where !p
        if constexpr (YSM) ld_shared_f64_if(p, ybuf_s + (uint32_t)r * 8u, v);
        else ld_global_f64_if(p, bx + r, v);
    };
    const int jt = ((n + NR - 1) / NR) * NR - 1;  // first step: a multiple of NR minus 1 (>= n-1)
    // lane t at step jt: e = (jt - t) mod G = G-1-t; yA = row jt-e, yB = row jt-e-G
    double yA = 0.0, yB = 0.0;
    {
        const int rA = jt - (G - 1 - t), rB = rA - G;
        yload(live && rA >= 0 && rA < n, rA, yA);
        yload(live && rB >= 0 && rB < n, rB, yB);
    }
    // staged refills, slot = step % PF; the lanes that merge during the first PF
    // steps (no staging has happened yet) merge the yB they already hold
    double stg[PF];
#pragma unroll
    for (int k = 0; k < PF; ++k) stg[k] = (t == ((G - 1 - k + PF) & (G - 1))) ? yB : 0.0;
    // U prefetch ring: uA[k], uB[k] = U(row at distance e / e+G, step jt - k).  A
    // distance <= kv beyond row 0 reads a corner position of the same band column
    // (in bounds, value unused: it only ever updates rows < 0); distances > kv and
    // columns outside [0, n) are not read.
    double uA[PF], uB[PF];
    const double *abk = live ? ab : g_dummy;
    int cof = (jt + 1) * ldab + KV;  // element offset of AB(KV, jp + 1) for the next jp (decremented per step)
    auto uload = [&](int jp, int e, double &a, double &b) {
        cof -= ldab;
        const bool col = live && jp >= 0 && jp < n;
        const double *p = abk + (cof - e);
        a = 0.0;
        b = 0.0;
        ld_global_f64_if(col && e <= KV, p, a);  // e <= KV: compile-time true when KV >= G - 1
        if constexpr (G <= KV) ld_global_f64_if(col && e + G <= KV, p - G, b);
    };
#pragma unroll
    for (int k = 0; k < PF; ++k) uload(jt - k, (G - 1 - k - t) & (G - 1), uA[k], uB[k]);

#pragma unroll 1
    for (int jb = jt; jb >= 0; jb -= NR) {
#pragma unroll
        for (int k = 0; k < NR; ++k) {
            const int j = jb - k;
            const int kk = k % PF;
            const int e = (G - 1 - k - t) & (G - 1);            // distance of yA
            const int towner = (G - 1 - k) & (G - 1);           // lane holding row j (e == 0)
            const int tmerge = (G - 1 - k + PF) & (G - 1);      // lane that staged a row PF steps ago
            // ---- merge the row staged PF steps ago (before it enters the window)
            yB = (t == tmerge) ? stg[kk] : yB;
            // ---- the pivot row of step j: its lane divides (DTBSV skips y(j) == 0)
            const bool own = (t == towner);
            const bool nz = own && live && (yA != 0.0);
            const unsigned nzb = __ballot_sync(FULL, nz);
            const double xo = ddiv_rn_if(nz, yA, uA[kk]);
            const int src = gbase + towner;
            const double x = __shfl_sync(FULL, xo, src);
            const bool upd = (nzb >> src) & 1u;
            // ---- column update of the window rows
            fma_rn_if(upd && (unsigned)(e - 1) < (unsigned)KV, -x, uA[kk], yA);
            if constexpr (G <= KV) fma_rn_if(upd && e + G <= KV, -x, uB[kk], yB);
            // ---- owner: x(j) out, shift the window rows, stage row j - 2G
            st_global_f64_if(own && wr && j < n, bx + j, xo);
            yA = own ? yB : yA;
            {
                const int r2 = j - 2 * G;
                yload(own && live && r2 >= 0 && r2 < n, r2, stg[kk]);
            }
            // ---- prefetch step j - PF
            uload(j - PF, (G - 1 - k - PF - t) & (G - 1), uA[kk], uB[kk]);
        }
    }
}

}  // namespace bandlu
