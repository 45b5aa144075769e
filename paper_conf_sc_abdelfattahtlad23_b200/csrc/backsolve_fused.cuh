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
// i == t (mod G).  A lane keeps S = ceil((kv+1)/G) rows in registers: slot s
// holds the row r == t + s*G (mod S*G) with d_s = j - r in [0, S*G); the row
// is in the active window while d_s <= kv, it is the pivot row of step j when
// d_s == 0 (its lane divides and broadcasts x(j) with one shuffle), and when
// it retires the slot takes row r - S*G (read from the y buffer: shared
// memory, or B in global memory).  U(r_s, j) = AB(kv - d_s, j): the U column
// is contiguous in band storage, so a slot's loads over the group are one
// coalesced segment; they are issued PF steps ahead into a register ring.
#pragma once
#include "common.cuh"

#ifndef BANDLU_FUSED_PF
#define BANDLU_FUSED_PF 8
#endif

namespace bandlu {

// YSM: y(i) read from shared memory at ybuf_s + 8 i (else from bx[i]).
// wr: this group stores x into bx (false for dead groups and, for dgbsv, where info > 0).
// All 32 lanes of the warp must call (shuffles / ballots over the full warp).
template <int KV, int G, bool YSM>
__device__ __forceinline__ void backsolve_group(int n, const double *ab, int ldab, double *bx, uint32_t ybuf_s,
                                                bool live, bool wr, int t, int gbase) {
    constexpr int S = (KV + G) / G;  // ceil((KV + 1) / G)
    constexpr int SG = S * G;
    constexpr int PF = BANDLU_FUSED_PF;
    constexpr bool POW2 = (SG & (SG - 1)) == 0;
    constexpr unsigned FULL = 0xffffffffu;
    auto wrap = [](int x) -> int {  // x in (-SG, SG) -> [0, SG)
        if constexpr (POW2) return x & (SG - 1);
        else return x < 0 ? x + SG : x;
    };
    auto yget = [&](int r) -> double {
        if constexpr (YSM) return ld_shared_f64(ybuf_s + (uint32_t)r * 8u);
        else return bx[r];
    };
    const int jn = n - 1;
    int d[S];
    double y[S];
#pragma unroll
    for (int s = 0; s < S; ++s) {
        const int q = (jn - t - s * G) % SG;
        d[s] = q < 0 ? q + SG : q;
        const int r = jn - d[s];
        y[s] = (live && r >= 0) ? yget(r) : 0.0;
    }
    // U prefetch ring: uv[k][s] = U(row of slot s at step jb-k, jb-k) of the current block
    double uv[PF][S];
    const double *pre = live ? ab + (int64_t)jn * ldab + KV : nullptr;  // &AB(KV, j) of the next prefetch
#pragma unroll
    for (int k = 0; k < PF; ++k) {
        const int j = jn - k;
#pragma unroll
        for (int s = 0; s < S; ++s) {
            const int dd = wrap(d[s] - k % SG);
            const bool ok = live && j >= 0 && dd <= KV && j - dd >= 0;
            uv[k][s] = ok ? pre[-dd] : 0.0;
        }
        if (live) pre -= ldab;
    }
#pragma unroll 1
    for (int jb = jn; jb >= 0; jb -= PF) {
#pragma unroll
        for (int k = 0; k < PF; ++k) {
            const int j = jb - k;
            if (j < 0) break;
            // ---- the pivot row of step j: its lane divides (DTBSV skips y(j) == 0)
            double yo = 0.0, uo = 1.0;
            bool own = false;
#pragma unroll
            for (int s = 0; s < S; ++s) {
                if (d[s] == 0) {
                    yo = y[s];
                    uo = uv[k][s];
                    own = true;
                }
            }
            const bool nz = own && (yo != 0.0);
            const unsigned nzb = __ballot_sync(FULL, nz);
            const double xo = ddiv_rn_if(nz, yo, uo);
            const int src = gbase + (j & (G - 1));
            const double x = __shfl_sync(FULL, xo, src);
            const bool upd = (nzb >> src) & 1u;
            // ---- column update of the window rows, then retire / refill / prefetch
#pragma unroll
            for (int s = 0; s < S; ++s) {
                const int dc = d[s];
                if (upd && dc >= 1 && dc <= KV) y[s] = __fma_rn(-x, uv[k][s], y[s]);
                if (dc == 0) {
                    if (wr) bx[j] = xo;
                    const int r2 = j - SG;
                    y[s] = (live && r2 >= 0) ? yget(r2) : 0.0;
                }
                const int dd = wrap(dc - PF % SG);
                const int jp = j - PF;
                const bool ok = live && jp >= 0 && dd <= KV && jp - dd >= 0;
                uv[k][s] = ok ? pre[-dd] : 0.0;
                d[s] = (dc == 0) ? SG - 1 : dc - 1;
            }
            if (live) pre -= ldab;
        }
    }
}

}  // namespace bandlu
