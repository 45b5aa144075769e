// gbtrs_bwd.cuh -- sm_100a backward substitution U x = y for ONE right-hand
// side: the second launch of dgbtrfs (the forward substitution ran inside the
// factorization kernel, Sec. 7).
//
// What it computes: DTBSV('U','N','N') with bandwidth kv, exactly
// the oracle's order: for j = n-1..0: if x(j) != 0: x(j) = x(j) / U(j,j)
// (true division, reading Q9); x(i) = fma(-x(j), U(i,j), x(i)), i = j-1 ..
// max(0, j-kv).
//
// Why a separate kernel from gbtrs_window.cuh: the solve is
// latency-bound -- one lane per matrix runs a 512-step serial chain, ~8 lanes
// per warp, ~2 warps per scheduler -- so its time is the number of dependent
// instructions per step.  The general window kernel spends ~200 warp
// instructions per step on forward/backward/pair bookkeeping and recomputes
// every address; this one only runs the backward pass with nrhs = 1:
//  * per-lane column pointers advance by -ldab per step (no 64-bit recompute);
//  * a column's U entries (rows max(0,kv-j)..kv, contiguous) are 11 16-byte
//    chunks (kv = 20) copied by the 32/gpw lanes of the matrix's copy group
//    with fixed chunk indices, plus the RHS row entering the window (8 bytes,
//    zero-filled below row 0), into an NS-deep smem ring;
//  * slot pitch == 2 (mod 16) doubles so the gpw lanes' 64-bit reads of the
//    same slot offset fall in distinct banks.
#pragma once
#include "common.cuh"

#ifndef BANDLU_BWD_NS
#define BANDLU_BWD_NS 4
#endif

namespace bandlu {

template <int KL_, int KU_>
struct TrsBwd {
    static constexpr int KV = KL_ + KU_, WB = KV + 1;
    static constexpr int NCH = (WB + 2) / 2;                    // 16-byte chunks per column (any alignment)
    static constexpr int RHS = 2 * NCH;                         // slot offset of the entering RHS row
    static constexpr int SLOT = ((RHS + 1 + 13) / 16) * 16 + 2;  // doubles per (matrix, step), == 2 mod 16
    static constexpr int NS = BANDLU_BWD_NS;                    // steps in flight (power of 2)
    static constexpr int PAD = (KV + 3) & ~1;                   // rows < 0 of the last kv steps read before a slot
    static size_t smem_bytes(int gpw) { return (size_t)(PAD + NS * gpw * SLOT) * 8; }
    static_assert((NS & (NS - 1)) == 0, "ring depth");
};

template <int KL, int KU, int GPW, class AP, class BP>
__global__ void __launch_bounds__(32) gbtrs_bwd_kernel(int n, AP A, int ldab, BP Bv, int batch) {
    using C = TrsBwd<KL, KU>;
    constexpr int KV = C::KV, WB = C::WB, NCH = C::NCH, SLOT = C::SLOT, NS = C::NS;
    constexpr int gpw = GPW;  // matrices per warp
    extern __shared__ __align__(16) double smem[];
    const int lane = (int)lane_id();
    // [r2b] (-DBANDLU_BWD_REVERSE_ORDER) warps taking the batch from its end, where the preceding
    // factorization's last columns may still sit in L2, measured slower: C3 0.290 vs 0.286 ms
#ifdef BANDLU_BWD_REVERSE_ORDER
    const int64_t base = (int64_t)(gridDim.x - 1 - blockIdx.x) * gpw;
#else
    const int64_t base = (int64_t)blockIdx.x * gpw;
#endif

    // ---- copy role: lane -> (matrix cm of the warp, chunk phase cq)
    constexpr int CPG = 32 / GPW;
    const int cm = lane / CPG, cq = lane % CPG;
    const bool clive = cm < gpw && base + cm < batch;
    const double *cab = clive ? A.get(base + cm) : nullptr;
    const double *cbv = clive ? Bv.get(base + cm) : nullptr;
    double *ring = smem + C::PAD;
    const uint32_t ring_s = smem_u32(ring);
    const void *dummy = g_dummy;
    auto issue = [&](int k) {  // copies of step k (column j = n-1-k) for matrix cm
        const int j = n - 1 - k;
        const uint32_t dst = ring_s + (uint32_t)(((k & (NS - 1)) * gpw + cm) * SLOT * 8);
        if (clive && j >= 0) {
            const double *lo = cab + (int64_t)j * ldab + max(0, KV - j);
            const uintptr_t a0 = reinterpret_cast<uintptr_t>(lo) & ~(uintptr_t)15;
            const uintptr_t a1 = reinterpret_cast<uintptr_t>(cab + (int64_t)j * ldab + KV + 1);
            const int nch = (int)((a1 - a0 + 15) >> 4);
#pragma unroll
            for (int i = 0; i < (NCH + CPG - 1) / CPG; ++i) {
                const int q = cq + i * CPG;
                if (q < nch) cp_async16(dst + q * 16, reinterpret_cast<const void *>(a0 + q * 16), 16u);
            }
            if (cq == CPG - 1) {  // RHS row j - WB enters the window at this step (zero below row 0)
                const bool ok = j - WB >= 0;
                cp_async8(dst + C::RHS * 8, ok ? (const void *)(cbv + j - WB) : dummy, ok ? 8u : 0u);
            }
        }
    };

    // ---- compute role: lane m < gpw solves matrix base + m
    const bool live = lane < gpw && base + lane < batch;
    const double *ab = live ? A.get(base + lane) : nullptr;
    double *bv = live ? Bv.get(base + lane) : nullptr;
    const double *colp = live ? ab + (int64_t)(n - 1) * ldab : nullptr;  // column j of step k
    double *bj = live ? bv + (n - 1) : nullptr;                          // x(j)
    const double *slot0 = ring + (lane < gpw ? lane : 0) * SLOT;

#pragma unroll 1
    for (int k = 0; k < NS; ++k) {
        issue(k);
        cp_async_commit();
    }
    constexpr int UB = WB <= 12 ? WB : 4;  // steps per block; window shifts by UB slots after it
    constexpr int XS = WB + UB;
    double x[XS];
#pragma unroll
    for (int i = 0; i < XS; ++i) x[i] = (i < WB && live && n - 1 - i >= 0) ? bv[n - 1 - i] : 0.0;

#pragma unroll 1
    for (int k0 = 0; k0 < n; k0 += UB) {
#pragma unroll
        for (int s = 0; s < UB; ++s) {
            const int k = k0 + s, j = n - 1 - k;
            if (k >= n) break;
            cp_async_wait<NS - 1>();
            __syncwarp();
            // uc[r] = AB(r, j) for r >= max(0, KV - j); smaller r read the pad or a neighbouring
            // slot and only feed window rows < 0, which are never stored
            const int rlo = max(0, KV - j);
            const int delta = live ? (int)((reinterpret_cast<uintptr_t>(colp + rlo) >> 3) & 1) : 0;
            const double *uc = slot0 + (k & (NS - 1)) * gpw * SLOT + delta - rlo;
            const bool nz = (x[s] != 0.0);
            const double xj = ddiv_rn_if(nz, x[s], uc[KV]);
            if (nz) {
#pragma unroll
                for (int i = 1; i < WB; ++i) x[s + i] = __fma_rn(-xj, uc[KV - i], x[s + i]);
            }
            if (live) *bj = xj;
            x[s + WB] = slot0[(k & (NS - 1)) * gpw * SLOT + C::RHS];  // row j - WB (0 below row 0)
            colp -= ldab;
            --bj;
            __syncwarp();
            issue(k + NS);
            cp_async_commit();
        }
#pragma unroll
        for (int i = 0; i < XS; ++i) x[i] = (i + UB < XS) ? x[i + UB] : 0.0;
    }
    cp_async_wait<0>();
}

}  // namespace bandlu
