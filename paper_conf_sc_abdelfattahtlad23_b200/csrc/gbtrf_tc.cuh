// gbtrf_tc.cuh -- sm_100a band LU with partial pivoting whose rank-1 updates run
// on the FP64 tensor cores (DMMA m8n8k4), one warp per matrix, compiled per
// (KL, KU) for kl+1 <= 16.
//
// What it computes: LAPACK DGBTF2 (Sec. 5.1 pseudo-code P:350-367,
// ju rule P:492-494, right-only swap P:358) -- the same per-element fp64
// operation sequence as the oracle, so factors, ipiv and info equal it
// (readings 7, 9, 10: one FMA per (element, step), +-0 reading).
//
// Why tensor cores on a path that is "not a dense contraction": the row-owner
// kernel (gbtrf_window.cuh) is bound by moving every pivot row through shared
// memory three times per column step (record write, broadcast read, new-row
// read).  Here the window lives in DMMA accumulator fragments and each column
// step is ONE m8n8k4 per 8x8 tile with only two live k-slots:
//   k = 0: A = -l_i (multiplier of row i), B = u_c (pivot row)   -> rank-1 update
//   k = 1: A = +1 on the pivot row's slot, B = the incoming row  -> row replacement
// and A = -1 (k = 0) on the pivot row itself, so its slot becomes
// fma(1, new_c, fma(-1, u_c, u_c)) = new_c exactly.  Measured on B200
// (tools/probes/dmma_probe.cu): m8n8k4 f64 equals the chain of IEEE FMAs in k
// order, so every non-pivot element gets exactly fma(-l_i, u_c, a_ic) (+0 from
// the empty k-slots), i.e. the LAPACK update bit for bit.  The tensor core does
// the broadcast that costs the row-owner kernel its shared-memory bandwidth.
//
// Layout (m8n8k4: lane = 4*g + t4): accumulator tile (rt, k) holds rows slot
// rt*8 + g, columns j0 + 8k + 2*t4 (+1) of the block starting at column j0;
// RT = ceil((kl+1)/8) row tiles, CT column tiles (CT*8 >= kv+9).  Row slots are
// physical: interchanges are relabelings (a row carries its logical position,
// DESIGN.md reading 10); the incoming row j+kl+1 takes the pivot row's slot.
// Columns: column j is zeroed when it retires, tiles rotate every 8 steps.
// Global traffic moves in blocks of 8 rows: in band storage 8 consecutive rows
// of one column are 64 contiguous bytes (cp.async in, chunked stores out).
#pragma once
#include "common.cuh"

#ifndef BANDLU_TC_MINB
#define BANDLU_TC_MINB 5
#endif

namespace bandlu {

template <int KL_, int KU_>
struct TrfTc {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU, W = KV + 1;
    static constexpr int RT = (KL + 1 + 7) / 8;      // row tiles
    static constexpr int CT = (KV + 8) / 8 + 1;      // column tiles: CT*8 >= KV+9
    static constexpr int NPOS = CT * 8;              // ring / record positions (absolute column mod NPOS)
    // row pitch (doubles), == 4 mod 16; records: [NPOS U row][y, pos][KL multipliers]
    static constexpr int PR = ((NPOS + 2 + KL + 11) / 16) * 16 + 4;
    static constexpr int NB = 8;                     // steps per block (= tile width)
    static constexpr int RR = 16;                    // ring rows: this block's 8 + the next block's 8
    static constexpr int GROUP_DBL = (RR + NB) * PR; // per warp: ring + U records
    static constexpr int WARPS = 4;
    static constexpr int MINB = BANDLU_TC_MINB;
    static constexpr int SIT = (NPOS + NB - 1 + 3) / 4;  // staging iterations (8 rows x NPOS, 4 columns/instr)
    static constexpr int UIT = (NB + KV + 3) / 4;        // U-store iterations
    static_assert(RT <= 2, "kl+1 <= 16");
    static constexpr size_t smem_bytes() { return (size_t)WARPS * GROUP_DBL * sizeof(double); }
};

__device__ __forceinline__ void dmma_8x8x4(double2 &c, double a, double b) {
    asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
        : "+d"(c.x), "+d"(c.y)
        : "d"(a), "d"(b));
}

// FWD: also the forward substitution of DGBTRS('N') for one right-hand side
// (Sec. 7, augmented [A|B]); see gbtrf_window.cuh.
template <int KL, int KU, bool FWD, class AP, class PP, class BP>
__global__ void __launch_bounds__(TrfTc<KL, KU>::WARPS * 32, TrfTc<KL, KU>::MINB)
    gbtrf_tc_kernel(int m, int n, AP A, int ldab, PP P, int *__restrict__ info, int batch, BP Bv) {
    using C = TrfTc<KL, KU>;
    constexpr int KV = C::KV, RT = C::RT, CT = C::CT, NPOS = C::NPOS, PR = C::PR, NB = C::NB, RR = C::RR;
    constexpr unsigned FULL = 0xffffffffu;
    extern __shared__ __align__(16) double smem[];

    const int lane = (int)lane_id(), wib = (int)(threadIdx.x >> 5);
    const int g = lane >> 2, t4 = lane & 3;
    const int64_t mat = (int64_t)blockIdx.x * C::WARPS + wib;
    if (mat >= batch) return;  // one matrix per warp: the whole warp leaves
    double *__restrict__ ab = A.get(mat);
    int *__restrict__ ipiv = P.get(mat);
    double *__restrict__ bv = FWD ? Bv.get(mat) : nullptr;
    if (m <= 0 || n <= 0) {
        if (lane == 0) info[mat] = 0;
        return;
    }
    double *ring = smem + (size_t)wib * C::GROUP_DBL;
    const uint32_t ring_s = smem_u32(ring);
    const uint32_t rec_s = ring_s + RR * PR * 8;

    // ---- staging of rows qb..qb+7 (qb-KL-1 a multiple of 8): row q = qb+bs gets
    // ring positions (c mod NPOS) for the NPOS columns c = q-KL .. q-KL+NPOS-1:
    // A(q, c) inside the band and the matrix, zero elsewhere.  Lane (bs = lane%8,
    // cc = lane/8 + 4*it) copies column qb-KL+cc of row bs: 8 lanes = one 64-byte
    // column chunk.  colq = &AB(0, qb-KL).
    auto stage_block = [&](int qb, const double *colq) {
        const int bs = lane & 7;
        const int q = qb + bs;
#pragma unroll
        for (int it = 0; it < C::SIT; ++it) {
            const int cc = (lane >> 3) + 4 * it, c = cc - bs;  // c: offset inside the row's NPOS window
            if (c >= 0 && c < NPOS) {
                const int col = qb - KL + cc;
                const bool ok = (c <= KV) && (q < m) && (col < n);
                const uint32_t dst = ring_s + (uint32_t)(((q & (RR - 1)) * PR + (col % NPOS)) * 8);
                cp_async8(dst, ok ? (const void *)(colq + (int64_t)cc * (ldab - 1) + (KV + KL + bs)) : (const void *)g_dummy,
                          ok ? 8u : 0u);
            }
        }
        if constexpr (FWD) {
            if (lane < NB) {
                const int qq = qb + lane;
                const bool okb = qq < m;
                cp_async8(ring_s + (uint32_t)(((qq & (RR - 1)) * PR + NPOS) * 8),
                          okb ? (const void *)(bv + qq) : (const void *)g_dummy, okb ? 8u : 0u);
            }
        }
        cp_async_commit();
    };
    stage_block(KL + 1, ab + (int64_t)1 * ldab);

    // ---- window: rows 0..KL in slots 0..KL, columns 0..CT*8-1
    double2 Cw[RT][CT];
    int pos[RT];
    double bq[RT];
#pragma unroll
    for (int rt = 0; rt < RT; ++rt) {
        const int r = rt * 8 + g;
#pragma unroll
        for (int k = 0; k < CT; ++k) {
            const int c0 = 8 * k + 2 * t4, c1 = c0 + 1;
            const bool ok0 = (r <= KL) && (r < m) && (c0 < n) && (c0 <= r + KU);
            const bool ok1 = (r <= KL) && (r < m) && (c1 < n) && (c1 <= r + KU);
            Cw[rt][k].x = ok0 ? ab[(int64_t)c0 * ldab + (KV + r - c0)] : 0.0;
            Cw[rt][k].y = ok1 ? ab[(int64_t)c1 * ldab + (KV + r - c1)] : 0.0;
        }
        pos[rt] = (r <= KL) ? r : 0x7fffffff;
        bq[rt] = (FWD && r <= KL && r < m) ? bv[r] : 0.0;
    }

    int linfo = 0;
    const int mn = min(m, n);
    double *colb = ab;          // &AB(0, j0)
    // A-fragment constants: k-slot 0 carries -l (aneg = -1 on t4 == 0 lanes), the
    // pivot row's slot gets -1 (k=0) and +1 (k=1)
    const double aneg = (t4 == 0) ? -1.0 : 0.0;
    const double apiv = (t4 == 0) ? -1.0 : (t4 == 1 ? 1.0 : 0.0);
    const double *scol = ab + (int64_t)(1 + NB) * ldab;  // &AB(0, qb-KL) of the block staged next
    int tb = 0;                 // column tile of j0 in the position ring
#pragma unroll 1
    for (int j0 = 0; j0 < mn; j0 += NB) {
        int tpos[CT];  // ring/record position of tile k's first column
#pragma unroll
        for (int k = 0; k < CT; ++k) tpos[k] = ((tb + k) % CT) * 8;
        cp_async_wait<0>();  // this block's rows (staged one block ahead) landed (own copies);
                             // the __syncwarp after the record write publishes them
        stage_block(j0 + NB + KL + 1, scol);
        scol += (int64_t)NB * ldab;

        int gt[CT];  // this lane's B-fragment offset in a record / ring row for tile k
#pragma unroll
        for (int k = 0; k < CT; ++k) gt[k] = (tpos[k] + g) * 8;
        const int rr0 = j0 + KL + 1;  // ring row of the row entering at step j0

#pragma unroll
        for (int s = 0; s < NB; ++s) {
            const int j = j0 + s;
            if (j >= mn) break;
            const int cs = s >> 1;  // lanes t4 == cs hold column j (register s & 1 of tile 0)

            // ---- IAMAX over the candidates (logical rows j..min(j+KL, m-1)), first max
            double x[RT];
            bool cand[RT];
            uint64_t key[RT];
            unsigned lhi = 0;
#pragma unroll
            for (int rt = 0; rt < RT; ++rt) {
                x[rt] = (s & 1) ? Cw[rt][0].y : Cw[rt][0].x;
                cand[rt] = (t4 == cs) && (pos[rt] < m);
                key[rt] = cand[rt] ? abs_key(x[rt]) : 0ull;
                if (cand[rt]) lhi = max(lhi, (unsigned)(key[rt] >> 32));
            }
            const unsigned mhi = __reduce_max_sync(FULL, lhi);
            unsigned bt[RT];  // lanes whose row-tile-rt candidate reaches the max high word
#pragma unroll
            for (int rt = 0; rt < RT; ++rt) bt[rt] = __ballot_sync(FULL, cand[rt] && (unsigned)(key[rt] >> 32) == mhi);
            int hits = 0;
#pragma unroll
            for (int rt = 0; rt < RT; ++rt) hits += __popc(bt[rt]);
            if (hits != 1) {
                // exact tie-break: low word, then smallest logical row (first index)
                unsigned llo = 0;
#pragma unroll
                for (int rt = 0; rt < RT; ++rt)
                    if (bt[rt] >> lane & 1u) llo = max(llo, (unsigned)key[rt]);
                const unsigned mlo = __reduce_max_sync(FULL, llo);
                unsigned lp = 0xffffffffu;
#pragma unroll
                for (int rt = 0; rt < RT; ++rt)
                    if ((bt[rt] >> lane & 1u) && (unsigned)key[rt] == mlo) lp = min(lp, (unsigned)pos[rt]);
                const unsigned mp = __reduce_min_sync(FULL, lp);
#pragma unroll
                for (int rt = 0; rt < RT; ++rt) bt[rt] = __ballot_sync(FULL, cand[rt] && (unsigned)pos[rt] == mp);
            }
            const int tp = (RT > 1 && bt[RT - 1]) ? RT - 1 : 0;
            const int gp = (__ffs(RT > 1 ? (bt[0] | bt[RT - 1]) : bt[0]) - 1) >> 2;
            bool prow[RT];  // this lane holds (part of) the pivot row
#pragma unroll
            for (int rt = 0; rt < RT; ++rt) prow[rt] = (g == gp) && (rt == tp);

            // ---- pivot row (U row j: NPOS positions) + (y, logical row) -> record s
            const uint32_t rec_j = rec_s + (uint32_t)(s * PR * 8);
            const int KLO = (s + 1) / 8;                    // first tile touched by columns j+1..
            const int KHI = min((s + KV + 1) / 8, CT - 1);  // last tile touched by columns ..j+KV+1
#pragma unroll
            for (int k = 0; k <= KHI; ++k)
#pragma unroll
                for (int rt = 0; rt < RT; ++rt) st_shared_v2_if(prow[rt], rec_j + (uint32_t)((tpos[k] + 2 * t4) * 8), Cw[rt][k]);
#pragma unroll
            for (int rt = 0; rt < RT; ++rt)
                st_shared_v2_if(prow[rt] && t4 == 0, rec_j + NPOS * 8,
                                make_double2(bq[rt], __longlong_as_double((long long)pos[rt])));
            __syncwarp();

            // ---- reads: pivot value, (y, logical row), B fragments (k=0: pivot row, k=1: new row)
            const double p = ld_shared_f64(rec_j + (uint32_t)((tpos[0] + s) * 8));
            const double2 yp = ld_shared_v2(rec_j + NPOS * 8);
            const int ppos = (int)__double_as_longlong(yp.y);
            const uint32_t rrow = ring_s + (uint32_t)(((rr0 + s) & (RR - 1)) * PR * 8);
            const uint32_t bsrc = (t4 == 0) ? rec_j : rrow;
            double bfr[CT];
#pragma unroll
            for (int k = KLO; k <= KHI; ++k) {
                bfr[k] = 0.0;
                ld_shared_f64_if(t4 < 2, bsrc + (uint32_t)gt[k], bfr[k]);
            }

            const bool zp = (p == 0.0);  // exact zero pivot: all candidates are +-0
            linfo = (zp && linfo == 0) ? j + 1 : linfo;
#pragma unroll
            for (int rt = 0; rt < RT; ++rt)
                if (pos[rt] == j && !prow[rt]) pos[rt] = ppos;  // interchange = relabel

            // ---- SCAL: multiplier = x * RN(1/p) (DSCAL(ONE/pivot), Q7); zero pivot: stored
            // unscaled, no update.  L entries go to the record, stored per block.
            const double rinv = zp ? 0.0 : __drcp_rn(p);
            double a[RT];
#pragma unroll
            for (int rt = 0; rt < RT; ++rt) {
                const double lu = __dmul_rn(x[rt], rinv);
                st_shared_f64_if(cand[rt] && !prow[rt], rec_j + (uint32_t)((NPOS + 1 + pos[rt] - j) * 8), zp ? x[rt] : lu);
                const double lr = __shfl_sync(FULL, lu, (lane & ~3) | cs);  // this quad's row multiplier
                a[rt] = prow[rt] ? apiv : __dmul_rn(lr, aneg);
                if constexpr (FWD) bq[rt] = __fma_rn(lr, -yp.x, bq[rt]);
            }
            if constexpr (FWD) {
                const double nb = ld_shared_f64(rrow + NPOS * 8);
#pragma unroll
                for (int rt = 0; rt < RT; ++rt) bq[rt] = prow[rt] ? nb : bq[rt];
            }

            // ---- rank-1 update + row replacement on the tensor cores.  Retired
            // columns of tile 0 keep bounded garbage until the tile rotates out.
#pragma unroll
            for (int rt = 0; rt < RT; ++rt)
#pragma unroll
                for (int k = KLO; k <= KHI; ++k) dmma_8x8x4(Cw[rt][k], a[rt], bfr[k]);
#pragma unroll
            for (int rt = 0; rt < RT; ++rt) pos[rt] = prow[rt] ? j + KL + 1 : pos[rt];
        }

        // ---- block outputs from the records: U rows j0..j0+7 (64-byte column
        // chunks), L columns j0..j0+7 (contiguous), ipiv, y
        __syncwarp();
        {
            const int bs = lane & 7;
#pragma unroll
            for (int it = 0; it < C::UIT; ++it) {
                const int bk = (lane >> 3) + 4 * it;  // column offset from j0; tile it/2
                if (bk - bs >= 0 && bk - bs <= KV && j0 + bs < mn && j0 + bk < n)
                    colb[(int64_t)bk * ldab + (KV + bs - bk)] =
                        ld_shared_f64(rec_s + (uint32_t)((bs * PR + tpos[it / 2] + (lane >> 3) + 4 * (it & 1)) * 8));
            }
#pragma unroll
            for (int it = 0; it < (NB * KL + 31) / 32; ++it) {
                const int e = lane + 32 * it, sc = e / KL, i = e - sc * KL;  // column j0+sc, row j0+sc+1+i
                if (sc < NB && j0 + sc < mn && j0 + sc + 1 + i < m)
                    colb[(int64_t)sc * ldab + (KV + 1 + i)] = ld_shared_f64(rec_s + (uint32_t)((sc * PR + NPOS + 2 + i) * 8));
            }
            if (lane < NB && j0 + lane < mn) {
                const double2 yq = ld_shared_v2(rec_s + (uint32_t)((lane * PR + NPOS) * 8));
                ipiv[j0 + lane] = (int)__double_as_longlong(yq.y) + 1;
                if constexpr (FWD) bv[j0 + lane] = yq.x;
            }
        }
        colb += (int64_t)NB * ldab;
        __syncwarp();  // records are rewritten by the next block
        // rotate column tiles: tile 0 (all its columns retired) becomes the last, zeroed
#pragma unroll
        for (int rt = 0; rt < RT; ++rt) {
#pragma unroll
            for (int k = 0; k + 1 < CT; ++k) Cw[rt][k] = Cw[rt][k + 1];
            Cw[rt][CT - 1] = make_double2(0.0, 0.0);
        }
        tb = (tb + 1 == CT) ? 0 : tb + 1;
    }
    cp_async_wait<0>();
    __syncwarp();

    // LAPACK's SET_FILLIN also zeroes fill-row positions whose matrix row is
    // >= m when m < n (those rows are never pivot rows here).
    if (m < n) {
        for (int c = m + KU + 1 + lane; c <= min(n - 1, m + KV - 1); c += 32) {
#pragma unroll 1
            for (int rr = 0; rr < KL; ++rr) {
                const int i = c - KV + rr;
                const bool zeroed = (c >= KU + 1 && c <= min(KV, n) - 1 && rr >= KV - c) || (c >= KV && c - KV < mn);
                if (i >= m && zeroed) ab[(int64_t)c * ldab + rr] = 0.0;
            }
        }
    }
    if (lane == 0) info[mat] = linfo;
}

}  // namespace bandlu
