// gbtrf_thin.cuh -- sm_100a band LU with partial pivoting for THIN bands: one
// thread per matrix with the whole (kl+1) x (kl+ku+1) window in registers, and
// every byte of the band moved by the warp cooperatively as whole, contiguous
// band columns through shared memory.
//
// What it computes: LAPACK DGBTF2 exactly (Sec. 5.1 pseudo-code
// P:350-367, right-only swaps P:358/P:369-374), the oracle's fp64 operation
// sequence => bitwise-equal factors, ipiv, info.  FL & 1 (FWD): the forward
// substitution of DGBTRS('N') for one right-hand side rides along (y into B);
// FL & 2 (BWD): then the backward substitution by the same thread, the U
// columns and y read back in reverse (one launch for dgbtrf + dgbtrs: the
// fused gbsv kernel of PAPER.md Sec. 7; B solved also where
// info > 0, as dgbtrfs specifies).
//
// Why: for a tridiagonal-like band a column step is a
// handful of flops, so the warp-cooperative row-slot kernel spends it on
// cross-lane traffic (~25 warp instructions per matrix-step at C2), and the
// round-1 thread-per-matrix kernel spent it on uncoalesced memory instructions
// (every thread its own sectors: ~23 M single-sector L1 requests at C2).  Here
// a thread owns its matrix's window (IAMAX, interchange, SCAL and update are
// thread-local, no warp collectives) and memory moves in blocks of P steps:
//  * in: the band columns the next block's entering rows live in (P whole
//    columns = one contiguous P*ldab-double chunk per matrix) are copied by the
//    warp with 8-byte cp.async, 32 consecutive doubles of one matrix per
//    instruction, into a per-matrix circular column window in shared memory,
//    one block ahead;
//  * out: the thread writes its U row / L column entries into that window in
//    place (every input element is read before its output overwrites it) and
//    after each block the P finished columns go back to global memory the same
//    cooperative way; b, y, ipiv are staged per block likewise.
//  Corner and padding positions travel in and out unchanged.
#pragma once
#include "common.cuh"

namespace bandlu {

template <int KL_, int KU_>
struct TrfThin {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU, W = KV + 1, R = KL + 1;
    static constexpr int P = 8;                           // steps (columns) per block
    static constexpr int NC = pow2_ceil(2 * P + KV + 1);  // circular column window
    // per-matrix window stride (doubles) for a run-time ldab: odd, so the 32 threads'
    // same-offset accesses hit distinct 8-byte bank pairs
    __host__ __device__ static constexpr int mstride(int ldab) { return (NC * ldab) | 1; }
    static constexpr int BS = 2 * P + 1;  // per-matrix b / y / x staging (doubles)
    __host__ __device__ static constexpr size_t smem_bytes(int ldab) {
        return (size_t)32 * (mstride(ldab) + BS) * 8 + (size_t)32 * (P + 1) * 4;
    }
};

template <int KL, int KU, int FL, class AP, class PP, class BP>
__global__ void __launch_bounds__(32) gbtrf_thin_kernel(int n, AP A, int ldab, PP Pv, int *__restrict__ info,
                                                      int batch, BP Bv) {
    using C = TrfThin<KL, KU>;
    constexpr int KV = C::KV, W = C::W, R = C::R, P = C::P, NC = C::NC, BS = C::BS;
    constexpr bool FWD = FL & 1, BWD = FL & 2;
    static_assert(!BWD || FWD, "the backward pass needs the forward pass");
    extern __shared__ __align__(16) double smem[];
    const int lane = (int)threadIdx.x;
    const int64_t base = (int64_t)blockIdx.x * 32;
    const int64_t mat = base + lane;
    const bool live = mat < batch;
    const int nm = (int)min((int64_t)32, batch - base);  // matrices of this warp
    const int m = n;  // square (dgbtrfs / dgbsv / square dgbtrf)
    if (n <= 0) {
        if (live) info[mat] = 0;
        return;
    }
    const int MS = C::mstride(ldab);
    double *win = smem;                                          // [32][MS]
    double *bst = smem + 32 * MS;                                // [32][BS]: b / y in at [0,P), y / x out at [P,2P)
    int *ist = reinterpret_cast<int *>(bst + 32 * BS);           // [32][P+1]: ipiv out
    double *mw = win + lane * MS;
    double *mb = bst + lane * BS;
    int *mi = ist + lane * (P + 1);
    auto col = [&](int c) -> double * { return mw + (c & (NC - 1)) * ldab; };

    // ---- cooperative whole-column copies: lane l moves elements e = l + 32k of each
    // matrix's chunk of columns c0 .. c0+ncol-1 (contiguous in band storage)
    const int q32 = 32 / ldab, r32 = 32 - q32 * ldab;
    const int dc0 = lane / ldab, rr0 = lane - dc0 * ldab;
    auto copy_in = [&](int c0, int ncol) {
        if (c0 < 0) {
            ncol += c0;
            c0 = 0;
        }
        if (c0 + ncol > n) ncol = n - c0;
        if (ncol <= 0) return;
        const int ne = ncol * ldab;
        for (int mm = 0; mm < nm; ++mm) {
            const double *src = A.get(base + mm) + (int64_t)c0 * ldab;
            double *dstm = win + mm * MS;
            int dc = dc0, r = rr0;
            for (int e = lane; e < ne; e += 32) {
                cp_async8(smem_u32(dstm + ((c0 + dc) & (NC - 1)) * ldab + r), src + e, 8u);
                dc += q32;
                r += r32;
                if (r >= ldab) {
                    r -= ldab;
                    ++dc;
                }
            }
        }
    };
    auto copy_out = [&](int c0, int ncol) {  // after a __syncwarp
        if (c0 + ncol > n) ncol = n - c0;
        if (ncol <= 0) return;
        const int ne = ncol * ldab;
        for (int mm = 0; mm < nm; ++mm) {
            double *dst = A.get(base + mm) + (int64_t)c0 * ldab;
            const double *srcm = win + mm * MS;
            int dc = dc0, r = rr0;
            for (int e = lane; e < ne; e += 32) {
                dst[e] = srcm[((c0 + dc) & (NC - 1)) * ldab + r];
                dc += q32;
                r += r32;
                if (r >= ldab) {
                    r -= ldab;
                    ++dc;
                }
            }
        }
    };
    // P values of B in (rows q0 + sgn*o, o = 0..P-1 -> bst[mm][o]; rows outside [0, m) -> 0)
    auto b_in = [&](int q0, int sgn) {
        for (int i = lane; i < nm * P; i += 32) {
            const int mm = i / P, o = i - mm * P, q = q0 + sgn * o;
            const bool ok = q >= 0 && q < m;
            cp_async8(smem_u32(bst + mm * BS + o), ok ? Bv.get(base + mm) + q : g_dummy, ok ? 8u : 0u);
        }
    };
    // P staged values bst[mm][P + o] -> B rows q0 + sgn*o (o < cnt); after a __syncwarp
    auto b_out = [&](int q0, int sgn, int cnt) {
        for (int i = lane; i < nm * P; i += 32) {
            const int mm = i / P, o = i - mm * P;
            if (o < cnt) Bv.get(base + mm)[q0 + sgn * o] = bst[mm * BS + P + o];
        }
    };
    auto ipiv_out = [&](int j0, int cnt) {
        for (int i = lane; i < nm * P; i += 32) {
            const int mm = i / P, o = i - mm * P;
            if (o < cnt) Pv.get(base + mm)[j0 + o] = ist[mm * (P + 1) + o];
        }
    };

    // ---- prologue: columns 0 .. P+KV (first window + block 0's entering rows); b of the
    // rows entering during block 0
    copy_in(0, P + KV + 1);
    if constexpr (FWD) b_in(KL + 1, 1);
    cp_async_commit();
    cp_async_wait<0>();
    __syncwarp();
    double w[R][W], y[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
#pragma unroll
        for (int c = 0; c < W; ++c)  // A(r, c) at band row KV + r - c; fill (c > r + KU) starts 0
            w[r][c] = (live && r < m && c < n && c <= r + KU) ? col(c)[KV + r - c] : 0.0;
        y[r] = 0.0;
        if constexpr (FWD) ld_global_f64_if(live && r < m, live ? Bv.get(mat) + r : g_dummy, y[r]);
    }

    int linfo = 0;
#pragma unroll 1
    for (int j0 = 0; j0 < n; j0 += P) {
        cp_async_wait<0>();  // this block's entering columns and b (issued one block ago)
        __syncwarp();
        double bin[P];
#pragma unroll
        for (int s = 0; s < P; ++s) bin[s] = FWD ? mb[s] : 0.0;
        __syncwarp();
        // next block's entering columns and b, one block ahead
        if (j0 + P < n) {
            copy_in(j0 + P + KV + 1, P);
            if constexpr (FWD) b_in(j0 + P + KL + 1, 1);
        }
        cp_async_commit();
#pragma unroll
        for (int s = 0; s < P; ++s) {
            const int j = j0 + s;
            if (j >= n) break;
            const int km = min(KL, m - 1 - j);
            // ---- IAMAX: first max |w[r][0]|, r = 0..km (BLAS IDAMAX, reading 2)
            int jp = 0;
            double best = fabs(w[0][0]);
#pragma unroll
            for (int r = 1; r < R; ++r) {
                const double a = fabs(w[r][0]);
                if (r <= km && a > best) {
                    best = a;
                    jp = r;
                }
            }
            mi[s] = j + jp + 1;
            double p = w[0][0];
#pragma unroll
            for (int r = 1; r < R; ++r) p = (jp == r) ? w[r][0] : p;
            if (p != 0.0) {
                // ---- interchange rows j and j+jp (whole rows == right-only swap, reading 10)
#pragma unroll
                for (int r = 1; r < R; ++r) {
                    if (jp == r) {
#pragma unroll
                        for (int c = 0; c < W; ++c) {
                            const double t = w[0][c];
                            w[0][c] = w[r][c];
                            w[r][c] = t;
                        }
                        const double t = y[0];
                        y[0] = y[r];
                        y[r] = t;
                    }
                }
                // ---- SCAL (x * RN(1/p), reading 6) and rank-1 update (FMA, readings 7, 9)
                const double rinv = __drcp_rn(w[0][0]);
#pragma unroll
                for (int r = 1; r < R; ++r) {
                    if (r <= km) {
                        const double l = __dmul_rn(w[r][0], rinv);
                        w[r][0] = l;
#pragma unroll
                        for (int c = 1; c < W; ++c) w[r][c] = __fma_rn(l, -w[0][c], w[r][c]);
                    }
                }
            } else if (live && linfo == 0) {
                linfo = j + 1;  // zero pivot: no interchange, no scaling, no update (reading 3)
            }
            if constexpr (FWD) {  // forward substitution with column j of L (DGER skips y == 0)
                if (y[0] != 0.0) {
#pragma unroll
                    for (int r = 1; r < R; ++r)
                        if (r <= km) y[r] = __fma_rn(w[r][0], -y[0], y[r]);
                }
                mb[P + s] = y[0];
            }
            // ---- retire into the column window: L column j, U row j (AB[KV-c][j+c])
            {
                double *cj = col(j);
#pragma unroll
                for (int r = 1; r < R; ++r)
                    if (r <= km) cj[KV + r] = w[r][0];
#pragma unroll
                for (int c = 0; c < W; ++c)
                    if (j + c < n) col(j + c)[KV - c] = w[0][c];
            }
            // ---- slide: rows up, columns left; row q = j+KL+1 enters from the window
#pragma unroll
            for (int r = 0; r < R - 1; ++r) {
#pragma unroll
                for (int c = 0; c < W; ++c) w[r][c] = (c + 1 < W) ? w[r + 1][c + 1] : 0.0;
                y[r] = y[r + 1];
            }
            {
                const int q = j + KL + 1;  // A(q, j+1+c) at band row KV + KL - c of column j+1+c
#pragma unroll
                for (int c = 0; c < W; ++c)
                    w[R - 1][c] = (live && q < m && j + 1 + c < n) ? col(j + 1 + c)[KV + KL - c] : 0.0;
                y[R - 1] = (q < m) ? bin[s] : 0.0;
            }
        }
        // ---- block done: columns j0 .. j0+P-1 are final; ipiv and y out
        __syncwarp();
        const int cnt = min(P, n - j0);
        copy_out(j0, cnt);
        ipiv_out(j0, cnt);
        if constexpr (FWD) b_out(j0, 1, cnt);
        __syncwarp();
    }
    cp_async_wait<0>();
    __syncwarp();

    if constexpr (BWD) {
        // ---- backward substitution U x = y (DTBSV column order, reading 8), P columns
        // per block from the top; U columns and the entering y rows read back one block
        // ahead (the writes above are this warp's own, ordered by the __syncwarp).
        // Window xw[d] = y(j - d), d = 0..KV.
        const int jt = n - 1;
        copy_in(jt - P + 1, P);
        b_in(jt - KV - 1, -1);  // y rows entering during the first block: jt-KV-1-o
        cp_async_commit();
        double xw[W];
#pragma unroll
        for (int d = 0; d < W; ++d) {
            xw[d] = 0.0;
            ld_global_f64_if(live && jt - d >= 0, live ? Bv.get(mat) + (jt - d) : g_dummy, xw[d]);
        }
#pragma unroll 1
        for (int jb = jt; jb >= 0; jb -= P) {
            cp_async_wait<0>();
            __syncwarp();
            double yin[P];
#pragma unroll
            for (int s = 0; s < P; ++s) yin[s] = mb[s];
            __syncwarp();
            if (jb - P >= 0) {
                copy_in(jb - 2 * P + 1, P);
                b_in(jb - P - KV - 1, -1);
            }
            cp_async_commit();
#pragma unroll
            for (int s = 0; s < P; ++s) {
                const int j = jb - s;
                if (j < 0) break;
                const double *cj = col(j);
                const double yj = xw[0];
                double xj = yj;
                if (yj != 0.0) {
                    xj = __ddiv_rn(yj, cj[KV]);
#pragma unroll
                    for (int d = 1; d < W; ++d)
                        if (j - d >= 0) xw[d] = __fma_rn(-xj, cj[KV - d], xw[d]);
                }
                mb[P + s] = xj;
#pragma unroll
                for (int d = 0; d < W - 1; ++d) xw[d] = xw[d + 1];
                xw[W - 1] = yin[s];  // y(j - KV - 1) (0 below row 0)
            }
            __syncwarp();
            b_out(jb, -1, min(P, jb + 1));
            __syncwarp();
        }
        cp_async_wait<0>();
    }
    if (live) info[mat] = linfo;
}

}  // namespace bandlu
