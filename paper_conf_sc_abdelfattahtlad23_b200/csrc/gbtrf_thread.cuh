// gbtrf_thread.cuh -- sm_100a band LU with partial pivoting, ONE THREAD PER
// MATRIX, for thin bands ((kl+1)·(kl+ku+1) register window).
//
// What it computes: LAPACK DGBTF2 exactly (Sec. 5.1 pseudo-code
// P:350-367, right-only swaps P:358/P:369-374), the oracle's fp64 operation
// sequence => bitwise-equal factors, ipiv, info; with FWD the forward
// substitution of dgbtrs('N') rides along (paper Sec. 7).
//
// Why: for a tridiagonal-like band the per-column work is a
// handful of flops, and the warp-cooperative kernels spend their step on
// cross-lane traffic (ballot/redux pivot search, the pivot-row record through
// shared memory) -- C2's factorization took ~1,200 cycles per column step.  A
// thread owns its matrix's whole (kl+1) x (kv+1) window in registers: the
// pivot search, the interchange (a register select), the scaling and the
// rank-1 update are thread-local, and the only communication is with memory:
//  * the band row entering the window (kv+1 entries, a diagonal of the band
//    array: stride ldab-1) is loaded P steps ahead into a register ring;
//  * the retired pivot row (U row j), the multipliers (L column j), ipiv[j]
//    and y(j) are stored as they retire.  Each thread's stores of one column
//    land in the same 32-byte sectors within a few steps, so L2 merges them.
// No warp collectives: threads of a warp run independent matrices.
#pragma once
#include "common.cuh"

namespace bandlu {

template <int KL_, int KU_>
struct TrfThread {
    static constexpr int KL = KL_, KU = KU_, KV = KL + KU, W = KV + 1, R = KL + 1;
    // steps of prefetch (input rows in flight per thread): ~24 doubles of ring
    static constexpr int P = (24 / W) < 2 ? 2 : ((24 / W) > 8 ? 8 : 24 / W);
    static constexpr int THREADS = 128;
    static constexpr size_t smem_bytes() { return (size_t)P * (W + 1) * THREADS * sizeof(double); }
};

template <int KL, int KU, bool FWD, class AP, class PP, class BP>
__global__ void __launch_bounds__(TrfThread<KL, KU>::THREADS)
    gbtrf_thread_kernel(int m, int n, AP A, int ldab, PP Pv, int *__restrict__ info, int batch, BP Bv) {
    using C = TrfThread<KL, KU>;
    constexpr int KV = C::KV, W = C::W, R = C::R, P = C::P;
    const int64_t mat = (int64_t)blockIdx.x * C::THREADS + threadIdx.x;
    if (mat >= batch) return;  // no collectives: threads are independent
    double *__restrict__ ab = A.get(mat);
    int *__restrict__ ipiv = Pv.get(mat);
    double *__restrict__ bv = FWD ? Bv.get(mat) : nullptr;
    if (m <= 0 || n <= 0) {
        info[mat] = 0;
        return;
    }
    const int mn = min(m, n);

    // window w[r][c] = A(j + r, j + c) at step j; rows >= m and columns >= n hold 0
    double w[R][W];
#pragma unroll
    for (int r = 0; r < R; ++r)
#pragma unroll
        for (int c = 0; c < W; ++c) {
            const bool ok = r < m && c < n && c <= r + KU;  // c > r + KU: fill (never read, starts 0)
            w[r][c] = ok ? ab[(int64_t)c * ldab + KV + r - c] : 0.0;
        }
    double y[R];
    if constexpr (FWD) {
#pragma unroll
        for (int r = 0; r < R; ++r) y[r] = (r < m) ? bv[r] : 0.0;
    }

    // input row q = j + KL + 1 (enters at the end of step j): A(q, q-KL+c), c = 0..KV,
    // at ab[(q-KL)*ldab + KV+KL + c*(ldab-1)], copied P steps ahead by cp.async into this
    // thread's slots of a shared-memory ring (a register ring gets rotated by moves that
    // wait on the loads).  Slot (s, c) of thread t at ((s*(W+1) + c)*THREADS + t) doubles;
    // c = W holds the row's B entry.
    extern __shared__ __align__(16) double smem[];
    const uint32_t ring_s = smem_u32(smem) + (uint32_t)(threadIdx.x * 8);
    auto slot = [&](int s, int c) { return ring_s + (uint32_t)(((s * (W + 1) + c) * C::THREADS) * 8); };
    const void *dummy = g_dummy;
    auto issue_row = [&](int q, int s) {
#pragma unroll
        for (int c = 0; c < W; ++c) {
            const int col = q - KL + c;
            const bool ok = q < m && col < n;
            cp_async8(slot(s, c), ok ? (const void *)(ab + (int64_t)col * ldab + (KV + KL - c)) : dummy, ok ? 8u : 0u);
        }
        if constexpr (FWD) {
            const bool ok = q < m;
            cp_async8(slot(s, W), ok ? (const void *)(bv + q) : dummy, ok ? 8u : 0u);
        }
        cp_async_commit();
    };
#pragma unroll
    for (int s = 0; s < P; ++s) issue_row(KL + 1 + s, s);

    int linfo = 0;
#pragma unroll 1
    for (int j0 = 0; j0 < mn; j0 += P) {
#pragma unroll
        for (int s = 0; s < P; ++s) {
            const int j = j0 + s;
            if (j < mn) {  // (uniform: every thread runs the same m, n)
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
                ipiv[j] = j + jp + 1;
                double p = w[0][0];
#pragma unroll
                for (int r = 1; r < R; ++r) p = (jp == r) ? w[r][0] : p;
                if (p != 0.0) {
                    // ---- interchange rows j and j+jp (whole rows == LAPACK's right-only swap, reading 10)
#pragma unroll
                    for (int r = 1; r < R; ++r) {
                        if (jp == r) {
#pragma unroll
                            for (int c = 0; c < W; ++c) {
                                const double t = w[0][c];
                                w[0][c] = w[r][c];
                                w[r][c] = t;
                            }
                            if constexpr (FWD) {
                                const double t = y[0];
                                y[0] = y[r];
                                y[r] = t;
                            }
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
                } else if (linfo == 0) {
                    linfo = j + 1;  // zero pivot: no interchange, no scaling, no update (reading 3)
                }
                if constexpr (FWD) {  // forward substitution with column j of L
                    if (y[0] != 0.0) {
#pragma unroll
                        for (int r = 1; r < R; ++r)
                            if (r <= km) y[r] = __fma_rn(w[r][0], -y[0], y[r]);
                    }
                    bv[j] = y[0];
                }
                // ---- retire: L column j, U row j (AB[KV-c][j+c])
#pragma unroll
                for (int r = 1; r < R; ++r)
                    if (r <= km) ab[(int64_t)j * ldab + KV + r] = w[r][0];
#pragma unroll
                for (int c = 0; c < W; ++c)
                    if (j + c < n) ab[(int64_t)j * ldab + KV + c * (ldab - 1)] = w[0][c];
                // ---- slide: rows up, columns left; the row j+KL+1 enters at the bottom
#pragma unroll
                for (int r = 0; r < R - 1; ++r) {
#pragma unroll
                    for (int c = 0; c < W; ++c) w[r][c] = (c + 1 < W) ? w[r + 1][c + 1] : 0.0;
                    if constexpr (FWD) y[r] = y[r + 1];
                }
                cp_async_wait<P - 1>();  // this thread's copies of row j+KL+1 (issued P steps ago)
#pragma unroll
                for (int c = 0; c < W; ++c) w[R - 1][c] = ld_shared_f64(slot(s, c));
                if constexpr (FWD) y[R - 1] = ld_shared_f64(slot(s, W));
                issue_row(j + KL + 1 + P, s);
            }
        }
    }

    cp_async_wait<0>();
    // LAPACK's SET_FILLIN also zeroes fill-row positions whose matrix row is
    // >= m when m < n (those rows are never pivot rows here).
    if (m < n) {
        for (int c = m + KU + 1; c <= min(n - 1, m + KV - 1); ++c) {
#pragma unroll 1
            for (int r = 0; r < KL; ++r) {
                const int i = c - KV + r;
                const bool zeroed = (c >= KU + 1 && c <= min(KV, n) - 1 && r >= KV - c) || (c >= KV && c - KV < mn);
                if (i >= m && zeroed) ab[(int64_t)c * ldab + r] = 0.0;
            }
        }
    }
    info[mat] = linfo;
}

}  // namespace bandlu
