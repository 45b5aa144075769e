// generic.cuh -- the "safeguard" kernels (Sec. 5.4: "the
// reference implementation is kept as a safe guard"): correct for ANY m, n,
// kl, ku, nrhs, ldab, at modest speed.  Unlike the paper's reference path
// (a host loop launching ~5 kernels per column) each is ONE launch.
//
//  gbtrf_generic: one warp per matrix, factorization in place in global memory
//    (L1-resident working set), per column j:
//      SET_FILLIN -> IAMAX (warp argmax, first index) -> ipiv/info ->
//      GET_UPDATE_BOUND (ju) -> SWAP cols j..ju -> SCAL(1/pivot) ->
//      RANK_ONE_UPDATE over the (km x (ju-j)) block, lanes over elements.
//  gbtrs_generic: one thread per (matrix, RHS column), forward pass with the
//    pivots applied progressively, then the column-wise banded
//    back-substitution with bandwidth kv.
//
// Arithmetic per element is exactly the LAPACK operation sequence (FMA in the
// rank-1 update and both solves, multiplier = x * RN(1/p), true division in
// the back-solve), so results equal the oracle bitwise.
#pragma once
#include "common.cuh"

namespace bandlu {

template <class AP, class PP>
__global__ void __launch_bounds__(128) gbtrf_generic_kernel(int m, int n, int kl, int ku, AP A, int ldab,
                                                            PP P, int *__restrict__ info, int batch) {
    const int warp = (int)((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    const int lane = (int)lane_id();
    if (warp >= batch) return;
    // quick return first: with m == 0 or n == 0 the pointer arrays may be NULL
    if (m == 0 || n == 0) {
        if (lane == 0) info[warp] = 0;
        return;
    }
    double *__restrict__ ab = A.get(warp);
    int *__restrict__ ipiv = P.get(warp);
    const int kv = kl + ku;
    auto AB = [&](int r, int c) -> double & { return ab[(int64_t)c * ldab + r]; };
    // initial fill-in zeroing, columns ku+1 .. min(kv,n)-1, rows kv-j .. kl-1
    for (int j = ku + 1; j <= min(kv, n) - 1; ++j)
        for (int r = kv - j + lane; r <= kl - 1; r += 32) AB(r, j) = 0.0;
    __syncwarp();

    int ju = 0, linfo = 0;
    const int mn = min(m, n);
    for (int j = 0; j < mn; ++j) {
        if (j + kv < n)
            for (int r = lane; r < kl; r += 32) AB(r, j + kv) = 0.0;
        const int km = min(kl, m - 1 - j);
        // IAMAX: first index of max |x| over AB(kv..kv+km, j)
        uint64_t best = 0;
        int bidx = 0x7fffffff;
        for (int t = lane; t <= km; t += 32) {
            uint64_t k = abs_key(AB(kv + t, j));
            if (bidx == 0x7fffffff || k > best) { best = k; bidx = t; }
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) {
            uint64_t ob = __shfl_xor_sync(0xffffffffu, best, off);
            int oi = __shfl_xor_sync(0xffffffffu, bidx, off);
            if (oi != 0x7fffffff && (bidx == 0x7fffffff || ob > best || (ob == best && oi < bidx))) {
                best = ob;
                bidx = oi;
            }
        }
        const int jp = bidx;
        if (lane == 0) ipiv[j] = j + jp + 1;
        const double piv = AB(kv + jp, j);
        __syncwarp();
        if (piv != 0.0) {
            ju = max(ju, min(j + ku + jp, n - 1));
            if (jp != 0)
                for (int c = lane; c <= ju - j; c += 32) {
                    double t = AB(kv + jp - c, j + c);
                    AB(kv + jp - c, j + c) = AB(kv - c, j + c);
                    AB(kv - c, j + c) = t;
                }
            __syncwarp();
            if (km > 0) {
                const double rcp = 1.0 / AB(kv, j);
                for (int i = 1 + lane; i <= km; i += 32) AB(kv + i, j) = AB(kv + i, j) * rcp;
                __syncwarp();
                // lanes over rows i (multiplier in a register), loop over columns c:
                // U(j, j+c) is one broadcast load, rows i of column j+c are contiguous
                const int w = ju - j;
                for (int i0 = 1; i0 <= km; i0 += 32) {
                    const int i = i0 + lane;
                    const bool row = i <= km;
                    const double l = row ? AB(kv + i, j) : 0.0;
                    double *a = &AB(kv + i - 1, j + 1);  // AB(kv+i-c, j+c) for c = 1
#pragma unroll 4
                    for (int c = 1; c <= w; ++c, a += ldab - 1) {
                        const double y = AB(kv - c, j + c);
                        if (y != 0.0 && row) *a = __fma_rn(l, -y, *a);
                    }
                }
                __syncwarp();
            }
        } else if (linfo == 0) {
            linfo = j + 1;
        }
    }
    if (lane == 0) info[warp] = linfo;
}

// one thread per (matrix, rhs column); matrices with info != 0 are skipped
// when skip_info != nullptr (dgbsv composition, LAPACK DGBSV).
template <class AP, class PP, class BP>
__global__ void __launch_bounds__(128) gbtrs_generic_kernel(int n, int kl, int ku, int nrhs, AP A, int ldab, PP P,
                                                            BP B, int ldb, const int *__restrict__ skip_info,
                                                            int batch) {
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (tid >= (int64_t)batch * nrhs) return;
    const int mi = (int)(tid / nrhs), r = (int)(tid % nrhs);
    if (skip_info != nullptr && skip_info[mi] != 0) return;
    const double *__restrict__ ab = A.get(mi);
    const int *__restrict__ ipiv = P.get(mi);
    double *__restrict__ b = B.get(mi) + (int64_t)r * ldb;
    const int kv = kl + ku;
    if (kl > 0) {
        for (int j = 0; j < n - 1; ++j) {
            const int lm = min(kl, n - 1 - j);
            const int l = ipiv[j] - 1;
            if (l != j) {
                double t = b[l];
                b[l] = b[j];
                b[j] = t;
            }
            const double y = b[j];
            if (y != 0.0) {
                const double *col = ab + (int64_t)j * ldab + kv;
                for (int i = 1; i <= lm; ++i) b[j + i] = __fma_rn(col[i], -y, b[j + i]);
            }
        }
    }
    for (int j = n - 1; j >= 0; --j) {
        if (b[j] != 0.0) {
            const double *col = ab + (int64_t)j * ldab + kv - j;  // col[i] = AB(kv+i-j, j)
            const double x = __ddiv_rn(b[j], col[j]);
            b[j] = x;
            for (int i = j - 1; i >= max(0, j - kv); --i) b[i] = __fma_rn(-x, col[i], b[i]);
        }
    }
}

// Transposed solve A^T X = B (LAPACK DGBTRS 'T'/'C' branch; SURVEY 8(f) f2,
// the transA argument of the paper's dgbtrs_batch).  One thread per
// (matrix, RHS column), reference-BLAS operation order (one fma per term):
//   U^T: x_j = (b_j - sum_{i=max(0,j-kv)}^{j-1} U(i,j) x_i) / U(j,j), i ascending
//   L^T: for j = n-2..0: b_j -= sum_{i=1}^{lm} L(j+i,j) b_{j+i} (dot from 0, i
//        ascending), then swap b_j <-> b_{ipiv[j]-1}.
template <class AP, class PP, class BP>
__global__ void __launch_bounds__(128) gbtrs_t_generic_kernel(int n, int kl, int ku, int nrhs, AP A, int ldab, PP P,
                                                              BP B, int ldb, int batch) {
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (tid >= (int64_t)batch * nrhs) return;
    const int mi = (int)(tid / nrhs), r = (int)(tid % nrhs);
    const double *__restrict__ ab = A.get(mi);
    const int *__restrict__ ipiv = P.get(mi);
    double *__restrict__ b = B.get(mi) + (int64_t)r * ldb;
    const int kv = kl + ku;
    for (int j = 0; j < n; ++j) {
        const double *col = ab + (int64_t)j * ldab + kv - j;  // col[i] = AB(kv+i-j, j) = U(i, j)
        double temp = b[j];
        for (int i = max(0, j - kv); i <= j - 1; ++i) temp = __fma_rn(-col[i], b[i], temp);
        b[j] = __ddiv_rn(temp, col[j]);
    }
    if (kl > 0) {
        for (int j = n - 2; j >= 0; --j) {
            const int lm = min(kl, n - 1 - j);
            const double *lc = ab + (int64_t)j * ldab + kv;  // lc[i] = L(j+i, j)
            double temp = 0.0;
            for (int i = 1; i <= lm; ++i) temp = __fma_rn(b[j + i], lc[i], temp);
            b[j] = __dsub_rn(b[j], temp);
            const int l = ipiv[j] - 1;
            if (l != j) {
                const double t = b[l];
                b[l] = b[j];
                b[j] = t;
            }
        }
    }
}

}  // namespace bandlu
