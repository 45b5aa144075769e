// bandlu.cu -- C ABI host layer (include/bandlu.h): argument checking with
// LAPACK error numbering, quick returns, kernel-variant dispatch (the B200
// counterpart of the paper's "complete picture", Sec. 5.4
// P:558-567, and its tuning sweep P:526-556), launches.  No allocation and no
// host synchronisation on the device entry points.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <type_traits>
#include <cstdio>
#include <cstdlib>
#include <mutex>

#include "../../include/bandlu.h"
#include "common.cuh"
#include "gbtrf_rows.cuh"
#include "gbtrf_wide.cuh"
#include "gbtrf_tc.cuh"
#include "gbtrf_thread.cuh"
#include "gbtrf_thin.cuh"
#include "gbtrf_tpm.cuh"
#include "gbtrf_window.cuh"
#include "gbtrs_bwd.cuh"
#include "gbtrs_rows.cuh"
#include "gbtrs_t.cuh"
#include "gbtrs_blk.cuh"
#include "gbtrs_window.cuh"
#include "generic.cuh"
#include "gbtrf_cols.cuh"
#include "jit.cuh"

using namespace bandlu;

namespace {

// (KL, KU) pairs compiled into register-resident window kernels (PAPER.md
// Sec. 8.1 P:897-929 proposes per-(kl, ku) specialisation; we instantiate the
// bands of the paper's sweeps and of BASELINE.json's configs).
#ifdef BANDLU_ONLY_C3  // experiment builds: only the (10,10) and (1,1) windows
#define BANDLU_WINDOW_LIST(X) \
    X(1, 1)                   \
    X(10, 10)
#define BANDLU_TC_LIST(X) X(10, 10)
#else
#define BANDLU_WINDOW_LIST(X) \
    X(0, 0)                   \
    X(0, 3)                   \
    X(1, 1)                   \
    X(2, 2)                   \
    X(2, 3)                   \
    X(3, 0)                   \
    X(3, 2)                   \
    X(4, 4)                   \
    X(10, 7)                  \
    X(10, 10)                 \
    X(2, 32)
// (KL, KU) pairs also compiled as tensor-core (DMMA) factorization kernels
// (kl+1 <= 16; preferred by AUTO where compiled).
// opt-in experiment (-DBANDLU_WITH_TC): measured slower than the row-slot kernel, AUTO never picks it
#ifdef BANDLU_WITH_TC
#define BANDLU_TC_LIST(X) X(10, 10)
#else
#define BANDLU_TC_LIST(X)
#endif
#endif

// (KL, KU, G, R): bands compiled as row-slot kernels (gbtrf_rows.cuh, G lanes x
// R rows per matrix, block-preloaded incoming rows); a subset of the window
// list (the solve launches reuse the window trs kernels).  AUTO prefers them.
// Only bands where the kernel keeps the window kernel's matrices per warp
// (G*R >= kl+1+4 with the same G) are listed; R = 2 (4 matrices per warp at
// (10,10)) needs ~250 registers and measured slower.
#ifndef BANDLU_ROWS_C3_G
#define BANDLU_ROWS_C3_G 16
#endif
#ifndef BANDLU_ROWS_C3_R
#define BANDLU_ROWS_C3_R 1
#endif
#if defined(BANDLU_NO_ROWS)
#define BANDLU_ROWS_LIST(X)
#elif defined(BANDLU_ONLY_C3)
#define BANDLU_ROWS_LIST(X) X(10, 10, BANDLU_ROWS_C3_G, BANDLU_ROWS_C3_R)
#else
// thin bands as row-slot kernels too (G*R >= kl+1+4 with the window kernel's G): measured
// C2 (1,1) 0.156 -> 0.149 ms, C1 (2,2) 0.028 -> 0.026 ms, XGC-like (4,4) 0.077 -> 0.058 ms
#ifdef BANDLU_NO_ROWS_THIN
#define BANDLU_ROWS_THIN_LIST(X)
#else
#define BANDLU_ROWS_THIN_LIST(X) X(1, 1, 8, 1) X(2, 2, 8, 1) X(2, 3, 8, 1) X(4, 4, 16, 1)
#endif
#define BANDLU_ROWS_LIST(X)                              \
    X(10, 10, BANDLU_ROWS_C3_G, BANDLU_ROWS_C3_R)        \
    X(10, 7, 16, 1)                                      \
    X(2, 32, 8, 1)                                       \
    BANDLU_ROWS_THIN_LIST(X)
#endif

// (KL, KU, GL, CPL) compiled as column-owner kernels (gbtrf_cols.cuh; kl <= 4, square): GL lanes
// per matrix with CPL column slots each (GL*CPL >= kl+ku+1); AUTO's choice where compiled.
#ifndef BANDLU_COLS_C4_GL  // (2,32): lanes per matrix x column slots per lane (experiments: 32 x 2)
#define BANDLU_COLS_C4_GL 16
#define BANDLU_COLS_C4_CPL 3
#endif
#if defined(BANDLU_NO_COLS)
#define BANDLU_COLS_LIST(X)
#elif defined(BANDLU_ONLY_C3)
#define BANDLU_COLS_LIST(X) X(1, 1, 4, 1)
#else
#define BANDLU_COLS_LIST(X) \
    X(0, 0, 4, 1)           \
    X(0, 3, 4, 1)           \
    X(1, 1, 4, 1)           \
    X(2, 2, 4, 2)           \
    X(2, 3, 4, 2)           \
    X(3, 0, 4, 1)           \
    X(3, 2, 4, 2)           \
    X(2, 32, BANDLU_COLS_C4_GL, BANDLU_COLS_C4_CPL) \
    BANDLU_COLS_EXTRA(X)
#endif
// the same bands with the forward substitution riding along (dgbtrfs): (2,32) with 32 lanes x 2
// slots there (one lane per right-hand side up to 32; C4: 1.62 vs 1.73 ms for 16 x 3), while the
// factorization alone runs 16 x 3 (1.10 vs 1.54 ms for 32 x 2)
#ifndef BANDLU_COLS_C4F_GL
#define BANDLU_COLS_C4F_GL 32
#define BANDLU_COLS_C4F_CPL 2
#endif
#if defined(BANDLU_NO_COLS) || defined(BANDLU_ONLY_C3)
#define BANDLU_COLS_FWD_LIST(X) BANDLU_COLS_LIST(X)
#else
#define BANDLU_COLS_FWD_LIST(X) \
    X(0, 0, 4, 1)               \
    X(0, 3, 4, 1)               \
    X(1, 1, 4, 1)               \
    X(2, 2, 4, 2)               \
    X(2, 3, 4, 2)               \
    X(3, 0, 4, 1)               \
    X(3, 2, 4, 2)               \
    X(2, 32, BANDLU_COLS_C4F_GL, BANDLU_COLS_C4F_CPL) \
    BANDLU_COLS_EXTRA(X)
#endif
// opt-in (measured): (4,4) slower than the row-slot kernel (XGC-like 0.096 vs
// 0.072 ms, (4,4) n = 512 x 10,000: 0.576 vs 0.545 ms)
#ifdef BANDLU_COLS_WIDE
#define BANDLU_COLS_EXTRA(X) X(4, 4, 4, 3)
#else
#define BANDLU_COLS_EXTRA(X)
#endif

// (KL, KU, MPW) compiled as thread-per-matrix shared-memory-window kernels with rank-4
// panel updates (gbtrf_tpm.cuh; square matrices), MPW matrices per CTA.
#ifndef BANDLU_TPM_MPW
#define BANDLU_TPM_MPW 16
#endif
// opt-in experiment (-DBANDLU_WITH_TPM): bitwise equal, but measured 2.95 vs 0.93 ms at C3
// and 1.18 vs 0.23 ms at 1,250 matrices -- AUTO never picks it
#if defined(BANDLU_WITH_TPM)
#define BANDLU_TPM_LIST(X) X(10, 10, BANDLU_TPM_MPW)
#else
#define BANDLU_TPM_LIST(X)
#endif

// (KL, KU) compiled as thin-band thread-per-matrix kernels with cooperative whole-column
// staging (gbtrf_thin.cuh; square matrices).  Opt-in experiment (-DBANDLU_WITH_THIN): bitwise
// equal, but measured slower than the row-slot kernels -- C2 one-launch 0.483 vs 0.242 ms, C2
// factorization 0.318 vs 0.145 ms, C1 0.174 vs 0.035 ms
#if !defined(BANDLU_WITH_THIN)
#define BANDLU_THIN_LIST(X)
#elif defined(BANDLU_ONLY_C3)
#define BANDLU_THIN_LIST(X) X(1, 1)
#else
#define BANDLU_THIN_LIST(X) \
    X(0, 0)                 \
    X(0, 3)                 \
    X(1, 1)                 \
    X(2, 2)                 \
    X(2, 3)                 \
    X(3, 0)                 \
    X(3, 2)                 \
    X(4, 4)
#endif

// (KL, KU) compiled as thread-per-matrix factorization kernels (gbtrf_thread.cuh, thin
// bands); BANDLU_THREAD_AUTO_LIST: the ones AUTO prefers (measured)
// opt-in experiment (-DBANDLU_WITH_THREAD): measured slower than the row-slot kernels for every
// thin band, AUTO never picks it
#if !defined(BANDLU_WITH_THREAD)
#define BANDLU_THREAD_LIST(X)
#elif defined(BANDLU_ONLY_C3)
#define BANDLU_THREAD_LIST(X) X(1, 1)
#else
#define BANDLU_THREAD_LIST(X) \
    X(0, 0)                   \
    X(0, 3)                   \
    X(1, 1)                   \
    X(2, 2)                   \
    X(2, 3)                   \
    X(3, 0)                   \
    X(3, 2)                   \
    X(4, 4)
#endif
#if defined(BANDLU_THREAD_AUTO_ALL)  // experiments: every compiled thin band
#define BANDLU_THREAD_AUTO_LIST(X) BANDLU_THREAD_LIST(X)
#elif !defined(BANDLU_THREAD_AUTO_LIST)
#define BANDLU_THREAD_AUTO_LIST(X)
#endif

// (KL, KU) with kl+1 > 32: two-warp row-slot kernel (gbtrf_wide.cuh), dispatched as
// BANDLU_ROWS; the solve uses the window trs kernel (BANDLU_TRS_LIST).
#if defined(BANDLU_NO_ROWS) || defined(BANDLU_ONLY_C3)
#define BANDLU_WIDE_LIST(X)
#else
#define BANDLU_WIDE_LIST(X) X(32, 32)
#endif
#define BANDLU_TRS_LIST(X) \
    BANDLU_WINDOW_LIST(X)  \
    BANDLU_WIDE_LIST(X)
// (KL, KU) with kl+ku+1 <= 32 compiled as lane-per-row solve kernels
// (gbtrs_rows.cuh); AUTO's choice for nrhs == 1.
#ifdef BANDLU_ONLY_C3
#define BANDLU_TRS_ROWS_LIST(X) \
    X(1, 1)                     \
    X(10, 10)
#else
#define BANDLU_TRS_ROWS_LIST(X) \
    X(0, 0)                     \
    X(0, 3)                     \
    X(1, 1)                     \
    X(2, 2)                     \
    X(2, 3)                     \
    X(3, 0)                     \
    X(3, 2)                     \
    X(4, 4)                     \
    X(10, 7)                    \
    X(10, 10)
#endif

// trs launch geometry: target resident warps (148 SMs x 8)
#ifndef BANDLU_TRS_WPSM
#define BANDLU_TRS_WPSM 8
#endif
constexpr int64_t kTrsWarpsTarget = 148 * BANDLU_TRS_WPSM;
#ifndef BANDLU_TRST_WPSM
#define BANDLU_TRST_WPSM BANDLU_TRS_WPSM
#endif
constexpr int64_t kTrsTWarpsTarget = 148 * BANDLU_TRST_WPSM;  // transposed solve (gbtrs_t.cuh)
// ring solves: matrices per warp also bounded by shared memory, so that BANDLU_TRS_WPSM one-warp
// CTAs still fit on an SM (a 32-matrix (32,32) ring is 142 KB: one warp per SM)
constexpr size_t kTrsSmemPerWarp = 227 * 1024 / BANDLU_TRS_WPSM;
template <class F>
int trs_fit_gpw(int gpw, F smem_of) {
#ifndef BANDLU_TRS_NO_FIT
    while (gpw > 1 && smem_of(gpw) > kTrsSmemPerWarp) gpw >>= 1;
#endif
    return gpw;
}

inline int cuda_ret(cudaError_t e) { return e == cudaSuccess ? 0 : BANDLU_ERR_CUDA + (int)e; }

template <class K>
int set_smem(K kernel, size_t bytes) {
    if (bytes > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
        if (e != cudaSuccess) return cuda_ret(e);
    }
    return 0;
}

// ------------------------------------------------------------------ trf
template <int KL, int KU, bool FWD, class AP, class PP, class BP>
int launch_trf_window(int m, int n, AP A, int ldab, PP P, int *info, int batch, cudaStream_t st, BP B) {
    using C = TrfWin<KL, KU>;
    auto k = gbtrf_window_kernel<KL, KU, FWD, AP, PP, BP>;
    size_t sm = C::smem_bytes();
    if (int r = set_smem(k, sm)) return r;
    const int64_t per_block = (int64_t)C::WARPS * C::GPW;
    const unsigned grid = (unsigned)((batch + per_block - 1) / per_block);
    k<<<grid, C::WARPS * 32, sm, st>>>(m, n, A, ldab, P, info, batch, B);
    return cuda_ret(cudaGetLastError());
}

template <int KL, int KU, int G, int R, int FL, class AP, class PP, class BP>
int launch_trf_rows(int m, int n, AP A, int ldab, PP P, int *info, int batch, cudaStream_t st, BP B) {
    using C = TrfRows<KL, KU, G, R>;
    auto k = gbtrf_rows_kernel<KL, KU, G, R, FL, AP, PP, BP>;
    size_t sm = (FL & FL_YSM) ? C::smem_bytes_y(n) : C::smem_bytes();
    if (int r = set_smem(k, sm)) return r;
    const int64_t per_block = (int64_t)C::WARPS * C::GPW;
    const unsigned grid = (unsigned)((batch + per_block - 1) / per_block);
    k<<<grid, C::WARPS * 32, sm, st>>>(m, n, A, ldab, P, info, batch, B);
    return cuda_ret(cudaGetLastError());
}

template <int KL, int KU, int GL, int CPL, int FL, class AP, class PP, class BP>
int launch_trf_cols(int n, AP A, int ldab, PP P, int *info, int batch, cudaStream_t st, BP B, int nrhs = 0,
                    int ldb = 1) {
    using C = TrfCols<KL, KU, GL, CPL>;
    auto k = gbtrf_cols_kernel<KL, KU, GL, CPL, FL, AP, PP, BP>;
    // the right-hand-side staging is allocated in both modes: for (2,32) it also holds the
    // factorization alone at 3 CTAs/SM (1.10 ms; 4 CTAs with the smaller layout: 1.18 ms)
    const size_t sm = C::smem_bytes(true);
    if (int r = set_smem(k, sm)) return r;
    const int64_t per_block = (int64_t)C::WARPS * C::GPW;
    const unsigned grid = (unsigned)((batch + per_block - 1) / per_block);
    k<<<grid, C::WARPS * 32, sm, st>>>(n, A, ldab, P, info, batch, B, nrhs, ldb);
    return cuda_ret(cudaGetLastError());
}

template <int KL, int KU, bool FWD, class AP, class PP, class BP>
int launch_trf_wide(int m, int n, AP A, int ldab, PP P, int *info, int batch, cudaStream_t st, BP B) {
    using C = TrfWide<KL, KU>;
    auto k = gbtrf_wide_kernel<KL, KU, FWD, AP, PP, BP>;
    size_t sm = C::smem_bytes();
    if (int r = set_smem(k, sm)) return r;
    k<<<(unsigned)batch, 64, sm, st>>>(m, n, A, ldab, P, info, batch, B);
    return cuda_ret(cudaGetLastError());
}

template <int KL, int KU, bool FWD, class AP, class PP, class BP>
int launch_trf_thread(int m, int n, AP A, int ldab, PP P, int *info, int batch, cudaStream_t st, BP B) {
    using C = TrfThread<KL, KU>;
    const unsigned grid = (unsigned)((batch + C::THREADS - 1) / C::THREADS);
    auto k = gbtrf_thread_kernel<KL, KU, FWD, AP, PP, BP>;
    if (int r = set_smem(k, C::smem_bytes())) return r;
    k<<<grid, C::THREADS, C::smem_bytes(), st>>>(m, n, A, ldab, P, info, batch, B);
    return cuda_ret(cudaGetLastError());
}

template <int KL, int KU, int FL, class AP, class PP, class BP>
int launch_trf_thin(int n, AP A, int ldab, PP P, int *info, int batch, cudaStream_t st, BP B) {
    using C = TrfThin<KL, KU>;
    auto k = gbtrf_thin_kernel<KL, KU, FL, AP, PP, BP>;
    const size_t sm = C::smem_bytes(ldab);
    if (sm > 227 * 1024) return BANDLU_ERR_UNSUPPORTED;
    if (int r = set_smem(k, sm)) return r;
    const unsigned grid = (unsigned)((batch + 31) / 32);
    k<<<grid, 32, sm, st>>>(n, A, ldab, P, info, batch, B);
    return cuda_ret(cudaGetLastError());
}

bool trf_thin_available(int kl, int ku) {
#define X(a, b) \
    if (kl == a && ku == b) return true;
    BANDLU_THIN_LIST(X)
#undef X
    return false;
}

template <int KL, int KU, int MPW, bool FWD, class AP, class PP, class BP>
int launch_trf_tpm(int n, AP A, int ldab, PP P, int *info, int batch, cudaStream_t st, BP B) {
    using C = TrfTpm<KL, KU, MPW>;
    auto k = gbtrf_tpm_kernel<KL, KU, MPW, FWD, AP, PP, BP>;
    const size_t sm = C::cta_bytes();
    if (int r = set_smem(k, sm)) return r;
    const unsigned grid = (unsigned)((batch + MPW - 1) / MPW);
    k<<<grid, MPW, sm, st>>>(n, A, ldab, P, info, batch, B);
    return cuda_ret(cudaGetLastError());
}

bool trf_tpm_available(int kl, int ku) {
#define X(a, b, w) \
    if (kl == a && ku == b) return true;
    BANDLU_TPM_LIST(X)
#undef X
    return false;
}

template <class AP, class PP>
int launch_trf_generic(int m, int n, int kl, int ku, AP A, int ldab, PP P, int *info, int batch, cudaStream_t st) {
    const unsigned grid = (unsigned)(((int64_t)batch * 32 + 127) / 128);
    gbtrf_generic_kernel<AP, PP><<<grid, 128, 0, st>>>(m, n, kl, ku, A, ldab, P, info, batch);
    return cuda_ret(cudaGetLastError());
}

bool trf_window_available(int kl, int ku) {
#define X(a, b) \
    if (kl == a && ku == b) return true;
    BANDLU_WINDOW_LIST(X)
#undef X
    return false;
}

bool trf_wide_available(int kl, int ku) {
#define X(a, b) \
    if (kl == a && ku == b) return true;
    BANDLU_WIDE_LIST(X)
#undef X
    return false;
}

bool trf_rows_available(int kl, int ku) {
#define X(a, b, g, r) \
    if (kl == a && ku == b) return true;
    BANDLU_ROWS_LIST(X)
#undef X
    return trf_wide_available(kl, ku);
}

bool trf_cols_available(int kl, int ku) {
#define X(a, b, g, c) \
    if (kl == a && ku == b) return true;
    BANDLU_COLS_LIST(X)
#undef X
    return false;
}
// the column-owner kernel with the fused backward solve (nrhs = 1): one launch for dgbtrfs.
// Opt-in (-DBANDLU_COLS_FUSED): bitwise, but the 4-lane backward pass (y re-read from B, prefetch
// distance 2-4 steps) measured slower than the separate backward kernel: C2 0.59 vs 0.245 ms,
// C1 0.049 vs 0.034 ms (the row-slot fused kernel).
bool trf_cols_fused(int kl, int ku) {
#ifdef BANDLU_COLS_FUSED
#define X(a, b, g, c) \
    if (kl == a && ku == b) return FusedSolveAny<a + b, g>::ok;
    BANDLU_COLS_FWD_LIST(X)
#undef X
#endif
    (void)kl, (void)ku;
    return false;
}
#ifndef BANDLU_COLS_MIN_NRHS
#define BANDLU_COLS_MIN_NRHS 1  // 2: one right-hand side keeps the row-slot / window plan
#endif
// right-hand sides the column-owner kernel can carry through its forward substitution (one per lane)
int trf_cols_rhs(int kl, int ku) {
#define X(a, b, g, c) \
    if (kl == a && ku == b) return g;
    BANDLU_COLS_FWD_LIST(X)
#undef X
    return 0;
}

bool trs_window_available(int kl, int ku) {
#define X(a, b) \
    if (kl == a && ku == b) return true;
    BANDLU_TRS_LIST(X)
#undef X
    return false;
}

bool trs_rows_available(int kl, int ku) {
#define X(a, b) \
    if (kl == a && ku == b) return true;
    BANDLU_TRS_ROWS_LIST(X)
#undef X
    return false;
}

bool trf_thread_available(int kl, int ku) {
#define X(a, b) \
    if (kl == a && ku == b) return true;
    BANDLU_THREAD_LIST(X)
#undef X
    return false;
}
bool trf_thread_preferred(int kl, int ku) {
#define X(a, b) \
    if (kl == a && ku == b) return true;
    BANDLU_THREAD_AUTO_LIST(X)
#undef X
    return false;
}

bool trf_tc_available(int kl, int ku) {
#define X(a, b) \
    if (kl == a && ku == b) return true;
    BANDLU_TC_LIST(X)
#undef X
    return false;
}

// ---- run-time compiled bands (jit.cuh): any (kl, ku) that no list above instantiates
// takes the row-slot kernel (kl + 5 <= 32 lanes: G = pow2 >= kl + 5) or the two-warp
// wide kernel (kl + 5 <= 64), compiled on first use; strided entry points only.
bool trf_compiled(int kl, int ku) { return trf_rows_available(kl, ku) || trf_window_available(kl, ku); }
int jit_rows_g(int kl) {
    int g = 8;
    while (g < kl + 5) g *= 2;
    return g <= 32 ? g : 0;
}
bool jit_band(int kl, int ku) {
    return !trf_compiled(kl, ku) && (jit_rows_g(kl) > 0 || kl + 5 <= 64) && bandlu_jit::nvrtc().ok;
}
const bandlu_jit::Kern &jit_trf(int kl, int ku, int fl) {
    const int g = jit_rows_g(kl);
    return g ? bandlu_jit::rows(kl, ku, g, fl) : bandlu_jit::wide(kl, ku, (fl & FL_FWD) != 0);
}
int jit_launch_trf(const bandlu_jit::Kern &K, int kl, int fl, int m, int n, Strided<double> A, int ldab,
                   Strided<int> P, int *info, int batch, cudaStream_t st, Strided<double> B) {
    void *args[] = {&m, &n, &A, &ldab, &P, &info, &batch, &B};
    if (jit_rows_g(kl)) {
        const long long W = K.geo[0], GPW = K.geo[1], GD = K.geo[3];
        const size_t sm = (size_t)(W * GPW * (GD + ((fl & FL_YSM) ? ((n + 15) & ~15) : 0)) * 8);
        if (sm > 48 * 1024) {
            cudaError_t e = cudaFuncSetAttribute((const void *)K.k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
            if (e != cudaSuccess) return cuda_ret(e);
        }
        const unsigned grid = (unsigned)((batch + W * GPW - 1) / (W * GPW));
        return cuda_ret(cudaLaunchKernel((const void *)K.k, dim3(grid), dim3((unsigned)(W * 32)), args, sm, st));
    }
    const size_t sm = (size_t)K.geo[0];
    if (sm > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute((const void *)K.k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        if (e != cudaSuccess) return cuda_ret(e);
    }
    return cuda_ret(cudaLaunchKernel((const void *)K.k, dim3((unsigned)batch), dim3(64), args, sm, st));
}
// run-time compiled window solve (any nrhs); skip: info array (dgbsv) or nullptr; fwd 0: backward only
int jit_launch_trs_window(int kl, int ku, int n, int nrhs, Strided<const double> A, int ldab, Strided<const int> P,
                          Strided<double> B, int ldb, const int *skip, int batch, cudaStream_t st, int fwd) {
    int R = nrhs >= 32 ? 32 : pow2_ceil(nrhs);
    int chunks = (nrhs + 31) / 32;
    const bool pairs = R >= 2;
    if (nrhs == 1 && fwd) {  // the block-granular solve, as for compiled bands
        const bandlu_jit::Kern &K = bandlu_jit::blk(kl, ku);
        if (!K.ok) return BANDLU_ERR_UNSUPPORTED;
        int gpw = 32;
        while (gpw > 1 && (int64_t)batch < (int64_t)gpw * kTrsWarpsTarget) gpw >>= 1;
        gpw = trs_fit_gpw(gpw, [&](int x) { return (size_t)(K.geo[0] + (long long)x * K.geo[1]) * 8; });
        const size_t sm = (size_t)(K.geo[0] + (long long)gpw * K.geo[1]) * 8;
        if (sm > 48 * 1024) {
            cudaError_t e = cudaFuncSetAttribute((const void *)K.k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
            if (e != cudaSuccess) return cuda_ret(e);
        }
        const unsigned grid = (unsigned)((batch + gpw - 1) / gpw);
        void *args[] = {&n, &nrhs, &A, &ldab, &P, &B, &ldb, &skip, &batch, &R, &chunks, &gpw, &fwd};
        return cuda_ret(cudaLaunchKernel((const void *)K.k, dim3(grid), dim3(32), args, sm, st));
    }
    const bandlu_jit::Kern &K = bandlu_jit::window(kl, ku, pairs);
    if (!K.ok) return BANDLU_ERR_UNSUPPORTED;
    const int64_t units = (int64_t)batch * chunks;
    int gpw = 32 / R;
    while (gpw > 1 && units < (int64_t)gpw * kTrsWarpsTarget) gpw >>= 1;
    int li = 0;
    while ((1 << li) < R) ++li;
    gpw = trs_fit_gpw(gpw, [&](int x) { return (size_t)(K.geo[0] + (long long)x * K.geo[1 + li]) * 8; });
    const size_t sm = (size_t)(K.geo[0] + (long long)gpw * K.geo[1 + li]) * 8;
    if (sm > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute((const void *)K.k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        if (e != cudaSuccess) return cuda_ret(e);
    }
    const unsigned grid = (unsigned)((units + gpw - 1) / gpw);
    void *args[] = {&n, &nrhs, &A, &ldab, &P, &B, &ldb, &skip, &batch, &R, &chunks, &gpw, &fwd};
    return cuda_ret(cudaLaunchKernel((const void *)K.k, dim3(grid), dim3(32), args, sm, st));
}
// run-time compiled backward-only solve (kl + ku + 1 <= 32), matrices per warp as launch_trs_bwd_lean
int jit_launch_trs_bwd(int kl, int ku, int n, Strided<const double> A, int ldab, Strided<double> B, int batch,
                       cudaStream_t st) {
    int gpw = 32;
    while (gpw > 1 && batch < (int64_t)gpw * kTrsWarpsTarget) gpw >>= 1;
    gpw = gpw < 2 ? 2 : gpw;
    const bandlu_jit::Kern &K = bandlu_jit::bwd(kl, ku, gpw);
    if (!K.ok) return BANDLU_ERR_UNSUPPORTED;
    const size_t sm = (size_t)(K.geo[0] + K.geo[1] * gpw) * 8;
    if (sm > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute((const void *)K.k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        if (e != cudaSuccess) return cuda_ret(e);
    }
    const unsigned grid = (unsigned)((batch + gpw - 1) / gpw);
    void *args[] = {&n, &A, &ldab, &B, &batch};
    return cuda_ret(cudaLaunchKernel((const void *)K.k, dim3(grid), dim3(32), args, sm, st));
}

int pick_trf(int m, int n, int kl, int ku) {
    if (m <= 0 || n <= 0) return BANDLU_GENERIC;
    if (jit_band(kl, ku)) return BANDLU_ROWS;  // compiled on first use (jit.cuh)
    if (m == n && trf_cols_available(kl, ku)) return BANDLU_COLS;
    // BANDLU_TC is opt-in: measured slower than the row-owner window at C3
    // (1.54 vs 1.10 ms), so AUTO never picks it.
    if (trf_thread_preferred(kl, ku)) return BANDLU_THREAD;
    if (trf_rows_available(kl, ku)) return BANDLU_ROWS;
    return trf_window_available(kl, ku) ? BANDLU_WINDOW : BANDLU_GENERIC;
}

template <int KL, int KU, bool FWD, class AP, class PP, class BP>
int launch_trf_tc(int m, int n, AP A, int ldab, PP P, int *info, int batch, cudaStream_t st, BP B) {
    using C = TrfTc<KL, KU>;
    auto k = gbtrf_tc_kernel<KL, KU, FWD, AP, PP, BP>;
    size_t sm = C::smem_bytes();
    if (int r = set_smem(k, sm)) return r;
    const unsigned grid = (unsigned)((batch + C::WARPS - 1) / C::WARPS);
    k<<<grid, C::WARPS * 32, sm, st>>>(m, n, A, ldab, P, info, batch, B);
    return cuda_ret(cudaGetLastError());
}

template <class AP, class PP>
int run_trf(int m, int n, int kl, int ku, AP A, int ldab, PP P, int *info, int batch, cudaStream_t st, int variant) {
    if (batch == 0) return 0;
    if (variant == BANDLU_AUTO) variant = pick_trf(m, n, kl, ku);
    if (variant == BANDLU_TC && m > 0 && n > 0) {
#define X(a, b) \
    if (kl == a && ku == b) return launch_trf_tc<a, b, false>(m, n, A, ldab, P, info, batch, st, Strided<double>{nullptr, 0});
        BANDLU_TC_LIST(X)
#undef X
        return BANDLU_ERR_UNSUPPORTED;
    }
    if (variant == BANDLU_COLS && m > 0 && n > 0) {
        if (m != n) return BANDLU_ERR_UNSUPPORTED;
#define X(a, b, g, c) \
    if (kl == a && ku == b) return launch_trf_cols<a, b, g, c, 0>(n, A, ldab, P, info, batch, st, Strided<double>{nullptr, 0});
        BANDLU_COLS_LIST(X)
#undef X
        return BANDLU_ERR_UNSUPPORTED;
    }
    if (variant == BANDLU_THIN && m > 0 && n > 0) {
        if (m != n) return BANDLU_ERR_UNSUPPORTED;
        if constexpr (std::is_same_v<AP, Strided<double>>) {
#define X(a, b) \
    if (kl == a && ku == b) return launch_trf_thin<a, b, 0>(n, A, ldab, P, info, batch, st, Strided<double>{nullptr, 0});
            BANDLU_THIN_LIST(X)
#undef X
        }
        return BANDLU_ERR_UNSUPPORTED;
    }
    if (variant == BANDLU_TPM && m > 0 && n > 0) {
        if (m != n) return BANDLU_ERR_UNSUPPORTED;
#define X(a, b, w) \
    if (kl == a && ku == b) return launch_trf_tpm<a, b, w, false>(n, A, ldab, P, info, batch, st, Strided<double>{nullptr, 0});
        BANDLU_TPM_LIST(X)
#undef X
        return BANDLU_ERR_UNSUPPORTED;
    }
    if (variant == BANDLU_THREAD && m > 0 && n > 0) {
#define X(a, b) \
    if (kl == a && ku == b) return launch_trf_thread<a, b, false>(m, n, A, ldab, P, info, batch, st, Strided<double>{nullptr, 0});
        BANDLU_THREAD_LIST(X)
#undef X
        return BANDLU_ERR_UNSUPPORTED;
    }
    if (variant == BANDLU_ROWS && m > 0 && n > 0) {
#define X(a, b, g, r) \
    if (kl == a && ku == b) return launch_trf_rows<a, b, g, r, 0>(m, n, A, ldab, P, info, batch, st, Strided<double>{nullptr, 0});
        BANDLU_ROWS_LIST(X)
#undef X
#define X(a, b) \
    if (kl == a && ku == b) return launch_trf_wide<a, b, false>(m, n, A, ldab, P, info, batch, st, Strided<double>{nullptr, 0});
        BANDLU_WIDE_LIST(X)
#undef X
        if constexpr (std::is_same_v<AP, Strided<double>>) {
            if (jit_band(kl, ku)) {
                const bandlu_jit::Kern &K = jit_trf(kl, ku, 0);
                if (K.ok) return jit_launch_trf(K, kl, 0, m, n, A, ldab, P, info, batch, st, Strided<double>{nullptr, 0});
            }
            if (jit_band(kl, ku)) return launch_trf_generic(m, n, kl, ku, A, ldab, P, info, batch, st);
        } else {
            if (jit_band(kl, ku)) return launch_trf_generic(m, n, kl, ku, A, ldab, P, info, batch, st);
        }
        return BANDLU_ERR_UNSUPPORTED;
    }
    if (variant == BANDLU_WINDOW && m > 0 && n > 0) {
#define X(a, b) \
    if (kl == a && ku == b) return launch_trf_window<a, b, false>(m, n, A, ldab, P, info, batch, st, Strided<double>{nullptr, 0});
        BANDLU_WINDOW_LIST(X)
#undef X
        return BANDLU_ERR_UNSUPPORTED;
    }
    if (variant != BANDLU_GENERIC && variant != BANDLU_WINDOW && variant != BANDLU_TC && variant != BANDLU_ROWS &&
        variant != BANDLU_THREAD && variant != BANDLU_TPM && variant != BANDLU_THIN && variant != BANDLU_COLS)
        return BANDLU_ERR_UNSUPPORTED;
    return launch_trf_generic(m, n, kl, ku, A, ldab, P, info, batch, st);
}

// ------------------------------------------------------------------ trs
// block-granular ring solve (gbtrs_blk.cuh), lane per (matrix, RHS column)
template <int KL, int KU, class AP, class PP, class BP>
int launch_trs_blk(int n, int nrhs, AP A, int ldab, PP P, BP B, int ldb, const int *skip, int batch,
                   cudaStream_t st, int fwd = 1) {
    using C = TrsBlk<KL, KU>;
    const int R = nrhs >= 32 ? 32 : pow2_ceil(nrhs);
    const int chunks = (nrhs + 31) / 32;
    auto k = gbtrs_blk_kernel<KL, KU, AP, PP, BP>;
    const int64_t units = (int64_t)batch * chunks;
    int gpw = 32 / R;
    while (gpw > 1 && units < (int64_t)gpw * kTrsWarpsTarget) gpw >>= 1;
    gpw = trs_fit_gpw(gpw, [&](int x) { return C::smem_bytes(R, x); });
    const size_t sm = C::smem_bytes(R, gpw);
    if (int r = set_smem(k, sm)) return r;
    const unsigned grid = (unsigned)((units + gpw - 1) / gpw);
    k<<<grid, 32, sm, st>>>(n, nrhs, A, ldab, P, B, ldb, skip, batch, R, chunks, gpw, fwd);
    return cuda_ret(cudaGetLastError());
}

template <int KL, int KU, class AP, class PP, class BP>
int launch_trs_window(int n, int nrhs, AP A, int ldab, PP P, BP B, int ldb, const int *skip, int batch,
                      cudaStream_t st, int fwd = 1) {
    // one RHS, full solve: the block-granular solve (C3 0.54 vs 0.61 ms, (32,32) n = 2048 5.3 vs
    // 9.4 ms); nrhs >= 2 (C4 2.03 vs 2.10 ms) and the backward-only pass after a forward-fused
    // factorization ((32,32) C5 points 1-4% faster) keep the row-pair window solve -- DESIGN.md Sec. 6
#if defined(BANDLU_TRS_BLK_ALL)
    return launch_trs_blk<KL, KU>(n, nrhs, A, ldab, P, B, ldb, skip, batch, st, fwd);
#elif !defined(BANDLU_TRS_NO_BLK)
    if (nrhs == 1 && fwd) return launch_trs_blk<KL, KU>(n, nrhs, A, ldab, P, B, ldb, skip, batch, st, fwd);
#endif
    using C = TrsWin<KL, KU>;
    const int R = nrhs >= 32 ? 32 : pow2_ceil(nrhs);
    const int chunks = (nrhs + 31) / 32;
    const bool pairs = R >= 2;
    auto k = pairs ? gbtrs_window_kernel<KL, KU, true, AP, PP, BP> : gbtrs_window_kernel<KL, KU, false, AP, PP, BP>;
    const int64_t units = (int64_t)batch * chunks;
    // Each lane runs a long serial chain: spread the units over >= ~8 warps per
    // SM (all four schedulers busy) before packing more of them into a warp.
    int gpw = 32 / R;
    while (gpw > 1 && units < (int64_t)gpw * kTrsWarpsTarget) gpw >>= 1;
    gpw = trs_fit_gpw(gpw, [&](int x) { return C::smem_bytes(R, x, pairs); });
    const size_t sm = C::smem_bytes(R, gpw, pairs);
    if (int r = set_smem(k, sm)) return r;
    const unsigned grid = (unsigned)((units + gpw - 1) / gpw);
    k<<<grid, 32, sm, st>>>(n, nrhs, A, ldab, P, B, ldb, skip, batch, R, chunks, gpw, fwd);
    return cuda_ret(cudaGetLastError());
}

template <int KL, int KU, class AP, class PP, class BP>
int launch_trs_rows(int n, int nrhs, AP A, int ldab, PP P, BP B, int ldb, const int *skip, int batch,
                    cudaStream_t st, int fwd = 1) {
    using C = TrsRows<KL, KU>;
    auto k = fwd ? gbtrs_rows_kernel<KL, KU, true, AP, PP, BP> : gbtrs_rows_kernel<KL, KU, false, AP, PP, BP>;
    const int64_t units = (int64_t)batch * nrhs, per_block = (int64_t)C::WARPS * C::GPW;
    const unsigned grid = (unsigned)((units + per_block - 1) / per_block);
    k<<<grid, C::WARPS * 32, 0, st>>>(n, nrhs, A, ldab, P, B, ldb, skip, batch);
    return cuda_ret(cudaGetLastError());
}

template <class AP, class PP, class BP>
int launch_trs_generic(int n, int kl, int ku, int nrhs, AP A, int ldab, PP P, BP B, int ldb, const int *skip,
                       int batch, cudaStream_t st) {
    const int64_t threads = (int64_t)batch * nrhs;
    const unsigned grid = (unsigned)((threads + 127) / 128);
    gbtrs_generic_kernel<AP, PP, BP><<<grid, 128, 0, st>>>(n, kl, ku, nrhs, A, ldab, P, B, ldb, skip, batch);
    return cuda_ret(cudaGetLastError());
}

// The lane-per-row solve issues one division and one broadcast per matrix-step
// (the window solve one per 32/R matrices); it only wins where a warp packs
// >= 8 matrices (kl+ku+1 <= 4): measured C2 (1,1) 0.097 vs 0.105 ms, but C3
// (10,10) 0.78 vs 0.32 ms and PELE-like (10,10) 0.083 vs 0.039 ms.
#ifdef BANDLU_NO_TRS_ROWS_AUTO  // experiments
bool trs_rows_preferred(int, int) { return false; }
#else
bool trs_rows_preferred(int kl, int ku) { return kl + ku + 1 <= 4 && trs_rows_available(kl, ku); }
#endif

// run-time compiled window solve for bands without a compiled one (jit.cuh)
bool jit_trs_band(int kl, int ku) {
    return !trs_window_available(kl, ku) && kl + ku <= 64 && bandlu_jit::nvrtc().ok;
}

int pick_trs(int n, int kl, int ku, int nrhs) {
    (void)n;
    if (nrhs == 1 && trs_rows_preferred(kl, ku)) return BANDLU_ROWS;
    return (trs_window_available(kl, ku) || jit_trs_band(kl, ku)) ? BANDLU_WINDOW : BANDLU_GENERIC;
}

template <class AP, class PP, class BP>
int launch_trs_t_generic(int n, int kl, int ku, int nrhs, AP A, int ldab, PP P, BP B, int ldb, int batch,
                         cudaStream_t st) {
    const int64_t threads = (int64_t)batch * nrhs;
    const unsigned grid = (unsigned)((threads + 127) / 128);
    gbtrs_t_generic_kernel<AP, PP, BP><<<grid, 128, 0, st>>>(n, kl, ku, nrhs, A, ldab, P, B, ldb, batch);
    return cuda_ret(cudaGetLastError());
}

// ring-staged transposed solve (gbtrs_t.cuh), lane per (matrix, RHS column) as the window solve
template <int KL, int KU, class AP, class PP, class BP>
int launch_trs_t(int n, int nrhs, AP A, int ldab, PP P, BP B, int ldb, int batch, cudaStream_t st) {
    using C = TrsT<KL, KU>;
    const int R = nrhs >= 32 ? 32 : pow2_ceil(nrhs);
    const int chunks = (nrhs + 31) / 32;
    auto k = gbtrs_t_kernel<KL, KU, AP, PP, BP>;
    const int64_t units = (int64_t)batch * chunks;
    int gpw = 32 / R;
    while (gpw > 1 && units < (int64_t)gpw * kTrsTWarpsTarget) gpw >>= 1;
    gpw = trs_fit_gpw(gpw, [&](int x) { return C::smem_bytes(R, x); });
    const size_t sm = C::smem_bytes(R, gpw);
    if (int r = set_smem(k, sm)) return r;
    const unsigned grid = (unsigned)((units + gpw - 1) / gpw);
    k<<<grid, 32, sm, st>>>(n, nrhs, A, ldab, P, B, ldb, batch, R, chunks, gpw);
    return cuda_ret(cudaGetLastError());
}
// run-time compiled transposed solve (bands without a compiled one)
int jit_launch_trs_t(int kl, int ku, int n, int nrhs, Strided<const double> A, int ldab, Strided<const int> P,
                     Strided<double> B, int ldb, int batch, cudaStream_t st) {
    int R = nrhs >= 32 ? 32 : pow2_ceil(nrhs);
    int chunks = (nrhs + 31) / 32;
    const bandlu_jit::Kern &K = bandlu_jit::trst(kl, ku);
    if (!K.ok) return BANDLU_ERR_UNSUPPORTED;
    const int64_t units = (int64_t)batch * chunks;
    int gpw = 32 / R;
    while (gpw > 1 && units < (int64_t)gpw * kTrsTWarpsTarget) gpw >>= 1;
    int li = 0;
    while ((1 << li) < R) ++li;
    gpw = trs_fit_gpw(gpw, [&](int x) { return (size_t)(K.geo[0] + (long long)x * K.geo[1 + li]) * 8; });
    const size_t sm = (size_t)(K.geo[0] + (long long)gpw * K.geo[1 + li]) * 8;
    if (sm > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute((const void *)K.k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        if (e != cudaSuccess) return cuda_ret(e);
    }
    const unsigned grid = (unsigned)((units + gpw - 1) / gpw);
    void *args[] = {&n, &nrhs, &A, &ldab, &P, &B, &ldb, &batch, &R, &chunks, &gpw};
    return cuda_ret(cudaLaunchKernel((const void *)K.k, dim3(grid), dim3(32), args, sm, st));
}

template <class AP, class PP, class BP>
int run_trs(int n, int kl, int ku, int nrhs, AP A, int ldab, PP P, BP B, int ldb, const int *skip, int batch,
            cudaStream_t st, int variant, char trans = 'N') {
    if (batch == 0 || n == 0 || nrhs == 0) return 0;
    if (trans != 'N' && trans != 'n') {  // A^T X = B ('C' == 'T' for real data)
        if (variant == BANDLU_AUTO) variant = (trs_window_available(kl, ku) || jit_trs_band(kl, ku)) ? BANDLU_WINDOW
                                                                                                     : BANDLU_GENERIC;
        if (variant == BANDLU_WINDOW) {
#define X(a, b) \
    if (kl == a && ku == b) return launch_trs_t<a, b>(n, nrhs, A, ldab, P, B, ldb, batch, st);
            BANDLU_TRS_LIST(X)
#undef X
            if (jit_trs_band(kl, ku)) {
                if constexpr (std::is_same_v<AP, Strided<const double>>) {
                    const int r = jit_launch_trs_t(kl, ku, n, nrhs, A, ldab, P, B, ldb, batch, st);
                    if (r != BANDLU_ERR_UNSUPPORTED) return r;
                }
                return launch_trs_t_generic(n, kl, ku, nrhs, A, ldab, P, B, ldb, batch, st);
            }
            return BANDLU_ERR_UNSUPPORTED;
        }
        if (variant != BANDLU_GENERIC) return BANDLU_ERR_UNSUPPORTED;
        return launch_trs_t_generic(n, kl, ku, nrhs, A, ldab, P, B, ldb, batch, st);
    }
    if (variant == BANDLU_AUTO) variant = pick_trs(n, kl, ku, nrhs);
    if (variant == BANDLU_WINDOW) {
#define X(a, b) \
    if (kl == a && ku == b) return launch_trs_window<a, b>(n, nrhs, A, ldab, P, B, ldb, skip, batch, st);
        BANDLU_TRS_LIST(X)
#undef X
        if (jit_trs_band(kl, ku)) {
            if constexpr (std::is_same_v<AP, Strided<const double>>) {
                const int r = jit_launch_trs_window(kl, ku, n, nrhs, A, ldab, P, B, ldb, skip, batch, st, 1);
                if (r != BANDLU_ERR_UNSUPPORTED) return r;
            }
            return launch_trs_generic(n, kl, ku, nrhs, A, ldab, P, B, ldb, skip, batch, st);
        }
        return BANDLU_ERR_UNSUPPORTED;
    }
    if (variant == BANDLU_ROWS) {
#define X(a, b) \
    if (kl == a && ku == b) return launch_trs_rows<a, b>(n, nrhs, A, ldab, P, B, ldb, skip, batch, st);
        BANDLU_TRS_ROWS_LIST(X)
#undef X
        return BANDLU_ERR_UNSUPPORTED;
    }
    if (variant != BANDLU_GENERIC) return BANDLU_ERR_UNSUPPORTED;
    return launch_trs_generic(n, kl, ku, nrhs, A, ldab, P, B, ldb, skip, batch, st);
}

// lean backward-only solve (gbtrs_bwd.cuh); matrices per warp as the window solve
template <int KL, int KU, class AP, class BP>
int launch_trs_bwd_lean(int n, AP A, int ldab, BP B, int batch, cudaStream_t st) {
    using C = TrsBwd<KL, KU>;
    int gpw = 32;
    while (gpw > 1 && batch < (int64_t)gpw * kTrsWarpsTarget) gpw >>= 1;
    gpw = gpw < 2 ? 2 : gpw;
    const size_t sm = C::smem_bytes(gpw);
    const unsigned grid = (unsigned)((batch + gpw - 1) / gpw);
    auto go = [&](auto k) -> int {
        if (int r = set_smem(k, sm)) return r;
        k<<<grid, 32, sm, st>>>(n, A, ldab, B, batch);
        return cuda_ret(cudaGetLastError());
    };
    switch (gpw) {
        case 2: return go(gbtrs_bwd_kernel<KL, KU, 2, AP, BP>);
        case 4: return go(gbtrs_bwd_kernel<KL, KU, 4, AP, BP>);
        case 8: return go(gbtrs_bwd_kernel<KL, KU, 8, AP, BP>);
        case 16: return go(gbtrs_bwd_kernel<KL, KU, 16, AP, BP>);
        default: return go(gbtrs_bwd_kernel<KL, KU, 32, AP, BP>);
    }
}

// backward-only solve after the fused factorization (nrhs == 1)
template <int KL, int KU, class AP, class PP, class BP>
int launch_trs_bwd(int n, AP A, int ldab, PP P, BP B, int ldb, int batch, cudaStream_t st) {
#ifndef BANDLU_TRS_BWD_WINDOW
    if constexpr (KL + KU + 1 <= 32) {
        if (trs_rows_preferred(KL, KU)) return launch_trs_rows<KL, KU>(n, 1, A, ldab, P, B, ldb, nullptr, batch, st, 0);
    }
#endif
#ifdef BANDLU_TRS_BWD_BLK
    return launch_trs_blk<KL, KU>(n, 1, A, ldab, P, B, ldb, nullptr, batch, st, 0);
#endif
#ifndef BANDLU_TRS_BWD_WINDOW
    if constexpr (std::is_same_v<AP, Strided<const double>> && KL + KU + 1 <= 32)
        return launch_trs_bwd_lean<KL, KU>(n, A, ldab, B, batch, st);
#endif
    return launch_trs_window<KL, KU>(n, 1, A, ldab, P, B, ldb, nullptr, batch, st, 0);
}

// ------------------------------------- fused factor + solve (dgbtrf; dgbtrs)
// nrhs == 1 on a band with a row-slot kernel: ONE launch (the fused gbsv
// kernel: factorization, forward substitution on the fly, backward
// substitution by the same lanes, Sec. 7).
// y(0..n-1) sits in shared memory when it fits next to the row ring at the
// kernel's resident-CTA target, else in B.  Other compiled bands with
// nrhs == 1: the factorization kernel with the forward substitution, then the
// backward-only solve launch.  Otherwise the plain trf + trs pair.
// Results equal dgbtrf followed by dgbtrs('N') for every matrix (dgbtrfs
// solves B even where info > 0; dgbsv leaves B untouched there).
// phase: 0 = every launch, 1 = first launch only, 2 = second launch only (the
// bench times them separately); | TRFS_TWO_LAUNCH forces the two-launch plan.
constexpr int TRFS_TWO_LAUNCH = BANDLU_TRFS_TWO_LAUNCH, TRFS_FUSED = BANDLU_TRFS_FUSED, TRFS_THIN = BANDLU_TRFS_THIN;
constexpr size_t kSmemPerSM = 227 * 1024;

template <int KL, int KU, int G, int R>
bool rows_ysm_fits(int n) {
#ifdef BANDLU_FUSED_NO_YSM  // experiments: y always in B
    if (n > 0) return false;
#endif
    using C = TrfRows<KL, KU, G, R>;
    const size_t b = C::smem_bytes_y(n);
    return b <= kSmemPerSM && b * (size_t)C::MINB <= kSmemPerSM;
}

// the fused backward solve keeps two right-hand-side rows per lane (backsolve_fused.cuh)
bool rows_fused_available(int kl, int ku) {
#define X(a, b, g, r) \
    if (kl == a && ku == b) return FusedSolve<a + b, g>::ok;
    BANDLU_ROWS_LIST(X)
#undef X
    return false;
}

// Matrices one wave of the fused kernel holds (SMs x resident CTAs x matrices per CTA).
// The fused kernel wins while the batch fits in one wave (the backward pass adds
// latency but no wave); beyond that the factorization + forward kernel followed by
// the bandwidth-bound backward kernel (8-32 matrices per warp) is faster -- measured
// C3 1.30 vs 1.25 ms, PELE-like 0.147 vs 0.140 ms, C2 0.262 vs 0.242 ms; XGC-like
// (512 matrices) 0.092 vs 0.115 ms, C1 0.035 vs 0.043 ms.  The
// choice depends on the batch, the results do not (same operation sequence).
int sm_count() {
    int d = 0, c = 148;
    if (cudaGetDevice(&d) == cudaSuccess) cudaDeviceGetAttribute(&c, cudaDevAttrMultiProcessorCount, d);
    return c;
}
int64_t rows_wave(int kl, int ku) {
#define X(a, b, g, r) \
    if (kl == a && ku == b) return (int64_t)sm_count() * TrfRows<a, b, g, r>::MINB * TrfRows<a, b, g, r>::WARPS * TrfRows<a, b, g, r>::GPW;
    BANDLU_ROWS_LIST(X)
#undef X
    return 0;
}
// dgbtrfs, nrhs = 1, a column-owner band: the column-owner kernel with the forward and backward
// substitutions in the same launch (AUTO; TRFS_FUSED forces the row-slot fused kernel instead,
// TRFS_TWO_LAUNCH the column-owner factorization + a backward launch)
bool cols_fused_pick(int n, int kl, int ku, int nrhs, int phase) {
    return n > 0 && nrhs == 1 && trf_cols_fused(kl, ku) && !(phase & (TRFS_TWO_LAUNCH | TRFS_FUSED));
}

bool trfs_fused_pick(int n, int kl, int ku, int nrhs, int64_t batch, int phase) {
    if (n <= 0 || nrhs != 1 || !rows_fused_available(kl, ku)) return false;
    if (phase & TRFS_TWO_LAUNCH) return false;
    if (phase & TRFS_FUSED) return true;
    if (cols_fused_pick(n, kl, ku, nrhs, phase)) return false;
    return batch <= rows_wave(kl, ku);
}

bool rows_ysm_fits_rt(int n, int kl, int ku) {
#define X(a, b, g, r) \
    if (kl == a && ku == b) return rows_ysm_fits<a, b, g, r>(n);
    BANDLU_ROWS_LIST(X)
#undef X
    return false;
}

// kernel ids / byte classes reported by bandlu_trfs_plan (include/bandlu.h)
enum { KN_TRF_ROWS = 1, KN_TRF_WINDOW, KN_TRF_WIDE, KN_TRF_THREAD, KN_TRF_GENERIC, KN_TRS_BWD, KN_TRS_ROWS,
       KN_TRS_WINDOW, KN_TRS_GENERIC, KN_TRF_THIN, KN_TRS_BLK, KN_TRF_COLS };
enum { KB_TRF = 1, KB_TRF_FWD, KB_TRS_BWD, KB_TRS, KB_GBSV };

// run-time compiled bands, nrhs == 1: is the fused kernel picked?  (geometry from the
// compiled module: [0] WARPS, [1] GPW, [2] MINB, [3] GROUP_DBL, [4] fused solve ok)
bool jit_fused_pick(const bandlu_jit::Kern &K, int kl, int64_t batch, int phase) {
    if (!K.ok || !jit_rows_g(kl) || !K.geo[4] || (phase & TRFS_TWO_LAUNCH)) return false;
    return (phase & TRFS_FUSED) || batch <= (int64_t)sm_count() * K.geo[2] * K.geo[0] * K.geo[1];
}
bool jit_ysm_fits(const bandlu_jit::Kern &K, int n) {
    const size_t b = (size_t)(K.geo[0] * K.geo[1] * (K.geo[3] + ((n + 15) & ~15)) * 8);
    return b <= kSmemPerSM && b * (size_t)K.geo[2] <= kSmemPerSM;
}

// the launches one dgbtrfs call makes for the shape (what run_trfs does)
int trfs_plan(int n, int kl, int ku, int nrhs, int64_t batch, int phase, int *kinds) {
    int k = 0;
    auto put = [&](int name, int bytes) { if (kinds) kinds[k] = name * 16 + bytes; ++k; };
    if (n <= 0 || nrhs <= 0) return 0;
    if ((phase & TRFS_THIN) && nrhs == 1 && trf_thin_available(kl, ku)) {
        put(KN_TRF_THIN, KB_GBSV);
        return k;
    }
    phase &= ~TRFS_THIN;
    if (nrhs == 1 && jit_band(kl, ku)) {
        const bandlu_jit::Kern &K = jit_trf(kl, ku, FL_FWD);
        if (K.ok) {
            if (jit_fused_pick(K, kl, batch, phase)) {
                put(KN_TRF_ROWS, KB_GBSV);
                return k;
            }
            put(jit_rows_g(kl) ? KN_TRF_ROWS : KN_TRF_WIDE, KB_TRF_FWD);
            put(kl + ku + 1 <= 32 ? KN_TRS_BWD : KN_TRS_WINDOW, KB_TRS_BWD);
            return k;
        }
    }
    if (cols_fused_pick(n, kl, ku, nrhs, phase)) {
        put(KN_TRF_COLS, KB_GBSV);
        return k;
    }
    if (trfs_fused_pick(n, kl, ku, nrhs, batch, phase)) {
        put(KN_TRF_ROWS, KB_GBSV);
        return k;
    }
    if (nrhs >= BANDLU_COLS_MIN_NRHS && nrhs <= trf_cols_rhs(kl, ku)) {
        put(KN_TRF_COLS, KB_TRF_FWD);
        put(nrhs > 1 ? KN_TRS_WINDOW
            : kl + ku + 1 <= 4 && trs_rows_preferred(kl, ku) ? KN_TRS_ROWS
            : kl + ku + 1 <= 32 ? KN_TRS_BWD : KN_TRS_WINDOW, KB_TRS_BWD);
        return k;
    }
    if (nrhs == 1 && (trf_window_available(kl, ku) || trf_wide_available(kl, ku))) {
        const int tv = trf_thread_preferred(kl, ku) ? KN_TRF_THREAD
                       : trf_wide_available(kl, ku) ? KN_TRF_WIDE
                       : trf_rows_available(kl, ku) ? KN_TRF_ROWS : KN_TRF_WINDOW;
        put(tv, KB_TRF_FWD);
        put(kl + ku + 1 <= 4 && trs_rows_preferred(kl, ku) ? KN_TRS_ROWS
            : kl + ku + 1 <= 32 ? KN_TRS_BWD : KN_TRS_WINDOW, KB_TRS_BWD);
        return k;
    }
    const int tv = pick_trf(n, n, kl, ku);
    put(tv == BANDLU_COLS ? KN_TRF_COLS : tv == BANDLU_ROWS ? (trf_wide_available(kl, ku) ? KN_TRF_WIDE : KN_TRF_ROWS)
        : tv == BANDLU_WINDOW ? KN_TRF_WINDOW : tv == BANDLU_THREAD ? KN_TRF_THREAD : KN_TRF_GENERIC, KB_TRF);
    const int sv = pick_trs(n, kl, ku, nrhs);
    put(sv == BANDLU_ROWS ? KN_TRS_ROWS : sv == BANDLU_WINDOW ? (nrhs == 1 ? KN_TRS_BLK : KN_TRS_WINDOW) : KN_TRS_GENERIC,
        KB_TRS);
    return k;
}

template <class AP, class PP, class BP>
int run_trfs(int n, int kl, int ku, int nrhs, AP A, int ldab, PP P, BP B, int ldb, int *info, int batch,
             cudaStream_t st, int phase) {
    if (batch == 0) return 0;
    if ((phase & TRFS_THIN) && n > 0 && nrhs == 1 && trf_thin_available(kl, ku)) {
        if ((phase & 3) == 2) return 0;  // one launch
#define X(a, b) \
    if (kl == a && ku == b) return launch_trf_thin<a, b, 3>(n, A, ldab, P, info, batch, st, B);
        BANDLU_THIN_LIST(X)
#undef X
    }
    phase &= ~TRFS_THIN;
    const bool fused = trfs_fused_pick(n, kl, ku, nrhs, batch, phase);
    const bool cfused = cols_fused_pick(n, kl, ku, nrhs, phase);
    const int pflags = phase & (TRFS_TWO_LAUNCH | TRFS_FUSED);
    phase &= ~(TRFS_TWO_LAUNCH | TRFS_FUSED);
    if (cfused) {
        if (phase == 2) return 0;  // one launch
#define X(a, b, g, c)                                                                                             \
    if (kl == a && ku == b) {                                                                                     \
        if constexpr (FusedSolveAny<a + b, g>::ok)                                                                \
            return launch_trf_cols<a, b, g, c, FL_FWD | FL_BWD>(n, A, ldab, P, info, batch, st, B, nrhs, ldb);   \
    }
        BANDLU_COLS_FWD_LIST(X)
#undef X
        return BANDLU_ERR_UNSUPPORTED;
    }
    if (fused) {
        if (phase == 2) return 0;  // the whole path is the first (only) launch
        const bool ysm = rows_ysm_fits_rt(n, kl, ku);
#define X(a, b, g, rr)                                                                                                   \
    if (kl == a && ku == b) {                                                                                            \
        if constexpr (FusedSolve<a + b, g>::ok)                                                                          \
            return ysm ? launch_trf_rows<a, b, g, rr, FL_FWD | FL_BWD | FL_YSM>(n, n, A, ldab, P, info, batch, st, B) \
                       : launch_trf_rows<a, b, g, rr, FL_FWD | FL_BWD>(n, n, A, ldab, P, info, batch, st, B);       \
    }
        BANDLU_ROWS_LIST(X)
#undef X
        return BANDLU_ERR_UNSUPPORTED;
    }
    // a column-owner band beyond one wave of the fused row-slot kernel: factorization + forward
    // substitution of up to GL right-hand sides, then the backward solve (C4: 3.48 -> 3.19 ms; C2's
    // factorization + forward 0.144 -> 0.135 ms once y is stored per 4-row block)
    if (n > 0 && nrhs >= BANDLU_COLS_MIN_NRHS && nrhs <= trf_cols_rhs(kl, ku)) {
        int r = BANDLU_ERR_UNSUPPORTED;
        Strided<const double> Ac{A.base, A.stride};
        Strided<const int> Pc{P.base, P.stride};
#define X(a, b, g, c)                                                                                       \
    if (kl == a && ku == b) {                                                                               \
        r = 0;                                                                                              \
        if (phase != 2) r = launch_trf_cols<a, b, g, c, FL_FWD>(n, A, ldab, P, info, batch, st, B, nrhs, ldb); \
        if (r == 0 && phase != 1)                                                                           \
            r = nrhs == 1 ? launch_trs_bwd<a, b>(n, Ac, ldab, Pc, B, ldb, batch, st)                        \
                          : launch_trs_window<a, b>(n, nrhs, Ac, ldab, Pc, B, ldb, nullptr, batch, st, 0);  \
    }
        BANDLU_COLS_FWD_LIST(X)
#undef X
        return r;
    }
    if (n > 0 && nrhs == 1 && (trf_window_available(kl, ku) || trf_wide_available(kl, ku))) {
        int r = BANDLU_ERR_UNSUPPORTED;
        Strided<const double> Ac{A.base, A.stride};
        Strided<const int> Pc{P.base, P.stride};
        if (trf_thread_preferred(kl, ku)) {
#define X(a, b)                                                                                           \
    if (kl == a && ku == b) {                                                                             \
        r = 0;                                                                                            \
        if (phase != 2) r = launch_trf_thread<a, b, true>(n, n, A, ldab, P, info, batch, st, B);          \
        if (r == 0 && phase != 1) r = launch_trs_bwd<a, b>(n, Ac, ldab, Pc, B, ldb, batch, st);           \
    }
            BANDLU_THREAD_LIST(X)
#undef X
            return r;
        }
        if (trf_rows_available(kl, ku)) {
#define X(a, b, g, rr)                                                                                    \
    if (kl == a && ku == b) {                                                                             \
        r = 0;                                                                                            \
        if (phase != 2) r = launch_trf_rows<a, b, g, rr, FL_FWD>(n, n, A, ldab, P, info, batch, st, B);   \
        if (r == 0 && phase != 1) r = launch_trs_bwd<a, b>(n, Ac, ldab, Pc, B, ldb, batch, st);           \
    }
            BANDLU_ROWS_LIST(X)
#undef X
#define X(a, b)                                                                                           \
    if (kl == a && ku == b) {                                                                             \
        r = 0;                                                                                            \
        if (phase != 2) r = launch_trf_wide<a, b, true>(n, n, A, ldab, P, info, batch, st, B);           \
        if (r == 0 && phase != 1) r = launch_trs_bwd<a, b>(n, Ac, ldab, Pc, B, ldb, batch, st);           \
    }
            BANDLU_WIDE_LIST(X)
#undef X
            return r;
        }
#define X(a, b)                                                                                           \
    if (kl == a && ku == b) {                                                                             \
        r = 0;                                                                                            \
        if (phase != 2) r = launch_trf_window<a, b, true>(n, n, A, ldab, P, info, batch, st, B);          \
        if (r == 0 && phase != 1) r = launch_trs_bwd<a, b>(n, Ac, ldab, Pc, B, ldb, batch, st);           \
    }
        BANDLU_WINDOW_LIST(X)
#undef X
        return r;
    }
    if (n > 0 && nrhs == 1 && jit_band(kl, ku)) {  // run-time compiled band (jit.cuh)
        const bandlu_jit::Kern &K = jit_trf(kl, ku, FL_FWD);
        if (K.ok) {
            const int ph = phase;
            if (jit_fused_pick(K, kl, batch, pflags)) {
                if (ph == 2) return 0;
                const int fl = FL_FWD | FL_BWD | (jit_ysm_fits(K, n) ? FL_YSM : 0);
                const bandlu_jit::Kern &KF = jit_trf(kl, ku, fl);
                if (KF.ok) return jit_launch_trf(KF, kl, fl, n, n, A, ldab, P, info, batch, st, B);
            } else {
                int r = 0;
                if (ph != 2) r = jit_launch_trf(K, kl, FL_FWD, n, n, A, ldab, P, info, batch, st, B);
                if (r == 0 && ph != 1) {
                    Strided<const double> Ac{A.base, A.stride};
                    Strided<const int> Pc{P.base, P.stride};
                    r = (kl + ku + 1 <= 32) ? jit_launch_trs_bwd(kl, ku, n, Ac, ldab, B, batch, st)
                                            : jit_launch_trs_window(kl, ku, n, 1, Ac, ldab, Pc, B, ldb, nullptr, batch,
                                                                    st, 0);
                }
                return r;
            }
        }
    }
    if (phase != 2)
        if (int r = run_trf(n, n, kl, ku, A, ldab, P, info, batch, st, BANDLU_AUTO)) return r;
    if (phase == 1) return 0;
    return run_trs(n, kl, ku, nrhs, Strided<const double>{A.base, A.stride}, ldab, Strided<const int>{P.base, P.stride},
                   B, ldb, nullptr, batch, st, BANDLU_AUTO);
}

// dgbsv (strided): the fused single-launch kernel writes B only where info == 0
// (FL_SKIPI, y in shared memory); otherwise trf, then trs skipping info > 0.
template <class AP, class PP, class BP>
int run_gbsv(int n, int kl, int ku, int nrhs, AP A, int ldab, PP P, BP B, int ldb, int *info, int batch,
             cudaStream_t st) {
    if (batch == 0) return 0;
    if (trfs_fused_pick(n, kl, ku, nrhs, batch, 0) && rows_ysm_fits_rt(n, kl, ku)) {
#define X(a, b, g, rr)                                                                                      \
    if (kl == a && ku == b) {                                                                               \
        if constexpr (FusedSolve<a + b, g>::ok)                                                             \
            return launch_trf_rows<a, b, g, rr, FL_FWD | FL_BWD | FL_YSM | FL_SKIPI>(n, n, A, ldab, P, info, \
                                                                                     batch, st, B);         \
    }
        BANDLU_ROWS_LIST(X)
#undef X
    }
    if (n > 0 && nrhs == 1 && jit_band(kl, ku)) {  // run-time compiled band: the fused kernel (jit.cuh)
        const bandlu_jit::Kern &K = jit_trf(kl, ku, FL_FWD);
        if (K.ok && jit_fused_pick(K, kl, batch, 0) && jit_ysm_fits(K, n)) {
            const int fl = FL_FWD | FL_BWD | FL_YSM | FL_SKIPI;
            const bandlu_jit::Kern &KF = jit_trf(kl, ku, fl);
            if (KF.ok) return jit_launch_trf(KF, kl, fl, n, n, A, ldab, P, info, batch, st, B);
        }
    }
    if (int r = run_trf(n, n, kl, ku, A, ldab, P, info, batch, st, BANDLU_AUTO)) return r;
    return run_trs(n, kl, ku, nrhs, Strided<const double>{A.base, A.stride}, ldab,
                   Strided<const int>{P.base, P.stride}, B, ldb, info, batch, st, BANDLU_AUTO);
}

// ------------------------------------------------------------ arg checks
int check_trf(int m, int n, int kl, int ku, const void *A, int ldab, int64_t strideA, const void *P,
              int64_t strideP, const void *info, int batch, bool strided) {
    if (m < 0) return -1;
    if (n < 0) return -2;
    if (kl < 0) return -3;
    if (ku < 0) return -4;
    if (ldab < 2 * kl + ku + 1) return -6;
    if (strided) {  // (m,n,kl,ku,dA,ldab,strideA,dipiv,strideP,dinfo,batch)
        if (batch < 0) return -11;
        if (batch > 0) {
            if (!A) return -5;
            if (strideA < (int64_t)ldab * n) return -7;
            if (!P && m > 0 && n > 0) return -8;
            if (strideP < (int64_t)(m < n ? m : n)) return -9;
            if (!info) return -10;
        }
    } else {  // (m,n,kl,ku,dA_array,ldab,dipiv_array,dinfo,batch)
        if (batch < 0) return -9;
        if (batch > 0) {
            if (!A) return -5;
            if (!P && m > 0 && n > 0) return -7;
            if (!info) return -8;
        }
    }
    return 0;
}

int check_trs(char trans, int n, int kl, int ku, int nrhs, const void *A, int ldab, int64_t strideA, const void *P,
              int64_t strideP, const void *B, int ldb, int64_t strideB, int batch, bool strided) {
    if (trans != 'N' && trans != 'n' && trans != 'T' && trans != 't' && trans != 'C' && trans != 'c') return -1;
    if (n < 0) return -2;
    if (kl < 0) return -3;
    if (ku < 0) return -4;
    if (nrhs < 0) return -5;
    if (ldab < 2 * kl + ku + 1) return -7;
    if (strided) {  // (trans,n,kl,ku,nrhs,dA,ldab,strideA,dipiv,strideP,dB,ldb,strideB,batch)
        if (ldb < (n > 1 ? n : 1)) return -12;
        if (batch < 0) return -14;
        if (batch > 0 && n > 0 && nrhs > 0) {
            if (!A) return -6;
            if (strideA < (int64_t)ldab * n) return -8;
            if (!P) return -9;
            if (strideP < n) return -10;
            if (!B) return -11;
            if (strideB < (int64_t)ldb * nrhs) return -13;
        }
    } else {
        if (ldb < (n > 1 ? n : 1)) return -10;  // (trans,n,kl,ku,nrhs,dA_array,ldab,dipiv_array,dB_array,ldb,batch)
        if (batch < 0) return -11;
        if (batch > 0 && n > 0 && nrhs > 0) {
            if (!A) return -6;
            if (!P) return -8;
            if (!B) return -9;
        }
    }
    return 0;
}

}  // namespace

// =================================================================== ABI
extern "C" {

int bandlu_version(void) { return 1; }

int bandlu_trf_variant(int m, int n, int kl, int ku) { return pick_trf(m, n, kl, ku); }
int bandlu_tc_available(int kl, int ku) { return trf_tc_available(kl, ku) ? 1 : 0; }
int bandlu_rows_available(int kl, int ku) { return trf_rows_available(kl, ku) ? 1 : 0; }
int bandlu_thread_available(int kl, int ku) { return trf_thread_available(kl, ku) ? 1 : 0; }
int bandlu_tpm_available(int kl, int ku) { return trf_tpm_available(kl, ku) ? 1 : 0; }
int bandlu_thin_available(int kl, int ku) { return trf_thin_available(kl, ku) ? 1 : 0; }
int bandlu_cols_available(int kl, int ku) { return trf_cols_available(kl, ku) ? 1 : 0; }

// 1 if (kl, ku) is served by run-time compiled kernels (jit.cuh), else 0 (no compilation)
int bandlu_jit_band(int kl, int ku) { return jit_band(kl, ku) ? 1 : 0; }

// NVRTC-compile (no load, no GPU needed) the kernels a run-time compiled band uses: the
// factorization (plain, + forward, fused) and the solves.  0 = every kernel compiled;
// otherwise 1 and the first error in log (truncated to loglen).
int bandlu_jit_check(int kl, int ku, char *log, int loglen) {
    std::vector<bandlu_jit::Spec> specs;
    const int g = jit_rows_g(kl);
    if (g) {
        specs.push_back(bandlu_jit::rows_spec(kl, ku, g, 0));
        specs.push_back(bandlu_jit::rows_spec(kl, ku, g, FL_FWD));
        if (kl + ku + 1 + BANDLU_FUSED_PF <= 2 * g)  // FusedSolve<kv, g>::ok
            specs.push_back(bandlu_jit::rows_spec(kl, ku, g, FL_FWD | FL_BWD | FL_YSM));
    } else {
        specs.push_back(bandlu_jit::wide_spec(kl, ku, true));
    }
    if (kl + ku + 1 <= 32) specs.push_back(bandlu_jit::bwd_spec(kl, ku, 8));
    specs.push_back(bandlu_jit::window_spec(kl, ku, true));
    specs.push_back(bandlu_jit::window_spec(kl, ku, false));
    specs.push_back(bandlu_jit::blk_spec(kl, ku));
    specs.push_back(bandlu_jit::trst_spec(kl, ku));
    for (const auto &sp : specs) {
        std::vector<char> bin;
        std::string low;
        const std::string err = bandlu_jit::compile(sp.first, sp.second, bin, low);
        if (!err.empty()) {
            if (log && loglen > 0) {
                std::strncpy(log, err.c_str(), (size_t)loglen - 1);
                log[loglen - 1] = '\0';
            }
            return 1;
        }
    }
    return 0;
}
int bandlu_trs_rows_available(int kl, int ku) { return trs_rows_available(kl, ku) ? 1 : 0; }
int bandlu_trs_variant(int n, int kl, int ku, int nrhs) { return pick_trs(n, kl, ku, nrhs); }
int bandlu_trfs_plan(int n, int kl, int ku, int nrhs, int batch, int phase, int *kinds) {
    if (n < 0 || kl < 0 || ku < 0 || nrhs < 0 || batch < 0) return -1;
    if ((phase & TRFS_TWO_LAUNCH) && (phase & TRFS_FUSED)) return -1;
    return trfs_plan(n, kl, ku, nrhs, batch, phase, kinds);  // phase flags as for dgbtrfs
}

int dgbtrf_strided_batched_ex(int m, int n, int kl, int ku, double *dA, int ldab, int64_t strideA, int *dipiv,
                              int64_t strideP, int *dinfo, int batch, bandlu_stream_t stream, int variant) {
    if (int r = check_trf(m, n, kl, ku, dA, ldab, strideA, dipiv, strideP, dinfo, batch, true)) return r;
    return run_trf(m, n, kl, ku, Strided<double>{dA, strideA}, ldab, Strided<int>{dipiv, strideP}, dinfo, batch,
                   (cudaStream_t)stream, variant);
}

int dgbtrf_strided_batched(int m, int n, int kl, int ku, double *dA, int ldab, int64_t strideA, int *dipiv,
                           int64_t strideP, int *dinfo, int batch, bandlu_stream_t stream) {
    return dgbtrf_strided_batched_ex(m, n, kl, ku, dA, ldab, strideA, dipiv, strideP, dinfo, batch, stream,
                                     BANDLU_AUTO);
}

int dgbtrf_batched(int m, int n, int kl, int ku, double *const *dA_array, int ldab, int *const *dipiv_array,
                   int *dinfo, int batch, bandlu_stream_t stream) {
    if (int r = check_trf(m, n, kl, ku, dA_array, ldab, 0, dipiv_array, 0, dinfo, batch, false)) return r;
    return run_trf(m, n, kl, ku, PtrArray<double>{dA_array}, ldab, PtrArray<int>{dipiv_array}, dinfo, batch,
                   (cudaStream_t)stream, BANDLU_AUTO);
}

int dgbtrs_strided_batched_ex(char trans, int n, int kl, int ku, int nrhs, const double *dA, int ldab,
                              int64_t strideA, const int *dipiv, int64_t strideP, double *dB, int ldb,
                              int64_t strideB, int batch, bandlu_stream_t stream, int variant) {
    if (int r = check_trs(trans, n, kl, ku, nrhs, dA, ldab, strideA, dipiv, strideP, dB, ldb, strideB, batch, true))
        return r;
    return run_trs(n, kl, ku, nrhs, Strided<const double>{dA, strideA}, ldab, Strided<const int>{dipiv, strideP},
                   Strided<double>{dB, strideB}, ldb, nullptr, batch, (cudaStream_t)stream, variant, trans);
}

int dgbtrs_strided_batched(char trans, int n, int kl, int ku, int nrhs, const double *dA, int ldab,
                           int64_t strideA, const int *dipiv, int64_t strideP, double *dB, int ldb, int64_t strideB,
                           int batch, bandlu_stream_t stream) {
    return dgbtrs_strided_batched_ex(trans, n, kl, ku, nrhs, dA, ldab, strideA, dipiv, strideP, dB, ldb, strideB,
                                     batch, stream, BANDLU_AUTO);
}

int dgbtrs_batched(char trans, int n, int kl, int ku, int nrhs, const double *const *dA_array, int ldab,
                   const int *const *dipiv_array, double *const *dB_array, int ldb, int batch,
                   bandlu_stream_t stream) {
    if (int r = check_trs(trans, n, kl, ku, nrhs, dA_array, ldab, 0, dipiv_array, 0, dB_array, ldb, 0, batch, false))
        return r;
    return run_trs(n, kl, ku, nrhs, PtrArray<const double>{dA_array}, ldab, PtrArray<const int>{dipiv_array},
                   PtrArray<double>{dB_array}, ldb, nullptr, batch, (cudaStream_t)stream, BANDLU_AUTO, trans);
}

int dgbsv_strided_batched(int n, int kl, int ku, int nrhs, double *dA, int ldab, int64_t strideA, int *dipiv,
                          int64_t strideP, double *dB, int ldb, int64_t strideB, int *dinfo, int batch,
                          bandlu_stream_t stream) {
    // (n,kl,ku,nrhs,dA,ldab,strideA,dipiv,strideP,dB,ldb,strideB,dinfo,batch)
    if (n < 0) return -1;
    if (kl < 0) return -2;
    if (ku < 0) return -3;
    if (nrhs < 0) return -4;
    if (ldab < 2 * kl + ku + 1) return -6;
    if (ldb < (n > 1 ? n : 1)) return -11;
    if (batch < 0) return -14;
    if (batch > 0) {
        if (!dA) return -5;
        if (strideA < (int64_t)ldab * n) return -7;
        if (!dipiv && n > 0) return -8;
        if (strideP < n) return -9;
        if (!dB && n > 0 && nrhs > 0) return -10;
        if (strideB < (int64_t)ldb * nrhs) return -12;
        if (!dinfo) return -13;
    }
    return run_gbsv(n, kl, ku, nrhs, Strided<double>{dA, strideA}, ldab, Strided<int>{dipiv, strideP},
                    Strided<double>{dB, strideB}, ldb, dinfo, batch, (cudaStream_t)stream);
}

int dgbtrfs_strided_batched_ex(int n, int kl, int ku, int nrhs, double *dA, int ldab, int64_t strideA, int *dipiv,
                               int64_t strideP, double *dB, int ldb, int64_t strideB, int *dinfo, int batch,
                               bandlu_stream_t stream, int phase) {
    // same argument list / numbering as dgbsv_strided_batched
    if (n < 0) return -1;
    if (kl < 0) return -2;
    if (ku < 0) return -3;
    if (nrhs < 0) return -4;
    if (ldab < 2 * kl + ku + 1) return -6;
    if (ldb < (n > 1 ? n : 1)) return -11;
    if (batch < 0) return -14;
    if (batch > 0) {
        if (!dA) return -5;
        if (strideA < (int64_t)ldab * n) return -7;
        if (!dipiv && n > 0) return -8;
        if (strideP < n) return -9;
        if (!dB && n > 0 && nrhs > 0) return -10;
        if (strideB < (int64_t)ldb * nrhs) return -12;
        if (!dinfo) return -13;
    }
    if ((phase & TRFS_TWO_LAUNCH) && (phase & TRFS_FUSED)) return -16;
    {
        const int ph = phase & ~(TRFS_TWO_LAUNCH | TRFS_FUSED | TRFS_THIN);
        if (ph < 0 || ph > 2) return -16;
    }
    return run_trfs(n, kl, ku, nrhs, Strided<double>{dA, strideA}, ldab, Strided<int>{dipiv, strideP},
                    Strided<double>{dB, strideB}, ldb, dinfo, batch, (cudaStream_t)stream, phase);
}

int dgbtrfs_strided_batched(int n, int kl, int ku, int nrhs, double *dA, int ldab, int64_t strideA, int *dipiv,
                            int64_t strideP, double *dB, int ldb, int64_t strideB, int *dinfo, int batch,
                            bandlu_stream_t stream) {
    return dgbtrfs_strided_batched_ex(n, kl, ku, nrhs, dA, ldab, strideA, dipiv, strideP, dB, ldb, strideB, dinfo,
                                      batch, stream, 0);
}

int dgbsv_batched(int n, int kl, int ku, int nrhs, double *const *dA_array, int ldab, int *const *dipiv_array,
                  double *const *dB_array, int ldb, int *dinfo, int batch, bandlu_stream_t stream) {
    // (n,kl,ku,nrhs,dA_array,ldab,dipiv_array,dB_array,ldb,dinfo,batch)
    if (n < 0) return -1;
    if (kl < 0) return -2;
    if (ku < 0) return -3;
    if (nrhs < 0) return -4;
    if (ldab < 2 * kl + ku + 1) return -6;
    if (ldb < (n > 1 ? n : 1)) return -9;
    if (batch < 0) return -11;
    if (batch > 0) {
        if (!dA_array) return -5;
        if (!dipiv_array && n > 0) return -7;
        if (!dB_array && n > 0 && nrhs > 0) return -8;
        if (!dinfo) return -10;
    }
    cudaStream_t st = (cudaStream_t)stream;
    if (int r = run_trf(n, n, kl, ku, PtrArray<double>{dA_array}, ldab, PtrArray<int>{dipiv_array}, dinfo, batch, st,
                        BANDLU_AUTO))
        return r;
    return run_trs(n, kl, ku, nrhs, PtrArray<const double>{(const double *const *)dA_array}, ldab,
                   PtrArray<const int>{(const int *const *)dipiv_array}, PtrArray<double>{dB_array}, ldb, dinfo,
                   batch, st, BANDLU_AUTO);
}

}  // extern "C"

// ============================================= host-buffer end-to-end path
// Pipelined over batch chunks on NS internal streams: H2D(A_c, B_c) ->
// dgbsv (one fused launch where available) -> D2H(A_c, ipiv_c, B_c, info_c);
// chunk c+1's copies overlap chunk c's kernels (separate copy engines for each
// direction).
namespace {
// Device-side state of the host-buffer entry point, kept across calls so an
// e2e call pays no allocation: per device, NS streams and one staging buffer
// per stream (grown on demand).  A process that alternates devices keeps one
// set per device instead of abandoning the previous one.
struct DevPipe {
    static constexpr int NSMAX = 8;
    int NS = 0;  // 0 = not created yet
    cudaStream_t s[NSMAX] = {};
    cudaEvent_t done[NSMAX] = {};
    cudaEvent_t start = nullptr;
    void *buf[NSMAX] = {};
    size_t cap = 0;
    cudaError_t prepare(size_t need) {
        cudaError_t e;
        if (NS == 0) {
            int ns = 4;
            if (const char *v = std::getenv("BANDLU_HOST_STREAMS")) ns = std::max(1, std::min(NSMAX, atoi(v)));
            for (int i = 0; i < ns; ++i) {
                if ((e = cudaStreamCreateWithFlags(&s[i], cudaStreamNonBlocking)) != cudaSuccess) return e;
                if ((e = cudaEventCreateWithFlags(&done[i], cudaEventDisableTiming)) != cudaSuccess) return e;
            }
            if ((e = cudaEventCreateWithFlags(&start, cudaEventDisableTiming)) != cudaSuccess) return e;
            NS = ns;
        }
        if (need > cap) {
            for (int i = 0; i < NS; ++i) {
                if (buf[i]) {
                    cudaStreamSynchronize(s[i]);
                    cudaFree(buf[i]);
                    buf[i] = nullptr;
                }
            }
            cap = 0;
            for (int i = 0; i < NS; ++i)
                if ((e = cudaMalloc(&buf[i], need)) != cudaSuccess) return e;
            cap = need;
        }
        return cudaSuccess;
    }
};
struct HostPipe {
    static constexpr int MAXDEV = 64;
    std::mutex mu;
    DevPipe dev[MAXDEV];
};
HostPipe g_pipe;
}  // namespace

extern "C" int dgbsv_strided_batched_host(int n, int kl, int ku, int nrhs, double *hA, int ldab, int64_t strideA,
                                          int *hipiv, int64_t strideP, double *hB, int ldb, int64_t strideB,
                                          int *hinfo, int batch, bandlu_stream_t stream) {
    if (n < 0) return -1;
    if (kl < 0) return -2;
    if (ku < 0) return -3;
    if (nrhs < 0) return -4;
    if (ldab < 2 * kl + ku + 1) return -6;
    if (ldb < (n > 1 ? n : 1)) return -11;
    if (batch < 0) return -14;
    if (batch == 0) return 0;
    if (!hA) return -5;
    if (strideA < (int64_t)ldab * n) return -7;
    if (!hipiv && n > 0) return -8;
    if (strideP < n) return -9;
    if (!hB && n > 0 && nrhs > 0) return -10;
    if (strideB < (int64_t)ldb * nrhs) return -12;
    if (!hinfo) return -13;

    cudaStream_t user = (cudaStream_t)stream;
    const int64_t bytes_per = strideA * 8 + strideB * 8 + strideP * 4 + 4;
    // ~32 MB chunks over NS = 4 streams: H2D of chunk c+1, the kernels of chunk c
    // and D2H of chunk c-1 overlap (PCIe copy engines run both directions at once)
    static const long long chunk_mb = [] {
        const char *v = std::getenv("BANDLU_HOST_CHUNK_MB");
        return v ? std::max(1ll, atoll(v)) : 32ll;  // measured at C3: 4 x 32 MB 32.0 ms, 3 x 64 MB 33.4 ms
    }();
    int64_t ch = (int64_t)((chunk_mb << 20) / (bytes_per > 0 ? bytes_per : 1));
    ch = ch < 1 ? 1 : (ch > batch ? batch : ch);
    const int nchunks = (int)((batch + ch - 1) / ch);
    const size_t offB = (size_t)ch * strideA * 8, offP = offB + (((size_t)ch * strideB * 8 + 15) & ~(size_t)15);
    const size_t offI = offP + (((size_t)ch * strideP * 4 + 15) & ~(size_t)15);
    const size_t need = offI + (size_t)ch * 4 + 16;

    std::lock_guard<std::mutex> lock(g_pipe.mu);
    int ret = 0, d = 0;
    cudaError_t e;
    if ((e = cudaGetDevice(&d)) != cudaSuccess) return cuda_ret(e);
    if (d < 0 || d >= HostPipe::MAXDEV) return BANDLU_ERR_UNSUPPORTED;
    DevPipe &pp = g_pipe.dev[d];
    if ((e = pp.prepare(need)) != cudaSuccess) return cuda_ret(e);
    cudaEvent_t ev0 = pp.start;
    cudaEventRecord(ev0, user);
    for (int i = 0; i < pp.NS; ++i) cudaStreamWaitEvent(pp.s[i], ev0, 0);
    for (int c = 0; c < nchunks; ++c) {
        const int i = c % pp.NS;
        cudaStream_t si = pp.s[i];
        char *base = (char *)pp.buf[i];
        double *dA = (double *)base, *dB = (double *)(base + offB);
        int *dP = (int *)(base + offP), *dI = (int *)(base + offI);
        const int64_t b0 = (int64_t)c * ch;
        const int cb = (int)((batch - b0) < ch ? (batch - b0) : ch);
        const size_t aN = (size_t)((cb - 1) * strideA + (int64_t)ldab * n);
        const size_t bN = (size_t)((cb - 1) * strideB + (int64_t)ldb * nrhs);
        const size_t pN = (size_t)((cb - 1) * strideP + n);
        cudaMemcpyAsync(dA, hA + b0 * strideA, aN * 8, cudaMemcpyHostToDevice, si);
        if (bN) cudaMemcpyAsync(dB, hB + b0 * strideB, bN * 8, cudaMemcpyHostToDevice, si);
        int r = dgbsv_strided_batched(n, kl, ku, nrhs, dA, ldab, strideA, dP, strideP, dB, ldb, strideB, dI, cb,
                                      (bandlu_stream_t)si);
        if (r) { ret = r; break; }
        cudaMemcpyAsync(hA + b0 * strideA, dA, aN * 8, cudaMemcpyDeviceToHost, si);
        if (pN && n > 0) cudaMemcpyAsync(hipiv + b0 * strideP, dP, pN * 4, cudaMemcpyDeviceToHost, si);
        if (bN) cudaMemcpyAsync(hB + b0 * strideB, dB, bN * 8, cudaMemcpyDeviceToHost, si);
        cudaMemcpyAsync(hinfo + b0, dI, (size_t)cb * 4, cudaMemcpyDeviceToHost, si);
        if ((e = cudaGetLastError()) != cudaSuccess) { ret = cuda_ret(e); break; }
    }
    for (int i = 0; i < pp.NS; ++i) {
        cudaEventRecord(pp.done[i], pp.s[i]);
        cudaStreamWaitEvent(user, pp.done[i], 0);
    }
    if ((e = cudaStreamSynchronize(user)) != cudaSuccess && !ret) ret = cuda_ret(e);
    return ret;
}
