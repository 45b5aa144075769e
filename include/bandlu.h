/*
 * bandlu.h -- C ABI of the B200-native batched band LU / solve library.
 *
 * Operations (PAPER.md = Abdelfattah et al., SC-W 2023, text at
 * /root/reference/PAPER.md; "P:<line>"):
 *   dgbtrf : LU factorization with partial pivoting of a batch of m x n band
 *            matrices, kl sub- / ku super-diagonals (Sec. 5, P:336-567;
 *            interface P:314-318; column algorithm).
 *   dgbtrs : solve A X = B with the factors (Sec. 6; interface
 *            P:320-326), TRANS = 'N'.
 *   dgbsv  : dgbtrf then dgbtrs (Sec. 3, Sec. 7 P:686-702;
 *            interface P:328-333).
 * Semantics are LAPACK DGBTRF(DGBTF2)/DGBTRS/DGBSV, which the paper adopts
 * (P:26-27): results equal the reference CPU oracle (oracle/) --
 * pivots and info bit-exact; factors and solutions bitwise in practice
 * (same fp64 operation sequence), criterion 1e-12 relative entrywise.
 *
 * ---------------------------------------------------------------- layout
 * A (band storage, LAPACK, P:286-304 and Fig. 2): each matrix is a
 *   column-major array AB(ldab, n), ldab >= 2*kl+ku+1.  With kv = kl+ku and
 *   0-based indices, A(i,j) is stored at AB[j*ldab + kv+i-j].  Rows 0..kl-1
 *   are fill-in space: their input values are never read.  On exit rows
 *   0..kv hold U (upper bandwidth kv) and rows kv+1..2kl+ku hold the
 *   multipliers of L (not permuted by later interchanges, "swap to the right
 *   only").  Positions whose matrix row is outside [0, m) ("corners")
 *   and padding rows ldab > 2kl+ku+1 are never read and never written, except
 *   that -- exactly as LAPACK DGBTF2's fill-in zeroing does -- fill-row
 *   positions of columns < n whose matrix row is >= m are set to 0 when m < n.
 * ipiv: min(m,n) int32 per matrix, 1-based LAPACK convention:
 *   row j was interchanged with row ipiv[j]-1, ipiv[j] in [j+1, min(m,j+1+kl)].
 * info: one int32 per matrix ("dedicated return code in the info
 *   array"): 0 = success, k > 0 = U(k,k) (1-based) is exactly zero; the
 *   factorization is still completed.  Written for every matrix when
 *   batch > 0, also on the quick return m = 0 or n = 0.
 * B: each right-hand side block is column-major B(ldb, nrhs), ldb >= max(1,n);
 *   rows n..ldb-1 are untouched.
 *
 * ------------------------------------------------------- memory / calls
 * All array arguments are DEVICE pointers (pointer-array variants: a device
 * array of device pointers) unless the name ends in _host.  Calls
 * are asynchronous on `stream` (a cudaStream_t; NULL = legacy default
 * stream); results are valid after the stream is synchronized.  The caller
 * owns all memory; the device entry points keep no state and allocate
 * nothing.  Thread-safe, re-entrant, deterministic (no atomics in the
 * arithmetic); per-matrix results do not depend on batch, its sharding, or
 * the kernel variant chosen.
 * Strided variants: matrix b starts at dA + b*strideA (strideA >= ldab*n),
 * dipiv + b*strideP (strideP >= min(m,n)), dB + b*strideB (strideB >=
 * ldb*nrhs); overlapping matrices are undefined behaviour.
 *
 * ------------------------------------------------------------- errors
 * Return 0: work enqueued.  Return -k: argument k (1-based position in the
 * C signature) is illegal; batch < 0, a NULL array with batch > 0, or a
 * too-small stride return the position of that argument too.  For the
 * pointer-array variants the positions are LAPACK's numbering (trf: -1 m,
 * -2 n, -3 kl, -4 ku, -6 ldab; trs: -1 trans, -2 n, -3 kl, -4 ku, -5 nrhs,
 * -7 ldab, -10 ldb; gbsv: -1 n, -2 kl, -3 ku, -4 nrhs, -6 ldab, -9 ldb).
 * The strided variants insert stride arguments, so later positions shift:
 * dgbtrf_strided -5 dA, -6 ldab, -7 strideA, -8 dipiv, -9 strideP, -10 dinfo,
 * -11 batch; dgbtrs_strided -7 ldab, -8 strideA, -9 dipiv, -10 strideP,
 * -11 dB, -12 ldb, -13 strideB, -14 batch; dgbsv_strided / dgbtrfs_strided /
 * dgbsv_strided_host -5 dA, -6 ldab, -7 strideA, -8 dipiv, -9 strideP,
 * -10 dB, -11 ldb, -12 strideB, -13 dinfo, -14 batch.  Nothing is enqueued
 * when the return is nonzero.  BANDLU_ERR_UNSUPPORTED: a forced
 * variant that is not compiled for the shape.  BANDLU_ERR_CUDA +
 * (cudaError_t) : a launch/runtime error (enqueue failed).
 */
#ifndef BANDLU_H
#define BANDLU_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* binary compatible with cudaStream_t */
typedef struct CUstream_st *bandlu_stream_t;

#define BANDLU_ERR_UNSUPPORTED 1000
#define BANDLU_ERR_CUDA 2000

/* Kernel variant selector for the *_ex entry points (testing / profiling).
 * AUTO = the library heuristic (what the plain entry points use). */
enum bandlu_variant {
    BANDLU_AUTO = 0,
    BANDLU_GENERIC = 1, /* warp-per-matrix in-place kernel, any m, n, kl, ku (safeguard) */
    BANDLU_WINDOW = 2,  /* register-resident sliding window, compiled (kl, ku) only (Sec. 5.3 / 8.1) */
    BANDLU_TC = 3,      /* dgbtrf only, opt-in: window in FP64 tensor-core (DMMA) fragments, compiled
                           (kl, ku) with kl+1 <= 16 (bandlu_tc_available); same LAPACK operation
                           sequence, bitwise equal results */
    BANDLU_ROWS = 4     /* dgbtrf: register window with R row slots per lane and block-preloaded
                           band rows, compiled (kl, ku) only (bandlu_rows_available); AUTO prefers it
                           where compiled.  dgbtrs ('N'): one lane per RHS row, a group of
                           pow2 >= kl+ku+1 lanes per (matrix, RHS column), compiled (kl, ku) with
                           kl+ku+1 <= 32 only (bandlu_trs_rows_available); AUTO's choice for
                           nrhs == 1 with kl+ku+1 <= 4.  Bitwise equal results */,
    BANDLU_THREAD = 5,  /* dgbtrf only: one thread per matrix, the whole (kl+1) x (kl+ku+1) window in
                           registers, thin compiled bands (bandlu_thread_available); bitwise equal
                           results */
    BANDLU_TPM = 6,     /* dgbtrf only, square (m == n): one thread per matrix, the window in shared
                           memory, 4-column panels factored in registers and a rank-4 trailing
                           update per panel (bandlu_tpm_available); bitwise equal results */
    BANDLU_THIN = 7     /* dgbtrf only, square, strided: thin bands, one thread per matrix with the
                           window in registers and whole band columns staged cooperatively through
                           shared memory (bandlu_thin_available); bitwise equal results */,
    BANDLU_COLS = 8     /* dgbtrf (and dgbtrfs' factorization), square: thin lower bands (kl <= 4),
                           the lanes of a group own the window's columns (gbtrf_cols.cuh);
                           compiled (kl, ku) only (bandlu_cols_available); AUTO's choice where
                           compiled.  Bitwise equal results */
};

/* ---- dgbtrf: band LU with partial pivoting ---- */
int dgbtrf_batched(int m, int n, int kl, int ku,
                   double *const *dA_array, int ldab,
                   int *const *dipiv_array, int *dinfo,
                   int batch, bandlu_stream_t stream);
int dgbtrf_strided_batched(int m, int n, int kl, int ku,
                           double *dA, int ldab, int64_t strideA,
                           int *dipiv, int64_t strideP, int *dinfo,
                           int batch, bandlu_stream_t stream);

/* ---- dgbtrs: A X = B (trans 'N'/'n') or A^T X = B (trans 'T'/'t'/'C'/'c',
 * identical for real data) with the dgbtrf factors (transA).
 * LAPACK DGBTRS semantics: no singularity check (singular U gives Inf/NaN).
 * 'T' follows the reference-BLAS operation order of DTBSV('U','T') and
 * DGEMV('T') (dot products accumulated in increasing index order).  For
 * 'T', AUTO and BANDLU_WINDOW run the ring-staged transposed solve (lane per
 * (matrix, RHS column); compiled bands, others compiled at run time when
 * kl + ku <= 64); BANDLU_GENERIC runs one thread per (matrix, RHS column).
 * Both give bitwise the same result. */
int dgbtrs_batched(char trans, int n, int kl, int ku, int nrhs,
                   const double *const *dA_array, int ldab,
                   const int *const *dipiv_array,
                   double *const *dB_array, int ldb,
                   int batch, bandlu_stream_t stream);
int dgbtrs_strided_batched(char trans, int n, int kl, int ku, int nrhs,
                           const double *dA, int ldab, int64_t strideA,
                           const int *dipiv, int64_t strideP,
                           double *dB, int ldb, int64_t strideB,
                           int batch, bandlu_stream_t stream);

/* ---- dgbsv: dgbtrf + dgbtrs.  B is untouched for every matrix
 * with info > 0 (LAPACK DGBSV).  Strided, nrhs == 1, a band with a fused
 * row-slot kernel, a batch within one wave of it and y(0..n-1) fitting in
 * shared memory: ONE launch of the fused gbsv kernel (factorization, forward substitution on the fly, backward
 * substitution by the same lanes; Sec. 7 P:686-702 generalised to any n).
 * Otherwise a factorization launch and a solve launch. ---- */
int dgbsv_batched(int n, int kl, int ku, int nrhs,
                  double *const *dA_array, int ldab, int *const *dipiv_array,
                  double *const *dB_array, int ldb, int *dinfo,
                  int batch, bandlu_stream_t stream);
int dgbsv_strided_batched(int n, int kl, int ku, int nrhs,
                          double *dA, int ldab, int64_t strideA,
                          int *dipiv, int64_t strideP,
                          double *dB, int ldb, int64_t strideB, int *dinfo,
                          int batch, bandlu_stream_t stream);

/* ---- dgbtrfs: dgbtrf followed by dgbtrs('N') on every matrix, as one call
 * (the bench's hot-path step).  Same arguments and numbering as
 * dgbsv_strided_batched.  nrhs == 1, a band with a fused row-slot kernel and a
 * batch that fits in one wave of it (SMs x resident matrices): ONE launch (the
 * fused kernel, as dgbsv; y in shared memory when it fits, else in B).  Other
 * nrhs == 1 cases with a compiled (kl, ku): the factorization kernel applies the
 * forward substitution (the paper's augmented [A|B], Sec. 7), then
 * one backward-substitution launch.  Results are bitwise
 * those of the separate calls.  Unlike dgbsv, B is solved also where
 * info > 0 (as dgbtrs would: singular U gives Inf/NaN). ---- */
int dgbtrfs_strided_batched(int n, int kl, int ku, int nrhs,
                            double *dA, int ldab, int64_t strideA,
                            int *dipiv, int64_t strideP,
                            double *dB, int ldb, int64_t strideB, int *dinfo,
                            int batch, bandlu_stream_t stream);
/* phase (profiling): 0 = everything, 1 = the first launch only, 2 = the second
 * launch only (nothing when the plan has one launch); + BANDLU_TRFS_TWO_LAUNCH
 * forces the two-launch plan (factorization + forward, then backward), +
 * BANDLU_TRFS_FUSED the fused kernel where it exists; any other value (or
 * both flags) returns -16. */
#define BANDLU_TRFS_TWO_LAUNCH 16
#define BANDLU_TRFS_FUSED 32
#define BANDLU_TRFS_THIN 64 /* the thin-band thread-per-matrix fused kernel (bandlu_thin_available) */
int dgbtrfs_strided_batched_ex(int n, int kl, int ku, int nrhs,
                               double *dA, int ldab, int64_t strideA,
                               int *dipiv, int64_t strideP,
                               double *dB, int ldb, int64_t strideB, int *dinfo,
                               int batch, bandlu_stream_t stream, int phase);

/* ---- host-buffer end-to-end variant of dgbsv_strided_batched: hA, hipiv,
 * hB, hinfo are HOST pointers (pinned memory recommended).  The library keeps,
 * per device, four streams and four staging buffers of one ~32 MB batch chunk
 * each (created on first use on that device, grown on demand, never freed;
 * BANDLU_HOST_STREAMS / BANDLU_HOST_CHUNK_MB override the defaults), copies
 * A and B in, factors and solves, copies A (factors), ipiv, B (solution) and
 * info back, and synchronizes `stream` before returning.  Batch chunks are
 * pipelined so host->device copies, kernels and device->host copies overlap.
 * Calls are serialized by a process-wide lock.  Returns as above, or
 * BANDLU_ERR_CUDA + err on an allocation / copy failure. */
int dgbsv_strided_batched_host(int n, int kl, int ku, int nrhs,
                               double *hA, int ldab, int64_t strideA,
                               int *hipiv, int64_t strideP,
                               double *hB, int ldb, int64_t strideB, int *hinfo,
                               int batch, bandlu_stream_t stream);

/* ---- variant-forcing entry points (tests / profiling).  variant is an
 * enum bandlu_variant; forcing BANDLU_WINDOW for a (kl, ku) that is not
 * compiled returns BANDLU_ERR_UNSUPPORTED. ---- */
int dgbtrf_strided_batched_ex(int m, int n, int kl, int ku,
                              double *dA, int ldab, int64_t strideA,
                              int *dipiv, int64_t strideP, int *dinfo,
                              int batch, bandlu_stream_t stream, int variant);
int dgbtrs_strided_batched_ex(char trans, int n, int kl, int ku, int nrhs,
                              const double *dA, int ldab, int64_t strideA,
                              const int *dipiv, int64_t strideP,
                              double *dB, int ldb, int64_t strideB,
                              int batch, bandlu_stream_t stream, int variant);

/* Which variant AUTO picks for a shape (no launch). */
int bandlu_trf_variant(int m, int n, int kl, int ku);
int bandlu_trs_variant(int n, int kl, int ku, int nrhs);
/* 1 if a tensor-core (BANDLU_TC) factorization kernel is compiled for (kl, ku),
 * else 0 (no launch).  BANDLU_TC is never chosen by AUTO; force it with
 * dgbtrf_strided_batched_ex.  Compiled only in -DBANDLU_WITH_TC builds. */
int bandlu_tc_available(int kl, int ku);
/* 1 if a row-slot (BANDLU_ROWS) factorization kernel is compiled for (kl, ku), else 0. */
int bandlu_rows_available(int kl, int ku);
/* 1 if a thread-per-matrix factorization kernel (BANDLU_THREAD) is compiled for (kl, ku), else 0
 * (only in -DBANDLU_WITH_THREAD builds: measured slower, AUTO never picks it). */
int bandlu_thread_available(int kl, int ku);
/* 1 if a thread-per-matrix shared-memory-window kernel (BANDLU_TPM) is compiled for (kl, ku), else 0. */
int bandlu_tpm_available(int kl, int ku);
/* 1 if a column-owner (BANDLU_COLS) factorization kernel is compiled for (kl, ku), else 0. */
int bandlu_cols_available(int kl, int ku);
/* 1 if a thin-band thread-per-matrix kernel (BANDLU_THIN) is compiled for (kl, ku), else 0
 * (only in -DBANDLU_WITH_THIN builds: measured slower, AUTO never picks it). */
int bandlu_thin_available(int kl, int ku);
/* Run-time compiled bands (Sec. 8.1: JIT-compiled register-resident
 * kernels).  A (kl, ku) that no ahead-of-time instantiation covers takes the same kernel
 * templates compiled with NVRTC for sm_100a on the first call that needs them (seconds;
 * cached per process, and on disk when BANDLU_JIT_CACHE names a directory): the row-slot
 * factorization for kl <= 27, the two-warp one for kl <= 59, the backward / window
 * solves; strided entry points only (pointer arrays use the generic kernels).  Without
 * NVRTC (dlopen libnvrtc.so.12) or with BANDLU_JIT=0 such bands use the generic kernels.
 * bandlu_jit_band: 1 if (kl, ku) is served that way (no compilation).  bandlu_jit_check:
 * compile (no GPU needed, nothing loaded) every kernel the band uses; 0 on success, else 1
 * and the first compiler error in log (loglen bytes). */
int bandlu_jit_band(int kl, int ku);
int bandlu_jit_check(int kl, int ku, char *log, int loglen);
/* 1 if a lane-per-row solve kernel (dgbtrs BANDLU_ROWS) is compiled for (kl, ku), else 0. */
int bandlu_trs_rows_available(int kl, int ku);
/* The launches one dgbtrfs_strided_batched call with this phase flag set makes
 * for a shape and batch (no launch):
 * returns their number L (0..2; < 0 on a negative argument) and, if kinds is
 * not NULL, writes L codes kinds[i] = 16 * kernel + bytes, kernel: 1 gbtrf_rows,
 * 2 gbtrf_window, 3 gbtrf_wide, 4 gbtrf_thread, 5 gbtrf_generic, 6 gbtrs_bwd,
 * 7 gbtrs_rows, 8 gbtrs_window, 9 gbtrs_generic, 10 gbtrf_thin, 11 gbtrs_blk; bytes (what the launch must
 * move per matrix): 1 factorization, 2 factorization + forward
 * substitution, 3 backward substitution, 4 full solve, 5 fused gbsv.
 * phase: 0, BANDLU_TRFS_TWO_LAUNCH, BANDLU_TRFS_FUSED or BANDLU_TRFS_THIN (as for dgbtrfs). */
int bandlu_trfs_plan(int n, int kl, int ku, int nrhs, int batch, int phase, int *kinds);
/* ABI version of this library. */
int bandlu_version(void);

#ifdef __cplusplus
}
#endif
#endif /* BANDLU_H */
