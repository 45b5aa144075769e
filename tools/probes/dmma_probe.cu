// Probe: semantics of mma.sync.m8n8k4 f64 on sm_100a -- is D = C + sum_k A_k B_k
// rounded like a chain of IEEE FMAs (and in which order)?
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void dmma_kernel(const double* A, const double* B, const double* C, double* D, int reps) {
    // A: 8x4 row-major, B: 4x8 (col layout: B[k][n]), C,D: 8x8 row-major; one warp.
    int t = threadIdx.x;
    for (int r = 0; r < reps; ++r) {
        const double* a = A + r * 32; const double* b = B + r * 32; const double* c = C + r * 64; double* d = D + r * 64;
        double a0 = a[(t / 4) * 4 + (t % 4)];          // A[row=t/4][k=t%4]
        double b0 = b[(t % 4) * 8 + (t / 4)];          // B[k=t%4][n=t/4]
        double c0 = c[(t / 4) * 8 + 2 * (t % 4)], c1 = c[(t / 4) * 8 + 2 * (t % 4) + 1];
        double d0, d1;
        asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%4,%5};\n"
                     : "=d"(d0), "=d"(d1) : "d"(a0), "d"(b0), "d"(c0), "d"(c1));
        d[(t / 4) * 8 + 2 * (t % 4)] = d0; d[(t / 4) * 8 + 2 * (t % 4) + 1] = d1;
    }
}

static double rnd(uint64_t* s) { *s = *s * 6364136223846793005ULL + 1442695040888963407ULL; return ((*s >> 11) * (1.0 / 9007199254740992.0)) * 2 - 1; }

int main() {
    const int R = 4000;
    size_t na = 32 * R, nc = 64 * R;
    double *A = (double*)malloc(na * 8), *B = (double*)malloc(na * 8), *C = (double*)malloc(nc * 8), *D = (double*)malloc(nc * 8);
    uint64_t s = 12345;
    for (size_t i = 0; i < na; ++i) { A[i] = rnd(&s); B[i] = rnd(&s); }
    for (size_t i = 0; i < nc; ++i) C[i] = rnd(&s) * (i % 7 == 0 ? 1e-3 : 1.0);
    // make a fraction of reps "rank-1": only k=0 nonzero
    for (int r = 0; r < R / 2; ++r) for (int i = 0; i < 8; ++i) for (int k = 1; k < 4; ++k) { A[r * 32 + i * 4 + k] = 0; B[r * 32 + k * 8 + i] = 0; }
    double *dA, *dB, *dC, *dD;
    cudaMalloc(&dA, na * 8); cudaMalloc(&dB, na * 8); cudaMalloc(&dC, nc * 8); cudaMalloc(&dD, nc * 8);
    cudaMemcpy(dA, A, na * 8, cudaMemcpyHostToDevice); cudaMemcpy(dB, B, na * 8, cudaMemcpyHostToDevice); cudaMemcpy(dC, C, nc * 8, cudaMemcpyHostToDevice);
    dmma_kernel<<<1, 32>>>(dA, dB, dC, dD, R);
    cudaError_t e = cudaDeviceSynchronize();
    printf("kernel: %s\n", cudaGetErrorString(e));
    cudaMemcpy(D, dD, nc * 8, cudaMemcpyDeviceToHost);
    long eq_fwd = 0, eq_bwd = 0, eq_r1 = 0, n_r1 = 0, n_full = 0, eq_exactish = 0;
    for (int r = 0; r < R; ++r) for (int i = 0; i < 8; ++i) for (int j = 0; j < 8; ++j) {
        double c = C[r * 64 + i * 8 + j], d = D[r * 64 + i * 8 + j];
        double f = c; for (int k = 0; k < 4; ++k) f = fma(A[r * 32 + i * 4 + k], B[r * 32 + k * 8 + j], f);
        double g = c; for (int k = 3; k >= 0; --k) g = fma(A[r * 32 + i * 4 + k], B[r * 32 + k * 8 + j], g);
        long double x = c; for (int k = 0; k < 4; ++k) x += (long double)A[r * 32 + i * 4 + k] * (long double)B[r * 32 + k * 8 + j];
        if (r < R / 2) { n_r1++; eq_r1 += (d == fma(A[r * 32 + i * 4], B[r * 32 + j], c)); }
        else { n_full++; eq_fwd += (d == f); eq_bwd += (d == g); eq_exactish += (d == (double)x); }
    }
    printf("rank-1 (k=0 only): %ld / %ld equal to fma(a0,b0,c)\n", eq_r1, n_r1);
    printf("full k=4: fma chain k=0..3: %ld/%ld   k=3..0: %ld/%ld   round(extended sum): %ld/%ld\n", eq_fwd, n_full, eq_bwd, n_full, eq_exactish, n_full);
    return 0;
}
