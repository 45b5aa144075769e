// DMMA m8n8k4 f64 and DFMA throughput/latency microbenchmark on one B200.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void dmma_tp(double* out, int iters) {
    double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
    double c[8][2];
    for (int i = 0; i < 8; ++i) { c[i][0] = i; c[i][1] = -i; }
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i)
            asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                         : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
    }
    double s = 0; for (int i = 0; i < 8; ++i) s += c[i][0] + c[i][1];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void dmma_lat(double* out, int iters) {
    double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4, c0 = 1, c1 = 2;
    for (int it = 0; it < iters; ++it)
        asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n" : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
    out[threadIdx.x] = c0 + c1;
}
__global__ void dfma_tp(double* out, int iters) {
    double x[8]; double a = threadIdx.x * 1e-3, b = 1.0 - threadIdx.x * 1e-5;
    for (int i = 0; i < 8; ++i) x[i] = i;
    for (int it = 0; it < iters; ++it)
#pragma unroll
        for (int i = 0; i < 8; ++i) x[i] = fma(x[i], b, a);
    double s = 0; for (int i = 0; i < 8; ++i) s += x[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void dfma_lat(double* out, int iters) {
    double x = threadIdx.x, a = 1e-3, b = 0.999;
    for (int it = 0; it < iters; ++it) x = fma(x, b, a);
    out[threadIdx.x] = x;
}
int main() {
    double* d; cudaMalloc(&d, 1 << 24);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
    int iters = 4096;
    for (int wps : {4, 8, 16}) {
        dmma_tp<<<148, 32 * wps>>>(d, 16); cudaDeviceSynchronize();
        cudaEventRecord(e0); dmma_tp<<<148, 32 * wps>>>(d, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        double n = 148.0 * wps * iters * 8; printf("DMMA: %2d warps/SM: %.3f ms, %.2f TFLOP/s (k=4 counted), %.2f cycles/DMMA/SM @1.965GHz\n", wps, ms, n * 512 / (ms * 1e-3) / 1e12, (ms * 1e-3 * 1.965e9) / (n / 148));
        dfma_tp<<<148, 32 * wps>>>(d, 16); cudaDeviceSynchronize();
        cudaEventRecord(e0); dfma_tp<<<148, 32 * wps>>>(d, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        double nf = 148.0 * wps * 32 * iters * 8; printf("DFMA: %2d warps/SM: %.3f ms, %.2f TFLOP/s\n", wps, ms, nf * 2 / (ms * 1e-3) / 1e12);
    }
    cudaEventRecord(e0); dmma_lat<<<1, 32>>>(d, iters); cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
    printf("DMMA dependent latency: %.1f cycles\n", ms * 1e-3 * 1.965e9 / iters);
    cudaEventRecord(e0); dfma_lat<<<1, 32>>>(d, iters * 16); cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
    printf("DFMA dependent latency: %.1f cycles\n", ms * 1e-3 * 1.965e9 / (iters * 16));
    return 0;
}
