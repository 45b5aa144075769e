// Throughput of LDS.64 broadcast, STS.64 single-lane, SHFL, and LDS+SHFL mixed on one SM set.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k_lds(double* out, int iters) {
    __shared__ double s[4096];
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) s[i] = i;
    __syncthreads();
    double acc = 0; int base = (threadIdx.x >> 4) * 64;  // 2 distinct addresses per warp (like 2 groups)
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 16; ++k) acc += s[(base + k + it) & 4095];
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_shfl(double* out, int iters) {
    unsigned v = threadIdx.x, acc = 0;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 16; ++k) acc += __shfl_sync(0xffffffffu, v + k, (threadIdx.x & 16) + k);
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_mix(double* out, int iters) {
    __shared__ double s[4096];
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) s[i] = i;
    __syncthreads();
    double acc = 0; unsigned v = threadIdx.x, acc2 = 0; int base = (threadIdx.x >> 4) * 64;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 16; ++k) { acc += s[(base + k + it) & 4095]; acc2 += __shfl_sync(0xffffffffu, v + k, (threadIdx.x & 16) + k); }
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc + acc2;
}
__global__ void k_sts(double* out, int iters) {
    __shared__ double s[4096];
    double acc = threadIdx.x; int lane = threadIdx.x & 31; int w = threadIdx.x >> 5;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 16; ++k) if (lane == ((it + k) & 15) || lane == 16 + ((it * 3 + k) & 15)) s[(w * 128 + k * 8 + lane) & 4095] = acc + k;
    }
    __syncthreads();
    out[blockIdx.x * blockDim.x + threadIdx.x] = s[threadIdx.x];
}
int main() {
    double* d; cudaMalloc(&d, 1 << 24);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
    int iters = 2048, warps = 16;
    void (*ks[4])(double*, int) = {k_lds, k_shfl, k_mix, k_sts};
    const char* names[4] = {"LDS.64 bcast(2 addr)", "SHFL.32", "LDS.64+SHFL", "STS.64 (2 lanes)"};
    for (int i = 0; i < 4; ++i) {
        ks[i]<<<148, 32 * warps>>>(d, 8); cudaDeviceSynchronize();
        cudaEventRecord(e0); ks[i]<<<148, 32 * warps>>>(d, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        double ninstr = (double)warps * iters * 16;  // per SM, of the named op (mix: pairs)
        printf("%-22s: %.3f ms, %.2f cycles per instr(pair) per SM\n", names[i], ms, ms * 1e-3 * 1.965e9 / ninstr);
    }
    return 0;
}
