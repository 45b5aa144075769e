// Dependent-chain latencies on one B200 SM (one warp): DFMA, DMUL, MUFU.RCP64H-based RN(1/x)
// (__drcp_rn), SHFL.IDX, LDS.  nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/lat tools/probes/lat_probe.cu
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k(double *out, long long *cyc, int iters) {
    double x = 1.0 + threadIdx.x * 1e-9, a = 0.999999, b = 1e-7;
    __shared__ double sm[64];
    sm[threadIdx.x] = x;
    __syncwarp();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) x = fma(x, a, b);
    long long t1 = clock64();
    for (int i = 0; i < iters; ++i) x = __drcp_rn(x);
    long long t2 = clock64();
    for (int i = 0; i < iters; ++i) x = __shfl_sync(0xffffffffu, x, (threadIdx.x + 1) & 31);
    long long t3 = clock64();
    unsigned addr = (unsigned)__cvta_generic_to_shared(sm + threadIdx.x);
    for (int i = 0; i < iters; ++i) {
        double y;
        asm volatile("ld.shared.f64 %0, [%1];" : "=d"(y) : "r"(addr));
        addr = (unsigned)__cvta_generic_to_shared(sm + ((int)y & 31));
        x += y;
    }
    long long t4 = clock64();
    for (int i = 0; i < iters; ++i) x = x * a;
    long long t5 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) { cyc[0] = t1 - t0; cyc[1] = t2 - t1; cyc[2] = t3 - t2; cyc[3] = t4 - t3; cyc[4] = t5 - t4; }
}
int main() {
    double *o; long long *c, h[5];
    cudaMalloc(&o, 4096); cudaMalloc(&c, 64);
    const int it = 4096;
    k<<<1, 32>>>(o, c, it); cudaDeviceSynchronize();
    k<<<1, 32>>>(o, c, it); cudaMemcpy(h, c, 40, cudaMemcpyDeviceToHost);
    printf("cycles per dependent op: DFMA %.1f  __drcp_rn %.1f  SHFL.IDX(64-bit) %.1f  LDS.64(+DADD) %.1f  DMUL %.1f\n",
           h[0] / (double)it, h[1] / (double)it, h[2] / (double)it, h[3] / (double)it, h[4] / (double)it);
    return 0;
}
