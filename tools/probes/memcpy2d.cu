// H2D/D2H bandwidth of contiguous vs 2-D (row-subset) copies from pinned host memory:
// does skipping the never-read fill rows of a band matrix (cudaMemcpy2DAsync, width < pitch)
// keep the PCIe rate?   nvcc -O2 -o /tmp/memcpy2d tools/probes/memcpy2d.cu && /tmp/memcpy2d
#include <cstdio>
#include <cuda_runtime.h>
int main() {
    const size_t ldab = 31, n = 512, batch = 2500, cols = n * batch;  // C3 shape, 1/4 of the batch
    const size_t bytes = ldab * cols * 8;
    double *h, *d;
    cudaMallocHost(&h, bytes);
    cudaMalloc(&d, bytes);
    for (size_t i = 0; i < bytes / 8; ++i) h[i] = 1.0;
    cudaStream_t s; cudaStreamCreate(&s);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    float ms;
    for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(e0, s);
        cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice, s);
        cudaEventRecord(e1, s); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf("H2D contiguous %.1f MB: %.2f ms = %.1f GB/s\n", bytes / 1e6, ms, bytes / ms / 1e6);
        for (size_t skip : {10, 8, 6}) {
            const size_t w = (ldab - skip) * 8;
            cudaEventRecord(e0, s);
            cudaMemcpy2DAsync(d + skip, ldab * 8, h + skip, ldab * 8, w, cols, cudaMemcpyHostToDevice, s);
            cudaEventRecord(e1, s); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
            printf("H2D 2-D rows %zu..%zu (%zu B of %zu): %.2f ms = %.1f GB/s useful, %.2f of contiguous time\n", skip,
                   ldab - 1, w, ldab * 8, ms, w * cols / ms / 1e6, 0.0);
        }
        cudaEventRecord(e0, s);
        cudaMemcpyAsync(h, d, bytes, cudaMemcpyDeviceToHost, s);
        cudaEventRecord(e1, s); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf("D2H contiguous: %.2f ms = %.1f GB/s\n", ms, bytes / ms / 1e6);
    }
    return 0;
}
