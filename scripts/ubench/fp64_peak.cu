// Measured FP64 FMA throughput of the GPU (the roofline peak of the on-the-fly Green's kernels):
// every SM full of warps, each thread running 8 independent DFMA chains.  2 flops per DFMA.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a fp64_peak.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void __launch_bounds__(256) dfma_peak(double* out, int iters) {
    double a[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) a[k] = 1.0 + 1e-6 * (threadIdx.x + k);
    const double b = 0.999999, c = 1e-9;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int k = 0; k < 8; ++k) a[k] = fma(a[k], b, c);
    }
    double s = 0.0;
#pragma unroll
    for (int k = 0; k < 8; ++k) s += a[k];
    if (s == 12345.0) out[0] = s;  // keep the chains alive
}

int main() {
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    double* d;
    cudaMalloc(&d, 8);
    const int blocks = sms * 8, threads = 256, iters = 20000;
    dfma_peak<<<blocks, threads>>>(d, 100);
    cudaDeviceSynchronize();
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    float best = 1e30f;
    for (int r = 0; r < 5; ++r) {
        cudaEventRecord(e0);
        dfma_peak<<<blocks, threads>>>(d, iters);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    const double flops = 2.0 * 8.0 * iters * (double)blocks * threads;
    printf("FP64 DFMA peak: %.2f TFLOP/s (%d SMs, best of 5, %.3f ms)\n", flops / (best * 1e-3) / 1e12, sms, best);
    return 0;
}
