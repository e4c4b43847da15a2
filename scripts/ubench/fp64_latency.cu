// Dependent-chain latency (cycles per operation) of FP64 operations and warp shuffles on the GPU:
// one warp, a chain of N dependent operations timed with clock64.  Explains the serial kernels
// (LSQ Cholesky, Newton searches) in DESIGN.md.  nvcc -O3 -arch=sm_100a fp64_latency.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int N = 4096;

template <int OP>
__global__ void chain(double* out, long long* cyc, double x0) {
    double x = x0 + threadIdx.x * 1e-9;
    const double a = 1.0000001, b = 1e-12;
    __syncwarp();
    long long t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < N; ++i) {
        if (OP == 0) x = fma(x, a, b);
        if (OP == 1) x = x * a;
        if (OP == 2) x = x + b;
        if (OP == 3) x = sqrt(x) + 1.0;             // sqrt + add
        if (OP == 4) x = 1.0 / x + 1.0;             // division + add
        if (OP == 5) x = rsqrt(x) + 1.0;            // rsqrt + add
        if (OP == 6) x = __shfl_sync(0xffffffffu, x, (threadIdx.x + 1) & 31) + b;  // shuffle + add
        if (OP == 7) x = x / 1.0000001 + 1e-12;    // division by a constant + add
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) { out[0] = x; cyc[0] = t1 - t0; }
}

int main() {
    double* d; long long* c;
    cudaMalloc(&d, 8); cudaMalloc(&c, 8);
    const char* names[8] = {"DFMA", "DMUL", "DADD", "sqrt+DADD", "1/x+DADD", "rsqrt+DADD", "shfl(f64)+DADD", "x/c+DADD"};
    for (int op = 0; op < 8; ++op) {
        for (int rep = 0; rep < 2; ++rep) {
            switch (op) {
                case 0: chain<0><<<1, 32>>>(d, c, 1.5); break;
                case 1: chain<1><<<1, 32>>>(d, c, 1.5); break;
                case 2: chain<2><<<1, 32>>>(d, c, 1.5); break;
                case 3: chain<3><<<1, 32>>>(d, c, 1.5); break;
                case 4: chain<4><<<1, 32>>>(d, c, 1.5); break;
                case 5: chain<5><<<1, 32>>>(d, c, 1.5); break;
                case 6: chain<6><<<1, 32>>>(d, c, 1.5); break;
                case 7: chain<7><<<1, 32>>>(d, c, 1.5); break;
            }
            cudaDeviceSynchronize();
        }
        long long h = 0;
        cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
        printf("%-16s %7.1f cycles per dependent op\n", names[op], (double)h / N);
    }
    return 0;
}
