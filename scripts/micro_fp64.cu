// Microbenchmark: FP64 vector FMA (DFMA) vs FP64 tensor-core MMA (mma.sync m8n8k4 f64, DMMA)
// throughput on sm_100a, run for ~2 s each so nvidia-smi can record the power draw.
// Informs whether the element tangent (a sum of small G^T C G products) is worth
// moving onto DMMA under the 1000 W power cap.  Not part of the product.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/micro_fp64 scripts/micro_fp64.cu
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

__global__ void dfma_loop(double *out, long iters, double a, double b) {
    double x[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) x[k] = threadIdx.x * 1e-9 + k;
    for (long it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 8; ++k) x[k] = fma(x[k], a, b);
    }
    double s = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) s += x[k];
    if (s == 12345.678) out[0] = s;
}

__device__ __forceinline__ void dmma(double &d0, double &d1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
                 : "+d"(d0), "+d"(d1)
                 : "d"(a), "d"(b));
}

__global__ void dmma_loop(double *out, long iters, double a, double b) {
    double c[4][2];
#pragma unroll
    for (int k = 0; k < 4; ++k) c[k][0] = c[k][1] = threadIdx.x * 1e-9 + k;
    const double av = a + threadIdx.x * 1e-12, bv = b - threadIdx.x * 1e-12;
    for (long it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 4; ++k) dmma(c[k][0], c[k][1], av, bv);
    }
    double s = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) s += c[k][0] + c[k][1];
    if (s == 12345.678) out[0] = s;
}

int main(int argc, char **argv) {
    const char *mode = argc > 1 ? argv[1] : "dfma";
    const double seconds = argc > 2 ? atof(argv[2]) : 2.0;
    const int warps = argc > 3 ? atoi(argv[3]) : 16;  // warps per SM
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    double *out;
    cudaMalloc(&out, 8);
    const bool mm = mode[1] == 'm';
    const dim3 grid(sms * warps / 4), block(128);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    long iters = 1 << 14;
    float ms = 0;
    for (;;) {  // calibrate one launch to ~50 ms
        cudaEventRecord(e0);
        if (mm) dmma_loop<<<grid, block>>>(out, iters, 0.999999, 1e-7);
        else dfma_loop<<<grid, block>>>(out, iters, 0.999999, 1e-7);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms > 40) break;
        iters *= 2;
    }
    const int reps = (int)(seconds * 1000 / ms) + 1;
    cudaEventRecord(e0);
    for (int r = 0; r < reps; ++r) {
        if (mm) dmma_loop<<<grid, block>>>(out, iters, 0.999999, 1e-7);
        else dfma_loop<<<grid, block>>>(out, iters, 0.999999, 1e-7);
    }
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    const double threads = (double)grid.x * block.x;
    // DFMA: 8 FMA per thread-iteration; DMMA: 4 mma of 8x8x4 = 256 FMA per warp -> 32 per thread
    const double fma_per_thread_iter = mm ? 4 * 256.0 / 32 : 8.0;
    const double tflops = 2 * fma_per_thread_iter * threads * (double)iters * reps / (ms * 1e-3) / 1e12;
    printf("{\"mode\": \"%s\", \"warps_per_sm\": %d, \"ms\": %.1f, \"tflops\": %.3f, \"err\": \"%s\"}\n", mode, warps,
           ms, tflops, cudaGetErrorString(cudaGetLastError()));
    return 0;
}
