// Microbenchmark: fp64 FMA throughput on sm_100a -- vector DFMA vs the fp64 tensor-core mma.sync
// shapes (m8n8k4, m16n8k4, m16n8k8, m16n8k16), and a mix of both in one warp (do they share a pipe?).
// Informs whether the element-Jacobian contraction J = sum_q G_q^T D_q G_q should move to DMMA.
// Not part of the product.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/micro_dmma scripts/micro_dmma.cu
//   ./build/micro_dmma   -> one JSON line per variant
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

constexpr int ITERS = 4096;

__global__ void dfma_kernel(double *out, double s) {
    double a[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) a[k] = threadIdx.x * 1e-3 + k;
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int k = 0; k < 8; ++k) a[k] = fma(a[k], s, 1e-9);
    }
    double t = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) t += a[k];
    if (t == 12345.0) out[0] = t;
}

__device__ __forceinline__ void mma884(double (&d)[2], double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                 : "+d"(d[0]), "+d"(d[1])
                 : "d"(a), "d"(b));
}
__device__ __forceinline__ void mma1684(double (&d)[4], double a0, double a1, double b) {
    asm volatile("mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
                 : "+d"(d[0]), "+d"(d[1]), "+d"(d[2]), "+d"(d[3])
                 : "d"(a0), "d"(a1), "d"(b));
}
__device__ __forceinline__ void mma1688(double (&d)[4], const double (&a)[4], const double (&b)[2]) {
    asm volatile("mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
                 "{%0,%1,%2,%3};"
                 : "+d"(d[0]), "+d"(d[1]), "+d"(d[2]), "+d"(d[3])
                 : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(b[0]), "d"(b[1]));
}
__device__ __forceinline__ void mma16816(double (&d)[4], const double (&a)[8], const double (&b)[4]) {
    asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, "
                 "{%4,%5,%6,%7,%8,%9,%10,%11}, {%12,%13,%14,%15}, {%0,%1,%2,%3};"
                 : "+d"(d[0]), "+d"(d[1]), "+d"(d[2]), "+d"(d[3])
                 : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(a[4]), "d"(a[5]), "d"(a[6]), "d"(a[7]),
                   "d"(b[0]), "d"(b[1]), "d"(b[2]), "d"(b[3]));
}

template <int NACC>
__global__ void mma884_kernel(double *out, double s) {
    double d[NACC][2];
    const double a = threadIdx.x * 1e-6, b = s;
#pragma unroll
    for (int k = 0; k < NACC; ++k) d[k][0] = d[k][1] = k;
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int k = 0; k < NACC; ++k) mma884(d[k], a, b);
    }
    double t = 0;
#pragma unroll
    for (int k = 0; k < NACC; ++k) t += d[k][0] + d[k][1];
    if (t == 12345.0) out[0] = t;
}

template <int NACC>
__global__ void mma1684_kernel(double *out, double s) {
    double d[NACC][4];
    const double a = threadIdx.x * 1e-6, b = s;
#pragma unroll
    for (int k = 0; k < NACC; ++k) d[k][0] = d[k][1] = d[k][2] = d[k][3] = k;
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int k = 0; k < NACC; ++k) mma1684(d[k], a, a + 1, b);
    }
    double t = 0;
#pragma unroll
    for (int k = 0; k < NACC; ++k) t += d[k][0] + d[k][1] + d[k][2] + d[k][3];
    if (t == 12345.0) out[0] = t;
}

template <int NACC>
__global__ void mma1688_kernel(double *out, double s) {
    double d[NACC][4];
    double a[4], b[2];
#pragma unroll
    for (int k = 0; k < 4; ++k) a[k] = threadIdx.x * 1e-6 + k;
    b[0] = s;
    b[1] = s * 0.5;
#pragma unroll
    for (int k = 0; k < NACC; ++k) d[k][0] = d[k][1] = d[k][2] = d[k][3] = k;
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int k = 0; k < NACC; ++k) mma1688(d[k], a, b);
    }
    double t = 0;
#pragma unroll
    for (int k = 0; k < NACC; ++k) t += d[k][0] + d[k][1] + d[k][2] + d[k][3];
    if (t == 12345.0) out[0] = t;
}

template <int NACC>
__global__ void mma16816_kernel(double *out, double s) {
    double d[NACC][4];
    double a[8], b[4];
#pragma unroll
    for (int k = 0; k < 8; ++k) a[k] = threadIdx.x * 1e-6 + k;
#pragma unroll
    for (int k = 0; k < 4; ++k) b[k] = s * k;
#pragma unroll
    for (int k = 0; k < NACC; ++k) d[k][0] = d[k][1] = d[k][2] = d[k][3] = k;
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int k = 0; k < NACC; ++k) mma16816(d[k], a, b);
    }
    double t = 0;
#pragma unroll
    for (int k = 0; k < NACC; ++k) t += d[k][0] + d[k][1] + d[k][2] + d[k][3];
    if (t == 12345.0) out[0] = t;
}

// m8n8k4 DMMA interleaved with RATIO vector DFMA per mma: does the mix exceed either alone?
template <int RATIO>
__global__ void mixed_kernel(double *out, double s) {
    double d[4][2];
    double v[8];
    const double a = threadIdx.x * 1e-6, b = s;
#pragma unroll
    for (int k = 0; k < 4; ++k) d[k][0] = d[k][1] = k;
#pragma unroll
    for (int k = 0; k < 8; ++k) v[k] = k;
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            mma884(d[k], a, b);
#pragma unroll
            for (int r = 0; r < RATIO; ++r) v[(k * RATIO + r) & 7] = fma(v[(k * RATIO + r) & 7], s, 1e-9);
        }
    }
    double t = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) t += d[k][0] + d[k][1];
#pragma unroll
    for (int k = 0; k < 8; ++k) t += v[k];
    if (t == 12345.0) out[0] = t;
}

int main() {
    double *out;
    cudaMalloc(&out, 8);
    int dev = 0, sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    auto run = [&](const char *name, void (*k)(double *, double), int warps_per_block, int blocks_per_sm,
                   double fma_per_warp_iter, double mma_per_warp_iter, double dfma_per_warp_iter) {
        const int blocks = sms * blocks_per_sm, threads = 32 * warps_per_block;
        float best = 1e30f;
        for (int rep = 0; rep < 3; ++rep) {
            cudaEventRecord(e0);
            k<<<blocks, threads>>>(out, 0.999999);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (ms < best) best = ms;
        }
        const double warps = (double)blocks * warps_per_block;
        const double fma = warps * ITERS * fma_per_warp_iter;
        const double tflops = 2.0 * fma / (best * 1e-3) * 1e-12;
        const double per_sm_clk = fma / (best * 1e-3) / sms / (clk * 1e3);
        printf("{\"variant\": \"%s\", \"warps_per_sm\": %d, \"ms\": %.3f, \"fp64_tflops\": %.2f, "
               "\"fma_per_sm_per_clk_at_max\": %.1f, \"mma_per_warp_iter\": %.0f, \"dfma_per_warp_iter\": %.0f, "
               "\"err\": \"%s\"}\n",
               name, warps_per_block * blocks_per_sm, best, tflops, per_sm_clk, mma_per_warp_iter,
               dfma_per_warp_iter, cudaGetErrorString(cudaGetLastError()));
        fflush(stdout);
    };
    for (int wps : {4, 8, 16, 32}) {
        run("dfma 8 chains", dfma_kernel, 4, wps / 4, 8 * 32, 0, 8);
        run("mma m8n8k4 x4 acc", mma884_kernel<4>, 4, wps / 4, 4 * 256, 4, 0);
        run("mma m8n8k4 x8 acc", mma884_kernel<8>, 4, wps / 4, 8 * 256, 8, 0);
        run("mma m16n8k4 x4 acc", mma1684_kernel<4>, 4, wps / 4, 4 * 512, 4, 0);
        run("mma m16n8k8 x4 acc", mma1688_kernel<4>, 4, wps / 4, 4 * 1024, 4, 0);
        run("mma m16n8k16 x4 acc", mma16816_kernel<4>, 4, wps / 4, 4 * 2048, 4, 0);
        run("mixed m8n8k4 + 4 dfma", mixed_kernel<4>, 4, wps / 4, 4 * 256 + 16 * 32, 4, 16);
        run("mixed m8n8k4 + 8 dfma", mixed_kernel<8>, 4, wps / 4, 4 * 256 + 32 * 32, 4, 32);
    }
    printf("{\"sms\": %d, \"clock_khz\": %d}\n", sms, clk);
    return 0;
}
