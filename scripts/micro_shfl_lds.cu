// Microbenchmark: do warp shuffles (SHFL) and shared-memory loads (LDS.64) share
// the L1/shared data path on sm_100a?  Times a loop of LDS.64 only, SHFL only and
// both interleaved; if "both" takes ~max(lds, shfl) they are separate pipes.
// Informs whether the eval kernel's redundant G_j shared loads (the L1 data pipe
// is its busiest unit) could move to shuffles.  Not part of the product.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/micro_shfl_lds scripts/micro_shfl_lds.cu
#include <cstdio>
#include <cuda_runtime.h>

template <int MODE>  // 0 = LDS only, 1 = SHFL only, 2 = both, 3 = LDS.128 with lane pairs on one 16-B chunk,
                     // 4 = LDS.128 all lanes distinct
__global__ void loop(double *out, int iters) {
    __shared__ double sm[32 * 16 + 32];
    const int l = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 32 * 16 + 32; i += blockDim.x) sm[i] = i * 0.5;
    __syncthreads();
    double acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    double v = l * 1.0;
    const double *base = sm + ((w & 7) * 32);
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            if (MODE == 0 || MODE == 2) acc[k] += base[(l + k + it) & 31];      // conflict-free LDS.64
            if (MODE == 1 || MODE == 2) acc[k] += __shfl_sync(0xffffffffu, v, (l + k) & 31);  // SHFL x2
            if (MODE == 3) {  // lanes 2m, 2m+1 read chunk m: 16 distinct 16-B chunks per warp
                const double2 t = reinterpret_cast<const double2 *>(sm)[((l >> 1) + k + it) & 15];
                acc[k] += t.x * t.y;
            }
            if (MODE == 4) {  // 32 distinct 16-B chunks
                const double2 t = reinterpret_cast<const double2 *>(sm)[(l + k + it) & 31];
                acc[k] += t.x * t.y;
            }
        }
        v += 1.0;
    }
    double s = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) s += acc[k];
    if (s == 1234.5) out[0] = s;
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    double *out;
    cudaMalloc(&out, 8);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int iters = 1 << 16;
    const char *names[5] = {"lds64", "shfl64", "both", "lds128_pairs", "lds128_distinct"};
    for (int rep = 0; rep < 2; ++rep)
        for (int m = 0; m < 5; ++m) {
            cudaEventRecord(e0);
            const dim3 g(sms * 4), b(256);
            if (m == 0) loop<0><<<g, b>>>(out, iters);
            if (m == 1) loop<1><<<g, b>>>(out, iters);
            if (m == 2) loop<2><<<g, b>>>(out, iters);
            if (m == 3) loop<3><<<g, b>>>(out, iters);
            if (m == 4) loop<4><<<g, b>>>(out, iters);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            // warp-instructions of the measured op per SM per cycle at the observed time (clock from attribute)
            int clk_khz = 0;
            cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
            const double warp_ops = (double)sms * 4 * 8 * iters * 8;  // warps x iters x 8 ops
            printf("{\"mode\": \"%s\", \"ms\": %.3f, \"warp_ops_per_sm_cycle\": %.3f}\n", names[m], ms,
                   warp_ops / sms / (ms * 1e-3 * clk_khz * 1e3));
        }
    return 0;
}
