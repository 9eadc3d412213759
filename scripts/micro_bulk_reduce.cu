// Microbenchmark: small fp64 scatter-add throughput on sm_100a -- per-lane red.global.add.f64
// vs TMA bulk reductions (cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f64) of 32 / 64 B
// runs issued by one lane or by every lane of a warp.  Informs the fused CSR assembly (NEXT-2):
// an extruded hex8 cell adds its 16 x 16 element matrix to the CSR values as 64 runs of 4
// contiguous doubles (the two levels of one neighbour vertex column).  Not part of the product.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/micro_bulk_reduce scripts/micro_bulk_reduce.cu
//   ./build/micro_bulk_reduce   -> one JSON line per variant
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void bulk_red_add_f64(double *dst, const double *src, uint32_t bytes) {
    asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f64 [%0], [%1], %2;" ::"l"(dst),
                 "r"(smem_u32(src)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }

// target of op o of warp w: runs of `len` doubles; pattern 0 = streaming (consecutive runs),
// pattern 1 = scattered inside a sliding 32 MB window (L2-resident reuse, like the CSR rows of
// nodes whose cells are processed close in time)
__device__ __forceinline__ int64_t target(int64_t w, int64_t o, int64_t ops_per_warp, int len, int pattern,
                                          int64_t nv) {
    const int64_t g = w * ops_per_warp + o;
    if (pattern == 0) return (g * len) % nv;
    const int64_t win = (32ll << 20) / 8;  // doubles in the window
    const int64_t base = ((g / 4096) * 4096 * len) % nv;
    uint64_t h = (uint64_t)g * 0x9E3779B97F4A7C15ull;
    h ^= h >> 29;
    return (base + (int64_t)(h % (uint64_t)(win / len)) * len) % nv;
}

__global__ void red_kernel(double *v, int64_t nv, int64_t ops_per_warp, int len, int pattern) {
    const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int l = threadIdx.x & 31;
    // lanes take consecutive ops; each op = len scalar reds
    for (int64_t o = l; o < ops_per_warp; o += 32) {
        double *p = v + target(w, o, ops_per_warp, len, pattern, nv);
        for (int k = 0; k < len; ++k) asm volatile("red.global.add.f64 [%0], %1;" ::"l"(p + k), "d"(1.0) : "memory");
    }
}

template <bool ALL_LANES>
__global__ void bulk_kernel(double *v, int64_t nv, int64_t ops_per_warp, int len, int pattern) {
    __shared__ __align__(128) double src[8][256];
    const int wl = threadIdx.x >> 5, l = threadIdx.x & 31;
    const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    for (int k = l; k < 256; k += 32) src[wl][k] = 1.0;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncwarp();
    if (ALL_LANES) {
        for (int64_t o = l; o < ops_per_warp; o += 32)
            bulk_red_add_f64(v + target(w, o, ops_per_warp, len, pattern, nv), &src[wl][(l * len) % 256],
                             len * 8);
    } else if (l == 0) {
        for (int64_t o = 0; o < ops_per_warp; ++o)
            bulk_red_add_f64(v + target(w, o, ops_per_warp, len, pattern, nv), &src[wl][0], len * 8);
    }
    bulk_commit();
    bulk_wait0();
}

int main() {
    const int64_t nv = 1ll << 28;  // 2 GiB of doubles
    double *v;
    cudaMalloc(&v, nv * 8);
    const int blocks = 148 * 8, threads = 256;
    const int64_t warps = (int64_t)blocks * threads / 32;
    double *h = new double[1 << 20];
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int pattern = 0; pattern < 2; ++pattern)
        for (int variant = 0; variant < 3; ++variant)
            for (int len : {4, 8}) {
                const int64_t ops_per_warp = variant == 0 ? 2048 : 4096;
                for (int rep = 0; rep < 2; ++rep) {
                    cudaMemset(v, 0, nv * 8);
                    cudaEventRecord(e0);
                    if (variant == 0) red_kernel<<<blocks, threads>>>(v, nv, ops_per_warp, len, pattern);
                    else if (variant == 1) bulk_kernel<false><<<blocks, threads>>>(v, nv, ops_per_warp, len, pattern);
                    else bulk_kernel<true><<<blocks, threads>>>(v, nv, ops_per_warp, len, pattern);
                    cudaEventRecord(e1);
                    cudaEventSynchronize(e1);
                    float ms = 0;
                    cudaEventElapsedTime(&ms, e0, e1);
                    // checksum over a prefix: every added value is 1.0
                    cudaMemcpy(h, v, (1 << 20) * 8, cudaMemcpyDeviceToHost);
                    double s = 0;
                    for (int i = 0; i < (1 << 20); ++i) s += h[i];
                    if (rep == 1) {
                        const double ops = (double)warps * ops_per_warp;
                        printf("{\"variant\": \"%s\", \"pattern\": \"%s\", \"run_doubles\": %d, \"ops\": %.0f, "
                               "\"ms\": %.3f, \"Gops_per_s\": %.2f, \"Gdoubles_added_per_s\": %.2f, \"prefix_sum\": %.0f, "
                               "\"err\": \"%s\"}\n",
                               variant == 0 ? "red.f64 per lane" : variant == 1 ? "bulk reduce, lane 0" : "bulk reduce, all lanes",
                               pattern ? "scattered in 32 MB window" : "streaming", len, ops, ms, ops / ms * 1e-6,
                               ops * len / ms * 1e-6, s, cudaGetErrorString(cudaGetLastError()));
                        fflush(stdout);
                    }
                }
            }
    return 0;
}
