// sfo_common.cuh -- element traits, per-tile record layout and sm_100a PTX
// helpers (1-D TMA bulk copies, mbarriers) for libstokesfo.so.
//
// Independent of oracle/: the reference-element tables below are generated
// here from the basis formulas, not shared.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace sfo {

// ---------------------------------------------------------------------------
// Element traits.  N nodes, Q quadrature points, TC cells per tile.
// Tile sizes are chosen so that one CTA holds TC*N threads (phase-2 mapping)
// = TC*Q threads (phase-1 mapping); see DESIGN.md "Kernels".
// ---------------------------------------------------------------------------
struct Hex8 {
    static constexpr int N = 8, Q = 8, TC = 16, ELEM = 0;
    // phase-2 mapping: thread <-> (cell t/N, node t%N): the 8 threads of a cell
    // share one warp quarter, so per-(cell,qp) scalars are read as broadcasts.
    static constexpr bool NODE_MAJOR_P2 = false;
    static constexpr int JPITCH = 4 * N * N;  // J staging pitch per cell (dense: one bulk store per tile)
    // Swizzles (cell index within the tile), chosen with a bank model of 64-bit
    // shared loads served per half-warp: every phase-1/phase-2 GradBF load and
    // every conn load is conflict-free.
    __host__ __device__ static constexpr int gswz(int c, int n) { return c ^ ((2 * n) & 15); }
    __host__ __device__ static constexpr int cswz(int c, int n) { return c ^ (4 * ((n >> 1) & 3)); }
};
struct Wedge6 {
    static constexpr int N = 6, Q = 6, TC = 32, ELEM = 1;
    // phase-2 mapping: thread <-> (cell t%TC, node t/TC) (node-major: 6 does not
    // divide a warp); J staging uses a padded pitch (73 x 16 B) and per-cell
    // bulk stores so the 16-byte staging stores are conflict-free.
    static constexpr bool NODE_MAJOR_P2 = true;
    static constexpr int JPITCH = 4 * N * N + 2;
    __host__ __device__ static constexpr int gswz(int c, int) { return c; }
    __host__ __device__ static constexpr int cswz(int c, int) { return c; }
};

__host__ __device__ constexpr int64_t round_up(int64_t x, int64_t m) { return (x + m - 1) / m * m; }

// Per-tile record in the workspace (and, identically, in shared memory):
//   conn  int32 [N][TC]          node ids, cell fastest
//   kc    fp64  [TC]             Glen prefactor per cell
//   wm    fp64  [Q][TC]          w_q det J_q
//   G     fp64  [N][Q][3][TC]    GradBF, cell fastest
// One 1-D TMA bulk copy moves a whole record (size multiple of 128 B).
template <class E>
struct Rec {
    static constexpr int N = E::N, Q = E::Q, TC = E::TC;
    static constexpr int CONN_OFF = 0;
    static constexpr int CONN_BYTES = (int)round_up(N * TC * 4, 16);
    static constexpr int KC_OFF = CONN_OFF + CONN_BYTES;
    static constexpr int WM_OFF = KC_OFF + TC * 8;
    static constexpr int G_OFF = WM_OFF + Q * TC * 8;
    static constexpr int BYTES = (int)round_up(G_OFF + N * Q * 3 * TC * 8, 128);
    // light record (on-the-fly geometry mode): conn + k_c only
    static constexpr int LIGHT_BYTES = (int)round_up(KC_OFF + TC * 8, 128);
    // index helpers (in elements of the respective type)
    __host__ __device__ static constexpr int conn(int n, int c) { return n * TC + E::cswz(c, n); }
    __host__ __device__ static constexpr int wm(int q, int c) { return q * TC + c; }
    __host__ __device__ static constexpr int g(int n, int q, int d, int c) { return ((n * Q + q) * 3 + d) * TC + E::gswz(c, n); }
};

// Workspace: [0, 256) header (error flag), then ntiles records.
constexpr int64_t WS_HEADER = 256;
enum : int { ERR_DETJ = 1, ERR_CONN = 2, ERR_CSR = 4 };

// ---------------------------------------------------------------------------
// PTX helpers (sm_90+/sm_100a): mbarrier + 1-D bulk async copies (TMA engine)
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
// global -> shared bulk copy, completion via mbarrier transaction count
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar,
                                         uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
        : "memory");
}
// shared -> global bulk copy (bulk-group completion)
__device__ __forceinline__ void bulk_s2g(void *dst, const void *src, uint32_t bytes, uint64_t pol) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(dst),
                 "r"(smem_u32(src)), "r"(bytes), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void cp_async16(void *dst, const void *src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async8(void *dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

}  // namespace sfo
