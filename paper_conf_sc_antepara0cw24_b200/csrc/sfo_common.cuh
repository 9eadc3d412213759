// sfo_common.cuh -- element traits, per-tile record layout and sm_100a PTX
// helpers (1-D TMA bulk copies, mbarriers) for libstokesfo.so.
//
// Independent of oracle/: the reference-element tables below are generated
// here from the basis formulas, not shared.
#pragma once
#include <cstdint>
#include <cuda.h>  // CUtensorMap (type only; the encoder is fetched through cudaGetDriverEntryPoint)
#include <cuda_runtime.h>

namespace sfo {

// ---------------------------------------------------------------------------
// Element traits.  N nodes, Q quadrature points (N == Q for both elements),
// TC cells per tile.  One tile is processed by ONE warp (one CTA = one warp):
// lane l <-> (cell l / N, node-or-qp l % N), TC = floor(32 / N) cells, so every
// exchange between the per-QP and per-node phases stays inside a warp
// (__syncwarp only; no CTA-wide barriers).  See DESIGN.md "Kernels".
// ---------------------------------------------------------------------------
struct Hex8 {
    static constexpr int N = 8, Q = 8, TC = 4, ELEM = 0;
    static constexpr int SLAB = 32;        // doubles per (qp, dir) slab of GradBF in a record
    static constexpr int JPITCH = 4 * N * N;  // J staging pitch per cell = the global image (one bulk store)
    // lane l <-> (cell l / 8, node-or-qp l % 8): a quarter-warp is one cell
    __host__ __device__ static constexpr int lane_cell(int l) { return l / N; }
    __host__ __device__ static constexpr int lane_sub(int l) { return l % N; }
    __host__ __device__ static constexpr int lane_of(int c, int sub) { return c * N + sub; }
    // slot of (cell c, node n) in the slab of qp q (a slab is 32 doubles = 2 x 16 bank pairs):
    // 16 (c >> 1) + a 4-bit bank-pair index linear over GF(2) in the bits of (c, n, q),
    //   b0 = q0 ^ n1, b1 = q1 ^ n2, b2 = q2 ^ n0, b3 = c0 ^ n1,
    // chosen so that three access patterns each hit 16 distinct bank pairs per half-warp:
    // the per-QP loads (fixed n, lanes over (c, q)), the vector per-node loads (fixed q, lanes
    // over (c, j)) and the DMMA operand loads (fixed c, lanes over (n = l >> 2, q = l & 3 (+4)))
    __host__ __device__ static constexpr int slot(int c, int n, int q) {
        return 16 * (c >> 1) + (((q ^ (n >> 1)) & 1) | (((q >> 1) ^ (n >> 2)) & 1) << 1 |
                                (((q >> 2) ^ n) & 1) << 2 | ((c ^ (n >> 1)) & 1) << 3);
    }
    // gathered U/s per (cell, node) in shared memory: node slot rotated by the cell, (n + c) mod 8, so
    // that the per-QP phase's broadcast reads of one node (one address per cell) hit 4 distinct bank
    // groups: 1 wavefront per LDS.128 / LDS.64 instead of 4 / 2 (cell pitch 128 B put every cell's
    // node n in the same banks; ncu r2p1: the U reads were LDS.128 at 4 wavefronts)
    static constexpr int UPITCH = N;
    __host__ __device__ static constexpr int uidx(int c, int n) { return c * UPITCH + ((n + c) & 7); }
    // per-QP scalars (f, cell, qp): qp slot rotated by 2 c, so the node phase's broadcast (q, q+1)
    // pair reads (one LDS.128 per field and QP pair, one address per cell) are conflict-free (1
    // wavefront instead of 2) while the per-QP phase's stores stay conflict-free (each cell's 8
    // lanes still fill its own 16 banks); q even => the pair (q, q+1) is adjacent and 16-B aligned
    static constexpr bool QS_PAIRS = true;
    __host__ __device__ static constexpr int qsi(int f, int c, int q) { return (f * TC + c) * Q + ((q + 2 * c) & 7); }
};
#ifndef SFO_WEDGE_SLAB32
#define SFO_WEDGE_SLAB32 1
#endif
struct Wedge6 {
    static constexpr int N = 6, Q = 6, TC = 5, ELEM = 1;  // 30 active lanes
#if SFO_WEDGE_SLAB32
    // 32-double slabs (2 padding slots per (qp, dir): +288 B per 5-cell record) with the q-rotated slot map
    // (c + 5n + 5q) mod 32: per-QP-phase GradBF loads conflict-free (36 vs 57 wavefronts per tile in the bank
    // model), per-node loads 162 (same), and the slot arithmetic is a power-of-two mask
    static constexpr int SLAB = 32;
#else
    static constexpr int SLAB = 30;
#endif
    static constexpr int JPITCH = 4 * N * N + 2;  // odd 16-B pitch: conflict-free staging, per-cell bulk stores
    // lane l <-> (cell l % 5, node-or-qp l / 5) (node-major), slot (29c + 25n) mod 30:
    // chosen by a search over affine slot maps with the shared-memory bank model
    // (per-QP loads 57 vs 108 wavefronts per tile, per-node loads 162 vs 240)
    __host__ __device__ static constexpr int lane_cell(int l) { return l % TC; }
    __host__ __device__ static constexpr int lane_sub(int l) { return l / TC; }
    __host__ __device__ static constexpr int lane_of(int c, int sub) { return sub * TC + c; }
#if SFO_WEDGE_SLAB32
    // (an affine map with the DMMA operand loads conflict-free, (c + 5n + h(q)) mod 32 with h = (0, 4, 8, 12, 1,
    // 8), measured −1-2% on the C5 vector Jacobian and −4% on the C5 residual, same box: the wedge6 Jacobian
    // stays on the vector kernel)
    __host__ __device__ static constexpr int slot(int c, int n, int q) { return (c + 5 * n + 5 * q) & 31; }
#else
    __host__ __device__ static constexpr int slot(int c, int n, int) { return (29 * c + 25 * n) % 30; }
#endif
    // odd 16-B cell pitch for the gathered U rows; per-QP scalars qp-major
    // (lanes (c, q) of the per-QP phase then write consecutive addresses)
    static constexpr int UPITCH = 7;
    __host__ __device__ static constexpr int uidx(int c, int n) { return c * UPITCH + n; }
    static constexpr bool QS_PAIRS = false;
    __host__ __device__ static constexpr int qsi(int f, int c, int q) { return (f * Q + q) * TC + c; }
};

__host__ __device__ constexpr int64_t round_up(int64_t x, int64_t m) { return (x + m - 1) / m * m; }

// Per-tile record in the workspace (and, identically, in shared memory):
//   conn  int32 [TC][N]                 node ids
//   kc    fp64  [TC]                    Glen prefactor per cell
//   wm    fp64  [Q][TC]                 w_q det J_q
//   G     fp64  [Q][3][SLAB]            GradBF; (cell c, node n) of qp q sits at
//                                       slot E::slot(c, n, q) (hex8: c*N + (n+q) mod N)
// The slot map makes both the per-QP loads (fixed n, lanes over (c, q)) and
// the per-node loads (fixed q, lanes over (c, j)) conflict-free for hex8
// (bank model in DESIGN.md).  One 1-D TMA bulk
// copy moves a whole record (size multiple of 16 B: 6,560 B hex8, 4,736 B wedge6).
template <class E>
struct Rec {
    static constexpr int N = E::N, Q = E::Q, TC = E::TC, SLAB = E::SLAB;
    static constexpr int CONN_OFF = 0;
    static constexpr int CONN_BYTES = (int)round_up(N * TC * 4, 16);
    static constexpr int KC_OFF = CONN_OFF + CONN_BYTES;
    static constexpr int WM_OFF = KC_OFF + (int)round_up(TC * 8, 16);
    static constexpr int G_OFF = WM_OFF + (int)round_up(Q * TC * 8, 16);
    static constexpr int BYTES = G_OFF + Q * 3 * SLAB * 8;
    // index helpers (in elements of the respective type)
    __host__ __device__ static constexpr int conn(int n, int c) { return c * N + n; }
    __host__ __device__ static constexpr int wm(int q, int c) { return q * TC + c; }
    __host__ __device__ static constexpr int g(int n, int q, int d, int c) { return (q * 3 + d) * SLAB + E::slot(c, n, q); }
};

// Compact per-tile record (STOKESFO_GEOMETRY_COMPACT): the geometry as
// A_q = J_q^-T (9 doubles per (cell, qp), row-major, r = physical component, s =
// reference direction) instead of GradBF; the evaluation forms GradBF_n(q) =
// A_q grad_xi phi_n(xi_q) in registers (9 FMA per node).  Layout:
//   conn  int32 [TC][N]
//   kc    fp64  [TC]
//   wm    fp64  [Q][TC]
//   A     fp64  [9][Q][TC]      (k = 3 r + s; lanes (c, q) of one k read 32 consecutive doubles)
// 2,720 B per hex8 tile (680 B/cell instead of 1,640), 2,576 B per wedge6 tile.
template <class E>
struct RecC {
    static constexpr int N = E::N, Q = E::Q, TC = E::TC;
    static constexpr int CONN_OFF = 0;
    static constexpr int KC_OFF = (int)round_up(N * TC * 4, 16);
    static constexpr int WM_OFF = KC_OFF + (int)round_up(TC * 8, 16);
    static constexpr int A_OFF = WM_OFF + (int)round_up(Q * TC * 8, 16);
    static constexpr int BYTES = A_OFF + 9 * Q * TC * 8;
    __host__ __device__ static constexpr int conn(int n, int c) { return c * N + n; }
    __host__ __device__ static constexpr int wm(int q, int c) { return q * TC + c; }
    __host__ __device__ static constexpr int a(int k, int q, int c) { return (k * Q + q) * TC + c; }
};

// Workspace: [0, 256) header (error flag), then ntiles records.
constexpr int64_t WS_HEADER = 256;
enum : int { ERR_DETJ = 1, ERR_CONN = 2, ERR_CSR = 4, ERR_NONFINITE = 8 };

// ---------------------------------------------------------------------------
// PTX helpers (sm_90+/sm_100a): mbarrier + 1-D bulk async copies (TMA engine)
// ---------------------------------------------------------------------------
// R[i] += v for a pointer into global memory (local or NVLink-mapped peer):
// red.global.add.f64 straight away.  atomicAdd on a generic double* makes the
// compiler test the address space first (two QSPC + branches per call).
__device__ __forceinline__ void red_add(double *p, double v) {
    asm volatile("red.global.add.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}
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
// shared -> global 2-D tensor store (TMA; bulk-group completion); out-of-bound box elements are skipped
__device__ __forceinline__ void tensor_s2g_2d(const CUtensorMap *map, int x, int y, const void *src, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.tensor.2d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%1, %2}], [%3], %4;" ::"l"(
            reinterpret_cast<uint64_t>(map)),
        "r"(x), "r"(y), "r"(smem_u32(src)), "l"(pol)
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
