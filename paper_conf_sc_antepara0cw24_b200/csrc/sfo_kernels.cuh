// sfo_kernels.cuh -- sm_100a kernels of libstokesfo.so.
//
//   G1 geometry_kernel : basis/quadrature precompute into per-tile records
//   G2 gather_kernel   : U_cell[c][n][a] = U[2 conn + a]
//   G3/G4 eval_kernel  : fused gather -> Ugrad -> Glen mu -> stress -> QP sum
//                        (Fig. 2) -> scatter-add, and (JAC) the
//                        forward-mode tangent of the same chain
//                        written as element matrices through a TMA bulk store
//   G5 scatter kernels, G7 halo pack/unpack.
//
// Design: HBM-bound fp64, no tensor cores.  Persistent
// CTAs stream one record per tile (conn, k_c, wM, GradBF of TC cells, cell
// fastest) with 1-D TMA bulk copies into a 2-stage mbarrier ring; U and s are
// gathered through conn (L2-resident thanks to Hilbert-ordered columns);
// per-QP work runs with thread <-> (cell, qp); per-node work with thread <->
// (cell, node), accumulating locally in registers (the paper's "local
// accumulation") and issuing one red.global.add.f64 per dof.
#pragma once
#include "sfo_common.cuh"

namespace sfo {

// ---------------------------------------------------------------------------
// Reference element, evaluated in device code from the basis formulas.
// ---------------------------------------------------------------------------
template <class E>
__device__ __forceinline__ void qp_coords(int q, double &x, double &y, double &z, double &w);

template <>
__device__ __forceinline__ void qp_coords<Hex8>(int q, double &x, double &y, double &z, double &w) {
    const double g = 1.0 / sqrt(3.0);
    x = (q & 1) ? g : -g;
    y = (q & 2) ? g : -g;
    z = (q & 4) ? g : -g;
    w = 1.0;
}
template <>
__device__ __forceinline__ void qp_coords<Wedge6>(int q, double &x, double &y, double &z, double &w) {
    const double g = 1.0 / sqrt(3.0);
    const int t = q % 3;
    x = (t == 1) ? 2.0 / 3.0 : 1.0 / 6.0;
    y = (t == 2) ? 2.0 / 3.0 : 1.0 / 6.0;
    z = (q >= 3) ? g : -g;
    w = 1.0 / 6.0;
}

// phi_n and d phi_n / d xi at (x, y, z)
template <class E>
__device__ __forceinline__ void basis(int n, double x, double y, double z, double &phi, double &dx, double &dy,
                                      double &dz);
template <>
__device__ __forceinline__ void basis<Hex8>(int n, double x, double y, double z, double &phi, double &dx,
                                            double &dy, double &dz) {
    // Shards order: x-sign (-,+,+,-), y-sign (-,-,+,+), z-sign by n >= 4
    const double sx = ((n & 3) == 1 || (n & 3) == 2) ? 1.0 : -1.0;
    const double sy = ((n & 3) >= 2) ? 1.0 : -1.0;
    const double sz = (n >= 4) ? 1.0 : -1.0;
    const double a = 1.0 + sx * x, b = 1.0 + sy * y, c = 1.0 + sz * z;
    phi = 0.125 * a * b * c;
    dx = 0.125 * sx * b * c;
    dy = 0.125 * a * sy * c;
    dz = 0.125 * a * b * sz;
}
template <>
__device__ __forceinline__ void basis<Wedge6>(int n, double x, double y, double z, double &phi, double &dx,
                                              double &dy, double &dz) {
    const int t = n % 3;
    const double s = (n >= 3) ? 1.0 : -1.0;
    const double h = 0.5 * (1.0 + s * z);
    const double lam = (t == 0) ? 1.0 - x - y : (t == 1 ? x : y);
    const double lx = (t == 0) ? -1.0 : (t == 1 ? 1.0 : 0.0);
    const double ly = (t == 0) ? -1.0 : (t == 1 ? 0.0 : 1.0);
    phi = lam * h;
    dx = lx * h;
    dy = ly * h;
    dz = lam * 0.5 * s;
}

// Position of GradBF (n, q, d, c) inside a record (swizzled cell index, see
// the element traits in sfo_common.cuh).
template <class E>
__host__ __device__ __forceinline__ int gidx(int n, int q, int d, int c) {
    return Rec<E>::g(n, q, d, c);
}

// ---------------------------------------------------------------------------
// G1: geometry precompute.  Thread <-> (cell, qp).
//   OUT = GEO_RECORDS: full per-tile records (stored-geometry mode, at create)
//   OUT = GEO_CANON:   canonical grad_bf [C][N][Q][3], w_measure [C][Q] (export)
//   OUT = GEO_CHECK:   only the det J > 0 / conn range checks
//   OUT = GEO_ALBANY:  GradBF, wGradBF, wBF component-major [entry][cell] at
//                      grad_bf (NEXT-1 scratch, see sfo_albany.cuh)
// ---------------------------------------------------------------------------
//   OUT = GEO_COMPACT: compact per-tile records (A_q = J_q^-T, wM; RecC)
enum { GEO_RECORDS = 0, GEO_CANON = 1, GEO_CHECK = 2, GEO_ALBANY = 3, GEO_COMPACT = 4 };

template <class E, int OUT>
__global__ void geometry_kernel(int64_t ncells, int64_t nnodes, const int32_t *__restrict__ conn,
                                const double *__restrict__ coords, const double *__restrict__ kc_in, double kscal,
                                char *__restrict__ recs, double *__restrict__ grad_bf, double *__restrict__ w_measure,
                                int *__restrict__ err) {
    using R = Rec<E>;
    using RC = RecC<E>;
    constexpr int N = E::N, Q = E::Q, TC = E::TC;
    constexpr bool REC = OUT == GEO_RECORDS || OUT == GEO_COMPACT;
    const int64_t ntiles = (ncells + TC - 1) / TC;
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t nwork = (REC ? ntiles * TC : ncells) * Q;
    if (gid >= nwork) return;
    const int q = (int)(gid % Q);
    const int64_t cell = gid / Q;
    const int64_t tile = cell / TC;
    const int c = (int)(cell % TC);
    char *rec = REC ? recs + tile * (int64_t)(OUT == GEO_COMPACT ? RC::BYTES : R::BYTES) : nullptr;
    int32_t *rconn = reinterpret_cast<int32_t *>(rec + (OUT == GEO_COMPACT ? RC::CONN_OFF : R::CONN_OFF));
    double *rkc = reinterpret_cast<double *>(rec + (OUT == GEO_COMPACT ? RC::KC_OFF : R::KC_OFF));
    double *rwm = reinterpret_cast<double *>(rec + (OUT == GEO_COMPACT ? RC::WM_OFF : R::WM_OFF));
    double *rg = reinterpret_cast<double *>(rec + R::G_OFF);
    double *ra = reinterpret_cast<double *>(rec + RC::A_OFF);
    if (cell >= ncells) {  // padding cells of the ragged last tile: zero record
        if (REC) {
            if (q == 0) {
                for (int n = 0; n < N; ++n) rconn[R::conn(n, c)] = 0;
                rkc[c] = 0.0;
            }
            rwm[R::wm(q, c)] = 0.0;
            if constexpr (OUT == GEO_COMPACT) {
                for (int k = 0; k < 9; ++k) ra[RC::a(k, q, c)] = 0.0;
            } else {
                for (int n = 0; n < N; ++n)
                    for (int d = 0; d < 3; ++d) rg[gidx<E>(n, q, d, c)] = 0.0;
            }
        }
        return;
    }
    int32_t nid[N];
    bool bad_conn = false;
    for (int n = 0; n < N; ++n) {
        nid[n] = conn[cell * N + n];
        if (nid[n] < 0 || nid[n] >= nnodes) {
            bad_conn = true;
            nid[n] = 0;
        }
    }
    if (bad_conn) atomicOr(err, ERR_CONN);
    if (REC && q == 0) {
        for (int n = 0; n < N; ++n) rconn[R::conn(n, c)] = nid[n];
        rkc[c] = kc_in ? kc_in[cell] : kscal;
    }
    double xq, yq, zq, wq;
    qp_coords<E>(q, xq, yq, zq, wq);
    double dphi[N][3];
    double J[3][3] = {{0, 0, 0}, {0, 0, 0}, {0, 0, 0}};
    // cell-local coordinates x_n - x_0 (sum_n grad_xi phi_n = 0): avoids the
    // O(|x| eps) residue of ~10^3-km absolute coordinates on metre-thick cells
    const double o0 = coords[3 * (int64_t)nid[0] + 0];
    const double o1 = coords[3 * (int64_t)nid[0] + 1];
    const double o2 = coords[3 * (int64_t)nid[0] + 2];
#pragma unroll
    for (int n = 0; n < N; ++n) {
        double phi;
        basis<E>(n, xq, yq, zq, phi, dphi[n][0], dphi[n][1], dphi[n][2]);
        const double x0 = coords[3 * (int64_t)nid[n] + 0] - o0;
        const double x1 = coords[3 * (int64_t)nid[n] + 1] - o1;
        const double x2 = coords[3 * (int64_t)nid[n] + 2] - o2;
#pragma unroll
        for (int s = 0; s < 3; ++s) {
            J[0][s] += x0 * dphi[n][s];
            J[1][s] += x1 * dphi[n][s];
            J[2][s] += x2 * dphi[n][s];
        }
    }
    // inverse transpose by cofactors: (J^-T)[r][s] = cof[r][s] / det
    double cof[3][3];
    cof[0][0] = J[1][1] * J[2][2] - J[1][2] * J[2][1];
    cof[0][1] = J[1][2] * J[2][0] - J[1][0] * J[2][2];
    cof[0][2] = J[1][0] * J[2][1] - J[1][1] * J[2][0];
    cof[1][0] = J[0][2] * J[2][1] - J[0][1] * J[2][2];
    cof[1][1] = J[0][0] * J[2][2] - J[0][2] * J[2][0];
    cof[1][2] = J[0][1] * J[2][0] - J[0][0] * J[2][1];
    cof[2][0] = J[0][1] * J[1][2] - J[0][2] * J[1][1];
    cof[2][1] = J[0][2] * J[1][0] - J[0][0] * J[1][2];
    cof[2][2] = J[0][0] * J[1][1] - J[0][1] * J[1][0];
    const double det = J[0][0] * cof[0][0] + J[0][1] * cof[0][1] + J[0][2] * cof[0][2];
    if (!(det > 0.0)) atomicOr(err, ERR_DETJ);
    if (OUT == GEO_CHECK) return;
    const double idet = 1.0 / det;
    if constexpr (OUT == GEO_COMPACT) {  // A = J^-T = cof / det
#pragma unroll
        for (int r = 0; r < 3; ++r)
#pragma unroll
            for (int s2 = 0; s2 < 3; ++s2) ra[RC::a(3 * r + s2, q, c)] = cof[r][s2] * idet;
        rwm[RC::wm(q, c)] = wq * det;
        return;
    } else {
#pragma unroll
        for (int n = 0; n < N; ++n)
#pragma unroll
            for (int r = 0; r < 3; ++r) {
                const double g = (cof[r][0] * dphi[n][0] + cof[r][1] * dphi[n][1] + cof[r][2] * dphi[n][2]) * idet;
                if (OUT == GEO_RECORDS) {
                    rg[gidx<E>(n, q, r, c)] = g;
                } else if (OUT == GEO_ALBANY) {
                    grad_bf[((int64_t)(n * Q + q) * 3 + r) * ncells + cell] = g;
                    grad_bf[((int64_t)(N * Q * 3) + (n * Q + q) * 3 + r) * ncells + cell] = g * (wq * det);
                } else if (grad_bf) {
                    grad_bf[((cell * N + n) * Q + q) * 3 + r] = g;
                }
            }
    }
    if (OUT == GEO_ALBANY) {
#pragma unroll
        for (int n = 0; n < N; ++n) {
            double phi, dx, dy, dz;
            basis<E>(n, xq, yq, zq, phi, dx, dy, dz);
            grad_bf[((int64_t)(2 * N * Q * 3) + n * Q + q) * ncells + cell] = phi * (wq * det);
        }
        return;
    }
    if (OUT == GEO_RECORDS) rwm[R::wm(q, c)] = wq * det;
    else if (w_measure) w_measure[cell * Q + q] = wq * det;
}

// Export records -> canonical grad_bf [C][N][Q][3], w_measure [C][Q].
template <class E>
__global__ void geometry_export_kernel(int64_t ncells, const char *__restrict__ recs, double *__restrict__ grad_bf,
                                       double *__restrict__ w_measure) {
    using R = Rec<E>;
    constexpr int N = E::N, Q = E::Q, TC = E::TC;
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (gid >= ncells * Q) return;
    const int q = (int)(gid % Q);
    const int64_t cell = gid / Q;
    const char *rec = recs + (cell / TC) * (int64_t)R::BYTES;
    const int c = (int)(cell % TC);
    const double *rwm = reinterpret_cast<const double *>(rec + R::WM_OFF);
    const double *rg = reinterpret_cast<const double *>(rec + R::G_OFF);
    if (w_measure) w_measure[cell * Q + q] = rwm[R::wm(q, c)];
    if (grad_bf)
        for (int n = 0; n < N; ++n)
            for (int d = 0; d < 3; ++d) grad_bf[((cell * N + n) * Q + q) * 3 + d] = rg[gidx<E>(n, q, d, c)];
}

// Export compact records -> canonical grad_bf = A_q grad_xi phi_n, w_measure (what the
// compact evaluation forms in registers).
template <class E>
__global__ void geometry_export_compact_kernel(int64_t ncells, const char *__restrict__ recs,
                                               double *__restrict__ grad_bf, double *__restrict__ w_measure) {
    using RC = RecC<E>;
    constexpr int N = E::N, Q = E::Q, TC = E::TC;
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (gid >= ncells * Q) return;
    const int q = (int)(gid % Q);
    const int64_t cell = gid / Q;
    const char *rec = recs + (cell / TC) * (int64_t)RC::BYTES;
    const int c = (int)(cell % TC);
    const double *ra = reinterpret_cast<const double *>(rec + RC::A_OFF);
    if (w_measure) w_measure[cell * Q + q] = reinterpret_cast<const double *>(rec + RC::WM_OFF)[RC::wm(q, c)];
    if (!grad_bf) return;
    double A[9];
    for (int k = 0; k < 9; ++k) A[k] = ra[RC::a(k, q, c)];
    double xq, yq, zq, wq;
    qp_coords<E>(q, xq, yq, zq, wq);
    for (int n = 0; n < N; ++n) {
        double phi, d0, d1, d2;
        basis<E>(n, xq, yq, zq, phi, d0, d1, d2);
        for (int r = 0; r < 3; ++r)
            grad_bf[((cell * N + n) * Q + q) * 3 + r] = fma(A[3 * r + 0], d0, fma(A[3 * r + 1], d1, A[3 * r + 2] * d2));
    }
}

// ---------------------------------------------------------------------------
// G2: gather.  Thread <-> (cell, node).
// ---------------------------------------------------------------------------
template <int N>
__global__ void gather_kernel(int64_t ncells, const int32_t *__restrict__ conn, const double2 *__restrict__ U,
                              double2 *__restrict__ Ucell) {
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (gid >= ncells * N) return;
    Ucell[gid] = __ldg(&U[conn[gid]]);
}

// ---------------------------------------------------------------------------
// G3/G4: fused evaluation.  One CTA = one warp, persistent over tiles of TC
// cells; lane l <-> (cell E::lane_cell(l), node-or-qp E::lane_sub(l)).
// ---------------------------------------------------------------------------
struct EvalArgs {
    const char *recs;         // per-tile records (stored-geometry mode)
    const double4 *xyz4;      // node coordinates (x, y, z, 0) (on-the-fly mode)
    const int32_t *conn;      // caller conn [C][N] (on-the-fly mode)
    const double *kc;         // caller flow factor [C] or null (on-the-fly mode)
    double kscal;             // scalar k if kc == null
    int *err;                 // sticky device error flag
    int64_t ntiles, ncells;
    const double *U;          // [nodes][2]
    const double *surface;    // [nodes] or null
    const double *force_qp;   // [C][Q][2] or null (overrides surface)
    double rho_g, delta;
    double *mu_qp;            // [C][Q] or null
    double *R_cell;           // [C][N][2] or null
    double *R;                // [nodes][2] or null (+=)
    double *J_cell;           // [C][2N][2N] (M_JAC)
    const double *X;          // [nodes][2] direction (M_JVP)
    double *Y;                // [nodes][2] += J(U) X (M_JVP), or += diag J(U) (M_DIAG)
    // fused halo over peer memory (null = none): rem[node] = row of remtab or -1;
    // remtab[row] = {count, peer_0, idx_0, peer_1, idx_1, ...} (REM_ROW ints);
    // peers[p] = device pointer of peer p's R, mapped into this process
    const int32_t *rem;
    const int32_t *remtab;
    double *const *peers;
    double *const *peers_y;   // M_JVP / M_DIAG: the peers' Y (required when rem is set)
    // NEXT-2 fused CSR assembly (M_CSR): J contributions go straight into
    // csr_vals[rowptr[2 g_i + a] + 2 slot[c][i][j] + b] (no element matrices)
    const int64_t *rowptr;    // [2 nodes + 1]
    const uint64_t *slots;    // [C][N] rows of N uint8 slots (8-byte pitch)
    double *csr_vals;         // [nnz] (+=)
    int use_jmap;             // wedge6 M_JAC: J tile stored through the kernel's tensor-map parameter
    int packed;               // M_JAC on the DMMA kernels: J_cell holds the symmetric block-packed form
};

// Symmetric block-packed element matrix (stokesfo_jacobian_packed): the N(N+1)/2 upper 2 x 2 node blocks
// (i, j >= i) of J_cell[c], block index i N - i (i - 1) / 2 + (j - i), entries [a][b] = J[(i,a),(j,b)].
template <int N>
__host__ __device__ __forceinline__ constexpr int pk_block(int i, int j) {
    return i * N - i * (i - 1) / 2 + (j - i);
}
template <int N>
__host__ __device__ constexpr int pk_blocks() {
    return N * (N + 1) / 2;
}

constexpr int REM_MAX = 7;                 // remote copies of one node (<= 8 parts meet at a vertex)
constexpr int REM_ROW = 1 + 2 * REM_MAX;

// V[node] += (r0, r1) locally and, for nodes on a partition boundary, into the
// V of every other GPU that holds the node (red.global.add.f64 through the
// NVLink-mapped peer pointers `peers`): the halo sum happens inside the
// evaluation kernel, no pack / exchange / unpack (DESIGN.md
// "Multi-GPU").  V = R (peers) or the J.v output Y (peers_y).
__device__ __forceinline__ void scatter_node(const int32_t *rem, const int32_t *remtab, double *V,
                                             double *const *peers, int32_t node, double r0, double r1) {
    red_add(V + 2 * (int64_t)node + 0, r0);
    red_add(V + 2 * (int64_t)node + 1, r1);
    if (rem) {
        const int32_t row = __ldg(rem + node);
        if (row >= 0) {
            const int32_t *t = remtab + (int64_t)row * REM_ROW;
            const int cnt = t[0];
            for (int k = 0; k < cnt; ++k) {
                double *pr = peers[t[1 + 2 * k]] + 2 * (int64_t)t[2 + 2 * k];
                red_add(pr + 0, r0);
                red_add(pr + 1, r1);
            }
        }
    }
}

// Half-block split of the k = N/2 tangent block between the two lanes that
// both own it, and diagonal 2x2 blocks formed as symmetric (3 entries): the
// tangent then forms each of the N(N+1)/2 distinct blocks of a cell once
// (A/B switches; 1 = on)
#ifndef SFO_KSPLIT
#define SFO_KSPLIT 1
#endif
#ifndef SFO_DIAGSYM
#define SFO_DIAGSYM 1
#endif

// Evaluation modes of the fused kernels
// M_DIAG: residual + the diagonal of the assembled Jacobian only (Jacobi
// preconditioner of the Newton-Krylov driver): J[(i,a),(i,a)] of every cell
// scatter-added into Y, no element matrices.
enum { M_RESID = 0, M_JAC = 1, M_JVP = 2, M_CSR = 3, M_DIAG = 4 };
// modes that form the tangent blocks (element matrices or CSR contributions)
template <int MODE>
__host__ __device__ constexpr bool forms_jac() {
    return MODE == M_JAC || MODE == M_CSR;
}
// per-(cell, qp) scalars: beta00 beta01 beta02 beta11 beta12, wmu2, gamma, wf0, wf1
// (+ for M_JVP: dbeta00 dbeta01 dbeta02 dbeta11 dbeta12, gamma * tau)
constexpr int NQS = 9;
template <int MODE>
__host__ __device__ constexpr int nqs() {
    return MODE == M_JVP ? 15 : 9;
}

// per-QP scalar f of (cell c, qp q): [NQS][TC][Q] (qp fastest: the per-QP
// phase writes 32 consecutive doubles, the per-node phase reads broadcasts)
template <class E>
__device__ __forceinline__ int qsi(int f, int c, int q) {
    return E::qsi(f, c, q);
}

// Per-QP scalars in shared memory: fields [0, SPLIT) in the common region `lo`,
// fields [SPLIT, nqs) in `hi` (the unused tail of the current stage buffer,
// when it has room: one shared-memory region less per warp -> one more
// resident warp per SM for hex8 JAC; see EvalSmem).
template <class E, int SPLIT>
struct QsView {
    double *lo, *hi;
    __device__ __forceinline__ double &operator()(int f, int c, int q) const {
        return f < SPLIT ? lo[E::qsi(f, c, q)] : hi[E::qsi(f - SPLIT, c, q)];
    }
    // fields of QPs (q, q+1), q even, as one 16-B load (E::QS_PAIRS layouts keep the pair adjacent)
    __device__ __forceinline__ double2 pair(int f, int c, int q) const {
        return *reinterpret_cast<const double2 *>(&(*this)(f, c, q));
    }
};

// per-QP scalar fields the per-node phase of a mode reads (JVP: 0-5, 7-14; residual: 0-5, 7, 8; else 0-8)
template <int MODE>
__host__ __device__ constexpr bool qs_used(int f) {
    return MODE == M_JVP ? f != 6 : (MODE == M_RESID ? (f != 6 && f < 9) : f < 9);
}

// Per-QP scalars kept in registers (the residual-only and J.v modes of the
// stored-geometry kernel, which exchange per-node partial sums instead).
struct RegQs {
    double *v;
    __device__ __forceinline__ double &operator()(int f, int, int) const { return v[f]; }
};

// Partial-sum exchange of the residual / J.v modes: lane (c, q) writes, for
// every node n of its cell, P[c][n][q] = (G_n(q) . sigma_a(q) + wf_a(q) phi_n(q))_a
// (double2, a = 0, 1); lane (c, i) then sums P[c][i][(k + i) mod Q] over k.
// Row pitch 8 double2, cell pitch chosen with the bank model (writes and
// rotated reads conflict-free for hex8; 24 / 28 wavefronts for wedge6).
template <class E>
__host__ __device__ constexpr int psum_idx(int c, int n, int q) {
    return c * (E::N == 8 ? 64 : 53) + n * 8 + q;
}
template <class E>
constexpr int psum_bytes() {
    return (E::N == 8 ? E::TC * 64 : (E::TC - 1) * 53 + E::N * 8) * 16;
}

// ---- shared device pieces ---------------------------------------------------

// x^(-1/3) for x > 0 in full fp64 precision with a short dependency chain:
// a float approximation 2^(-log2(x)/3) (MUFU lg2/ex2, ~1e-7 relative) refined
// by one third-order step of (1 - e)^(-1/3) = 1 + e/3 + 2e^2/9 + O(e^3),
// e = 1 - x y^3 (truncation ~1e-21, rounding ~2e-16).  ~12 instructions
// instead of rcbrt's ~40, on the per-QP critical path (e2 -> mu -> scalars).
// Outside the float range the library rcbrt is used.
#ifndef SFO_FAST_RCBRT
#define SFO_FAST_RCBRT 1
#endif
__device__ __forceinline__ double rcbrt_fp64(double x) {
    if (!SFO_FAST_RCBRT || !(x > 1e-30 && x < 1e30)) return rcbrt(x);
    float l, y0;
    asm("lg2.approx.f32 %0, %1;" : "=f"(l) : "f"((float)x));
    asm("ex2.approx.f32 %0, %1;" : "=f"(y0) : "f"(l * (-1.0f / 3.0f)));
    const double y = (double)y0;
    const double e = fma(-x * y, y * y, 1.0);
    return fma(y * e, fma(e, 2.0 / 9.0, 1.0 / 3.0), y);
}

// Per-QP tail: given Ugrad and grad s_h at (cell c, qp q), evaluate the
// effective strain rate (Z2), Glen viscosity at n = 3 (Z1, Z3) and the per-QP
// scalars the per-node phase needs.  beta = B g so that sigma = 2 mu beta gives
// strs00..strs12 of Fig. 2.
template <class E, int MODE = M_RESID, class QS>
__device__ __forceinline__ void qp_tail(const EvalArgs &a, const QS &qs, int c, int q, int nvalid, int64_t cell0,
                                        bool have_s, double kc, double wm, double ux, double uy, double uz, double vx,
                                        double vy, double vz, double gs0, double gs1, const double *dg = nullptr) {
    constexpr int Q = E::Q;
    constexpr double P_EXP = -1.0 / 3.0;  // (1 - n) / (2 n) at n = 3
    const double uyvx = uy + vx;
    const double e2 = ux * ux + vy * vy + ux * vy + 0.25 * uyvx * uyvx + 0.25 * uz * uz + 0.25 * vz * vz;
    const double r = rcbrt_fp64(e2 + a.delta);  // (e2 + delta)^(-1/3)
    const double mu = kc * r;
    const double wmu2 = 2.0 * wm * mu;
    qs(0, c, q) = 2.0 * ux + vy;   // beta_(0,0) = strs00 / (2 mu)
    qs(1, c, q) = 0.5 * uyvx;      // beta_(0,1) = beta_(1,0) = strs01 / (2 mu)
    qs(2, c, q) = 0.5 * uz;        // beta_(0,2) = strs02 / (2 mu)
    qs(3, c, q) = ux + 2.0 * vy;   // beta_(1,1) = strs11 / (2 mu)
    qs(4, c, q) = 0.5 * vz;        // beta_(1,2) = strs12 / (2 mu)
    qs(5, c, q) = wmu2;
    // gamma = wM 2 mu p / (e2 + delta) = wmu2 p r^3  (d mu / d e2, reading Z5)
    qs(6, c, q) = wmu2 * P_EXP * (r * r * r);
    double wf0 = 0.0, wf1 = 0.0;
    if (a.force_qp) {
        if (c < nvalid) {
            const double2 f = *reinterpret_cast<const double2 *>(a.force_qp + ((cell0 + c) * Q + q) * 2);
            wf0 = wm * f.x;
            wf1 = wm * f.y;
        }
    } else if (have_s) {
        wf0 = wm * a.rho_g * gs0;
        wf1 = wm * a.rho_g * gs1;
    }
    qs(7, c, q) = wf0;
    qs(8, c, q) = wf1;
    if (MODE == M_JVP) {
        // directional derivative along X: dg = grad of X at the QP; d beta = B dg;
        // tau = (B g) . dg = d(eps_e^2); d sigma = 2 mu (d beta + p tau beta / (e2 + delta))
        const double dux = dg[0], duy = dg[1], duz = dg[2], dvx = dg[3], dvy = dg[4], dvz = dg[5];
        const double b00 = 2.0 * ux + vy, b01 = 0.5 * uyvx, b02 = 0.5 * uz, b11 = ux + 2.0 * vy, b12 = 0.5 * vz;
        const double tau = b00 * dux + b01 * (duy + dvx) + b02 * duz + b11 * dvy + b12 * dvz;
        qs(9, c, q) = 2.0 * dux + dvy;
        qs(10, c, q) = 0.5 * (duy + dvx);
        qs(11, c, q) = 0.5 * duz;
        qs(12, c, q) = dux + 2.0 * dvy;
        qs(13, c, q) = 0.5 * dvz;
        qs(14, c, q) = wmu2 * P_EXP * (r * r * r) * tau;
    }
    if (a.mu_qp && c < nvalid) a.mu_qp[(cell0 + c) * Q + q] = mu;
}

// Per-node phase, lane <-> (cell c2, node i): residual rows (i,0), (i,1) and,
// for JAC, the 2x2 tangent blocks J[(i,.),(j_k,.)], j_k = (i+k) mod N,
// k = 0..N/2, accumulated over QPs in registers (the paper's local
// accumulation).
// J_q[(i,a),(j,b)] = sum_e M_ab[e] G_j[e],
// M_ab = wM 2 mu (B-block (a,b) applied to G_i) + gamma h_(i,a) beta_(b,.)
// is the exact forward derivative of the chain (seed-sparse Sacado lanes).
// pf() is called once at q = Q/2 (prefetch hook).
template <class E, int MODE, class PF, class QS>
__device__ __forceinline__ void node_accumulate(const double *rg, const QS &qs, int c2, int i, const double *bfi,
                                                double &R0, double &R1, double (&Jb)[E::N / 2 + 1][2][2], double &dR0,
                                                double &dR1, PF pf) {
    constexpr int N = E::N, Q = E::Q, K = N / 2;
    constexpr bool JAC = forms_jac<MODE>();
    R0 = 0.0;
    R1 = 0.0;
    dR0 = 0.0;
    dR1 = 0.0;
    if (JAC) {
#pragma unroll
        for (int k = 0; k <= K; ++k) Jb[k][0][0] = Jb[k][0][1] = Jb[k][1][0] = Jb[k][1][1] = 0.0;
    }
    constexpr int NF = nqs<MODE>();
    double sq[NF], sq1[NF];  // this QP's scalars; the next QP's when they arrive as a (q, q+1) pair
#pragma unroll
    for (int q = 0; q < Q; ++q) {
        if (q == Q / 2) pf();
#pragma unroll
        for (int f = 0; f < NF; ++f) {
            if (!qs_used<MODE>(f)) {
                sq[f] = 0.0;
            } else if (E::QS_PAIRS && (q & 1) == 0) {
                const double2 v = qs.pair(f, c2, q);
                sq[f] = v.x;
                sq1[f] = v.y;
            } else if (E::QS_PAIRS) {
                sq[f] = sq1[f];
            } else {
                sq[f] = qs(f, c2, q);
            }
        }
        const double b00 = sq[0], b01 = sq[1], b02 = sq[2];
        const double b11 = sq[3], b12 = sq[4];
        const double b10 = b01;
        const double wmu2 = sq[5];
        const double wf0 = sq[7], wf1 = sq[8];
        const double gi0 = rg[gidx<E>(i, q, 0, c2)];
        const double gi1 = rg[gidx<E>(i, q, 1, c2)];
        const double gi2 = rg[gidx<E>(i, q, 2, c2)];
        // h_(i,a) = sum_d G_i[d] beta_(a,d);  residual row (i,a) += wmu2 h + wf_a BF_i
        const double h0 = fma(gi2, b02, fma(gi1, b01, gi0 * b00));
        const double h1 = fma(gi2, b12, fma(gi1, b11, gi0 * b10));
        R0 = fma(wf0, bfi[q], fma(wmu2, h0, R0));
        R1 = fma(wf1, bfi[q], fma(wmu2, h1, R1));
        if (MODE == M_JVP) {
            // dR_(i,a) += wmu2 G_i . dbeta_a + gamma tau h_(i,a)
            const double d00 = sq[9 % NF], d01 = sq[10 % NF], d02 = sq[11 % NF];
            const double d11 = sq[12 % NF], d12 = sq[13 % NF];
            const double gt = sq[14 % NF];
            const double e0 = fma(gi2, d02, fma(gi1, d01, gi0 * d00));
            const double e1 = fma(gi2, d12, fma(gi1, d11, gi0 * d01));
            dR0 = fma(gt, h0, fma(wmu2, e0, dR0));
            dR1 = fma(gt, h1, fma(wmu2, e1, dR1));
        }
        if (MODE == M_DIAG) {
            // J[(i,a),(i,a)] = wM 2 mu G_i^T B_aa G_i + gamma h_(i,a)^2,
            // B_00 = diag(2, 1/2, 1/2), B_11 = diag(1/2, 2, 1/2) (the k = 0 block's diagonal)
            const double gam = sq[6];
            const double t = 0.5 * fma(gi2, gi2, fma(gi1, gi1, gi0 * gi0));
            dR0 = fma(gam * h0, h0, fma(wmu2, fma(1.5 * gi0, gi0, t), dR0));
            dR1 = fma(gam * h1, h1, fma(wmu2, fma(1.5 * gi1, gi1, t), dR1));
        }
        if (JAC) {
            const double gam = sq[6];
            const double gh0 = gam * h0, gh1 = gam * h1;
            const double w0 = wmu2 * gi0, w1 = wmu2 * gi1, w2 = wmu2 * gi2;
            const double m00x = fma(2.0, w0, gh0 * b00), m00y = fma(0.5, w1, gh0 * b01),
                         m00z = fma(0.5, w2, gh0 * b02);
            const double m01x = fma(0.5, w1, gh0 * b10), m01y = fma(gh0, b11, w0), m01z = gh0 * b12;
            const double m10x = fma(gh1, b00, w1), m10y = fma(0.5, w0, gh1 * b01), m10z = gh1 * b02;
            const double m11x = fma(0.5, w0, gh1 * b10), m11y = fma(2.0, w1, gh1 * b11),
                         m11z = fma(0.5, w2, gh1 * b12);
#pragma unroll
            for (int k = 0; k <= K; ++k) {
                const int j = (i + k) % N;
                double gj0, gj1, gj2;
                if (k == 0) {
                    gj0 = gi0; gj1 = gi1; gj2 = gi2;
                } else {
                    gj0 = rg[gidx<E>(j, q, 0, c2)];
                    gj1 = rg[gidx<E>(j, q, 1, c2)];
                    gj2 = rg[gidx<E>(j, q, 2, c2)];
                }
                if (SFO_KSPLIT && k == K) {
                    // block (i, i+K) is also block (i+K, i)^T of the partner lane: each lane of
                    // the pair forms half of it (lanes i < K column b = 0: (0,0), (1,0); lanes
                    // i >= K row a = 1 of their own block: (1,1), (1,0)), so only the first
                    // operand differs between the two (m00 / m11); ksplit_exchange completes it
                    const bool lo = i < K;
                    const double ax = lo ? m00x : m11x, ay = lo ? m00y : m11y, az = lo ? m00z : m11z;
                    Jb[k][0][0] = fma(az, gj2, fma(ay, gj1, fma(ax, gj0, Jb[k][0][0])));
                    Jb[k][0][1] = fma(m10z, gj2, fma(m10y, gj1, fma(m10x, gj0, Jb[k][0][1])));
                    continue;
                }
                // explicit 3-deep DFMA chains into the accumulators (no DMUL/DADD)
                Jb[k][0][0] = fma(m00z, gj2, fma(m00y, gj1, fma(m00x, gj0, Jb[k][0][0])));
                Jb[k][0][1] = fma(m01z, gj2, fma(m01y, gj1, fma(m01x, gj0, Jb[k][0][1])));
                // the diagonal block is symmetric (J is a Hessian): (1,0) = (0,1), set after the loop
                if (!(SFO_DIAGSYM && k == 0))
                    Jb[k][1][0] = fma(m10z, gj2, fma(m10y, gj1, fma(m10x, gj0, Jb[k][1][0])));
                Jb[k][1][1] = fma(m11z, gj2, fma(m11y, gj1, fma(m11x, gj0, Jb[k][1][1])));
            }
        }
    }
    if (JAC && SFO_DIAGSYM) Jb[0][1][0] = Jb[0][0][1];
}

// Completes block k = K after node_accumulate's split (SFO_KSPLIT): lane i < K
// holds P00, P10 of P = J[(i,.),(i+K,.)], its partner lane i+K holds P11, P01
// (entries (1,1), (1,0) of its own block P^T).  One exchange of two doubles;
// every lane of the warp must call this.
template <class E>
__device__ __forceinline__ void ksplit_exchange(double (&Jb)[E::N / 2 + 1][2][2], int c, int i, bool act) {
    constexpr int N = E::N, K = N / 2;
    if (!SFO_KSPLIT) return;
    const int src = act ? E::lane_of(c, (i + K) % N) : (int)(threadIdx.x & 31);
    const double e0 = Jb[K][0][0], e1 = Jb[K][0][1];
    const double f0 = __shfl_sync(0xffffffffu, e0, src), f1 = __shfl_sync(0xffffffffu, e1, src);
    if (i < K) {  // e = (P00, P10), f = (P11, P01)
        Jb[K][0][0] = e0;
        Jb[K][0][1] = f1;
        Jb[K][1][0] = e1;
        Jb[K][1][1] = f0;
    } else {  // e = (P11, P01), f = (P00, P10); own block = P^T = [[P00, P10], [P01, P11]]
        Jb[K][0][0] = f0;
        Jb[K][0][1] = f1;
        Jb[K][1][0] = e1;
        Jb[K][1][1] = e0;
    }
}

// Write J[c2] rows (2i, 2i+1) into a staging image of the global layout:
// direct blocks (i, i+k), k = 0..K, and transposed blocks (i+k, i) for
// 0 < k < K (J is symmetric: the Hessian of the quadrature energy).  Rotating
// j with i keeps the 16-byte stores of a quarter-warp in distinct bank groups.
template <class E>
__device__ __forceinline__ void stage_J(double *base, int c2, int i, const double (&Jb)[E::N / 2 + 1][2][2]) {
    constexpr int N = E::N, K = N / 2, LD = 2 * N;
    double *Jc = base + c2 * E::JPITCH;
#pragma unroll
    for (int k = 0; k <= K; ++k) {
        const int j = (i + k) % N;
        *reinterpret_cast<double2 *>(Jc + (2 * i + 0) * LD + 2 * j) = make_double2(Jb[k][0][0], Jb[k][0][1]);
        *reinterpret_cast<double2 *>(Jc + (2 * i + 1) * LD + 2 * j) = make_double2(Jb[k][1][0], Jb[k][1][1]);
        if (k > 0 && k < K) {
            *reinterpret_cast<double2 *>(Jc + (2 * j + 0) * LD + 2 * i) = make_double2(Jb[k][0][0], Jb[k][1][0]);
            *reinterpret_cast<double2 *>(Jc + (2 * j + 1) * LD + 2 * i) = make_double2(Jb[k][0][1], Jb[k][1][1]);
        }
    }
}

// One lane issues the TMA store(s) of a staged tile of element Jacobians: one
// 1-D bulk copy when the staging pitch is the global image (hex8); for the
// padded wedge6 staging (pitch JPITCH > NN) one 2-D tensor store through the
// tensor map J viewed as [C][NN] doubles with a (JPITCH x TC) box -- the box's
// padding columns and the rows past C fall outside the tensor and are not
// written -- or, without a map, one bulk copy per cell.
template <class E>
__device__ __forceinline__ void store_J(double *J_cell, int64_t cell0, int nvalid, const char *stage, uint64_t pol,
                                        const CUtensorMap *jmap = nullptr) {
    constexpr int NN = 4 * E::N * E::N;
    if (E::JPITCH == NN) {
        bulk_s2g(J_cell + cell0 * NN, stage, (uint32_t)(nvalid * NN * 8), pol);
    } else if (jmap) {
        tensor_s2g_2d(jmap, 0, (int)cell0, stage, pol);
    } else {
        for (int c = 0; c < nvalid; ++c)
            bulk_s2g(J_cell + (cell0 + c) * NN, stage + c * E::JPITCH * 8, (uint32_t)(NN * 8), pol);
    }
    bulk_commit();
}

// NEXT-2 fused assembly: lane (c, i) adds its tangent blocks into the CSR
// values through the per-cell slot table -- direct blocks (i, i+k), k = 0..K,
// and, by symmetry, the transposed blocks (i+k, i) for 0 < k < K (the same
// split as stage_J).  Row bases rp = (rowptr[2 g_i], rowptr[2 g_i + 1]) and
// slot rows of the partner nodes come from their lanes by shuffle.  Every lane
// of the warp must call this (shuffles); `live` gates the atomics.
template <class E>
__device__ __forceinline__ void csr_scatter(double *vals, int c, int i, bool live, uint64_t srow, longlong2 rp,
                                            const double (&Jb)[E::N / 2 + 1][2][2]) {
    constexpr int N = E::N, K = N / 2;
    const int cc = c < E::TC ? c : 0;
#pragma unroll
    for (int k = 0; k <= K; ++k) {
        const int j = (i + k) % N;
        const int src = E::lane_of(cc, j);
        const uint64_t srow_j = __shfl_sync(0xffffffffu, srow, src);
        const long long rj0 = __shfl_sync(0xffffffffu, rp.x, src);
        const long long rj1 = __shfl_sync(0xffffffffu, rp.y, src);
        if (live) {
            const int sij = (int)((srow >> (8 * j)) & 0xff);
            double *p0 = vals + rp.x + 2 * sij, *p1 = vals + rp.y + 2 * sij;
            red_add(p0, Jb[k][0][0]);
            red_add(p0 + 1, Jb[k][0][1]);
            red_add(p1, Jb[k][1][0]);
            red_add(p1 + 1, Jb[k][1][1]);
            if (k > 0 && k < K) {  // J[(j,a),(i,b)] = J[(i,b),(j,a)]
                const int sji = (int)((srow_j >> (8 * i)) & 0xff);
                double *q0 = vals + rj0 + 2 * sji, *q1 = vals + rj1 + 2 * sji;
                red_add(q0, Jb[k][0][0]);
                red_add(q0 + 1, Jb[k][1][0]);
                red_add(q1, Jb[k][0][1]);
                red_add(q1 + 1, Jb[k][1][1]);
            }
        }
    }
}

// slot row and CSR row bases of lane (cell, node i), loaded ahead of use
__device__ __forceinline__ void csr_row_load(const EvalArgs &a, int64_t cell, int32_t g, bool live, uint64_t &srow,
                                             longlong2 &rp, int N, int i) {
    srow = 0;
    rp = make_longlong2(0, 0);
    if (live) {
        srow = __ldg(a.slots + cell * N + i);
        rp = __ldg(reinterpret_cast<const longlong2 *>(a.rowptr) + g);
    }
}

template <class E>
__device__ __forceinline__ void basis_row(int i, double (&bfi)[E::Q]) {
#pragma unroll
    for (int q = 0; q < E::Q; ++q) {
        double x, y, z, w, dx, dy, dz;
        qp_coords<E>(q, x, y, z, w);
        basis<E>(i, x, y, z, bfi[q], dx, dy, dz);
    }
}

// Resident 1-warp CTAs per SM the register budget is sized for (12 with the
// Jacobian accumulators, 16 for the residual-only kernels: <= 128 registers).
#ifndef SFO_WEDGE_JAC_WARPS
#define SFO_WEDGE_JAC_WARPS 16
#endif
template <class E, int MODE>
__host__ __device__ constexpr int warps_per_sm() {
    // wedge6 JAC: 16 (128 registers, 2-warp CTAs so that 16 x 13.7 KB of shared
    // memory fits next to the per-CTA driver reserve)
    return forms_jac<MODE>() ? (E::N == 6 && MODE == M_JAC ? SFO_WEDGE_JAC_WARPS : 12) : 16;
}
// Independent persistent warps per CTA (each warp runs its own tile loop and
// record ring in its own shared-memory slice; only __syncwarp is used).
template <class E, int MODE>
__host__ __device__ constexpr int warps_per_cta() {
    return (E::N == 6 && MODE == M_JAC && SFO_WEDGE_JAC_WARPS > 12) ? 2 : 1;
}

// ---- G3/G4 with stored geometry (the §8(a2) precompute streamed per tile) ----

// Shared memory: NSTAGE stage buffers + per-QP scalars + mbarriers.  A stage
// buffer holds [record | gathered U (double2 [TC][N]) | s ([TC][N])]; once the
// warp has consumed a tile's record, the same buffer stages the tile's element
// Jacobians (the global image) for one TMA bulk store.
template <class E, int MODE, int NSTAGE = 2>
struct EvalSmem {
    static constexpr int N = E::N, Q = E::Q, TC = E::TC;
    static constexpr int REC = Rec<E>::BYTES;
    static constexpr int U_OFF = (int)round_up(REC, 16);     // double2 [TC][UPITCH]
    static constexpr int S_OFF = U_OFF + TC * E::UPITCH * 16;  // double  [TC][UPITCH]
    static constexpr int X_OFF = (int)round_up(S_OFF + TC * E::UPITCH * 8, 16);  // double2 [TC][UPITCH] (M_JVP)
    static constexpr int IN_BYTES = X_OFF + (MODE == M_JVP ? TC * E::UPITCH * 16 : 0);
    static constexpr int J_BYTES = MODE == M_JAC ? TC * E::JPITCH * 8 : 0;
    static constexpr int STAGE = (int)round_up(IN_BYTES > J_BYTES ? IN_BYTES : J_BYTES, 128);
    // per-QP scalar fields that fit in the stage's tail past the inputs (free until the J staging)
    static constexpr int TAIL_OFF = (int)round_up(IN_BYTES, 16);
    static constexpr int FIELD = TC * Q * 8;
    static constexpr int TAIL_FIT = (STAGE - TAIL_OFF) / FIELD;
    static constexpr int TAIL_FIELDS = TAIL_FIT < 3 ? TAIL_FIT : 3;
    // residual-only and J.v modes keep the per-QP scalars in registers (partial-sum exchange)
    static constexpr bool PSUM = MODE == M_RESID || MODE == M_JVP;
    static constexpr int SPLIT = PSUM ? 0 : nqs<MODE>() - TAIL_FIELDS;   // fields [0, SPLIT) in the common region
    static constexpr int OFF_QS = NSTAGE * STAGE;            // double [SPLIT][TC][Q]
    static constexpr int OFF_BAR = (int)round_up(OFF_QS + SPLIT * FIELD, 8);
    static constexpr int BYTES = OFF_BAR + NSTAGE * 8;
    static constexpr int SLICE = (int)round_up(BYTES, 128);  // per-warp slice in multi-warp CTAs
    static_assert(!PSUM || Rec<E>::G_OFF + psum_bytes<E>() <= Rec<E>::BYTES, "partial sums overlay GradBF");
    static_assert(U_OFF % 16 == 0 && X_OFF % 16 == 0 && STAGE % 128 == 0 && OFF_QS % 16 == 0, "alignment");
};

// Gather of U (16 B) and s (8 B) of one tile through its conn (lane <->
// (cell, node)): loaded into registers at the prefetch point (one tile ahead,
// half a tile of latency slack) and stored to the tile's stage buffer with one
// conflict-free 16-B shared store per lane (a cp.async gather would cost one
// shared-memory wavefront per lane: the L1/shared data pipe is the busiest unit).
struct Gathered {
    double2 u;
    double s;
    double2 x;
};
template <class E, int MODE>
__device__ __forceinline__ Gathered gather_load(const char *stage, const double *U, const double *surface,
                                                bool have_s, const double *X) {
    using R = Rec<E>;
    Gathered v{make_double2(0.0, 0.0), 0.0, make_double2(0.0, 0.0)};
    const int l = threadIdx.x & 31;
    if (l < E::TC * E::N) {
        const int c = E::lane_cell(l), n = E::lane_sub(l);
        const int32_t g = reinterpret_cast<const int32_t *>(stage + R::CONN_OFF)[R::conn(n, c)];
        v.u = __ldg(reinterpret_cast<const double2 *>(U) + g);
        if (have_s) v.s = __ldg(surface + g);
        if (MODE == M_JVP) v.x = __ldg(reinterpret_cast<const double2 *>(X) + g);
    }
    return v;
}
template <class E, int MODE>
__device__ __forceinline__ void gather_store(char *stage, const Gathered &v) {
    using S = EvalSmem<E, MODE>;
    const int l = threadIdx.x & 31;
    if (l < E::TC * E::N) {
        const int e = E::uidx(E::lane_cell(l), E::lane_sub(l));  // [cell][node]
        reinterpret_cast<double2 *>(stage + S::U_OFF)[e] = v.u;
        reinterpret_cast<double *>(stage + S::S_OFF)[e] = v.s;
        if (MODE == M_JVP) reinterpret_cast<double2 *>(stage + S::X_OFF)[e] = v.x;
    }
}

template <class E, int MODE, int NSTAGE>
__global__ void __launch_bounds__(32 * warps_per_cta<E, MODE>(), (warps_per_sm<E, MODE>() / warps_per_cta<E, MODE>()))
    eval_kernel(EvalArgs a, const __grid_constant__ CUtensorMap jmap) {
    constexpr int N = E::N, Q = E::Q, TC = E::TC;
    constexpr bool JAC = MODE == M_JAC, JVP = MODE == M_JVP, CSR = MODE == M_CSR;
    static_assert(N == Q, "lane mappings assume N == Q");
    using R = Rec<E>;
    using S = EvalSmem<E, MODE, NSTAGE>;
    constexpr int WPC = warps_per_cta<E, MODE>();
    extern __shared__ __align__(128) char smem_all[];
    // this warp's virtual CTA: index vb of vg, its own shared-memory slice
    char *smem = smem_all + (threadIdx.x >> 5) * S::SLICE;
    const int64_t vb = (int64_t)blockIdx.x * WPC + (threadIdx.x >> 5);
    const int64_t vg = (int64_t)gridDim.x * WPC;
    double *qs_lo = reinterpret_cast<double *>(smem + S::OFF_QS);
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem + S::OFF_BAR);
    const int l = threadIdx.x & 31;
    const bool act = l < TC * N;
    const int c = act ? E::lane_cell(l) : TC, s = act ? E::lane_sub(l) : 0;  // (cell, node-or-qp)
    const bool have_s = (a.surface != nullptr) && (a.force_qp == nullptr);

    uint64_t pol_stream = 0;
    if (l == 0) {
        pol_stream = policy_evict_first();
        for (int k = 0; k < NSTAGE; ++k) mbar_init(&bar[k], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int k = 0; k < NSTAGE; ++k) {
            const int64_t tile = vb + (int64_t)k * vg;
            if (tile < a.ntiles) {
                mbar_arrive_expect_tx(&bar[k], R::BYTES);
                bulk_g2s(smem + k * S::STAGE, a.recs + tile * (int64_t)R::BYTES, R::BYTES, &bar[k], pol_stream);
            }
        }
    }
    __syncwarp();
    if (vb < a.ntiles) {
        mbar_wait(&bar[0], 0);
        gather_store<E, MODE>(smem, gather_load<E, MODE>(smem, a.U, a.surface, have_s, a.X));
    }
    double bfi[Q];
    basis_row<E>(act ? s : 0, bfi);
    double bq[N];  // phi_n at this lane's QP, every n (partial-sum modes)
    {
        double x, y, z, w, dx, dy, dz;
        qp_coords<E>(act ? s : 0, x, y, z, w);
#pragma unroll
        for (int n = 0; n < N; ++n) basis<E>(n, x, y, z, bq[n], dx, dy, dz);
    }

    int it = 0;
    for (int64_t tile = vb; tile < a.ntiles; tile += vg, ++it) {
        const int st = it % NSTAGE;
        char *stage = smem + st * S::STAGE;
        const int32_t *rconn = reinterpret_cast<const int32_t *>(stage + R::CONN_OFF);
        const double *rkc = reinterpret_cast<const double *>(stage + R::KC_OFF);
        const double *rwm = reinterpret_cast<const double *>(stage + R::WM_OFF);
        const double *rg = reinterpret_cast<const double *>(stage + R::G_OFF);
        const double2 *Us = reinterpret_cast<const double2 *>(stage + S::U_OFF);
        const double *ss = reinterpret_cast<const double *>(stage + S::S_OFF);
        const double2 *Xs = reinterpret_cast<const double2 *>(stage + S::X_OFF);
        const QsView<E, S::SPLIT> qs{qs_lo, reinterpret_cast<double *>(stage + S::TAIL_OFF)};
        const int64_t cell0 = tile * TC;
        const int nvalid = (a.ncells - cell0 < (int64_t)TC) ? (int)(a.ncells - cell0) : TC;

        __syncwarp();  // this tile's gathered U, s (stored by every lane) are visible

        // ---- per-QP phase: lane <-> (cell c, qp s) ----
        double gq[S::PSUM ? N : 1][3];  // G_n(q) kept for the partial sums (PSUM modes)
        double qv[S::PSUM ? 15 : 1];
        if (act) {
            const int q = s;
            double ux = 0, uy = 0, uz = 0, vx = 0, vy = 0, vz = 0, gs0 = 0, gs1 = 0;
            double dg[6] = {0, 0, 0, 0, 0, 0};
#pragma unroll
            for (int n = 0; n < N; ++n) {
                const double g0 = rg[gidx<E>(n, q, 0, c)];
                const double g1 = rg[gidx<E>(n, q, 1, c)];
                const double g2 = rg[gidx<E>(n, q, 2, c)];
                if constexpr (S::PSUM) {
                    gq[n][0] = g0;
                    gq[n][1] = g1;
                    gq[n][2] = g2;
                }
                const int e = E::uidx(c, n);
                const double2 uv = Us[e];
                ux = fma(uv.x, g0, ux); uy = fma(uv.x, g1, uy); uz = fma(uv.x, g2, uz);
                vx = fma(uv.y, g0, vx); vy = fma(uv.y, g1, vy); vz = fma(uv.y, g2, vz);
                if (have_s) {
                    const double sn = ss[e];
                    gs0 = fma(sn, g0, gs0); gs1 = fma(sn, g1, gs1);
                }
                if (JVP) {
                    const double2 xv = Xs[e];
                    dg[0] = fma(xv.x, g0, dg[0]); dg[1] = fma(xv.x, g1, dg[1]); dg[2] = fma(xv.x, g2, dg[2]);
                    dg[3] = fma(xv.y, g0, dg[3]); dg[4] = fma(xv.y, g1, dg[4]); dg[5] = fma(xv.y, g2, dg[5]);
                }
            }
            if constexpr (S::PSUM)
                qp_tail<E, MODE>(a, RegQs{qv}, c, q, nvalid, cell0, have_s, rkc[c], rwm[R::wm(q, c)], ux, uy, uz, vx,
                                 vy, vz, gs0, gs1, dg);
            else
                qp_tail<E, MODE>(a, qs, c, q, nvalid, cell0, have_s, rkc[c], rwm[R::wm(q, c)], ux, uy, uz, vx, vy,
                                 vz, gs0, gs1, dg);
        }
        __syncwarp();

        // ---- per-node phase (+ gather of the next tile at q = Q/2) ----
        const int32_t gnode = act ? rconn[R::conn(s, c)] : 0;
        const int64_t ntile = tile + vg;
        const int nst = (it + 1) % NSTAGE;
        Gathered nxt{make_double2(0.0, 0.0), 0.0, make_double2(0.0, 0.0)};
        auto prefetch = [&]() {
            if (ntile < a.ntiles) {
                mbar_wait(&bar[nst], (uint32_t)(((it + 1) / NSTAGE) & 1));
                nxt = gather_load<E, MODE>(smem + nst * S::STAGE, a.U, a.surface, have_s, a.X);
            }
            // NSTAGE >= 3: refill the previous tile's stage here, half a tile after
            // its J bulk store was issued (its SMEM read has long completed)
            if (NSTAGE >= 3 && l == 0 && it >= 1) {
                const int ps = (it - 1) % NSTAGE;
                const int64_t rt = tile + (int64_t)(NSTAGE - 1) * vg;
                if (JAC) bulk_wait_read0();
                if (rt < a.ntiles) {
                    mbar_arrive_expect_tx(&bar[ps], R::BYTES);
                    bulk_g2s(smem + ps * S::STAGE, a.recs + rt * (int64_t)R::BYTES, R::BYTES, &bar[ps], pol_stream);
                }
            }
        };
        double R0 = 0.0, R1 = 0.0, dR0 = 0.0, dR1 = 0.0;
        double Jb[N / 2 + 1][2][2];
        uint64_t srow = 0;
        longlong2 rp = make_longlong2(0, 0);
        if (CSR) csr_row_load(a, cell0 + c, gnode, act && c < nvalid, srow, rp, N, s);
        if constexpr (S::PSUM) {
            // partial sums over the GradBF region of this stage (its reads are done: __syncwarp above)
            double2 *P = reinterpret_cast<double2 *>(stage + R::G_OFF);
            // J.v without a residual output (the Newton-Krylov operator apply): skip the residual's exchange
            const bool resid_out = !JVP || a.R != nullptr || a.R_cell != nullptr;
            if (resid_out) {
                if (act) {
                    const double w = qv[5];
                    const double s00 = w * qv[0], s01 = w * qv[1], s02 = w * qv[2], s11 = w * qv[3], s12 = w * qv[4];
#pragma unroll
                    for (int n = 0; n < N; ++n) {
                        const double g0 = gq[n][0], g1 = gq[n][1], g2 = gq[n][2];
                        P[psum_idx<E>(c, n, s)] =
                            make_double2(fma(qv[7], bq[n], fma(g2, s02, fma(g1, s01, g0 * s00))),
                                         fma(qv[8], bq[n], fma(g2, s12, fma(g1, s11, g0 * s01))));
                    }
                }
                __syncwarp();
                prefetch();
                if (act) {
#pragma unroll
                    for (int k = 0; k < Q; ++k) {
                        const double2 v = P[psum_idx<E>(c, s, (k + s) % Q)];
                        R0 += v.x;
                        R1 += v.y;
                    }
                }
            } else {
                prefetch();
            }
            if (JVP) {
                __syncwarp();
                if (act) {
                    // d sigma_a = wmu2 d beta_a + gamma tau beta_a
                    const double w = qv[5], gt = qv[14];
                    const double d00 = fma(w, qv[9], gt * qv[0]), d01 = fma(w, qv[10], gt * qv[1]);
                    const double d02 = fma(w, qv[11], gt * qv[2]), d11 = fma(w, qv[12], gt * qv[3]);
                    const double d12 = fma(w, qv[13], gt * qv[4]);
#pragma unroll
                    for (int n = 0; n < N; ++n) {
                        const double g0 = gq[n][0], g1 = gq[n][1], g2 = gq[n][2];
                        P[psum_idx<E>(c, n, s)] = make_double2(fma(g2, d02, fma(g1, d01, g0 * d00)),
                                                               fma(g2, d12, fma(g1, d11, g0 * d01)));
                    }
                }
                __syncwarp();
                if (act) {
#pragma unroll
                    for (int k = 0; k < Q; ++k) {
                        const double2 v = P[psum_idx<E>(c, s, (k + s) % Q)];
                        dR0 += v.x;
                        dR1 += v.y;
                    }
                }
            }
        } else {
            if (act) node_accumulate<E, MODE>(rg, qs, c, s, bfi, R0, R1, Jb, dR0, dR1, prefetch);
            else prefetch();
            if (forms_jac<MODE>()) ksplit_exchange<E>(Jb, c, s, act);
        }
        __syncwarp();  // every lane is done with this stage's record and qs

        if (CSR) csr_scatter<E>(a.csr_vals, c, s, act && c < nvalid, srow, rp, Jb);
        if (JAC) {
            if (act) stage_J<E>(reinterpret_cast<double *>(stage), c, s, Jb);
            fence_proxy_async_smem();
            __syncwarp();
            if (l == 0) {
                store_J<E>(a.J_cell, cell0, nvalid, stage, pol_stream, a.use_jmap ? &jmap : nullptr);
                if (NSTAGE < 3) bulk_wait_read0();  // staging read -> the buffer may take the next record
            }
        }
        if (l == 0 && NSTAGE < 3) {
            const int64_t nt = tile + (int64_t)NSTAGE * vg;
            if (nt < a.ntiles) {
                mbar_arrive_expect_tx(&bar[st], R::BYTES);
                bulk_g2s(stage, a.recs + nt * (int64_t)R::BYTES, R::BYTES, &bar[st], pol_stream);
            }
        }
        if (act && c < nvalid) {
            if (a.R) scatter_node(a.rem, a.remtab, a.R, a.peers, gnode, R0, R1);
            if (a.R_cell) *reinterpret_cast<double2 *>(a.R_cell + ((cell0 + c) * N + s) * 2) = make_double2(R0, R1);
            if (JVP || MODE == M_DIAG) scatter_node(a.rem, a.remtab, a.Y, a.peers_y, gnode, dR0, dR1);
        }
        if (ntile < a.ntiles) gather_store<E, MODE>(smem + nst * S::STAGE, nxt);
    }
    if (JAC && l == 0) bulk_wait0();
}

// ---- G4 on the fp64 tensor cores (residual + element Jacobians; hex8 and wedge6) ----
// The per-node phase of a cell is a dense contraction over its QPs (reading Z5):
//   J[(i,a),(j,b)] = sum_q wmu2 G_i^T B_ab G_j + gamma h_(i,a) h_(j,b),  h_(i,a) = G_i . beta_a,
// B_00 = diag(2, 1/2, 1/2), B_11 = diag(1/2, 2, 1/2), B_01 = [[0,1,0],[1/2,0,0],[0,0,0]], B_10 = B_01^T.
// With S_dd = sum_q wmu2 G[d] G[d]^T and Gam_ab = sum_q gamma h_a h_b^T (N x N over node pairs):
//   J_00 = 2 S_00 + (S_11 + S_22) / 2 + Gam_00,  J_11 = 2 S_11 + (S_00 + S_22) / 2 + Gam_11,
//   J_01 = sum_q wmu2 (G[1] G[0]^T / 2 + G[0] G[1]^T) + Gam_01,  J_10 = J_01^T.
// Each N x N product over Q QPs is two m8n8k4 DMMAs (k = 4 QPs); both operands of every DMMA are the
// lane's own values in the layout lane l <-> (node i = l >> 2, qp q = (l & 3) + 4 kc), so a cell is 16
// DMMAs + ~50 vector FP64 ops per lane (the vector form: ~160 FP64 instructions per lane and cell).
// wedge6 pads the 6 x 6 node blocks to 8 x 8 and its 6 QPs to 8 (zero operands: lanes i >= 6, and
// q >= 6 in the second k step), the same 16 DMMAs per cell.
// The C fragments hold J rows (2i, 2i+1), columns 4 (l & 3) .. +3 after one transposing shuffle of J_01:
// two 256-bit stores per lane and cell straight to J_cell (no staging, no shared-memory round trip;
// J_cell 32-B aligned, else the vector kernels run).
// The per-QP phase (lane <-> (cell, qp)) and the record ring are the stored kernel's.
#ifndef SFO_MMA_SPLIT
#define SFO_MMA_SPLIT 1
#endif
// cells of a tile unrolled in the DMMA node phase: stored kernel 1 (2: -7% same box, it is at its HBM bound
// and the extra registers cost), compact kernel 2 (+3%, latency-bound; profiles/r2_samebox_mma_unroll.txt)
#ifndef SFO_MMA_UNROLL_STORED
#define SFO_MMA_UNROLL_STORED 1
#endif
#ifndef SFO_MMA_UNROLL_COMPACT
#define SFO_MMA_UNROLL_COMPACT 2
#endif
__device__ __forceinline__ void dmma884(double (&d)[2], double a, double b) {
    asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
        : "+d"(d[0]), "+d"(d[1])
        : "d"(a), "d"(b));
}
__device__ __forceinline__ void st_v4_hint(double *p, double x, double y, double z, double w, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.v4.f64 [%0], {%1, %2, %3, %4}, %5;" ::"l"(p), "d"(x), "d"(y), "d"(z),
                 "d"(w), "l"(pol)
                 : "memory");
}
// per-QP scalars of the DMMA kernels: [NQS][TC][8] with the QP pair (q, q + 4) adjacent (one LDS.128 per
// field gives a lane both of its QPs); wedge6's slots of q = 6, 7 are never written (the readers zero them)
template <class E>
struct QsMma {
    double *p;
    __device__ __forceinline__ static int idx(int f, int c, int q) { return (f * E::TC + c) * 8 + 2 * (q & 3) + (q >> 2); }
    __device__ __forceinline__ double &operator()(int f, int c, int q) const { return p[idx(f, c, q)]; }
    __device__ __forceinline__ double2 pair(int f, int c, int qq) const {
        return *reinterpret_cast<const double2 *>(p + idx(f, c, qq));
    }
};
template <class E>
constexpr int qs_mma_bytes() {
    return NQS * E::TC * 8 * 8;
}

// phi_ni at the lane's two DMMA QPs (qq, qq + 4): the body-force rows (0 on padding lanes / QPs)
template <class E>
__device__ __forceinline__ void mma_phi(int ni, int qq, double (&phi)[2]) {
    double x, y, z, w, dx, dy, dz;
#pragma unroll
    for (int kc = 0; kc < 2; ++kc) {
        const int q = qq + 4 * kc;
        phi[kc] = 0.0;
        if (ni < E::N && q < E::Q) {
            qp_coords<E>(q, x, y, z, w);
            basis<E>(ni, x, y, z, phi[kc], dx, dy, dz);
        }
    }
}

// The DMMA per-node phase of one tile: GradBF rg in the record slot layout (Rec<E>::g), per-QP scalars in
// the QsMma layout; lane (ni, qq) returns the residual rows of (cell qq, node ni) in Rm[0] (and, wedge6's
// fifth cell, of (cell 4, node ni) in Rm[1] on the lanes qq == 0) and writes the element Jacobians of the
// tile's valid cells straight to J_cell.  pf() is called once, before cell TC / 2.
template <class E, int UNROLL, class PF>
__device__ __forceinline__ void mma_node_phase(double *__restrict__ J_cell, const double *rg, const QsMma<E> &qs,
                                               const double (&phi)[2], int64_t cell0, int nvalid, int ni, int qq,
                                               uint64_t pol, double (&Rm)[2][2], bool packed, PF pf) {
    constexpr int N = E::N, Q = E::Q, TC = E::TC;
    static_assert(N <= 8 && Q <= 8 && Q > 4 && TC <= 5, "two k steps of 4 QPs, 8 x 8 node blocks");
    const bool node_ok = N == 8 || ni < N;
#pragma unroll(UNROLL)
    for (int cc = 0; cc < TC; ++cc) {
        if (cc == TC / 2) pf();
        double S00[2] = {0, 0}, S11[2] = {0, 0}, S22[2] = {0, 0}, X01[2] = {0, 0}, G00[2] = {0, 0},
               G11[2] = {0, 0};
        // J_01's three products in independent accumulators (dependent DMMA chains of 2, not 6; SFO_MMA_SPLIT)
        double Xb[2] = {0, 0}, Xc[2] = {0, 0};
        double r0 = 0.0, r1 = 0.0;
        const double2 b00 = qs.pair(0, cc, qq), b01 = qs.pair(1, cc, qq), b02 = qs.pair(2, cc, qq);
        const double2 b11 = qs.pair(3, cc, qq), b12 = qs.pair(4, cc, qq), wv = qs.pair(5, cc, qq);
        const double2 gv = qs.pair(6, cc, qq), f0 = qs.pair(7, cc, qq), f1 = qs.pair(8, cc, qq);
#pragma unroll
        for (int kc = 0; kc < 2; ++kc) {
            const int q = qq + 4 * kc;
            const bool q_ok = Q == 8 || q < Q;  // wedge6: QPs 6, 7 of the second k step are padding
            const bool ok = node_ok && q_ok;
            const double g0 = ok ? rg[gidx<E>(ni, q, 0, cc)] : 0.0;
            const double g1 = ok ? rg[gidx<E>(ni, q, 1, cc)] : 0.0;
            const double g2 = ok ? rg[gidx<E>(ni, q, 2, cc)] : 0.0;
            const double B00 = kc ? b00.y : b00.x, B01 = kc ? b01.y : b01.x, B02 = kc ? b02.y : b02.x;
            const double B11 = kc ? b11.y : b11.x, B12 = kc ? b12.y : b12.x;
            const double w = q_ok ? (kc ? wv.y : wv.x) : 0.0, gam = q_ok ? (kc ? gv.y : gv.x) : 0.0;
            const double wf0 = q_ok ? (kc ? f0.y : f0.x) : 0.0, wf1 = q_ok ? (kc ? f1.y : f1.x) : 0.0;
            const double h0 = q_ok ? fma(g2, B02, fma(g1, B01, g0 * B00)) : 0.0;
            const double h1 = q_ok ? fma(g2, B12, fma(g1, B11, g0 * B01)) : 0.0;
            r0 = fma(wf0, phi[kc], fma(w, h0, r0));
            r1 = fma(wf1, phi[kc], fma(w, h1, r1));
            const double wg0 = w * g0, wg1 = w * g1;
            dmma884(S00, g0, wg0);
            dmma884(S11, g1, wg1);
            dmma884(S22, g2, w * g2);
            dmma884(X01, g1, 0.5 * wg0);
            dmma884(SFO_MMA_SPLIT ? Xb : X01, g0, wg1);
            const double gh1 = gam * h1;
            dmma884(G00, h0, gam * h0);
            dmma884(G11, h1, gh1);
            dmma884(SFO_MMA_SPLIT ? Xc : X01, h0, gh1);
        }
        if (SFO_MMA_SPLIT) {
            X01[0] += Xb[0] + Xc[0];
            X01[1] += Xb[1] + Xc[1];
        }
        // residual rows of (cc, ni): sum over the 4 lanes of the node's QP quads
        r0 += __shfl_xor_sync(0xffffffffu, r0, 1);
        r1 += __shfl_xor_sync(0xffffffffu, r1, 1);
        r0 += __shfl_xor_sync(0xffffffffu, r0, 2);
        r1 += __shfl_xor_sync(0xffffffffu, r1, 2);
        if (qq == cc) {
            Rm[0][0] = r0;
            Rm[0][1] = r1;
        }
        if (TC > 4 && cc == 4 && qq == 0) {
            Rm[1][0] = r0;
            Rm[1][1] = r1;
        }
        // J_10[ni][2qq + e] = J_01[2qq + e][ni]: lane (2qq + e, ni >> 1), element ni & 1
        const int src0 = 8 * qq + (ni >> 1), src1 = src0 + 4;
        const double t00 = __shfl_sync(0xffffffffu, X01[0], src0), t01 = __shfl_sync(0xffffffffu, X01[1], src0);
        const double t10 = __shfl_sync(0xffffffffu, X01[0], src1), t11 = __shfl_sync(0xffffffffu, X01[1], src1);
        const double j10a = (ni & 1) ? t01 : t00, j10b = (ni & 1) ? t11 : t10;
        if (cc < nvalid && node_ok && (N == 8 || 2 * qq < N)) {
            double *Jr = J_cell + (cell0 + cc) * (4 * N * N) + (2 * ni) * (2 * N) + 4 * qq;
            const double j00a = fma(2.0, S00[0], fma(0.5, S11[0] + S22[0], G00[0]));
            const double j00b = fma(2.0, S00[1], fma(0.5, S11[1] + S22[1], G00[1]));
            const double j11a = fma(2.0, S11[0], fma(0.5, S00[0] + S22[0], G11[0]));
            const double j11b = fma(2.0, S11[1], fma(0.5, S00[1] + S22[1], G11[1]));
            if (!packed) {
                st_v4_hint(Jr, j00a, X01[0], j00b, X01[1], pol);
                st_v4_hint(Jr + 2 * N, j10a, j11a, j10b, j11b, pol);
            } else {  // the lane's blocks (ni, 2qq), (ni, 2qq + 1) that lie in the upper block triangle
                double *Jb = J_cell + (cell0 + cc) * (4 * pk_blocks<N>());
                const int j0 = 2 * qq, j1 = j0 + 1;
                if (j0 >= ni) st_v4_hint(Jb + 4 * pk_block<N>(ni, j0), j00a, X01[0], j10a, j11a, pol);
                if (j1 >= ni) st_v4_hint(Jb + 4 * pk_block<N>(ni, j1), j00b, X01[1], j10b, j11b, pol);
            }
        }
    }
}

// residual scatter of a DMMA tile: lane (ni, qq) owns (cell qq, node ni) and, wedge6, (cell 4, node ni)
template <class E>
__device__ __forceinline__ void mma_scatter_r(const EvalArgs &a, const int32_t (&gnode)[2], const double (&Rm)[2][2],
                                              int64_t cell0, int nvalid, int ni, int qq) {
    constexpr int N = E::N;
    if (ni >= N) return;
#pragma unroll
    for (int k = 0; k < (E::TC > 4 ? 2 : 1); ++k) {
        const int cc = k ? 4 : qq;
        if ((k == 0 || qq == 0) && cc < nvalid) {
            if (a.R) scatter_node(a.rem, a.remtab, a.R, a.peers, gnode[k], Rm[k][0], Rm[k][1]);
            if (a.R_cell)
                *reinterpret_cast<double2 *>(a.R_cell + ((cell0 + cc) * N + ni) * 2) = make_double2(Rm[k][0], Rm[k][1]);
        }
    }
}
// node ids the lane scatters to (read from the tile's record before its stage is refilled)
template <class E, class RR>
__device__ __forceinline__ void mma_gnodes(const int32_t *rconn, int ni, int qq, int32_t (&gnode)[2]) {
    const int n = ni < E::N ? ni : 0;
    gnode[0] = rconn[RR::conn(n, qq < E::TC ? qq : 0)];
    gnode[1] = E::TC > 4 ? rconn[RR::conn(n, 4 < E::TC ? 4 : 0)] : 0;
}

#ifndef SFO_MMA_JAC_WARPS
#define SFO_MMA_JAC_WARPS 12
#endif
template <class E, int NSTAGE>
struct MmaSmem {
    static constexpr int REC = Rec<E>::BYTES;
    static constexpr int U_OFF = (int)round_up(REC, 16);
    static constexpr int S_OFF = U_OFF + E::TC * E::UPITCH * 16;
    static constexpr int STAGE = (int)round_up(S_OFF + E::TC * E::UPITCH * 8, 128);
    static constexpr int OFF_QS = NSTAGE * STAGE;
    static constexpr int OFF_BAR = OFF_QS + qs_mma_bytes<E>();
    static constexpr int BYTES = OFF_BAR + NSTAGE * 8;
    static_assert(U_OFF == EvalSmem<E, M_JAC, NSTAGE>::U_OFF && S_OFF == EvalSmem<E, M_JAC, NSTAGE>::S_OFF,
                  "gather_store / gather_load share the stored kernel's stage layout");
};

template <class E, int NSTAGE>
__global__ void __launch_bounds__(32, SFO_MMA_JAC_WARPS) eval_mma_kernel(EvalArgs a) {
    constexpr int N = E::N, TC = E::TC;
    using R = Rec<E>;
    using S = MmaSmem<E, NSTAGE>;
    extern __shared__ __align__(128) char smem[];
    const int64_t vb = blockIdx.x, vg = gridDim.x;
    const QsMma<E> qs{reinterpret_cast<double *>(smem + S::OFF_QS)};
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem + S::OFF_BAR);
    const int l = threadIdx.x & 31;
    const bool act = l < TC * N;
    const int c = act ? E::lane_cell(l) : 0, s = act ? E::lane_sub(l) : 0;  // per-QP phase: (cell, qp)
    const int ni = l >> 2, qq = l & 3;                                      // DMMA fragments: (node, qp quad)
    const bool have_s = (a.surface != nullptr) && (a.force_qp == nullptr);

    const uint64_t pol_stream = policy_evict_first();
    if (l == 0) {
        for (int k = 0; k < NSTAGE; ++k) mbar_init(&bar[k], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int k = 0; k < NSTAGE; ++k) {
            const int64_t tile = vb + (int64_t)k * vg;
            if (tile < a.ntiles) {
                mbar_arrive_expect_tx(&bar[k], R::BYTES);
                bulk_g2s(smem + k * S::STAGE, a.recs + tile * (int64_t)R::BYTES, R::BYTES, &bar[k], pol_stream);
            }
        }
    }
    __syncwarp();
    if (vb < a.ntiles) {
        mbar_wait(&bar[0], 0);
        gather_store<E, M_JAC>(smem, gather_load<E, M_JAC>(smem, a.U, a.surface, have_s, nullptr));
    }
    double phi[2];
    mma_phi<E>(ni, qq, phi);

    int it = 0;
    for (int64_t tile = vb; tile < a.ntiles; tile += vg, ++it) {
        const int st = it % NSTAGE;
        char *stage = smem + st * S::STAGE;
        const int32_t *rconn = reinterpret_cast<const int32_t *>(stage + R::CONN_OFF);
        const double *rkc = reinterpret_cast<const double *>(stage + R::KC_OFF);
        const double *rwm = reinterpret_cast<const double *>(stage + R::WM_OFF);
        const double *rg = reinterpret_cast<const double *>(stage + R::G_OFF);
        const double2 *Us = reinterpret_cast<const double2 *>(stage + S::U_OFF);
        const double *ss = reinterpret_cast<const double *>(stage + S::S_OFF);
        const int64_t cell0 = tile * TC;
        const int nvalid = (a.ncells - cell0 < (int64_t)TC) ? (int)(a.ncells - cell0) : TC;

        __syncwarp();  // this tile's gathered U, s are visible

        // ---- per-QP phase: lane <-> (cell c, qp s), as in eval_kernel ----
        if (act) {
            const int q = s;
            double ux = 0, uy = 0, uz = 0, vx = 0, vy = 0, vz = 0, gs0 = 0, gs1 = 0;
#pragma unroll
            for (int n = 0; n < N; ++n) {
                const double g0 = rg[gidx<E>(n, q, 0, c)];
                const double g1 = rg[gidx<E>(n, q, 1, c)];
                const double g2 = rg[gidx<E>(n, q, 2, c)];
                const int e = E::uidx(c, n);
                const double2 uv = Us[e];
                ux = fma(uv.x, g0, ux); uy = fma(uv.x, g1, uy); uz = fma(uv.x, g2, uz);
                vx = fma(uv.y, g0, vx); vy = fma(uv.y, g1, vy); vz = fma(uv.y, g2, vz);
                if (have_s) {
                    const double sn = ss[e];
                    gs0 = fma(sn, g0, gs0); gs1 = fma(sn, g1, gs1);
                }
            }
            qp_tail<E, M_JAC>(a, qs, c, q, nvalid, cell0, have_s, rkc[c], rwm[R::wm(q, c)], ux, uy, uz, vx, vy, vz,
                              gs0, gs1);
        }
        __syncwarp();

        // ---- per-node phase on the tensor cores, one cell at a time ----
        int32_t gnode[2];
        mma_gnodes<E, R>(rconn, ni, qq, gnode);
        const int64_t ntile = tile + vg;
        const int nst = (it + 1) % NSTAGE;
        Gathered nxt{make_double2(0.0, 0.0), 0.0, make_double2(0.0, 0.0)};
        double Rm[2][2] = {{0.0, 0.0}, {0.0, 0.0}};
        mma_node_phase<E, SFO_MMA_UNROLL_STORED>(a.J_cell, rg, qs, phi, cell0, nvalid, ni, qq, pol_stream, Rm, a.packed != 0, [&]() {
            if (ntile < a.ntiles) {  // the next tile's gather, half a tile of latency slack
                mbar_wait(&bar[nst], (uint32_t)(((it + 1) / NSTAGE) & 1));
                nxt = gather_load<E, M_JAC>(smem + nst * S::STAGE, a.U, a.surface, have_s, nullptr);
            }
        });
        __syncwarp();  // every lane is done with this stage's record and per-QP scalars

        if (l == 0) {
            const int64_t nt = tile + (int64_t)NSTAGE * vg;
            if (nt < a.ntiles) {
                mbar_arrive_expect_tx(&bar[st], R::BYTES);
                bulk_g2s(stage, a.recs + nt * (int64_t)R::BYTES, R::BYTES, &bar[st], pol_stream);
            }
        }
        mma_scatter_r<E>(a, gnode, Rm, cell0, nvalid, ni, qq);
        if (ntile < a.ntiles) gather_store<E, M_JAC>(smem + nst * S::STAGE, nxt);
    }
}

// ---- G3/G4 with compact stored geometry (A_q = J_q^-T streamed per tile) ----
// The stored kernel's TMA record ring and register gather, with the compact
// record (RecC): the per-QP phase forms GradBF_n(q) = A_q grad_xi phi_n(xi_q)
// in registers (reference gradients at the lane's QP from its QP coordinates)
// and, for the tangent modes, stores it to a per-warp GradBF region in the
// stored kernel's slot layout, so the per-node phase is unchanged.  680 B/cell
// of geometry instead of 1,640 (hex8): the evaluation moves 26% fewer HBM bytes
// for 9 FMA per (node, QP) more.  Shared memory per warp: 2 record stages +
// GradBF region + per-QP scalars; the element-Jacobian staging overlays the
// GradBF + scalar regions (as in the on-the-fly kernel), so the next record can
// land while the TMA store drains.
template <class E, int MODE>
struct CompactSmem {
    static constexpr int N = E::N, Q = E::Q, TC = E::TC, SLAB = E::SLAB;
    static constexpr int REC = RecC<E>::BYTES;
    static constexpr int U_OFF = (int)round_up(REC, 16);                         // double2 [TC][UPITCH]
    static constexpr int S_OFF = U_OFF + TC * E::UPITCH * 16;                      // double  [TC][UPITCH]
    static constexpr int X_OFF = (int)round_up(S_OFF + TC * E::UPITCH * 8, 16);   // double2 [TC][UPITCH] (M_JVP)
    static constexpr int IN_BYTES = X_OFF + (MODE == M_JVP ? TC * E::UPITCH * 16 : 0);
    static constexpr int STAGE = (int)round_up(IN_BYTES, 128);
    static constexpr bool PSUM = MODE == M_RESID || MODE == M_JVP;
    static constexpr int G_BYTES = Q * 3 * SLAB * 8;                               // GradBF (or partial sums)
    static constexpr int OFF_G = 2 * STAGE;
    static constexpr int OFF_QS = OFF_G + G_BYTES;                                 // double [NQS][TC][Q]
    static constexpr int QS_BYTES = PSUM ? 0 : nqs<MODE>() * TC * Q * 8;
    static constexpr int J_BYTES = MODE == M_JAC ? TC * E::JPITCH * 8 : 0;         // J staging over G + qs
    static constexpr int TAIL = (G_BYTES + QS_BYTES > J_BYTES ? G_BYTES + QS_BYTES : J_BYTES);
    static constexpr int OFF_BAR = (int)round_up(OFF_G + TAIL, 8);
    static constexpr int BYTES = OFF_BAR + 2 * 8;
    static_assert(!PSUM || psum_bytes<E>() <= G_BYTES, "partial sums overlay the GradBF region");
    static_assert(U_OFF % 16 == 0 && X_OFF % 16 == 0 && STAGE % 128 == 0 && OFF_G % 128 == 0 && OFF_QS % 16 == 0,
                  "alignment");
};

template <class E, int MODE>
__device__ __forceinline__ Gathered gather_load_c(const char *stage, const double *U, const double *surface,
                                                  bool have_s, const double *X) {
    using R = RecC<E>;
    Gathered v{make_double2(0.0, 0.0), 0.0, make_double2(0.0, 0.0)};
    const int l = threadIdx.x & 31;
    if (l < E::TC * E::N) {
        const int c = E::lane_cell(l), n = E::lane_sub(l);
        const int32_t g = reinterpret_cast<const int32_t *>(stage + R::CONN_OFF)[R::conn(n, c)];
        v.u = __ldg(reinterpret_cast<const double2 *>(U) + g);
        if (have_s) v.s = __ldg(surface + g);
        if (MODE == M_JVP) v.x = __ldg(reinterpret_cast<const double2 *>(X) + g);
    }
    return v;
}
template <class E, int MODE>
__device__ __forceinline__ void gather_store_c(char *stage, const Gathered &v) {
    using S = CompactSmem<E, MODE>;
    const int l = threadIdx.x & 31;
    if (l < E::TC * E::N) {
        const int e = E::uidx(E::lane_cell(l), E::lane_sub(l));
        reinterpret_cast<double2 *>(stage + S::U_OFF)[e] = v.u;
        reinterpret_cast<double *>(stage + S::S_OFF)[e] = v.s;
        if (MODE == M_JVP) reinterpret_cast<double2 *>(stage + S::X_OFF)[e] = v.x;
    }
}

#ifndef SFO_COMPACT_JAC_WARPS
#define SFO_COMPACT_JAC_WARPS 12
#endif
template <class E, int MODE>
__global__ void __launch_bounds__(32, (forms_jac<MODE>() ? SFO_COMPACT_JAC_WARPS : 16))
    eval_compact_kernel(EvalArgs a, const __grid_constant__ CUtensorMap jmap) {
    constexpr int N = E::N, Q = E::Q, TC = E::TC;
    constexpr bool JAC = MODE == M_JAC, JVP = MODE == M_JVP, CSR = MODE == M_CSR;
    static_assert(N == Q, "lane mappings assume N == Q");
    using R = RecC<E>;
    using S = CompactSmem<E, MODE>;
    extern __shared__ __align__(128) char smem[];
    double *rg = reinterpret_cast<double *>(smem + S::OFF_G);
    const QsView<E, nqs<MODE>()> qs{reinterpret_cast<double *>(smem + S::OFF_QS), nullptr};
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem + S::OFF_BAR);
    const int l = threadIdx.x & 31;
    const bool act = l < TC * N;
    const int c = act ? E::lane_cell(l) : TC, s = act ? E::lane_sub(l) : 0;  // (cell, node-or-qp)
    const bool have_s = (a.surface != nullptr) && (a.force_qp == nullptr);
    const int64_t vb = blockIdx.x, vg = gridDim.x;

    uint64_t pol_stream = 0;
    if (l == 0) {
        pol_stream = policy_evict_first();
        for (int k = 0; k < 2; ++k) mbar_init(&bar[k], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int k = 0; k < 2; ++k) {
            const int64_t tile = vb + (int64_t)k * vg;
            if (tile < a.ntiles) {
                mbar_arrive_expect_tx(&bar[k], R::BYTES);
                bulk_g2s(smem + k * S::STAGE, a.recs + tile * (int64_t)R::BYTES, R::BYTES, &bar[k], pol_stream);
            }
        }
    }
    __syncwarp();
    if (vb < a.ntiles) {
        mbar_wait(&bar[0], 0);
        gather_store_c<E, MODE>(smem, gather_load_c<E, MODE>(smem, a.U, a.surface, have_s, a.X));
    }
    double xq, yq, zq, wq;  // this lane's QP (per-QP phase)
    qp_coords<E>(act ? s : 0, xq, yq, zq, wq);
    double bfi[Q];
    basis_row<E>(act ? s : 0, bfi);
    double bq[N];  // phi_n at this lane's QP, every n (partial-sum modes)
    {
        double dx, dy, dz;
#pragma unroll
        for (int n = 0; n < N; ++n) basis<E>(n, xq, yq, zq, bq[n], dx, dy, dz);
    }

    int it = 0;
    for (int64_t tile = vb; tile < a.ntiles; tile += vg, ++it) {
        const int st = it & 1;
        char *stage = smem + st * S::STAGE;
        const int32_t *rconn = reinterpret_cast<const int32_t *>(stage + R::CONN_OFF);
        const double *rkc = reinterpret_cast<const double *>(stage + R::KC_OFF);
        const double *rwm = reinterpret_cast<const double *>(stage + R::WM_OFF);
        const double *ra = reinterpret_cast<const double *>(stage + R::A_OFF);
        const double2 *Us = reinterpret_cast<const double2 *>(stage + S::U_OFF);
        const double *ss = reinterpret_cast<const double *>(stage + S::S_OFF);
        const double2 *Xs = reinterpret_cast<const double2 *>(stage + S::X_OFF);
        const int64_t cell0 = tile * TC;
        const int nvalid = (a.ncells - cell0 < (int64_t)TC) ? (int)(a.ncells - cell0) : TC;

        if (JAC && l == 0) bulk_wait_read0();  // the previous tile's J staging (over G + qs) has been read
        __syncwarp();                          // + this tile's gathered U, s are visible
        const int32_t gnode = act ? rconn[R::conn(s, c)] : 0;

        // ---- per-QP phase: lane <-> (cell c, qp s); GradBF = A grad_xi phi in registers ----
        double gq[S::PSUM ? N : 1][3];
        double qv[S::PSUM ? 15 : 1];
        if (act) {
            const int q = s;
            double A[9];
#pragma unroll
            for (int k = 0; k < 9; ++k) A[k] = ra[R::a(k, q, c)];
            double ux = 0, uy = 0, uz = 0, vx = 0, vy = 0, vz = 0, gs0 = 0, gs1 = 0;
            double dg[6] = {0, 0, 0, 0, 0, 0};
#pragma unroll
            for (int n = 0; n < N; ++n) {
                double phi, d0, d1, d2;
                basis<E>(n, xq, yq, zq, phi, d0, d1, d2);
                const double g0 = fma(A[0], d0, fma(A[1], d1, A[2] * d2));
                const double g1 = fma(A[3], d0, fma(A[4], d1, A[5] * d2));
                const double g2 = fma(A[6], d0, fma(A[7], d1, A[8] * d2));
                if constexpr (S::PSUM) {
                    gq[n][0] = g0;
                    gq[n][1] = g1;
                    gq[n][2] = g2;
                } else {
                    rg[gidx<E>(n, q, 0, c)] = g0;
                    rg[gidx<E>(n, q, 1, c)] = g1;
                    rg[gidx<E>(n, q, 2, c)] = g2;
                }
                const int e = E::uidx(c, n);
                const double2 uv = Us[e];
                ux = fma(uv.x, g0, ux); uy = fma(uv.x, g1, uy); uz = fma(uv.x, g2, uz);
                vx = fma(uv.y, g0, vx); vy = fma(uv.y, g1, vy); vz = fma(uv.y, g2, vz);
                if (have_s) {
                    const double sn = ss[e];
                    gs0 = fma(sn, g0, gs0); gs1 = fma(sn, g1, gs1);
                }
                if (JVP) {
                    const double2 xv = Xs[e];
                    dg[0] = fma(xv.x, g0, dg[0]); dg[1] = fma(xv.x, g1, dg[1]); dg[2] = fma(xv.x, g2, dg[2]);
                    dg[3] = fma(xv.y, g0, dg[3]); dg[4] = fma(xv.y, g1, dg[4]); dg[5] = fma(xv.y, g2, dg[5]);
                }
            }
            if constexpr (S::PSUM)
                qp_tail<E, MODE>(a, RegQs{qv}, c, q, nvalid, cell0, have_s, rkc[c], rwm[R::wm(q, c)], ux, uy, uz, vx,
                                 vy, vz, gs0, gs1, dg);
            else
                qp_tail<E, MODE>(a, qs, c, q, nvalid, cell0, have_s, rkc[c], rwm[R::wm(q, c)], ux, uy, uz, vx, vy,
                                 vz, gs0, gs1, dg);
        }
        __syncwarp();  // the stage (record, U, s) is consumed: refill it with the record two tiles ahead
        if (l == 0) {
            const int64_t nt = tile + 2 * vg;
            if (nt < a.ntiles) {
                mbar_arrive_expect_tx(&bar[st], R::BYTES);
                bulk_g2s(stage, a.recs + nt * (int64_t)R::BYTES, R::BYTES, &bar[st], pol_stream);
            }
        }

        // ---- per-node phase (+ gather of the next tile at q = Q/2) ----
        const int64_t ntile = tile + vg;
        const int nst = (it + 1) & 1;
        Gathered nxt{make_double2(0.0, 0.0), 0.0, make_double2(0.0, 0.0)};
        auto prefetch = [&]() {
            if (ntile < a.ntiles) {
                mbar_wait(&bar[nst], (uint32_t)(((it + 1) >> 1) & 1));
                nxt = gather_load_c<E, MODE>(smem + nst * S::STAGE, a.U, a.surface, have_s, a.X);
            }
        };
        double R0 = 0.0, R1 = 0.0, dR0 = 0.0, dR1 = 0.0;
        double Jb[N / 2 + 1][2][2];
        uint64_t srow = 0;
        longlong2 rp = make_longlong2(0, 0);
        if (CSR) csr_row_load(a, cell0 + c, gnode, act && c < nvalid, srow, rp, N, s);
        if constexpr (S::PSUM) {
            // partial sums over the (unused) GradBF region
            double2 *P = reinterpret_cast<double2 *>(rg);
            // J.v without a residual output (the Newton-Krylov operator apply): skip the residual's exchange
            const bool resid_out = !JVP || a.R != nullptr || a.R_cell != nullptr;
            if (resid_out) {
                if (act) {
                    const double w = qv[5];
                    const double s00 = w * qv[0], s01 = w * qv[1], s02 = w * qv[2], s11 = w * qv[3], s12 = w * qv[4];
#pragma unroll
                    for (int n = 0; n < N; ++n) {
                        const double g0 = gq[n][0], g1 = gq[n][1], g2 = gq[n][2];
                        P[psum_idx<E>(c, n, s)] =
                            make_double2(fma(qv[7], bq[n], fma(g2, s02, fma(g1, s01, g0 * s00))),
                                         fma(qv[8], bq[n], fma(g2, s12, fma(g1, s11, g0 * s01))));
                    }
                }
                __syncwarp();
                prefetch();
                if (act) {
#pragma unroll
                    for (int k = 0; k < Q; ++k) {
                        const double2 v = P[psum_idx<E>(c, s, (k + s) % Q)];
                        R0 += v.x;
                        R1 += v.y;
                    }
                }
            } else {
                prefetch();
            }
            if (JVP) {
                __syncwarp();
                if (act) {
                    const double w = qv[5], gt = qv[14];
                    const double d00 = fma(w, qv[9], gt * qv[0]), d01 = fma(w, qv[10], gt * qv[1]);
                    const double d02 = fma(w, qv[11], gt * qv[2]), d11 = fma(w, qv[12], gt * qv[3]);
                    const double d12 = fma(w, qv[13], gt * qv[4]);
#pragma unroll
                    for (int n = 0; n < N; ++n) {
                        const double g0 = gq[n][0], g1 = gq[n][1], g2 = gq[n][2];
                        P[psum_idx<E>(c, n, s)] = make_double2(fma(g2, d02, fma(g1, d01, g0 * d00)),
                                                               fma(g2, d12, fma(g1, d11, g0 * d01)));
                    }
                }
                __syncwarp();
                if (act) {
#pragma unroll
                    for (int k = 0; k < Q; ++k) {
                        const double2 v = P[psum_idx<E>(c, s, (k + s) % Q)];
                        dR0 += v.x;
                        dR1 += v.y;
                    }
                }
            }
        } else {
            if (act) node_accumulate<E, MODE>(rg, qs, c, s, bfi, R0, R1, Jb, dR0, dR1, prefetch);
            else prefetch();
            if (forms_jac<MODE>()) ksplit_exchange<E>(Jb, c, s, act);
        }
        __syncwarp();  // every lane is done with G and qs
        if (CSR) csr_scatter<E>(a.csr_vals, c, s, act && c < nvalid, srow, rp, Jb);
        if (JAC) {
            if (act) stage_J<E>(rg, c, s, Jb);
            fence_proxy_async_smem();
            __syncwarp();
            if (l == 0)
                store_J<E>(a.J_cell, cell0, nvalid, reinterpret_cast<const char *>(rg), pol_stream,
                           a.use_jmap ? &jmap : nullptr);
        }
        if (act && c < nvalid) {
            if (a.R) scatter_node(a.rem, a.remtab, a.R, a.peers, gnode, R0, R1);
            if (a.R_cell) *reinterpret_cast<double2 *>(a.R_cell + ((cell0 + c) * N + s) * 2) = make_double2(R0, R1);
            if (JVP || MODE == M_DIAG) scatter_node(a.rem, a.remtab, a.Y, a.peers_y, gnode, dR0, dR1);
        }
        if (ntile < a.ntiles) gather_store_c<E, MODE>(smem + nst * S::STAGE, nxt);
    }
    if (JAC && l == 0) bulk_wait0();
}

// ---- G4 with compact stored geometry on the fp64 tensor cores (hex8, wedge6) ----
// The compact kernel's record ring (A_q = J_q^-T) and register gather, the per-QP phase forming
// GradBF = A_q grad_xi phi into the per-warp GradBF region (record slot layout), and the DMMA per-node phase
// of eval_mma_kernel (mma_node_phase: J written straight from the accumulator fragments, no staging). The
// record stage is refilled right after the per-QP phase (GradBF lives in the per-warp region), so the TMA
// lead is 1.5 tiles. Shared memory per warp: 2 record stages + GradBF + per-QP scalars (hex8 15.6 KB).
template <class E>
struct CompactMmaSmem {
    using C = CompactSmem<E, M_JAC>;
    static constexpr int STAGE = C::STAGE;  // RecC + gathered U, s (gather_store_c's layout)
    static constexpr int OFF_G = 2 * STAGE;
    static constexpr int OFF_QS = OFF_G + E::Q * 3 * E::SLAB * 8;
    static constexpr int OFF_BAR = OFF_QS + qs_mma_bytes<E>();
    static constexpr int BYTES = OFF_BAR + 2 * 8;
    static_assert(OFF_G % 128 == 0 && OFF_QS % 16 == 0, "alignment");
};

template <class E>
__global__ void __launch_bounds__(32, SFO_MMA_JAC_WARPS) eval_compact_mma_kernel(EvalArgs a) {
    constexpr int N = E::N, TC = E::TC;
    using R = RecC<E>;
    using S = CompactMmaSmem<E>;
    extern __shared__ __align__(128) char smem[];
    double *rg = reinterpret_cast<double *>(smem + S::OFF_G);
    const QsMma<E> qs{reinterpret_cast<double *>(smem + S::OFF_QS)};
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem + S::OFF_BAR);
    const int64_t vb = blockIdx.x, vg = gridDim.x;
    const int l = threadIdx.x & 31;
    const bool act = l < TC * N;
    const int c = act ? E::lane_cell(l) : 0, s = act ? E::lane_sub(l) : 0;  // per-QP phase: (cell, qp)
    const int ni = l >> 2, qq = l & 3;                                      // DMMA fragments: (node, qp quad)
    const bool have_s = (a.surface != nullptr) && (a.force_qp == nullptr);

    const uint64_t pol_stream = policy_evict_first();
    if (l == 0) {
        for (int k = 0; k < 2; ++k) mbar_init(&bar[k], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int k = 0; k < 2; ++k) {
            const int64_t tile = vb + (int64_t)k * vg;
            if (tile < a.ntiles) {
                mbar_arrive_expect_tx(&bar[k], R::BYTES);
                bulk_g2s(smem + k * S::STAGE, a.recs + tile * (int64_t)R::BYTES, R::BYTES, &bar[k], pol_stream);
            }
        }
    }
    __syncwarp();
    if (vb < a.ntiles) {
        mbar_wait(&bar[0], 0);
        gather_store_c<E, M_JAC>(smem, gather_load_c<E, M_JAC>(smem, a.U, a.surface, have_s, nullptr));
    }
    double xq, yq, zq, wq;  // this lane's QP (per-QP phase)
    qp_coords<E>(s, xq, yq, zq, wq);
    double phi[2];
    mma_phi<E>(ni, qq, phi);

    int it = 0;
    for (int64_t tile = vb; tile < a.ntiles; tile += vg, ++it) {
        const int st = it & 1;
        char *stage = smem + st * S::STAGE;
        const int32_t *rconn = reinterpret_cast<const int32_t *>(stage + R::CONN_OFF);
        const double *rkc = reinterpret_cast<const double *>(stage + R::KC_OFF);
        const double *rwm = reinterpret_cast<const double *>(stage + R::WM_OFF);
        const double *ra = reinterpret_cast<const double *>(stage + R::A_OFF);
        const double2 *Us = reinterpret_cast<const double2 *>(stage + S::C::U_OFF);
        const double *ss = reinterpret_cast<const double *>(stage + S::C::S_OFF);
        const int64_t cell0 = tile * TC;
        const int nvalid = (a.ncells - cell0 < (int64_t)TC) ? (int)(a.ncells - cell0) : TC;

        __syncwarp();  // this tile's gathered U, s are visible; the previous node phase is done with G and qs
        int32_t gnode[2];
        mma_gnodes<E, R>(rconn, ni, qq, gnode);

        // ---- per-QP phase: lane <-> (cell c, qp s); GradBF = A grad_xi phi in registers -> G region ----
        if (act) {
            const int q = s;
            double A[9];
#pragma unroll
            for (int k = 0; k < 9; ++k) A[k] = ra[R::a(k, q, c)];
            double ux = 0, uy = 0, uz = 0, vx = 0, vy = 0, vz = 0, gs0 = 0, gs1 = 0;
#pragma unroll
            for (int n = 0; n < N; ++n) {
                double ph, d0, d1, d2;
                basis<E>(n, xq, yq, zq, ph, d0, d1, d2);
                const double g0 = fma(A[0], d0, fma(A[1], d1, A[2] * d2));
                const double g1 = fma(A[3], d0, fma(A[4], d1, A[5] * d2));
                const double g2 = fma(A[6], d0, fma(A[7], d1, A[8] * d2));
                rg[gidx<E>(n, q, 0, c)] = g0;
                rg[gidx<E>(n, q, 1, c)] = g1;
                rg[gidx<E>(n, q, 2, c)] = g2;
                const int e = E::uidx(c, n);
                const double2 uv = Us[e];
                ux = fma(uv.x, g0, ux); uy = fma(uv.x, g1, uy); uz = fma(uv.x, g2, uz);
                vx = fma(uv.y, g0, vx); vy = fma(uv.y, g1, vy); vz = fma(uv.y, g2, vz);
                if (have_s) {
                    const double sn = ss[e];
                    gs0 = fma(sn, g0, gs0); gs1 = fma(sn, g1, gs1);
                }
            }
            qp_tail<E, M_JAC>(a, qs, c, q, nvalid, cell0, have_s, rkc[c], rwm[R::wm(q, c)], ux, uy, uz, vx, vy, vz,
                              gs0, gs1);
        }
        __syncwarp();  // the stage (record, U, s) is consumed: refill it with the record two tiles ahead
        if (l == 0) {
            const int64_t nt = tile + 2 * vg;
            if (nt < a.ntiles) {
                mbar_arrive_expect_tx(&bar[st], R::BYTES);
                bulk_g2s(stage, a.recs + nt * (int64_t)R::BYTES, R::BYTES, &bar[st], pol_stream);
            }
        }

        // ---- per-node phase on the tensor cores (+ gather of the next tile before cell TC / 2) ----
        const int64_t ntile = tile + vg;
        const int nst = (it + 1) & 1;
        Gathered nxt{make_double2(0.0, 0.0), 0.0, make_double2(0.0, 0.0)};
        double Rm[2][2] = {{0.0, 0.0}, {0.0, 0.0}};
        mma_node_phase<E, SFO_MMA_UNROLL_COMPACT>(a.J_cell, rg, qs, phi, cell0, nvalid, ni, qq, pol_stream, Rm, a.packed != 0, [&]() {
            if (ntile < a.ntiles) {
                mbar_wait(&bar[nst], (uint32_t)(((it + 1) >> 1) & 1));
                nxt = gather_load_c<E, M_JAC>(smem + nst * S::STAGE, a.U, a.surface, have_s, nullptr);
            }
        });
        mma_scatter_r<E>(a, gnode, Rm, cell0, nvalid, ni, qq);
        if (ntile < a.ntiles) gather_store_c<E, M_JAC>(smem + nst * S::STAGE, nxt);
    }
}

// ---- G3/G4 with on-the-fly geometry ------------------------------------------
// Same evaluation; GradBF and wM are recomputed per tile from the gathered
// node coordinates (cell-local, reading Z17) instead of being streamed: 40
// streamed B/cell instead of 1,640 (hex8).  conn and k_c are read straight
// from the caller's arrays two tiles ahead; U, s and the node coordinates are
// gathered into registers one tile ahead (at the middle of the previous tile's
// node phase) and stored to shared memory after it, already cell-local
// (x_n - x_0 with x_0 from the cell's node-0 lane by shuffle): one conflict-free
// shared store per value instead of a cp.async gather, which costs one
// shared-memory wavefront per lane (ncu r2 p1: 32 per LDGSTS.128 vs 4 ideal).
// The reference gradients at the lane's QP are evaluated in registers from
// its QP coordinates (no shared table).

template <class E, int MODE>
struct OtfSmem {
    static constexpr int N = E::N, Q = E::Q, TC = E::TC, SLAB = E::SLAB;
    // gathered-input cell pitch: hex8 9 (the 4 cells' broadcast 16-B reads fall in distinct banks)
    static constexpr int UP = E::N == 8 ? 9 : E::UPITCH;
    static constexpr int IN_U = 0;                        // double2 [TC][UP]  U
    static constexpr int IN_XY = TC * UP * 16;            // double2 [TC][UP]  cell-local (x, y)
    static constexpr int IN_Z = 2 * TC * UP * 16;         // double  [TC][UP]  cell-local z
    static constexpr int IN_S = IN_Z + TC * UP * 8;       // double  [TC][UP]  s
    static constexpr int IN_X = (int)round_up(IN_S + TC * UP * 8, 16);  // double2 [TC][UP] X (M_JVP)
    static constexpr int IN_BYTES = (int)round_up(IN_X + (MODE == M_JVP ? TC * UP * 16 : 0), 128);
    static constexpr int OFF_G = 2 * IN_BYTES;                               // GradBF [Q][3][SLAB]
    static constexpr int OFF_QS = OFF_G + Q * 3 * SLAB * 8;                  // double [NQS][TC][Q]
    static constexpr int J_BYTES = MODE == M_JAC ? TC * E::JPITCH * 8 : 0;   // J staging overlays G + qs
    static_assert(J_BYTES <= OFF_QS + nqs<MODE>() * TC * Q * 8 - OFF_G, "J staging must fit over G + qs");
    static constexpr int BYTES = OFF_QS + nqs<MODE>() * TC * Q * 8;
    static_assert(IN_XY % 16 == 0 && IN_X % 16 == 0 && IN_BYTES % 128 == 0 && OFF_G % 128 == 0 && OFF_QS % 16 == 0,
                  "alignment");
};

struct OtfGathered {
    double2 u, xy, x;
    double z, s;
};

// lane (cell, node) loads its node's inputs into registers (zeros for dead lanes)
template <int MODE>
__device__ __forceinline__ OtfGathered otf_load(int32_t g, bool live, const double *U, const double4 *xyz4,
                                                const double *surface, bool have_s, const double *X) {
    OtfGathered v{make_double2(0.0, 0.0), make_double2(0.0, 0.0), make_double2(0.0, 0.0), 0.0, 0.0};
    if (live) {
        v.u = __ldg(reinterpret_cast<const double2 *>(U) + g);
        const double *p = reinterpret_cast<const double *>(xyz4 + g);
        v.xy = __ldg(reinterpret_cast<const double2 *>(p));
        v.z = __ldg(p + 2);
        if (have_s) v.s = __ldg(surface + g);
        if (MODE == M_JVP) v.x = __ldg(reinterpret_cast<const double2 *>(X) + g);
    }
    return v;
}

// store one tile's gathered inputs, coordinates made cell-local (reading Z17);
// every lane of the warp must call this (shuffles)
template <class E, int MODE>
__device__ __forceinline__ void otf_store(char *in, const OtfGathered &v, int c, int n, bool act) {
    using S = OtfSmem<E, MODE>;
    const int src = act ? E::lane_of(c, 0) : (int)(threadIdx.x & 31);
    const double x0 = __shfl_sync(0xffffffffu, v.xy.x, src);
    const double y0 = __shfl_sync(0xffffffffu, v.xy.y, src);
    const double z0 = __shfl_sync(0xffffffffu, v.z, src);
    if (act) {
        const int e = c * S::UP + n;
        reinterpret_cast<double2 *>(in + S::IN_U)[e] = v.u;
        reinterpret_cast<double2 *>(in + S::IN_XY)[e] = make_double2(v.xy.x - x0, v.xy.y - y0);
        reinterpret_cast<double *>(in + S::IN_Z)[e] = v.z - z0;
        reinterpret_cast<double *>(in + S::IN_S)[e] = v.s;
        if (MODE == M_JVP) reinterpret_cast<double2 *>(in + S::IN_X)[e] = v.x;
    }
}

// resident one-warp CTAs per SM the on-the-fly kernels' register budget is sized for
#ifndef SFO_OTF_JAC_WARPS
#define SFO_OTF_JAC_WARPS 12
#endif
template <class E, int MODE>
__global__ void __launch_bounds__(32, (forms_jac<MODE>() ? SFO_OTF_JAC_WARPS : 16)) eval_otf_kernel(EvalArgs a) {
    constexpr int N = E::N, Q = E::Q, TC = E::TC;
    static_assert(N == Q, "lane mappings assume N == Q");
    constexpr bool JAC = MODE == M_JAC, JVP = MODE == M_JVP, CSR = MODE == M_CSR;
    using S = OtfSmem<E, MODE>;
    extern __shared__ __align__(128) char smem[];
    double *rg = reinterpret_cast<double *>(smem + S::OFF_G);
    const QsView<E, nqs<MODE>()> qs{reinterpret_cast<double *>(smem + S::OFF_QS), nullptr};
    const int l = threadIdx.x;
    const bool act = l < TC * N;
    const int c = act ? E::lane_cell(l) : TC, s = act ? E::lane_sub(l) : 0;
    const bool have_s = (a.surface != nullptr) && (a.force_qp == nullptr);
    uint64_t pol_stream = 0;
    if (l == 0) pol_stream = policy_evict_first();

    // this lane's QP (per-QP phase) and phi_i at every QP (node phase)
    double xq, yq, zq, wq;
    qp_coords<E>(act ? s : 0, xq, yq, zq, wq);
    double bfi[Q];
    basis_row<E>(act ? s : 0, bfi);

    // conn / k_c of a tile, one lane per (cell, node); cells past the end -> node 0
    auto load_tile = [&](int64_t tile, int32_t &g, double &kcv, bool &live) {
        const int64_t cell = tile * TC + c;
        live = act && tile < a.ntiles && cell < a.ncells;
        g = live ? __ldg(a.conn + cell * N + s) : 0;
        kcv = live ? (a.kc ? __ldg(a.kc + cell) : a.kscal) : 0.0;
    };
    int32_t g_cur, g_nxt;
    double kc_cur, kc_nxt;
    bool live_cur, live_nxt;
    load_tile(blockIdx.x, g_cur, kc_cur, live_cur);
    load_tile(blockIdx.x + (int64_t)gridDim.x, g_nxt, kc_nxt, live_nxt);
    if ((int64_t)blockIdx.x < a.ntiles)
        otf_store<E, MODE>(smem, otf_load<MODE>(g_cur, live_cur, a.U, a.xyz4, a.surface, have_s, a.X), c, s, act);

    int it = 0;
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
        const char *in = smem + (it & 1) * S::IN_BYTES;
        const double2 *Us = reinterpret_cast<const double2 *>(in + S::IN_U);
        const double2 *XY = reinterpret_cast<const double2 *>(in + S::IN_XY);
        const double *Zs = reinterpret_cast<const double *>(in + S::IN_Z);
        const double *ss = reinterpret_cast<const double *>(in + S::IN_S);
        const double2 *Xs = reinterpret_cast<const double2 *>(in + S::IN_X);
        const int64_t cell0 = tile * TC;
        const int nvalid = (a.ncells - cell0 < (int64_t)TC) ? (int)(a.ncells - cell0) : TC;

        if (JAC && l == 0) bulk_wait_read0();  // previous tile's J staging (over G + qs) has been read
        __syncwarp();                          // + this tile's gathered inputs are visible

        // ---- per-QP phase: geometry, GradBF -> smem, then Ugrad etc. ----
        // every lane of cell c loaded its k_c; take it from the cell's node-0 lane
        const double kc = __shfl_sync(0xffffffffu, kc_cur, act ? E::lane_of(c, 0) : 0);
        if (act) {
            const int q = s;
            // reference gradients d phi_n / d xi at this lane's QP, in registers
            double dq[N][3];
#pragma unroll
            for (int n = 0; n < N; ++n) {
                double phi;
                basis<E>(n, xq, yq, zq, phi, dq[n][0], dq[n][1], dq[n][2]);
            }
            double J00 = 0, J01 = 0, J02 = 0, J10 = 0, J11 = 0, J12 = 0, J20 = 0, J21 = 0, J22 = 0;
#pragma unroll
            for (int n = 1; n < N; ++n) {  // cell-local: node 0 sits at the origin
                const double2 xy = XY[c * S::UP + n];
                const double z = Zs[c * S::UP + n];
                const double d0 = dq[n][0], d1 = dq[n][1], d2 = dq[n][2];
                J00 = fma(xy.x, d0, J00); J01 = fma(xy.x, d1, J01); J02 = fma(xy.x, d2, J02);
                J10 = fma(xy.y, d0, J10); J11 = fma(xy.y, d1, J11); J12 = fma(xy.y, d2, J12);
                J20 = fma(z, d0, J20); J21 = fma(z, d1, J21); J22 = fma(z, d2, J22);
            }
            // cofactors: (J^-T)[r][s] = cof[r][s] / det
            const double c00 = J11 * J22 - J12 * J21, c01 = J12 * J20 - J10 * J22, c02 = J10 * J21 - J11 * J20;
            const double c10 = J02 * J21 - J01 * J22, c11 = J00 * J22 - J02 * J20, c12 = J01 * J20 - J00 * J21;
            const double c20 = J01 * J12 - J02 * J11, c21 = J02 * J10 - J00 * J12, c22 = J00 * J11 - J01 * J10;
            const double det = J00 * c00 + J01 * c01 + J02 * c02;
            if (!(det > 0.0) && c < nvalid) atomicOr(a.err, ERR_DETJ);
            const double id = 1.0 / det;
            double ux = 0, uy = 0, uz = 0, vx = 0, vy = 0, vz = 0, gs0 = 0, gs1 = 0;
            double dg[6] = {0, 0, 0, 0, 0, 0};
#pragma unroll
            for (int n = 0; n < N; ++n) {
                const double d0 = dq[n][0], d1 = dq[n][1], d2 = dq[n][2];
                const double g0 = fma(c00, d0, fma(c01, d1, c02 * d2)) * id;
                const double g1 = fma(c10, d0, fma(c11, d1, c12 * d2)) * id;
                const double g2 = fma(c20, d0, fma(c21, d1, c22 * d2)) * id;
                rg[gidx<E>(n, q, 0, c)] = g0;
                rg[gidx<E>(n, q, 1, c)] = g1;
                rg[gidx<E>(n, q, 2, c)] = g2;
                const double2 uv = Us[c * S::UP + n];
                ux = fma(uv.x, g0, ux); uy = fma(uv.x, g1, uy); uz = fma(uv.x, g2, uz);
                vx = fma(uv.y, g0, vx); vy = fma(uv.y, g1, vy); vz = fma(uv.y, g2, vz);
                if (have_s) {
                    const double sn = ss[c * S::UP + n];
                    gs0 = fma(sn, g0, gs0); gs1 = fma(sn, g1, gs1);
                }
                if (JVP) {
                    const double2 xv = Xs[c * S::UP + n];
                    dg[0] = fma(xv.x, g0, dg[0]); dg[1] = fma(xv.x, g1, dg[1]); dg[2] = fma(xv.x, g2, dg[2]);
                    dg[3] = fma(xv.y, g0, dg[3]); dg[4] = fma(xv.y, g1, dg[4]); dg[5] = fma(xv.y, g2, dg[5]);
                }
            }
            qp_tail<E, MODE>(a, qs, c, q, nvalid, cell0, have_s, kc, wq * det, ux, uy, uz, vx, vy, vz, gs0, gs1,
                             dg);
        }
        __syncwarp();

        // ---- per-node phase (+ register gather of the next tile, conn of the one after) ----
        const int32_t gnode = g_cur;
        int32_t g_nn = 0;
        double kc_nn = 0.0;
        bool live_nn = false;
        OtfGathered nxt{make_double2(0.0, 0.0), make_double2(0.0, 0.0), make_double2(0.0, 0.0), 0.0, 0.0};
        auto prefetch = [&]() {
            if (tile + gridDim.x < a.ntiles)
                nxt = otf_load<MODE>(g_nxt, live_nxt, a.U, a.xyz4, a.surface, have_s, a.X);
            load_tile(tile + 2 * (int64_t)gridDim.x, g_nn, kc_nn, live_nn);
        };
        double R0 = 0.0, R1 = 0.0, dR0 = 0.0, dR1 = 0.0;
        double Jb[N / 2 + 1][2][2];
        uint64_t srow = 0;
        longlong2 rp = make_longlong2(0, 0);
        if (CSR) csr_row_load(a, cell0 + c, gnode, act && c < nvalid, srow, rp, N, s);
        if (act) node_accumulate<E, MODE>(rg, qs, c, s, bfi, R0, R1, Jb, dR0, dR1, prefetch);
        else prefetch();
        if (forms_jac<MODE>()) ksplit_exchange<E>(Jb, c, s, act);
        __syncwarp();  // G and qs are consumed
        if (CSR) csr_scatter<E>(a.csr_vals, c, s, act && c < nvalid, srow, rp, Jb);

        if (JAC) {
            if (act) stage_J<E>(rg, c, s, Jb);
            fence_proxy_async_smem();
            __syncwarp();
            if (l == 0) store_J<E>(a.J_cell, cell0, nvalid, reinterpret_cast<const char *>(rg), pol_stream);
        }
        if (act && c < nvalid) {
            if (a.R) scatter_node(a.rem, a.remtab, a.R, a.peers, gnode, R0, R1);
            if (JVP || MODE == M_DIAG) scatter_node(a.rem, a.remtab, a.Y, a.peers_y, gnode, dR0, dR1);
            if (a.R_cell) *reinterpret_cast<double2 *>(a.R_cell + ((cell0 + c) * N + s) * 2) = make_double2(R0, R1);
        }
        // the other input buffer was last read in the previous tile's per-QP phase
        if (tile + gridDim.x < a.ntiles) otf_store<E, MODE>(smem + ((it + 1) & 1) * S::IN_BYTES, nxt, c, s, act);
        g_cur = g_nxt; kc_cur = kc_nxt; live_cur = live_nxt;
        g_nxt = g_nn; kc_nxt = kc_nn; live_nxt = live_nn;
    }
    if (JAC && l == 0) bulk_wait0();
    (void)live_cur;
}

// ---- G4 with on-the-fly geometry on the fp64 tensor cores (residual + element Jacobians) ----
// eval_otf_kernel's input ring (register gather of U, s and cell-local coordinates one tile ahead, conn / k_c two
// tiles ahead) and per-QP phase (J_q from the coordinates, det J, cofactors, GradBF into the per-warp region in the
// record slot layout), with the DMMA per-node phase of eval_mma_kernel (mma_node_phase). No J staging: the
// shared memory per warp is the two input buffers + GradBF + per-QP scalars.
template <class E>
struct OtfMmaSmem {
    using O = OtfSmem<E, M_JAC>;
    static constexpr int IN_BYTES = O::IN_BYTES;
    static constexpr int OFF_G = 2 * IN_BYTES;
    static constexpr int OFF_QS = OFF_G + E::Q * 3 * E::SLAB * 8;
    static constexpr int BYTES = OFF_QS + qs_mma_bytes<E>();
    static_assert(OFF_G % 128 == 0 && OFF_QS % 16 == 0, "alignment");
};

template <class E>
__global__ void __launch_bounds__(32, SFO_MMA_JAC_WARPS) eval_otf_mma_kernel(EvalArgs a) {
    constexpr int N = E::N, TC = E::TC;
    using S = OtfMmaSmem<E>;
    using O = typename S::O;
    extern __shared__ __align__(128) char smem[];
    double *rg = reinterpret_cast<double *>(smem + S::OFF_G);
    const QsMma<E> qs{reinterpret_cast<double *>(smem + S::OFF_QS)};
    const int l = threadIdx.x;
    const bool act = l < TC * N;
    const int c = act ? E::lane_cell(l) : TC, s = act ? E::lane_sub(l) : 0;  // per-QP phase: (cell, qp)
    const int ni = l >> 2, qq = l & 3;                                       // DMMA fragments: (node, qp quad)
    const bool have_s = (a.surface != nullptr) && (a.force_qp == nullptr);
    const uint64_t pol_stream = policy_evict_first();

    double xq, yq, zq, wq;
    qp_coords<E>(act ? s : 0, xq, yq, zq, wq);
    double phi[2];
    mma_phi<E>(ni, qq, phi);

    auto load_tile = [&](int64_t tile, int32_t &g, double &kcv, bool &live) {
        const int64_t cell = tile * TC + c;
        live = act && tile < a.ntiles && cell < a.ncells;
        g = live ? __ldg(a.conn + cell * N + s) : 0;
        kcv = live ? (a.kc ? __ldg(a.kc + cell) : a.kscal) : 0.0;
    };
    int32_t g_cur, g_nxt;
    double kc_cur, kc_nxt;
    bool live_cur, live_nxt;
    load_tile(blockIdx.x, g_cur, kc_cur, live_cur);
    load_tile(blockIdx.x + (int64_t)gridDim.x, g_nxt, kc_nxt, live_nxt);
    if ((int64_t)blockIdx.x < a.ntiles)
        otf_store<E, M_JAC>(smem, otf_load<M_JAC>(g_cur, live_cur, a.U, a.xyz4, a.surface, have_s, nullptr), c, s,
                            act);

    int it = 0;
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
        const char *in = smem + (it & 1) * S::IN_BYTES;
        const double2 *Us = reinterpret_cast<const double2 *>(in + O::IN_U);
        const double2 *XY = reinterpret_cast<const double2 *>(in + O::IN_XY);
        const double *Zs = reinterpret_cast<const double *>(in + O::IN_Z);
        const double *ss = reinterpret_cast<const double *>(in + O::IN_S);
        const int64_t cell0 = tile * TC;
        const int nvalid = (a.ncells - cell0 < (int64_t)TC) ? (int)(a.ncells - cell0) : TC;

        __syncwarp();  // this tile's gathered inputs are visible; the previous node phase is done with G and qs

        // ---- per-QP phase: geometry, GradBF -> smem, then Ugrad etc. (as eval_otf_kernel) ----
        const double kc = __shfl_sync(0xffffffffu, kc_cur, act ? E::lane_of(c, 0) : 0);
        if (act) {
            const int q = s;
            double dq[N][3];
#pragma unroll
            for (int n = 0; n < N; ++n) {
                double ph;
                basis<E>(n, xq, yq, zq, ph, dq[n][0], dq[n][1], dq[n][2]);
            }
            double J00 = 0, J01 = 0, J02 = 0, J10 = 0, J11 = 0, J12 = 0, J20 = 0, J21 = 0, J22 = 0;
#pragma unroll
            for (int n = 1; n < N; ++n) {  // cell-local: node 0 sits at the origin
                const double2 xy = XY[c * O::UP + n];
                const double z = Zs[c * O::UP + n];
                const double d0 = dq[n][0], d1 = dq[n][1], d2 = dq[n][2];
                J00 = fma(xy.x, d0, J00); J01 = fma(xy.x, d1, J01); J02 = fma(xy.x, d2, J02);
                J10 = fma(xy.y, d0, J10); J11 = fma(xy.y, d1, J11); J12 = fma(xy.y, d2, J12);
                J20 = fma(z, d0, J20); J21 = fma(z, d1, J21); J22 = fma(z, d2, J22);
            }
            const double c00 = J11 * J22 - J12 * J21, c01 = J12 * J20 - J10 * J22, c02 = J10 * J21 - J11 * J20;
            const double c10 = J02 * J21 - J01 * J22, c11 = J00 * J22 - J02 * J20, c12 = J01 * J20 - J00 * J21;
            const double c20 = J01 * J12 - J02 * J11, c21 = J02 * J10 - J00 * J12, c22 = J00 * J11 - J01 * J10;
            const double det = J00 * c00 + J01 * c01 + J02 * c02;
            if (!(det > 0.0) && c < nvalid) atomicOr(a.err, ERR_DETJ);
            const double id = 1.0 / det;
            double ux = 0, uy = 0, uz = 0, vx = 0, vy = 0, vz = 0, gs0 = 0, gs1 = 0;
#pragma unroll
            for (int n = 0; n < N; ++n) {
                const double d0 = dq[n][0], d1 = dq[n][1], d2 = dq[n][2];
                const double g0 = fma(c00, d0, fma(c01, d1, c02 * d2)) * id;
                const double g1 = fma(c10, d0, fma(c11, d1, c12 * d2)) * id;
                const double g2 = fma(c20, d0, fma(c21, d1, c22 * d2)) * id;
                rg[gidx<E>(n, q, 0, c)] = g0;
                rg[gidx<E>(n, q, 1, c)] = g1;
                rg[gidx<E>(n, q, 2, c)] = g2;
                const double2 uv = Us[c * O::UP + n];
                ux = fma(uv.x, g0, ux); uy = fma(uv.x, g1, uy); uz = fma(uv.x, g2, uz);
                vx = fma(uv.y, g0, vx); vy = fma(uv.y, g1, vy); vz = fma(uv.y, g2, vz);
                if (have_s) {
                    const double sn = ss[c * O::UP + n];
                    gs0 = fma(sn, g0, gs0); gs1 = fma(sn, g1, gs1);
                }
            }
            qp_tail<E, M_JAC>(a, qs, c, q, nvalid, cell0, have_s, kc, wq * det, ux, uy, uz, vx, vy, vz, gs0, gs1);
        }
        __syncwarp();

        // ---- per-node phase on the tensor cores (+ register gather of the next tile, conn of the one after) ----
        int32_t gnode[2];  // lane (ni, qq) scatters (cell qq, node ni) [and wedge6's (cell 4, node ni)]
        {
            const int nn = ni < N ? ni : 0;
            gnode[0] = __shfl_sync(0xffffffffu, g_cur, E::lane_of(qq < TC ? qq : 0, nn));
            gnode[1] = __shfl_sync(0xffffffffu, g_cur, E::lane_of(TC > 4 ? 4 : 0, nn));
        }
        int32_t g_nn = 0;
        double kc_nn = 0.0;
        bool live_nn = false;
        OtfGathered nxt{make_double2(0.0, 0.0), make_double2(0.0, 0.0), make_double2(0.0, 0.0), 0.0, 0.0};
        double Rm[2][2] = {{0.0, 0.0}, {0.0, 0.0}};
        mma_node_phase<E, SFO_MMA_UNROLL_COMPACT>(a.J_cell, rg, qs, phi, cell0, nvalid, ni, qq, pol_stream, Rm,
                                                  a.packed != 0, [&]() {
            if (tile + gridDim.x < a.ntiles)
                nxt = otf_load<M_JAC>(g_nxt, live_nxt, a.U, a.xyz4, a.surface, have_s, nullptr);
            load_tile(tile + 2 * (int64_t)gridDim.x, g_nn, kc_nn, live_nn);
        });
        mma_scatter_r<E>(a, gnode, Rm, cell0, nvalid, ni, qq);
        // the other input buffer was last read in the previous tile's per-QP phase
        if (tile + gridDim.x < a.ntiles) otf_store<E, M_JAC>(smem + ((it + 1) & 1) * S::IN_BYTES, nxt, c, s, act);
        g_cur = g_nxt; kc_cur = kc_nxt; live_cur = live_nxt;
        g_nxt = g_nn; kc_nxt = kc_nn; live_nxt = live_nn;
    }
    (void)live_cur;
}

// Setup for the on-the-fly mode: node coordinates as double4.
__global__ void xyz4_kernel(int64_t nnodes, const double *__restrict__ coords, double4 *__restrict__ xyz4) {
    const int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (v < nnodes) xyz4[v] = make_double4(coords[3 * v], coords[3 * v + 1], coords[3 * v + 2], 0.0);
}

// ---------------------------------------------------------------------------
// NEXT-4: basal friction side-set term (PAPER.md P:L59 -> [24]; reading Z18).
// Bed = bottom face of each listed basal cell (local nodes 0..NB-1).  Thread
// <-> face: face QPs (2x2 Gauss / 3-point triangle), surface measure
// |dx/dxi x dx/deta| in face-local coordinates, beta_h and u_h interpolated
// with the face basis; R += int beta u phi_i, J_face = delta_ab int beta phi_i phi_j.
// ---------------------------------------------------------------------------
template <int NB>
__device__ __forceinline__ void face_basis(int q, double &w, double (&phi)[NB], double (&dxi)[NB], double (&deta)[NB]) {
    if (NB == 4) {
        const double g = 1.0 / sqrt(3.0);
        const double x = (q & 1) ? g : -g, y = (q & 2) ? g : -g;
        w = 1.0;
#pragma unroll
        for (int n = 0; n < NB; ++n) {
            const double sx = (n == 1 || n == 2) ? 1.0 : -1.0, sy = (n >= 2) ? 1.0 : -1.0;
            phi[n] = 0.25 * (1.0 + sx * x) * (1.0 + sy * y);
            dxi[n] = 0.25 * sx * (1.0 + sy * y);
            deta[n] = 0.25 * (1.0 + sx * x) * sy;
        }
    } else {
        const double x = (q == 1) ? 2.0 / 3.0 : 1.0 / 6.0, y = (q == 2) ? 2.0 / 3.0 : 1.0 / 6.0;
        w = 1.0 / 6.0;
        const double l[3] = {1.0 - x - y, x, y}, lx[3] = {-1.0, 1.0, 0.0}, ly[3] = {-1.0, 0.0, 1.0};
#pragma unroll
        for (int n = 0; n < NB; ++n) {
            phi[n] = l[n];
            dxi[n] = lx[n];
            deta[n] = ly[n];
        }
    }
}

template <class E>
__global__ void basal_friction_kernel(int64_t nfaces, const int32_t *__restrict__ cells, const int32_t *__restrict__ conn,
                                      const double *__restrict__ coords, const double *__restrict__ beta,
                                      const double *__restrict__ U, double *__restrict__ R, double *__restrict__ Jf) {
    constexpr int N = E::N, NB = N / 2, NQF = NB == 4 ? 4 : 3, ND = 2 * NB;
    const int64_t f = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (f >= nfaces) return;
    const int64_t cell = cells[f];
    int32_t nid[NB];
    double x[NB][3], b[NB], u[NB][2];
#pragma unroll
    for (int n = 0; n < NB; ++n) {
        nid[n] = conn[cell * N + n];
        b[n] = beta[nid[n]];
        u[n][0] = U[2 * (int64_t)nid[n]];
        u[n][1] = U[2 * (int64_t)nid[n] + 1];
    }
#pragma unroll
    for (int n = 0; n < NB; ++n)
#pragma unroll
        for (int r = 0; r < 3; ++r) x[n][r] = coords[3 * (int64_t)nid[n] + r] - coords[3 * (int64_t)nid[0] + r];
    double Rf[NB][2] = {};
    double M[NB][NB] = {};
#pragma unroll
    for (int q = 0; q < NQF; ++q) {
        double w, phi[NB], dxi[NB], deta[NB];
        face_basis<NB>(q, w, phi, dxi, deta);
        double t0[3] = {0, 0, 0}, t1[3] = {0, 0, 0};
#pragma unroll
        for (int n = 0; n < NB; ++n)
#pragma unroll
            for (int r = 0; r < 3; ++r) {
                t0[r] = fma(x[n][r], dxi[n], t0[r]);
                t1[r] = fma(x[n][r], deta[n], t1[r]);
            }
        const double cx = t0[1] * t1[2] - t0[2] * t1[1], cy = t0[2] * t1[0] - t0[0] * t1[2],
                     cz = t0[0] * t1[1] - t0[1] * t1[0];
        const double ds = sqrt(cx * cx + cy * cy + cz * cz) * w;
        double bq = 0.0, u0 = 0.0, u1 = 0.0;
#pragma unroll
        for (int n = 0; n < NB; ++n) {
            bq = fma(b[n], phi[n], bq);
            u0 = fma(u[n][0], phi[n], u0);
            u1 = fma(u[n][1], phi[n], u1);
        }
        const double wb = ds * bq;
#pragma unroll
        for (int i = 0; i < NB; ++i) {
            Rf[i][0] = fma(wb * u0, phi[i], Rf[i][0]);
            Rf[i][1] = fma(wb * u1, phi[i], Rf[i][1]);
#pragma unroll
            for (int j = 0; j < NB; ++j) M[i][j] = fma(wb * phi[i], phi[j], M[i][j]);
        }
    }
#pragma unroll
    for (int i = 0; i < NB; ++i) {
        red_add(R + 2 * (int64_t)nid[i], Rf[i][0]);
        red_add(R + 2 * (int64_t)nid[i] + 1, Rf[i][1]);
    }
    if (Jf) {
        double *J = Jf + f * ND * ND;
#pragma unroll
        for (int i = 0; i < NB; ++i)
#pragma unroll
            for (int a = 0; a < 2; ++a)
#pragma unroll
                for (int j = 0; j < NB; ++j)
#pragma unroll
                    for (int bb = 0; bb < 2; ++bb) J[(2 * i + a) * ND + 2 * j + bb] = (a == bb) ? M[i][j] : 0.0;
    }
}

// ---------------------------------------------------------------------------
// NEXT-4: lateral (calving-front) pressure side-set term (PAPER.md P:L59 ->
// [24]; reading Z19).  Thread <-> face (cell, side k): the quad over the
// footprint edge k -> k+1, local nodes (k, k+1, k+1+P, k+P) (P = N/2, mod P).
// 2x2 Gauss; n dGamma = dx/dxi x dx/deta (face-local coordinates, outward for
// CCW footprints); psi = rho_i g (s_h - z_h) - rho_w g max(z_sl - z_h, 0);
// R[i][a] -= sum_q psi n_a dGamma phi_i.  Independent of U (no Jacobian term).
// ---------------------------------------------------------------------------
template <class E>
__global__ void lateral_pressure_kernel(int64_t nfaces, int64_t ncells, const int32_t *__restrict__ faces,
                                        const int32_t *__restrict__ conn, const double *__restrict__ coords,
                                        const double *__restrict__ surface, double rho_i_g, double rho_w_g,
                                        double z_sl, double *__restrict__ R, int *__restrict__ err) {
    constexpr int N = E::N, P = N / 2;
    const int64_t f = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (f >= nfaces) return;
    const int2 cs = reinterpret_cast<const int2 *>(faces)[f];
    const int64_t cell = cs.x;
    const int k = cs.y;
    if (k < 0 || k >= P || cell < 0 || cell >= ncells) {
        atomicOr(err, ERR_CONN);
        return;
    }
    const int k1 = (k + 1 == P) ? 0 : k + 1;
    const int loc[4] = {k, k1, k1 + P, k + P};
    int32_t nid[4];
    double x[4][3], sn[4];
#pragma unroll
    for (int n = 0; n < 4; ++n) {
        nid[n] = __ldg(conn + cell * N + loc[n]);
        sn[n] = __ldg(surface + nid[n]);
#pragma unroll
        for (int r = 0; r < 3; ++r) x[n][r] = __ldg(coords + 3 * (int64_t)nid[n] + r);
    }
    const double z0 = x[0][2];
    const double g = 0.5773502691896257645;  // 1/sqrt(3)
    double Rf[4][2] = {};
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const double xi = (q & 1) ? g : -g, et = (q & 2) ? g : -g;
        double phi[4], dxi[4], det[4];
#pragma unroll
        for (int n = 0; n < 4; ++n) {
            const double sx = (n == 1 || n == 2) ? 1.0 : -1.0, sy = (n >= 2) ? 1.0 : -1.0;
            phi[n] = 0.25 * (1.0 + sx * xi) * (1.0 + sy * et);
            dxi[n] = 0.25 * sx * (1.0 + sy * et);
            det[n] = 0.25 * (1.0 + sx * xi) * sy;
        }
        double t0[3] = {0, 0, 0}, t1[3] = {0, 0, 0};
        double zq = 0.0, sq = 0.0;
#pragma unroll
        for (int n = 0; n < 4; ++n) {
#pragma unroll
            for (int r = 0; r < 3; ++r) {
                const double xl = x[n][r] - x[0][r];  // face-local (reading Z17)
                t0[r] = fma(xl, dxi[n], t0[r]);
                t1[r] = fma(xl, det[n], t1[r]);
            }
            zq = fma(x[n][2] - z0, phi[n], zq);
            sq = fma(sn[n], phi[n], sq);
        }
        zq += z0;  // sum_n phi_n = 1
        const double n0 = t0[1] * t1[2] - t0[2] * t1[1];
        const double n1 = t0[2] * t1[0] - t0[0] * t1[2];
        const double psi = rho_i_g * (sq - zq) - rho_w_g * fmax(z_sl - zq, 0.0);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            Rf[i][0] = fma(-psi * n0, phi[i], Rf[i][0]);
            Rf[i][1] = fma(-psi * n1, phi[i], Rf[i][1]);
        }
    }
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        red_add(R + 2 * (int64_t)nid[i], Rf[i][0]);
        red_add(R + 2 * (int64_t)nid[i] + 1, Rf[i][1]);
    }
}

// ---------------------------------------------------------------------------
// G5: assembly.  R part: thread <-> (cell, node).  CSR part: thread <-> (cell, row).
// ---------------------------------------------------------------------------
// With a peer table attached (stokesfo_set_remote) the same fused halo sum as
// the evaluation kernels' epilogue (scatter_node).
template <int N>
__global__ void scatter_r_kernel(int64_t ncells, const int32_t *__restrict__ conn, const double2 *__restrict__ Rc,
                                 double *__restrict__ R, const int32_t *rem, const int32_t *remtab,
                                 double *const *peers) {
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (gid >= ncells * N) return;
    const double2 v = Rc[gid];
    scatter_node(rem, remtab, R, peers, conn[gid], v.x, v.y);
}

template <int N>
__global__ void scatter_csr_kernel(int64_t ncells, const int32_t *__restrict__ conn, const double *__restrict__ Jc,
                                   const int64_t *__restrict__ rowptr, const int32_t *__restrict__ colidx,
                                   double *__restrict__ vals, int *__restrict__ err) {
    constexpr int ND = 2 * N;
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (gid >= ncells * ND) return;
    const int64_t cell = gid / ND;
    const int r = (int)(gid % ND);
    const int64_t row = 2 * (int64_t)conn[cell * N + r / 2] + (r & 1);
    const int64_t lo0 = rowptr[row], hi0 = rowptr[row + 1];
    for (int s = 0; s < ND; ++s) {
        const int32_t col = 2 * conn[cell * N + s / 2] + (s & 1);
        int64_t lo = lo0, hi = hi0;  // binary search in the sorted row
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if (colidx[mid] < col) lo = mid + 1; else hi = mid;
        }
        if (lo < hi0 && colidx[lo] == col)
            red_add(vals + lo, Jc[cell * ND * ND + r * ND + s]);
        else
            atomicOr(err, ERR_CSR);
    }
}

// NEXT-2: per-cell CSR slots (thread <-> (cell, i)): slot[c][i][j] = index of
// node g_j in the sorted neighbour list of g_i (binary search in row 2 g_i,
// once per mesh), packed as N bytes of one uint64 per (cell, i).
template <int N>
__global__ void csr_slots_kernel(int64_t ncells, const int32_t *__restrict__ conn,
                                 const int64_t *__restrict__ rowptr, const int32_t *__restrict__ colidx,
                                 uint64_t *__restrict__ slots, int *__restrict__ err) {
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (gid >= ncells * N) return;
    const int64_t cell = gid / N;
    const int64_t row = 2 * (int64_t)conn[gid];
    const int64_t lo0 = rowptr[row], hi0 = rowptr[row + 1];
    uint64_t w = 0;
    for (int j = 0; j < N; ++j) {
        const int32_t col = 2 * conn[cell * N + j];
        int64_t lo = lo0, hi = hi0;
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if (colidx[mid] < col) lo = mid + 1; else hi = mid;
        }
        const int64_t sl = (lo - lo0) >> 1;
        if (lo < hi0 && colidx[lo] == col && sl < 256) w |= (uint64_t)sl << (8 * j);
        else atomicOr(err, ERR_CSR);
    }
    slots[gid] = w;
}

// CSR assembly of element matrices through the slot table (thread <-> (cell, row)).
template <int N>
__global__ void scatter_csr_slots_kernel(int64_t ncells, const int32_t *__restrict__ conn,
                                         const double *__restrict__ Jc, const int64_t *__restrict__ rowptr,
                                         const uint64_t *__restrict__ slots, double *__restrict__ vals) {
    constexpr int ND = 2 * N;
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (gid >= ncells * ND) return;
    const int64_t cell = gid / ND;
    const int r = (int)(gid % ND);
    const int i = r >> 1;
    const uint64_t w = __ldg(slots + cell * N + i);
    double *base = vals + __ldg(rowptr + 2 * (int64_t)conn[cell * N + i] + (r & 1));
    const double2 *Jr = reinterpret_cast<const double2 *>(Jc + (cell * ND + r) * ND);
#pragma unroll
    for (int j = 0; j < N; ++j) {
        const double2 v = __ldcs(Jr + j);  // streamed once
        double *p = base + 2 * (int)((w >> (8 * j)) & 0xff);
        red_add(p, v.x);
        red_add(p + 1, v.y);
    }
}

// Deterministic, atomic-free CSR assembly of element matrices ("pull"): a
// warp owns the CSR rows 2v, 2v+1 (contiguous in vals) of NPW nodes v at once,
// accumulates the two rows of every incident cell's J (node -> (cell, local i)
// incidence, ascending cell order) in a shared-memory row buffer through the
// slot table, then adds the buffer to vals with coalesced stores.  Every
// J_cell element is read once (by the warp of its row's node); no two warps
// touch the same entry.  The NPW nodes' loads (incidence, up to 8 cells' J
// rows and slot rows each) are all issued before any is consumed: the kernel
// is a chain of dependent gathers, so memory-level parallelism per warp is
// what sets its speed.
constexpr int CSR_GATHER_MAXDEG = 64;   // neighbour nodes per node (else the atomic kernel)
constexpr int CSR_GATHER_WARPS = 8;
// Per element type: nodes per warp, incident cells handled in the batched path (an interior node of an
// extruded mesh has 2 x (cells around a footprint vertex): hex8 (quads) 8, wedge6 (triangles) 12 on the
// Voronoi-dual triangulation), and 64-bit words of the per-node pull record.
template <int N>
struct PullCfg {
    static constexpr int NPW = N == 8 ? 2 : 1;
    static constexpr int BATCH = N == 8 ? 8 : 12;
    static constexpr int WORDS = 32 / NPW;
    static constexpr int CI0 = 2, SR0 = CI0 + BATCH / 2, K0W = SR0 + BATCH;  // record word offsets
    static_assert(K0W < WORDS, "record fits");
};
template <int N>
__host__ __device__ constexpr int pull_npw() {
    return PullCfg<N>::NPW;
}
template <int N>
__host__ __device__ constexpr int pull_words() {
    return PullCfg<N>::WORDS;
}
// ACC = false: the rows are overwritten (vals = assembled J; no prior zeroing, no read of vals).
// row pair (2 i + a, columns 2 j, 2 j + 1) of cell `cell`'s element matrix: full [C][2N][2N] (streamed
// once) or symmetric block-packed (block (i, j) or the transpose of block (j, i); each off-diagonal
// block is read by two node warps, so the packed reads keep the default L2 policy)
template <int N, bool PACKED>
__device__ __forceinline__ double2 jrow2(const double *__restrict__ Jc, int64_t cell, int i, int a, int j) {
    if (!PACKED) return __ldcs(reinterpret_cast<const double2 *>(Jc + (cell * 2 * N + 2 * i + a) * 2 * N) + j);
    const double *b = Jc + cell * (4 * pk_blocks<N>());
    if (j >= i) return __ldg(reinterpret_cast<const double2 *>(b + 4 * pk_block<N>(i, j) + 2 * a));
    const double *t = b + 4 * pk_block<N>(j, i);
    return make_double2(__ldg(t + a), __ldg(t + 2 + a));
}
// Per-node pull record (built once by stokesfo_csr_slots; PullCfg<N>::WORDS 64-bit words per node: 128 B hex8,
// 256 B wedge6): everything the pull assembly needs before it can load element-matrix rows, in one coalesced
// load per node instead of the dependent chain rowptr / inc_ptr -> inc -> slots (three DRAM round trips per task;
// ncu r2g: long_sb 43-44%).
//   w0 CSR row base r0 (rowptr[2v]); w1 = len (both rows) | cnt << 32; w[CI0..) the first BATCH incidence
//   entries (cell N + i) as int32 pairs; w[SR0..) their slot rows; w[K0W] = incidence start k0 (> BATCH path)
template <int N>
__global__ void node_rec_kernel(int64_t nnodes, const int64_t *__restrict__ rowptr, const int64_t *__restrict__ inc_ptr,
                                const int32_t *__restrict__ inc, const uint64_t *__restrict__ slots,
                                uint64_t *__restrict__ rec) {
    using P = PullCfg<N>;
    const int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (v >= nnodes) return;
    const int64_t r0 = rowptr[2 * v], k0 = inc_ptr[v];
    const int len = (int)(rowptr[2 * v + 2] - r0), cnt = (int)(inc_ptr[v + 1] - k0);
    uint64_t w[P::WORDS];
    for (int k = 0; k < P::WORDS; ++k) w[k] = 0;
    w[0] = (uint64_t)r0;
    w[1] = (uint64_t)(uint32_t)len | ((uint64_t)(uint32_t)cnt << 32);
    for (int e = 0; e < P::BATCH && e < cnt; ++e) {
        const int32_t ci = inc[k0 + e];
        w[P::CI0 + e / 2] |= (uint64_t)(uint32_t)ci << (32 * (e & 1));
        w[P::SR0 + e] = slots[ci];
    }
    w[P::K0W] = (uint64_t)k0;
    uint4 *o = reinterpret_cast<uint4 *>(rec + v * P::WORDS);
    for (int k = 0; k < P::WORDS / 2; ++k) o[k] = make_uint4((uint32_t)w[2 * k], (uint32_t)(w[2 * k] >> 32),
                                                            (uint32_t)w[2 * k + 1], (uint32_t)(w[2 * k + 1] >> 32));
}

template <int N, bool ACC = true, bool PACKED = false>
__global__ void __launch_bounds__(32 * CSR_GATHER_WARPS, 4)
    csr_gather_kernel(int64_t nnodes, const double *__restrict__ Jc, const uint64_t *__restrict__ nrec,
                      const int32_t *__restrict__ inc, const uint64_t *__restrict__ slots, double *__restrict__ vals) {
    constexpr int LC = 2 * N;            // lanes per cell: each loads one (j, b = 0..1) pair of one row
    constexpr int CPI = 32 / LC;         // cells per load instruction (2 for hex8 and wedge6)
    using P = PullCfg<N>;
    constexpr int NPW = P::NPW, BATCH = P::BATCH, NI = BATCH / CPI, NREC_WORDS = P::WORDS;
    __shared__ __align__(16) double buf[CSR_GATHER_WARPS][NPW][4 * CSR_GATHER_MAXDEG];
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    const int64_t v0 = (blockIdx.x * (int64_t)CSR_GATHER_WARPS + w) * NPW;
    if (v0 >= nnodes) return;  // uniform per warp
    static_assert(NI * CPI == BATCH, "whole load groups");
    static_assert(NPW * NREC_WORDS == 32, "one record word per lane");
    // lane l holds word l % WORDS of node l / WORDS's pull record
    const int64_t vr = v0 + l / NREC_WORDS;
    const uint64_t rw = vr < nnodes ? __ldg(nrec + vr * NREC_WORDS + (l % NREC_WORDS)) : 0;
    int64_t r0[NPW], k0[NPW];
    int len[NPW], cnt[NPW];
#pragma unroll
    for (int n = 0; n < NPW; ++n) {
        r0[n] = (int64_t)__shfl_sync(0xffffffffu, rw, n * NREC_WORDS);
        const uint64_t lc = __shfl_sync(0xffffffffu, rw, n * NREC_WORDS + 1);
        len[n] = (int)(uint32_t)lc;  // both rows: 4 deg entries
        cnt[n] = (int)(uint32_t)(lc >> 32);
        k0[n] = (int64_t)__shfl_sync(0xffffffffu, rw, n * NREC_WORDS + P::K0W);
    }
    // pull the rows' vals lines into L2 now: the final read-modify-write then hits L2
    if (ACC) {
#pragma unroll
        for (int n = 0; n < NPW; ++n)
            for (int p = 16 * l; p < len[n]; p += 16 * 32)
                asm volatile("prefetch.global.L2 [%0];" ::"l"(vals + r0[n] + p));
    }
#pragma unroll
    for (int n = 0; n < NPW; ++n)
        for (int p = 2 * l; p < len[n]; p += 64) *reinterpret_cast<double2 *>(&buf[w][n][p]) = make_double2(0.0, 0.0);
    // lane l <-> (cell u = l / LC of the pair, row a, column node j); columns (j, 0..1) as one double2
    const int u = l / LC, a = (l % LC) / N, j = l % N;
    const bool lane_ok = l < CPI * LC;
    double2 x[NPW][NI];
    int sl[NPW][NI];  // this lane's slot byte (column node j) of its incident cell
    const uint8_t *sb = reinterpret_cast<const uint8_t *>(slots);
#pragma unroll
    for (int n = 0; n < NPW; ++n)
#pragma unroll
        for (int t = 0; t < NI; ++t) {
            const int e = CPI * t + (u < CPI ? u : 0);  // incidence entry of this lane
            const uint64_t cp = __shfl_sync(0xffffffffu, rw, n * NREC_WORDS + P::CI0 + (e >> 1));
            const uint64_t srow = __shfl_sync(0xffffffffu, rw, n * NREC_WORDS + P::SR0 + e);
            const int32_t ci = (int32_t)(uint32_t)((e & 1) ? (cp >> 32) : cp);
            const bool live = lane_ok && e < cnt[n];
            const int64_t cell = ci / N;
            const int i = ci - (int)(cell * N);
            x[n][t] = live ? jrow2<N, PACKED>(Jc, cell, i, a, j) : make_double2(0.0, 0.0);
            sl[n][t] = live ? (int)((srow >> (8 * j)) & 0xffu) : -1;
        }
    __syncwarp();
#pragma unroll
    for (int n = 0; n < NPW; ++n) {
        const int half = len[n] >> 1;
        // cells u = 0 and u = 1 of a pair may hit the same entries: add them in turn
#pragma unroll
        for (int t = 0; t < NI; ++t)
#pragma unroll
            for (int uu = 0; uu < CPI; ++uu) {
                if (u == uu && sl[n][t] >= 0) {
                    double2 *p = reinterpret_cast<double2 *>(&buf[w][n][a * half + 2 * sl[n][t]]);
                    double2 b = *p;
                    b.x += x[n][t].x;
                    b.y += x[n][t].y;
                    *p = b;
                }
                __syncwarp();
            }
        // rare: more than BATCH incident cells (not on extruded hex8 / wedge6 meshes)
        for (int64_t k = k0[n] + BATCH; k < k0[n] + cnt[n]; ++k) {
            const int32_t ci = __ldg(inc + k);
            const int64_t cell = ci / N;
            const int i = ci - (int)(cell * N);
            if (l < LC) {
                const int s = (int)__ldg(sb + 8 * (int64_t)ci + j);
                const double2 y = jrow2<N, PACKED>(Jc, cell, i, a, j);
                buf[w][n][a * half + 2 * s] += y.x;
                buf[w][n][a * half + 2 * s + 1] += y.y;
            }
            __syncwarp();
        }
    }
    __syncwarp();
#pragma unroll
    for (int n = 0; n < NPW; ++n)
        for (int p = 2 * l; p < len[n]; p += 64) {
            double2 *o = reinterpret_cast<double2 *>(vals + r0[n] + p);
            const double2 b = *reinterpret_cast<const double2 *>(&buf[w][n][p]);
            if (ACC) {
                double2 c = *o;
                c.x += b.x;
                c.y += b.y;
                *o = c;
            } else {
                __stcs(o, b);  // streamed: the assembled matrix is not re-read by this kernel
            }
        }
}

// ---------------------------------------------------------------------------
// Failure detection (STOKESFO_CHECK_FINITE=1): any non-finite value in an
// output raises the sticky ERR_NONFINITE flag (one atomic per warp).
// ---------------------------------------------------------------------------
__global__ void finite_check_kernel(int64_t n, const double *__restrict__ p, int *__restrict__ err) {
    bool bad = false;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        bad |= !isfinite(__ldcs(p + i));
    if (__any_sync(0xffffffffu, bad) && (threadIdx.x & 31) == 0) atomicOr(err, ERR_NONFINITE);
}

// ---------------------------------------------------------------------------
// G7: halo pack / unpack-add.
// ---------------------------------------------------------------------------
__global__ void halo_pack_kernel(int64_t n, const int32_t *__restrict__ nodes, const double2 *__restrict__ R,
                                 double2 *__restrict__ buf) {
    const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k < n) buf[k] = R[nodes[k]];
}
__global__ void halo_unpack_add_kernel(int64_t n, const int32_t *__restrict__ nodes, const double2 *__restrict__ buf,
                                       double2 *__restrict__ R) {
    const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k < n) {
        const double2 b = buf[k];
        double2 r = R[nodes[k]];
        r.x += b.x;
        r.y += b.y;
        R[nodes[k]] = r;
    }
}

}  // namespace sfo
