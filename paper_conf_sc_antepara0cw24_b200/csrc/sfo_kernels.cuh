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
// ---------------------------------------------------------------------------
template <class E>
__global__ void geometry_kernel(int64_t ncells, int64_t nnodes, const int32_t *__restrict__ conn,
                                const double *__restrict__ coords, const double *__restrict__ kc_in, double kscal,
                                char *__restrict__ recs, int *__restrict__ err) {
    using R = Rec<E>;
    constexpr int N = E::N, Q = E::Q, TC = E::TC;
    const int64_t ntiles = (ncells + TC - 1) / TC;
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (gid >= ntiles * TC * Q) return;
    const int q = (int)(gid % Q);
    const int64_t cell = gid / Q;
    const int64_t tile = cell / TC;
    const int c = (int)(cell % TC);
    char *rec = recs + tile * (int64_t)R::BYTES;
    int32_t *rconn = reinterpret_cast<int32_t *>(rec + R::CONN_OFF);
    double *rkc = reinterpret_cast<double *>(rec + R::KC_OFF);
    double *rwm = reinterpret_cast<double *>(rec + R::WM_OFF);
    double *rg = reinterpret_cast<double *>(rec + R::G_OFF);
    if (cell >= ncells) {  // padding cells of the ragged last tile: zero record
        if (q == 0) {
            for (int n = 0; n < N; ++n) rconn[R::conn(n, c)] = 0;
            rkc[c] = 0.0;
        }
        rwm[R::wm(q, c)] = 0.0;
        for (int n = 0; n < N; ++n)
            for (int d = 0; d < 3; ++d) rg[gidx<E>(n, q, d, c)] = 0.0;
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
    if (q == 0) {
        for (int n = 0; n < N; ++n) rconn[R::conn(n, c)] = nid[n];
        rkc[c] = kc_in ? kc_in[cell] : kscal;
    }
    double xq, yq, zq, wq;
    qp_coords<E>(q, xq, yq, zq, wq);
    double dphi[N][3];
    double J[3][3] = {{0, 0, 0}, {0, 0, 0}, {0, 0, 0}};
#pragma unroll
    for (int n = 0; n < N; ++n) {
        double phi;
        basis<E>(n, xq, yq, zq, phi, dphi[n][0], dphi[n][1], dphi[n][2]);
        const double x0 = coords[3 * (int64_t)nid[n] + 0];
        const double x1 = coords[3 * (int64_t)nid[n] + 1];
        const double x2 = coords[3 * (int64_t)nid[n] + 2];
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
    const double idet = 1.0 / det;
#pragma unroll
    for (int n = 0; n < N; ++n)
#pragma unroll
        for (int r = 0; r < 3; ++r)
            rg[gidx<E>(n, q, r, c)] =
                (cof[r][0] * dphi[n][0] + cof[r][1] * dphi[n][1] + cof[r][2] * dphi[n][2]) * idet;
    rwm[R::wm(q, c)] = wq * det;
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
// G3/G4: fused evaluation.
// ---------------------------------------------------------------------------
struct EvalArgs {
    const char *recs;
    int64_t ntiles, ncells;
    const double *U;          // [nodes][2]
    const double *surface;    // [nodes] or null
    const double *force_qp;   // [C][Q][2] or null (overrides surface)
    double rho_g, delta;
    double *mu_qp;            // [C][Q] or null
    double *R_cell;           // [C][N][2] or null
    double *R;                // [nodes][2] or null (+=)
    double *J_cell;           // [C][2N][2N] (JAC)
};

constexpr int NQS = 9;  // per-(cell, qp) scalars: beta00 beta01 beta02 beta11 beta12, wmu2, gamma, wf0, wf1

// Shared memory: two stage buffers + per-QP scalars + 2 mbarriers.
// A stage buffer holds [record | gathered U (double2 [N][TC]) | s ([N][TC])];
// once a tile's phase 2 has consumed its record, the same buffer stages the
// tile's element Jacobians for the TMA bulk store (JAC).
template <class E, bool JAC, int NSTAGE = 2>
struct EvalSmem {
    static constexpr int N = E::N, Q = E::Q, TC = E::TC;
    static constexpr int REC = Rec<E>::BYTES;
    static constexpr int U_OFF = REC;                        // double2 [N][TC]
    static constexpr int S_OFF = U_OFF + N * TC * 16;        // double  [N][TC]
    static constexpr int IN_BYTES = S_OFF + N * TC * 8;
    static constexpr int J_BYTES = JAC ? TC * E::JPITCH * 8 : 0;
    static constexpr int STAGE = (int)round_up(IN_BYTES > J_BYTES ? IN_BYTES : J_BYTES, 128);
    static constexpr int OFF_QS = NSTAGE * STAGE;            // double [NQS][Q][TC]
    static constexpr int OFF_BAR = OFF_QS + NQS * Q * TC * 8;
    static constexpr int BYTES = OFF_BAR + NSTAGE * 8;
};

// Issue the gather of U (16 B) and s (8 B) of one tile through its conn, as
// cp.async copies into the tile's stage buffer (thread <-> (cell, node)).
template <class E>
__device__ __forceinline__ void issue_gather(char *stage, const double *U, const double *surface, bool have_s) {
    using R = Rec<E>;
    using S = EvalSmem<E, false>;
    const int t = threadIdx.x;
    const int c = t % E::TC, n = t / E::TC;
    const int32_t g = reinterpret_cast<const int32_t *>(stage + R::CONN_OFF)[R::conn(n, c)];
    cp_async16(stage + S::U_OFF + (n * E::TC + c) * 16, U + 2 * (int64_t)g);
    if (have_s) cp_async8(stage + S::S_OFF + (n * E::TC + c) * 8, surface + g);
    cp_async_commit();
}

// Resident CTAs per SM the register budget is tuned for (shared memory permits
// this many for hex8 at the given stage count).
template <class E, bool JAC, int NSTAGE>
constexpr int min_blocks() {
    return E::N == 8 ? (NSTAGE == 2 ? 3 : 2) : 2;
}

template <class E, bool JAC, int NSTAGE>
__global__ void __launch_bounds__(E::TC *E::N, (min_blocks<E, JAC, NSTAGE>())) eval_kernel(EvalArgs a) {
    constexpr int N = E::N, Q = E::Q, TC = E::TC;
    static_assert(N == Q, "thread mappings assume N == Q");
    using R = Rec<E>;
    using S = EvalSmem<E, JAC, NSTAGE>;
    static_assert(S::U_OFF == EvalSmem<E, false>::U_OFF && S::S_OFF == EvalSmem<E, false>::S_OFF, "layout");
    extern __shared__ __align__(128) char smem[];
    double *qs = reinterpret_cast<double *>(smem + S::OFF_QS);
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem + S::OFF_BAR);
    const int t = threadIdx.x;
    const bool have_s = (a.surface != nullptr) && (a.force_qp == nullptr);

    uint64_t pol_stream = 0;
    if (t == 0) {
        pol_stream = policy_evict_first();
        for (int s = 0; s < NSTAGE; ++s) mbar_init(&bar[s], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (t == 0) {
        for (int s = 0; s < NSTAGE; ++s) {
            const int64_t tile = blockIdx.x + (int64_t)s * gridDim.x;
            if (tile < a.ntiles) {
                mbar_arrive_expect_tx(&bar[s], R::BYTES);
                bulk_g2s(smem + s * S::STAGE, a.recs + tile * (int64_t)R::BYTES, R::BYTES, &bar[s], pol_stream);
            }
        }
    }
    if ((int64_t)blockIdx.x < a.ntiles) {
        mbar_wait(&bar[0], 0);
        issue_gather<E>(smem, a.U, a.surface, have_s);
    }

    // phase-2 identity: thread <-> (cell c2, node i)
    const int c2 = E::NODE_MAJOR_P2 ? t % TC : t / N;
    const int i = E::NODE_MAJOR_P2 ? t / TC : t % N;
    double bfi[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) {
        double x, y, z, w, dx, dy, dz;
        qp_coords<E>(q, x, y, z, w);
        basis<E>(i, x, y, z, bfi[q], dx, dy, dz);
    }
    constexpr double P_EXP = -1.0 / 3.0;  // (1 - n) / (2 n) at n = 3

    int it = 0;
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
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

        cp_async_wait_all();  // this thread's gathers for this tile have landed
        __syncthreads();      // ... and everyone's

        // ---- phase 1: per-QP quantities (thread <-> (cell, qp)) ----
        {
            const int c = t % TC, q = t / TC;
            double ux = 0, uy = 0, uz = 0, vx = 0, vy = 0, vz = 0, gs0 = 0, gs1 = 0;
#pragma unroll
            for (int n = 0; n < N; ++n) {
                const double g0 = rg[gidx<E>(n, q, 0, c)];
                const double g1 = rg[gidx<E>(n, q, 1, c)];
                const double g2 = rg[gidx<E>(n, q, 2, c)];
                const double2 uv = Us[n * TC + c];
                ux += uv.x * g0; uy += uv.x * g1; uz += uv.x * g2;
                vx += uv.y * g0; vy += uv.y * g1; vz += uv.y * g2;
                if (have_s) {
                    const double sn = ss[n * TC + c];
                    gs0 += sn * g0; gs1 += sn * g1;
                }
            }
            const double uyvx = uy + vx;
            // effective strain rate^2 (reading Z2) and Glen viscosity, n = 3
            const double e2 = ux * ux + vy * vy + ux * vy + 0.25 * uyvx * uyvx + 0.25 * uz * uz + 0.25 * vz * vz;
            const double r = rcbrt(e2 + a.delta);  // (e2 + delta)^(-1/3)
            const double mu = rkc[c] * r;
            const double wm = rwm[R::wm(q, c)];
            const double wmu2 = 2.0 * wm * mu;
            // beta = B g: sigma = 2 mu beta reproduces strs00..strs12 of Fig. 2
            double *qq = qs + q * TC + c;
            qq[0 * Q * TC] = 2.0 * ux + vy;   // beta_(0,0) = strs00 / (2 mu)
            qq[1 * Q * TC] = 0.5 * uyvx;      // beta_(0,1) = beta_(1,0) = strs01 / (2 mu)
            qq[2 * Q * TC] = 0.5 * uz;        // beta_(0,2) = strs02 / (2 mu)
            qq[3 * Q * TC] = ux + 2.0 * vy;   // beta_(1,1) = strs11 / (2 mu)
            qq[4 * Q * TC] = 0.5 * vz;        // beta_(1,2) = strs12 / (2 mu)
            qq[5 * Q * TC] = wmu2;
            // gamma = wM 2 mu p / (e2 + delta) = wmu2 p r^3  (d mu / d e2 chain, reading Z5)
            qq[6 * Q * TC] = wmu2 * P_EXP * (r * r * r);
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
            qq[7 * Q * TC] = wf0;
            qq[8 * Q * TC] = wf1;
            if (a.mu_qp && c < nvalid) a.mu_qp[(cell0 + c) * Q + q] = mu;
        }
        __syncthreads();

        // ---- phase 2: per-node accumulation (thread <-> (cell c2, node i)) ----
        const int32_t gnode = rconn[R::conn(i, c2)];
        double R0 = 0.0, R1 = 0.0;
        constexpr int K = N / 2;            // symmetric block scheme: blocks (i, i+k), k = 0..K
        double Jb[JAC ? K + 1 : 1][2][2];   // Jb[k][a][b] = J[(i,a), (j_k,b)], j_k = (i+k) mod N
        if (JAC) {
#pragma unroll
            for (int k = 0; k <= K; ++k) Jb[k][0][0] = Jb[k][0][1] = Jb[k][1][0] = Jb[k][1][1] = 0.0;
        }
#pragma unroll
        for (int q = 0; q < Q; ++q) {
            if (q == Q / 2) {
                // prefetch: gather U, s of the next tile (its record was issued
                // NSTAGE-1 tiles ago) while the rest of this tile computes
                const int64_t nt = tile + gridDim.x;
                if (nt < a.ntiles) {
                    const int ns = (it + 1) % NSTAGE;
                    mbar_wait(&bar[ns], (uint32_t)(((it + 1) / NSTAGE) & 1));
                    issue_gather<E>(smem + ns * S::STAGE, a.U, a.surface, have_s);
                }
            }
            const double *qq = qs + q * TC + c2;
            const double b00 = qq[0 * Q * TC], b01 = qq[1 * Q * TC], b02 = qq[2 * Q * TC];
            const double b11 = qq[3 * Q * TC], b12 = qq[4 * Q * TC];
            const double b10 = b01;
            const double wmu2 = qq[5 * Q * TC];
            const double wf0 = qq[7 * Q * TC], wf1 = qq[8 * Q * TC];
            const double gi0 = rg[gidx<E>(i, q, 0, c2)];
            const double gi1 = rg[gidx<E>(i, q, 1, c2)];
            const double gi2 = rg[gidx<E>(i, q, 2, c2)];
            // h_(i,a) = sum_d G_i[d] beta_(a,d);  residual row (i,a) = wmu2 h + wf_a BF_i
            const double h0 = fma(gi2, b02, fma(gi1, b01, gi0 * b00));
            const double h1 = fma(gi2, b12, fma(gi1, b11, gi0 * b10));
            R0 = fma(wf0, bfi[q], fma(wmu2, h0, R0));
            R1 = fma(wf1, bfi[q], fma(wmu2, h1, R1));
            if (JAC) {
                // J_q[(i,a),(j,b)] = sum_e M_ab[e] G_j[e] with
                // M_ab = wmu2 * (B-block (a,b) applied to G_i) + gamma h_(i,a) beta_(b,.)
                const double gam = qq[6 * Q * TC];
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
                    // explicit 3-deep DFMA chains into the accumulators (no DMUL/DADD)
                    Jb[k][0][0] = fma(m00z, gj2, fma(m00y, gj1, fma(m00x, gj0, Jb[k][0][0])));
                    Jb[k][0][1] = fma(m01z, gj2, fma(m01y, gj1, fma(m01x, gj0, Jb[k][0][1])));
                    Jb[k][1][0] = fma(m10z, gj2, fma(m10y, gj1, fma(m10x, gj0, Jb[k][1][0])));
                    Jb[k][1][1] = fma(m11z, gj2, fma(m11y, gj1, fma(m11x, gj0, Jb[k][1][1])));
                }
            }
        }
        const bool valid = c2 < nvalid;
        const int64_t cell = cell0 + c2;
        __syncthreads();  // everyone is done with this stage's record and qs

        if (JAC) {
            // Stage J[c2] rows (2i, 2i+1) into this stage buffer: direct blocks
            // (i, i+k), k = 0..K, and transposed blocks (i+k, i) for 0 < k < K
            // (J is symmetric: the Hessian of the quadrature energy).
            double *Jc = reinterpret_cast<double *>(stage) + c2 * E::JPITCH;
            constexpr int LD = 2 * N;
#pragma unroll
            for (int k = 0; k <= K; ++k) {
                const int j = (i + k) % N;
                *reinterpret_cast<double2 *>(Jc + (2 * i + 0) * LD + 2 * j) = make_double2(Jb[k][0][0], Jb[k][0][1]);
                *reinterpret_cast<double2 *>(Jc + (2 * i + 1) * LD + 2 * j) = make_double2(Jb[k][1][0], Jb[k][1][1]);
                if (k > 0 && k < K) {
                    *reinterpret_cast<double2 *>(Jc + (2 * j + 0) * LD + 2 * i) =
                        make_double2(Jb[k][0][0], Jb[k][1][0]);
                    *reinterpret_cast<double2 *>(Jc + (2 * j + 1) * LD + 2 * i) =
                        make_double2(Jb[k][0][1], Jb[k][1][1]);
                }
            }
            fence_proxy_async_smem();
            __syncthreads();
            if (t == 0) {
                if (E::JPITCH == 4 * N * N) {
                    bulk_s2g(a.J_cell + cell0 * (4 * N * N), stage, (uint32_t)(nvalid * 4 * N * N * 8), pol_stream);
                } else {
                    for (int c = 0; c < nvalid; ++c)
                        bulk_s2g(a.J_cell + (cell0 + c) * (4 * N * N), stage + c * E::JPITCH * 8,
                                 (uint32_t)(4 * N * N * 8), pol_stream);
                }
                bulk_commit();
                bulk_wait_read0();  // staging read done -> the buffer may take the next record
            }
        }
        if (t == 0) {
            const int64_t nt = tile + (int64_t)NSTAGE * gridDim.x;
            if (nt < a.ntiles) {
                mbar_arrive_expect_tx(&bar[st], R::BYTES);
                bulk_g2s(stage, a.recs + nt * (int64_t)R::BYTES, R::BYTES, &bar[st], pol_stream);
            }
        }
        if (valid) {
            if (a.R) {
                atomicAdd(a.R + 2 * (int64_t)gnode + 0, R0);
                atomicAdd(a.R + 2 * (int64_t)gnode + 1, R1);
            }
            if (a.R_cell) *reinterpret_cast<double2 *>(a.R_cell + (cell * N + i) * 2) = make_double2(R0, R1);
        }
    }
    if (JAC && t == 0) bulk_wait0();
}

// ---------------------------------------------------------------------------
// G5: assembly.  R part: thread <-> (cell, node).  CSR part: thread <-> (cell, row).
// ---------------------------------------------------------------------------
template <int N>
__global__ void scatter_r_kernel(int64_t ncells, const int32_t *__restrict__ conn, const double2 *__restrict__ Rc,
                                 double *__restrict__ R) {
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (gid >= ncells * N) return;
    const int64_t g = conn[gid];
    const double2 v = Rc[gid];
    atomicAdd(R + 2 * g + 0, v.x);
    atomicAdd(R + 2 * g + 1, v.y);
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
            atomicAdd(vals + lo, Jc[cell * ND * ND + r * ND + s]);
        else
            atomicOr(err, ERR_CSR);
    }
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
