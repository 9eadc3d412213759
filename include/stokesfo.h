/*
 * stokesfo.h -- C ABI of libstokesfo.so: the B200 (sm_100a) Stokes-FO
 * (Blatter-Pattyn) per-cell residual + forward-AD Jacobian evaluator.
 *
 * The problem the ABI follows is PAPER.md eq. (3):
 *     F(U; {phi_i}, {grad phi_i}, H, ...) = 0,
 * the finite-element discretisation of the first-order Stokes equations
 * eq. (1) on a mesh extruded from a 2-D footprint,
 * with the per-cell evaluation of Fig. 2 (StokesFOResid, optimized
 * loop order) and its AD Jacobian (Sacado SFad, 16 derivative
 * components per hex8 cell = 8 nodes x 2 velocity components).
 *
 * Conventions (all readings listed in DESIGN.md):
 *   - dof = 2*node + comp (interleaved); local derivative index k = 2*n + a (Z9)
 *   - hex8: Shards node order, 2x2x2 Gauss, q = i + 2j + 4k (Z8, Z9)
 *   - wedge6: bottom triangle (0,0),(1,0),(0,1) then top; 3-point interior
 *     triangle rule x 2-point Gauss, q = t + 3k (Z8)
 *   - Glen's law (Z1-Z3): eps_e^2 = ux^2 + vy^2 + ux vy + 1/4 (uy+vx)^2
 *     + 1/4 uz^2 + 1/4 vz^2;  mu = k_c (eps_e^2 + delta)^((1-n)/(2n)); n = 3.
 *   - stresses exactly as Fig. 2; body force f = rho_g grad s_h
 *     with sign + (eq. (1); Z6), or a caller-given force_qp.
 *   - residual (Fig. 2):
 *       R[n][a] = sum_q wM_q (sum_d sigma_(a,d) GradBF[n][q][d] + f_a BF[n][q])
 *   - Jacobian J[(i,a),(j,b)] = dR_cell[i][a] / dU_cell[j][b] including
 *     d mu / dU (full Newton, Z5); row-major [2N][2N], row = 2i+a, col = 2j+b.
 *
 * Memory and ownership:
 *   - The caller owns ALL device memory (e.g. torch tensors via data_ptr()),
 *     including the workspace.  The library never calls cudaMalloc.
 *   - The ctx is a host object freed by stokesfo_destroy.  desc arrays (conn,
 *     coords, surface, force_qp, flow_factor) must stay valid and unchanged
 *     while the ctx lives (stokesfo_create snapshots geometry, conn and the
 *     flow factor into the workspace; surface and force_qp are re-read at
 *     every evaluation).
 *   - Every device pointer must be 16-byte aligned (workspace: 256-byte),
 *     otherwise EINVAL.
 *
 * Errors and execution:
 *   - Functions return stokesfo_status_t codes; no exception crosses the ABI.
 *   - Every call is asynchronous on desc.stream.  Device-side errors (det J <= 0,
 *     conn out of range, CSR entry missing) set a sticky flag in the workspace
 *     that stokesfo_sync reports as STOKESFO_EMESH.
 *   - glen_n != 3 returns STOKESFO_EUNSUPPORTED (the CPU oracle supports any n).
 *   - Element outputs (mu_qp, R_cell, J_cell, U_cell) are overwritten; global
 *     outputs (R, csr_vals) are accumulated (+=): the caller zeroes them.
 *   - A ctx is not thread-safe; distinct ctxs are independent.
 */
#ifndef STOKESFO_H
#define STOKESFO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define STOKESFO_ABI_VERSION 1

typedef struct stokesfo_ctx stokesfo_ctx; /* opaque host object */

typedef enum { STOKESFO_HEX8 = 0, STOKESFO_WEDGE6 = 1 } stokesfo_elem_t;

/* Where GradBF = J^-T grad_xi phi and wMeasure = w det J (eq. (3) inputs
 * {phi_i}, {grad phi_i}) come from during an evaluation:
 *   STORED:     precomputed once by stokesfo_create and streamed
 *               from the workspace at every evaluation (1,640 B/cell hex8);
 *   ON_THE_FLY: recomputed per tile from the gathered node coordinates inside
 *               the evaluation kernels (40 streamed B/cell hex8; det J <= 0 is
 *               re-checked at every evaluation).
 *   COMPACT:    precomputed once by stokesfo_create as A_q = J_q^-T and wMeasure
 *               (680 B/cell hex8, 515 B/cell wedge6) and streamed at every
 *               evaluation, which forms GradBF = A_q grad_xi phi_n in registers.
 * All give the same results up to rounding (parity-tested at 1e-12). */
typedef enum {
    STOKESFO_GEOMETRY_STORED = 0,
    STOKESFO_GEOMETRY_ON_THE_FLY = 1,
    STOKESFO_GEOMETRY_COMPACT = 2
} stokesfo_geometry_mode_t;

typedef enum {
    STOKESFO_OK = 0,
    STOKESFO_EINVAL = 1,       /* bad argument, size or alignment */
    STOKESFO_EMESH = 2,        /* det J <= 0, conn out of range, CSR entry missing */
    STOKESFO_ECUDA = 3,        /* a CUDA runtime error */
    STOKESFO_ENOMEM = 4,       /* workspace too small */
    STOKESFO_EUNSUPPORTED = 5, /* e.g. glen_n != 3 */
    STOKESFO_ENONFINITE = 6    /* NaN / Inf in an output (only with STOKESFO_CHECK_FINITE=1) */
} stokesfo_status_t;

typedef struct {
    uint32_t abi_version;        /* = STOKESFO_ABI_VERSION */
    int32_t elem;                /* stokesfo_elem_t */
    int64_t num_cells;           /* C, local to this device (may be 0) */
    int64_t num_nodes;           /* local to this device */
    const int32_t *conn;         /* dev [C][N] local node ids, N = 8 (hex8) / 6 (wedge6) */
    const double *coords;        /* dev [num_nodes][3] (x, y, z) */
    const double *surface;       /* dev [num_nodes] surface height s, or NULL */
    const double *force_qp;      /* dev [C][Q][2] body force at QPs, or NULL; overrides surface */
    const double *flow_factor;   /* dev [C] k_c = A_c^(-1/n)/2, or NULL (then scalar k) */
    double k;                    /* Glen prefactor used when flow_factor == NULL */
    double glen_n;               /* Glen exponent; must be 3 */
    double delta;                /* regularisation of eps_e^2 (Z3), > 0 */
    double rho_g;                /* rho * g multiplying grad s_h */
    void *workspace;             /* dev, caller-owned, >= stokesfo_workspace_size() bytes */
    size_t workspace_bytes;
    void *stream;                /* cudaStream_t used by every call (NULL = legacy default) */
    int32_t geometry_mode;       /* stokesfo_geometry_mode_t */
    int32_t reserved0;
} stokesfo_desc_t;

/* Bytes of workspace needed for desc (reads elem, num_cells, num_nodes and
 * geometry_mode). */
int stokesfo_workspace_size(const stokesfo_desc_t *d, size_t *bytes);

/* Validate desc and run the basis/quadrature precompute:
 * GradBF[c][n][q][:] = J_q^-T grad_xi phi_n(xi_q), wMeasure[c][q] = w_q det J_q
 * into the workspace (STORED mode; ON_THE_FLY mode stores node coordinates
 * instead and checks det J), plus a snapshot of conn and the flow factor.
 * Synchronises desc.stream once: a conn entry outside [0, num_nodes) returns
 * STOKESFO_EMESH here (no ctx is created), so no evaluation ever uses an
 * out-of-range conn as an address (conn must not change while the ctx lives);
 * det J <= 0 sets the sticky flag reported by stokesfo_sync. */
int stokesfo_create(const stokesfo_desc_t *d, stokesfo_ctx **out);

/* Gather: U_cell[c][n][a] = U[2 conn[c][n] + a].
 * U: dev [num_nodes][2]; U_cell: dev [C][N][2] (overwritten). */
int stokesfo_gather(stokesfo_ctx *c, const double *U, double *U_cell);

/* Residual evaluation, fused gather -> Ugrad -> mu -> stress -> QP sum ->
 * scatter (Fig. 2).  U: dev [num_nodes][2].  Optional
 * outputs (NULL to skip): mu_qp [C][Q] (overwritten), R_cell [C][N][2]
 * (overwritten), R [num_nodes][2] (+=). */
int stokesfo_viscosity_resid(stokesfo_ctx *c, const double *U, double *mu_qp, double *R_cell,
                             double *R);

/* Residual + forward-AD Jacobian in one pass.
 * J_cell: dev [C][2N][2N] row-major (required, overwritten); R_cell, R optional
 * as above. */
int stokesfo_jacobian(stokesfo_ctx *c, const double *U, double *J_cell, double *R_cell, double *R);

/* Matrix-free Jacobian-vector product (NEXT-3, Newton-Krylov operator apply):
 * Y += J(U) X with J = dR/dU assembled over all cells, computed as the forward
 * directional derivative of the fused chain along X (no element matrices are
 * formed); optionally R += R(U) in the same pass.  U, X: dev [num_nodes][2];
 * Y, R: dev [num_nodes][2] (+=).  With a peer table attached
 * (stokesfo_set_remote), Y is halo-summed like R and needs the peers' Y
 * pointers (stokesfo_set_remote_jvp), else EINVAL. */
int stokesfo_jvp(stokesfo_ctx *c, const double *U, const double *X, double *Y, double *R);

/* Diagonal of the assembled Jacobian (NEXT-3, the Jacobi preconditioner of the
 * Newton-Krylov driver): diag[2 node + a] += sum over the cells holding the node
 * of J_cell[(i,a),(i,a)] (the same forward derivative as stokesfo_jacobian,
 * P:L215-221; no element matrices are formed), optionally R += R(U) in the same
 * pass.  U: dev [num_nodes][2]; diag, R: dev [num_nodes][2] (+=).  With a peer
 * table attached it is halo-summed like stokesfo_jvp's Y (needs
 * stokesfo_set_remote_jvp, else EINVAL). */
int stokesfo_jacobian_diag(stokesfo_ctx *c, const double *U, double *diag, double *R);

/* Basal friction side-set term (NEXT-4; P:L59 -> [24]; reading Z18):
 * on the bottom face of each listed basal cell (local nodes 0..3 hex8 /
 * 0..2 wedge6), R[2 node_i + a] += int beta_h u_h,a phi_i dGamma and
 * J_face[f][(i,a)][(j,b)] = delta_ab int beta_h phi_i phi_j dGamma (row-major
 * [2NB][2NB], NB = 4 / 3; optional).  basal_cells: dev int32 [nfaces] cell
 * ids; beta: dev [num_nodes] friction coefficient; U, R: dev [num_nodes][2]. */
int stokesfo_basal_friction(stokesfo_ctx *c, const int32_t *basal_cells, int64_t nfaces, const double *beta,
                            const double *U, double *R, double *J_face);

/* Lateral (calving-front / ocean) pressure side-set term (NEXT-4; P:L59 ->
 * [24]; reading Z19).  On each listed lateral face -- the quad of
 * cell `cell` over its footprint polygon side k (local nodes k, k+1, k+1+P,
 * k+P; P = 4 hex8 / 3 wedge6, indices mod P; xi along the side, eta upward) --
 *     R[2 node_i + a] -= int psi(z) n_a phi_i dGamma,  a = 0, 1,
 *     psi(z) = rho_i_g (s_h - z) - rho_w_g max(sea_level - z, 0),
 * with 2x2 Gauss, n dGamma = dx/dxi x dx/deta (outward for counter-clockwise
 * footprint polygons) and s_h, z interpolated with the bilinear face basis.
 * The term does not depend on U (no Jacobian contribution).  faces: dev int32
 * [nfaces][2] = (cell, side), 8-B aligned (stokesfo_mesh_lateral_faces builds
 * the footprint boundary's list); surface: dev [num_nodes] s; R: dev
 * [num_nodes][2] (+=).  A side outside [0, P) or a cell outside [0, C) raises
 * the sticky EMESH flag. */
int stokesfo_lateral_pressure(stokesfo_ctx *c, const int32_t *faces, int64_t nfaces, const double *surface,
                              double rho_i_g, double rho_w_g, double sea_level, double *R);

/* Attach the lateral pressure term (same arguments as stokesfo_lateral_pressure,
 * minus R) to the ctx so that stokesfo_newton_solve solves
 * F = R_visc + R_basal + R_lateral = 0 (the term is U-independent: it enters F,
 * not J).  The arrays stay caller-owned and must outlive the solve;
 * nfaces = 0 detaches. */
int stokesfo_set_lateral(stokesfo_ctx *c, const int32_t *faces, int64_t nfaces, const double *surface,
                         double rho_i_g, double rho_w_g, double sea_level);

/* Assembly: the sum over cells of eq. (3)
 * into the global residual and into the global Jacobian matrix that the damped
 * Newton method computes at each nonlinear iteration and hands to GMRES with a
 * matrix-dependent AMG preconditioner (section III-A).
 * R[2 conn[c][n] + a] += R_cell[c][n][a] (if R_cell and R are non-NULL)
 * and csr_vals[pos(row, col)] += J_cell[c][k][l] (if J_cell and csr_vals are
 * non-NULL; requires an earlier stokesfo_csr_pattern call with non-NULL rowptr
 * and colidx, which must stay valid). */
int stokesfo_scatter_assemble(stokesfo_ctx *c, const double *R_cell, double *R,
                              const double *J_cell, double *csr_vals);

/* NEXT-2 global matrix from element matrices with the atomic-free pull
 * assembly (requires stokesfo_csr_slots; nodes with at most 64 neighbour nodes,
 * else EUNSUPPORTED): a warp owns a node's two CSR rows and sums the rows of
 * every incident cell's J_cell in ascending cell order (bitwise reproducible).
 * accumulate != 0: csr_vals += assembled J (as stokesfo_scatter_assemble);
 * accumulate == 0: csr_vals = assembled J -- every entry of the pattern is
 * written, so the caller needs no zeroing pass and the kernel never reads
 * csr_vals (15 GB less traffic per C4 fill).  J_cell: dev [C][2N][2N];
 * csr_vals: dev [nnz]. */
int stokesfo_assemble_csr(stokesfo_ctx *c, const double *J_cell, double *csr_vals, int accumulate);

/* NEXT-2 element Jacobians in symmetric block-packed form.  The element tangent
 * is the Hessian of the cell's quadrature energy sum_q wM Psi(eps_e^2) (Glen's law
 * is a potential flow law; section III-A; reading Z5), so
 * J_cell[c] is symmetric and its N(N+1)/2 upper 2 x 2 node blocks determine it:
 * Jp dev [C][N(N+1)/2][2][2], block (i, j >= i) at index i N - i (i - 1) / 2 +
 * (j - i), entries [a][b] = J[(i,a),(j,b)] (hex8 1,152 B per cell instead of
 * 2,048; wedge6 672 instead of 1,152).  Jp must be 32-B aligned.  R_cell and R
 * as stokesfo_jacobian.  Written by the fp64 tensor-core kernels (every
 * geometry mode): STOKESFO_JAC_MMA=0 at create returns EUNSUPPORTED. */
int stokesfo_jacobian_packed(stokesfo_ctx *c, const double *U, double *Jp, double *R_cell, double *R);

/* stokesfo_assemble_csr from the packed form: row (i, a) of cell c is block
 * (i, j) for j >= i and the transpose of block (j, i) for j < i.  Jp dev
 * [C][N(N+1)/2][2][2]; otherwise the same requirements, ordering and
 * accumulate semantics as stokesfo_assemble_csr. */
int stokesfo_assemble_csr_packed(stokesfo_ctx *c, const double *Jp, double *csr_vals, int accumulate);

/* CSR pattern of the global Jacobian matrix (NEXT-2; section III-A:
 * computed at each nonlinear iteration, used by the matrix-dependent AMG) over dofs
 * (rows = 2*num_nodes; columns of a row = sorted dofs of
 * every node sharing a cell with the row's node).  Size query: pass rowptr =
 * colidx = NULL to get *nnz.  Fill: rowptr dev [2*num_nodes+1] int64, colidx
 * dev [nnz] int32.  Synchronises the stream (host-side construction from a
 * copy of conn; an entry outside [0, num_nodes) returns EMESH). */
int stokesfo_csr_pattern(stokesfo_ctx *c, int64_t *nnz, int64_t *rowptr, int32_t *colidx);

/* NEXT-2 per-cell CSR slots: slot[c][i][j] (uint8, j = 0..N-1, byte j of the
 * uint64 slots[c*N + i]) = index of node conn[c][j] in the sorted neighbour-node
 * list of node conn[c][i], so that J_cell[c][(i,a)][(j,b)] lands at
 * csr_vals[rowptr[2 conn[c][i] + a] + 2 slot + b].  Requires an earlier
 * stokesfo_csr_pattern fill (rowptr 16-B aligned); computed on the device once
 * (binary searches in colidx) into caller-owned slots: dev uint64 [C][N]
 * followed by the node -> cell incidence and a record per node for the pull
 * assembly (row base, lengths, the first 8 (hex8) / 12 (wedge6) incident
 * cells and their slot rows: one coalesced load per node; 128 / 256 B) --
 * stokesfo_csr_slots_size bytes in all,
 * 16-B aligned, must stay valid.  Attaches
 * the table to the ctx: stokesfo_scatter_assemble then uses it instead of
 * per-entry searches, and stokesfo_jacobian_csr becomes available.  A node
 * with more than 256 neighbour nodes returns EUNSUPPORTED; a missing entry
 * raises the sticky EMESH flag.  A new stokesfo_csr_pattern fill detaches it. */
int stokesfo_csr_slots_size(stokesfo_ctx *c, size_t *bytes);
int stokesfo_csr_slots(stokesfo_ctx *c, uint64_t *slots);

/* NEXT-2 fused: residual + forward-AD Jacobian assembled straight into the
 * global CSR matrix in one pass (no element matrices in HBM; Albany's
 * ScatterResidual into a CrsMatrix): csr_vals[...] += every
 * cell's J contributions (red.global.add.f64 through the slot table), R += the
 * residual (optional).  Requires stokesfo_csr_slots.  csr_vals: dev [nnz]
 * (+=); U, R: dev [num_nodes][2].  Summation order is unspecified (atomics). */
int stokesfo_jacobian_csr(stokesfo_ctx *c, const double *U, double *csr_vals, double *R);

/* Export the precomputed geometry in the canonical layout:
 * grad_bf dev [C][N][Q][3], w_measure dev [C][Q] (either may be NULL). */
int stokesfo_geometry(stokesfo_ctx *c, double *grad_bf, double *w_measure);

/* Multi-GPU halo sum.  pack: buf[k][a] = R[2 send_nodes[k] + a];
 * unpack_add: R[2 recv_nodes[k] + a] += buf[k][a].  Node lists are local ids,
 * unique within a list; buf is dev [n][2]. */
int stokesfo_halo_pack(stokesfo_ctx *c, const double *R, const int32_t *send_nodes, int64_t n,
                       double *buf);
int stokesfo_halo_unpack_add(stokesfo_ctx *c, const double *buf, const int32_t *recv_nodes,
                             int64_t n, double *R);

/* Fused halo sum over peer memory: after
 * this call, the residual scatter of stokesfo_viscosity_resid / _jacobian /
 * _jvp (and the R part of stokesfo_scatter_assemble) also adds every contribution to a partition-boundary node into the R
 * of each other GPU holding that node, with atomics through NVLink-mapped
 * peer pointers, so no pack / exchange / unpack is needed (one stream-ordered
 * barrier per evaluation; R passed to the calls must be the buffer the peers
 * mapped).  rem: dev int32 [num_nodes], row of remtab or -1; remtab: dev int32
 * [rows][15] = {count <= 7, peer, remote_local_index, ...}; peers: dev array of
 * device pointers (one per peer index; entries for this rank unused).  All
 * stay owned by the caller and must outlive their use; rem = NULL detaches. */
int stokesfo_set_remote(stokesfo_ctx *c, const int32_t *rem, const int32_t *remtab, double *const *peers);
/* The peers' J.v output buffers for stokesfo_jvp under the same node table:
 * peers_y: dev array of device pointers (one per peer index), caller-owned;
 * requires stokesfo_set_remote first (else EINVAL); NULL detaches (jvp then
 * returns EINVAL while the table is attached).  stokesfo_set_remote(NULL)
 * detaches both. */
int stokesfo_set_remote_jvp(stokesfo_ctx *c, double *const *peers_y);
/* CUDA IPC plumbing for the above (handle = 64 opaque bytes).  A handle maps
 * the whole allocation containing dev_ptr; *offset = dev_ptr - allocation
 * base, to add to the pointer the peer obtains from stokesfo_ipc_open_handle. */
int stokesfo_ipc_get_handle(const void *dev_ptr, void *handle, int64_t *offset);
int stokesfo_ipc_open_handle(const void *handle, void **dev_ptr);
int stokesfo_ipc_close(void *dev_ptr);

/* Failure detection: with the environment variable STOKESFO_CHECK_FINITE=1 set
 * when the ctx is created, viscosity_resid / jacobian / jvp / jacobian_diag scan
 * the outputs they wrote for NaN / Inf (one extra read of each output) and raise
 * a sticky flag that stokesfo_sync reports as STOKESFO_ENONFINITE. */

/* Synchronise the ctx stream; returns ECUDA on a CUDA error, else EMESH if a
 * mesh error flag (det J <= 0, conn out of range, CSR entry missing) was raised
 * since create, else ENONFINITE if the finite check flagged an output, else OK. */
int stokesfo_sync(stokesfo_ctx *c);

/* Static string for a status code. */
const char *stokesfo_strerror(int status);

void stokesfo_destroy(stokesfo_ctx *c);

/* Launch/tiling facts for measurement (kernels launched per evaluation call,
 * cells per tile, grid size).  Any pointer may be NULL. */
int stokesfo_launch_info(stokesfo_ctx *c, int32_t *cells_per_tile, int32_t *grid_resid,
                         int32_t *grid_jac, int64_t *record_bytes_per_tile);

/* ---------------- NEXT-3: damped Newton-Krylov driver ---------------------- */

/* Solves F(U) = R_visc(U) + R_basal(U) [+ R_lateral, see stokesfo_set_lateral] = 0
 * (damped Newton, Jacobian at
 * every nonlinear step): per step, J dU = -F by Jacobi-preconditioned CG on the
 * matrix-free operator stokesfo_jvp + basal face term (J is SPD once basal
 * friction removes the rigid null space; Jacobi diagonal from
 * stokesfo_jacobian_diag and the basal face matrices), then Armijo backtracking
 * on ||F||.  The CG scalars stay on the device and blocks of 8 CG iterations are
 * replayed as one CUDA graph on a stream the solve creates (ordered after the
 * ctx stream's prior work and before its later work); convergence is checked
 * once per block.  Stops when ||F|| <= max(atol, rtol ||F_0||) or after
 * max_newton steps.  Single-GPU ctx (a ctx with stokesfo_set_remote attached
 * returns EINVAL).  Synchronous.  U: dev [num_nodes][2], initial guess in,
 * solution out.  work: dev, stokesfo_newton_work_size bytes, 256-B aligned.
 * hist_F: host [max_newton + 1] ||F|| per step; hist_cg: host [max_newton] CG
 * iterations to reach rtol_cg per step (the block may run up to 7 more, which
 * only refine the step; may be NULL); *iters = Newton steps taken. */
typedef struct {
    int32_t max_newton;   /* e.g. 8 */
    int32_t max_cg;       /* CG iterations per Newton step */
    int32_t max_ls;       /* backtracking halvings */
    int32_t reserved;
    double rtol_newton;   /* on ||F|| / ||F_0|| */
    double atol_newton;
    double rtol_cg;       /* linear solve ||r|| <= rtol_cg ||F|| (1e-6) */
    double ls_c;          /* Armijo constant, e.g. 1e-4 */
} stokesfo_newton_opts_t;
int stokesfo_newton_work_size(stokesfo_ctx *c, int64_t nbasal, size_t *bytes);
int stokesfo_newton_solve(stokesfo_ctx *c, const int32_t *basal_cells, int64_t nbasal, const double *beta,
                          double *U, void *work, const stokesfo_newton_opts_t *opts, double *hist_F,
                          int32_t *hist_cg, int32_t *iters);

/* ---------------- NEXT-1: the paper's evaluator chain on B200 -------------- */

/* Albany's unfused chain (SURVEY CS-1) with HBM intermediates, to reproduce
 * the paper's baseline-vs-optimized experiment (Table III/IV) on
 * B200:  GatherSolution -> DOFVecGradInterpolation (Ugrad) -> ViscosityFO
 * (muLandIce) -> StokesFOBodyForce (force) -> StokesFOResid (Fig. 2) ->
 * Residual.  derivs = 0: ScalarT = double (the Residual kernel); derivs = 1:
 * ScalarT = value + 2N derivative lanes, Sacado SFad<double,2N> (the Jacobian
 * kernel).  All intermediates live in a caller-owned device
 * scratch of stokesfo_albany_scratch_size bytes, component-major with the cell
 * index fastest (thread-per-cell kernels read coalesced).  The chain derives
 * the force from desc.surface (force_qp is EUNSUPPORTED here).  Results equal
 * stokesfo_viscosity_resid / stokesfo_jacobian up to rounding (parity-tested). */
typedef enum { STOKESFO_FIG2_BASELINE = 0, STOKESFO_FIG2_OPTIMIZED = 1 } stokesfo_fig2_variant_t;
int stokesfo_albany_scratch_size(stokesfo_ctx *c, int derivs, size_t *bytes);
/* GradBF, wGradBF = GradBF wM, wBF = BF wM into the scratch (once per mesh). */
int stokesfo_albany_setup(stokesfo_ctx *c, int derivs, double *scratch);
/* Gather (seeded), Ugrad, muLandIce, force into the scratch. U: dev [nodes][2]. */
int stokesfo_albany_evaluators(stokesfo_ctx *c, int derivs, const double *U, double *scratch);
/* StokesFOResid, Fig. 2 left (BASELINE: global accumulation, two QP passes) or
 * right column (OPTIMIZED: fused loop, local res0/res1, single store). */
int stokesfo_albany_resid(stokesfo_ctx *c, int derivs, int variant, double *scratch);
/* Residual -> R_cell [C][N][2] (opt) and, for derivs = 1, J_cell [C][2N][2N] (opt). */
int stokesfo_albany_extract(stokesfo_ctx *c, int derivs, const double *scratch, double *R_cell, double *J_cell);

/* ---------------- host-side mesh construction (no GPU needed) ------------- */

/* Extrude a footprint by L uniform-sigma layers:
 *   node(v,k) = v*(L+1)+k (k = 0 bed .. L surface); cell(f,k) = f*L+k;
 *   conn[cell] = [poly verts at level k, same at level k+1];
 *   coords[node] = (x_v, y_v, b_v + H_v * (k/L)).
 * Host arrays: xy [nv][2], polys [nf][npoly] (npoly = 4 -> hex8, 3 -> wedge6),
 * b, H [nv]; outputs conn [nf*L][2*npoly], coords [nv*(L+1)][3]. */
int stokesfo_mesh_extrude(int32_t npoly, int64_t nv, const double *xy, int64_t nf,
                          const int32_t *polys, const double *b, const double *H, int32_t L,
                          int32_t *conn, double *coords);

/* Column partition into nparts contiguous equal-count ranges:
 * part r owns columns [ranges[r], ranges[r+1]), ranges[r] = floor(r*nf/nparts). */
int stokesfo_mesh_partition_columns(int64_t nf, int32_t nparts, int64_t *ranges);

/* Localise the cells of one part: local node ids are the ranks of the touched
 * global ids in ascending order.  conn_global: host [ncells][npc].  Size query
 * with gids == NULL (sets *num_local_nodes); fill gids [num_local_nodes] and
 * conn_local [ncells][npc]. */
int stokesfo_mesh_localize(int32_t npc, int64_t ncells, const int32_t *conn_global,
                           int64_t *num_local_nodes, int64_t *gids, int32_t *conn_local);

/* Halo list of "mine" w.r.t. "other": local ids (in mine) of the global ids the
 * two sorted lists share, ordered by global id.  Size query with idx == NULL. */
int stokesfo_mesh_halo_list(int64_t n_mine, const int64_t *gids_mine, int64_t n_other,
                            const int64_t *gids_other, int64_t *n_shared, int32_t *idx);

/* Lateral faces of the extruded mesh: every footprint polygon side whose edge
 * belongs to exactly one polygon (the footprint boundary), times the L layers:
 * faces[m] = (cell f L + l, side k), ordered by (f, k, l).  polys: host
 * [nf][npoly].  Size query with faces == NULL (sets *nfaces); fill faces host
 * int32 [nfaces][2]. */
int stokesfo_mesh_lateral_faces(int32_t npoly, int64_t nf, const int32_t *polys, int32_t L, int64_t *nfaces,
                                int32_t *faces);

#ifdef __cplusplus
}
#endif
#endif /* STOKESFO_H */
