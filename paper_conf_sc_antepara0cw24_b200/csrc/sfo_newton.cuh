// sfo_newton.cuh -- NEXT-3: a damped Newton-Krylov driver consuming the fused
// evaluators ("A damped Newton's method solves the nonlinear
// system where a Jacobian matrix is computed at each nonlinear iteration").
//
// F(U) = R_visc(U) (+ body force) + R_basal(U) (stokesfo_viscosity_resid +
// stokesfo_basal_friction); each Newton step solves J dU = -F with Jacobi-
// preconditioned CG on the matrix-free operator J v = stokesfo_jvp(U; v) +
// R_basal(v) (the basal term is linear in U), the Jacobi diagonal coming from
// the element Jacobians (stokesfo_jacobian) and the basal face matrices; then
// Armijo backtracking on ||F||.  J is symmetric positive definite once basal
// friction removes the rigid null space.  Host loop in C++, vector algebra in
// the small kernels below; the evaluator kernels are the product's own.
#pragma once
#include "sfo_common.cuh"

namespace sfo {
namespace newton {

// sum(x * y) -> *out (out zeroed by the caller); grid-stride, warp + block reduce
__global__ void dot_kernel(int64_t n, const double *__restrict__ x, const double *__restrict__ y,
                           double *__restrict__ out) {
    __shared__ double part[32];
    double acc = 0.0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        acc = fma(x[i], y[i], acc);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = acc;
    __syncthreads();
    if (threadIdx.x < 32) {
        acc = threadIdx.x < (blockDim.x >> 5) ? part[threadIdx.x] : 0.0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
        if (threadIdx.x == 0) atomicAdd(out, acc);
    }
}

// y = a x + b y
__global__ void axpby_kernel(int64_t n, double a, const double *__restrict__ x, double b, double *__restrict__ y) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        y[i] = fma(a, x[i], b * y[i]);
}

// z = r / d (Jacobi)
__global__ void jacobi_kernel(int64_t n, const double *__restrict__ r, const double *__restrict__ d,
                             double *__restrict__ z) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        z[i] = r[i] / d[i];
}

// diag[dof(c, r)] += J_cell[c][r][r]
template <int N>
__global__ void diag_cells_kernel(int64_t C, const int32_t *__restrict__ conn, const double *__restrict__ J,
                                  double *__restrict__ diag) {
    constexpr int ND = 2 * N;
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (gid >= C * ND) return;
    const int64_t c = gid / ND;
    const int r = (int)(gid % ND);
    atomicAdd(diag + 2 * (int64_t)conn[c * N + r / 2] + (r & 1), J[(c * ND + r) * ND + r]);
}

// diag[dof] += J_face[f][r][r] (bottom face nodes 0..NB-1 of the basal cell)
template <int N>
__global__ void diag_faces_kernel(int64_t nf, const int32_t *__restrict__ cells, const int32_t *__restrict__ conn,
                                  const double *__restrict__ Jf, double *__restrict__ diag) {
    constexpr int NB = N / 2, ND = 2 * NB;
    const int64_t gid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (gid >= nf * ND) return;
    const int64_t f = gid / ND;
    const int r = (int)(gid % ND);
    atomicAdd(diag + 2 * (int64_t)conn[(int64_t)cells[f] * N + r / 2] + (r & 1), Jf[(f * ND + r) * ND + r]);
}

}  // namespace newton
}  // namespace sfo
