// sfo_newton.cuh -- NEXT-3: a damped Newton-Krylov driver consuming the fused
// evaluators ("A damped Newton's method solves the nonlinear
// system where a Jacobian matrix is computed at each nonlinear iteration").
//
// F(U) = R_visc(U) (+ body force) + R_basal(U) (stokesfo_viscosity_resid +
// stokesfo_basal_friction); each Newton step solves J dU = -F with Jacobi-
// preconditioned CG on the matrix-free operator J v = stokesfo_jvp(U; v) +
// R_basal(v) (the basal term is linear in U), the Jacobi diagonal coming from
// the diagonal-only evaluation (stokesfo_jacobian_diag) and the basal face
// matrices; then Armijo backtracking on ||F||.  J is symmetric positive
// definite once basal friction removes the rigid null space.  Host loop in
// C++; the CG scalars stay on the device and blocks of CG iterations replay
// as one CUDA graph; vector algebra in the small kernels below, the evaluator
// kernels are the product's own.
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

// CG scalars live on the device (slots of `s`), so a block of CG iterations runs
// without host round trips and is captured once into a CUDA graph:
//   s[RZ] = r.z, s[PAP] = p.Ap, s[RR] = r.r, s[RZN] = new r.z, s[ALPHA], s[BETA]
enum { S_RZ = 0, S_PAP = 1, S_RR = 2, S_RZN = 3, S_ALPHA = 4, S_BETA = 5, S_IT = 6, S_SLOTS = 8 };

// alpha = r.z / p.Ap (0 once the iteration has converged to p.Ap = 0: a no-op step)
__global__ void cg_alpha_kernel(double *s) {
    const double pap = s[S_PAP];
    s[S_ALPHA] = (pap != 0.0 && isfinite(pap)) ? s[S_RZ] / pap : 0.0;
}
// beta = r.z_new / r.z; r.z <- r.z_new; hist[it] = r.r (the block's residual history)
__global__ void cg_beta_kernel(double *s, double *hist) {
    const double rz = s[S_RZ];
    s[S_BETA] = (rz != 0.0 && isfinite(rz)) ? s[S_RZN] / rz : 0.0;
    s[S_RZ] = s[S_RZN];
    const int it = (int)s[S_IT];
    hist[it] = s[S_RR];
    s[S_IT] = it + 1;
}
// y += sign * (*a) * x
__global__ void axpy_dev_kernel(int64_t n, const double *__restrict__ a, double sign, const double *__restrict__ x,
                                double *__restrict__ y) {
    const double al = sign * *a;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        y[i] = fma(al, x[i], y[i]);
}
// y = x + (*b) y
__global__ void xpby_dev_kernel(int64_t n, const double *__restrict__ x, const double *__restrict__ b,
                                double *__restrict__ y) {
    const double be = *b;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        y[i] = fma(be, y[i], x[i]);
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
