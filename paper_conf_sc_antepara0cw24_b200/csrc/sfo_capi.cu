// sfo_capi.cu -- extern "C" entry points of libstokesfo.so (include/stokesfo.h).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <vector>

#include <nvtx3/nvToolsExt.h>  // header-only NVTX3 (no link dependency; inert without a tool attached)

#include "../../include/stokesfo.h"
#include "sfo_kernels.cuh"
#include "sfo_albany.cuh"
#include "sfo_newton.cuh"

using namespace sfo;

struct stokesfo_ctx {
    stokesfo_desc_t d;
    cudaStream_t stream;
    int N, Q, TC;
    int64_t ntiles;
    int *err;              // device flag in the workspace header
    char *recs;            // device records (full or light)
    double4 *xyz4;         // node coordinates (on-the-fly geometry mode)
    int mode;              // stokesfo_geometry_mode_t
    int grid_resid, grid_jac, grid_jvp, grid_csr, grid_diag;
    int rec_bytes;
    int nstage_resid, nstage_jac;  // TMA record ring depth of the eval kernels
    const int32_t *rem = nullptr;     // fused halo over peer memory (stokesfo_set_remote)
    const int32_t *remtab = nullptr;
    double *const *peers = nullptr;
    double *const *peers_y = nullptr;  // the peers' J.v outputs (stokesfo_set_remote_jvp)
    const int64_t *rowptr = nullptr;  // CSR pattern (set by stokesfo_csr_pattern)
    const int32_t *colidx = nullptr;
    int64_t csr_rows = 0;
    int64_t csr_maxdeg = 0;            // max neighbour nodes of a node (slots are uint8)
    const uint64_t *slots = nullptr;   // per-cell CSR slots (set by stokesfo_csr_slots)
    const int64_t *inc_ptr = nullptr;  // node -> (cell N + i) incidence on the device (in the slots buffer)
    const int32_t *inc = nullptr;
    const uint64_t *nrec = nullptr;    // per-node pull records (in the slots buffer; csr_gather_kernel)
    std::vector<int64_t> inc_ptr_h;    // host incidence from the last csr_pattern fill (until csr_slots)
    std::vector<int32_t> inc_h;
    // lateral pressure term attached for the Newton driver (stokesfo_set_lateral)
    const int32_t *lat_faces = nullptr;
    int64_t lat_n = 0;
    const double *lat_surface = nullptr;
    double lat_rho_i_g = 0.0, lat_rho_w_g = 0.0, lat_sea = 0.0;
    // wedge6 element-Jacobian tensor map (TMA 2-D store of a padded tile), re-encoded when J_cell moves
    CUtensorMap jmap;
    const double *jmap_ptr = nullptr;
    bool jmap_ok = false;
    bool check_finite = false;  // STOKESFO_CHECK_FINITE=1 at create: scan outputs for NaN / Inf
    bool jac_mma = false;       // Jacobian on the fp64 tensor cores (eval_mma_kernel / eval_compact_mma_kernel)
    bool mma_ok = false;        // the DMMA kernels are configured (stokesfo_jacobian_packed)
    int grid_mma = 0;           // their persistent grid
};

namespace {

// NVTX range around every C-ABI entry point when STOKESFO_PROFILE=1 (nsys / ncu --nvtx
// timelines of a multi-rank step); a no-op otherwise.
bool profile_on() {
    static const bool on = [] {
        const char *e = getenv("STOKESFO_PROFILE");
        return e && atoi(e) == 1;
    }();
    return on;
}
struct NvtxRange {
    bool on;
    explicit NvtxRange(const char *name) : on(profile_on()) {
        if (on) nvtxRangePushA(name);
    }
    ~NvtxRange() {
        if (on) nvtxRangePop();
    }
};
#define SFO_RANGE(name) NvtxRange sfo_nvtx_range_(name)

bool aligned(const void *p, size_t a) { return (reinterpret_cast<uintptr_t>(p) % a) == 0; }

// STOKESFO_CHECK_FINITE=1: scan an output (n doubles) for NaN / Inf after the call that wrote it
void check_finite(const stokesfo_ctx *c, const double *p, int64_t n) {
    if (!c->check_finite || !p || n <= 0) return;
    const int bs = 256;
    const unsigned g = (unsigned)std::min<int64_t>((n + bs - 1) / bs, 148 * 16);
    finite_check_kernel<<<g, bs, 0, c->stream>>>(n, p, c->err);
}

int cuda_status() {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        fprintf(stderr, "libstokesfo: CUDA error %s\n", cudaGetErrorString(e));
        return STOKESFO_ECUDA;
    }
    return STOKESFO_OK;
}

template <class E, bool JAC>
constexpr int default_stages() {
    return 2;
}

template <class E>
int64_t xyz4_bytes(int64_t nnodes) {
    return round_up(nnodes * 32, 256);
}

template <class E>
int64_t ws_bytes(int64_t ncells, int64_t nnodes, int mode) {
    const int64_t ntiles = (ncells + E::TC - 1) / E::TC;
    if (mode == STOKESFO_GEOMETRY_ON_THE_FLY) return WS_HEADER + xyz4_bytes<E>(nnodes);
    if (mode == STOKESFO_GEOMETRY_COMPACT) return WS_HEADER + ntiles * (int64_t)RecC<E>::BYTES;
    return WS_HEADER + ntiles * (int64_t)Rec<E>::BYTES;
}

template <class E, int MODE>
int configure_compact(int *grid) {
    auto fn = eval_compact_kernel<E, MODE>;
    constexpr int bytes = CompactSmem<E, MODE>::BYTES;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess)
        return cuda_status();
    int dev = 0, sms = 0, per_sm = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, 32, bytes) != cudaSuccess) return cuda_status();
    *grid = std::max(1, sms * std::max(1, per_sm));
    return STOKESFO_OK;
}

template <class E, int MODE>
int configure_otf(int *grid) {
    using S = OtfSmem<E, MODE>;
    auto fn = eval_otf_kernel<E, MODE>;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, S::BYTES) != cudaSuccess)
        return cuda_status();
    int dev = 0, sms = 0, per_sm = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, 32, S::BYTES) != cudaSuccess)
        return cuda_status();
    *grid = std::max(1, sms * std::max(1, per_sm));
    return STOKESFO_OK;
}

// Launch shape of eval_kernel: WPC independent warps per CTA, each with its own
// shared-memory slice (WPC = 1: exactly S::BYTES).
template <class E, int MODE, int NS>
constexpr int eval_smem_bytes() {
    using S = EvalSmem<E, MODE, NS>;
    return warps_per_cta<E, MODE>() == 1 ? S::BYTES : warps_per_cta<E, MODE>() * S::SLICE;
}

template <class E, int MODE, int NS>
int configure_eval(int *grid) {
    auto fn = eval_kernel<E, MODE, NS>;
    constexpr int bytes = eval_smem_bytes<E, MODE, NS>();
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess)
        return cuda_status();
    int dev = 0, sms = 0, per_sm = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, 32 * warps_per_cta<E, MODE>(), bytes) !=
        cudaSuccess)
        return cuda_status();
    *grid = std::max(1, sms * std::max(1, per_sm));
    return STOKESFO_OK;
}

template <class E>
int configure_mma(int *grid) {
    auto fn = eval_mma_kernel<E, 2>;
    constexpr int bytes = MmaSmem<E, 2>::BYTES;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess)
        return cuda_status();
    int dev = 0, sms = 0, per_sm = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, 32, bytes) != cudaSuccess) return cuda_status();
    *grid = std::max(1, sms * std::max(1, per_sm));
    return STOKESFO_OK;
}

template <class E>
int configure_compact_mma(int *grid) {
    auto fn = eval_compact_mma_kernel<E>;
    constexpr int bytes = CompactMmaSmem<E>::BYTES;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess)
        return cuda_status();
    int dev = 0, sms = 0, per_sm = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, 32, bytes) != cudaSuccess) return cuda_status();
    *grid = std::max(1, sms * std::max(1, per_sm));
    return STOKESFO_OK;
}

template <class E>
int configure_otf_mma(int *grid) {
    auto fn = eval_otf_mma_kernel<E>;
    constexpr int bytes = OtfMmaSmem<E>::BYTES;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess)
        return cuda_status();
    int dev = 0, sms = 0, per_sm = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, 32, bytes) != cudaSuccess) return cuda_status();
    *grid = std::max(1, sms * std::max(1, per_sm));
    return STOKESFO_OK;
}

// Element Jacobians on the fp64 tensor cores. STOKESFO_JAC_MMA unset: hex8 (the DMMA kernels cost the same per
// cell for both elements, which beats the vector kernel for hex8's 8 x 8 node blocks but not for wedge6's
// padded 6 x 6); 1: both elements; 0: neither (and no packed form). The DMMA kernels are configured
// unless 0: stokesfo_jacobian_packed always runs on them.
inline int jac_mma_env() {
    const char *e = getenv("STOKESFO_JAC_MMA");
    return e ? atoi(e) : -1;
}
template <class E>
bool want_jac_mma() {
    const int v = jac_mma_env();
    return v == 1 || (v < 0 && E::N == 8);
}

template <class E>
int create_impl(stokesfo_ctx *c) {
    c->N = E::N;
    c->Q = E::Q;
    c->TC = E::TC;
    c->ntiles = (c->d.num_cells + E::TC - 1) / E::TC;
    const bool otf = c->mode == STOKESFO_GEOMETRY_ON_THE_FLY;
    const bool compact = c->mode == STOKESFO_GEOMETRY_COMPACT;
    c->rec_bytes = otf ? 0 : (compact ? RecC<E>::BYTES : Rec<E>::BYTES);
    int st;
    if (compact) {
        c->nstage_resid = c->nstage_jac = 2;
        if ((st = configure_compact<E, M_RESID>(&c->grid_resid))) return st;
        if ((st = configure_compact<E, M_JAC>(&c->grid_jac))) return st;
        c->jac_mma = want_jac_mma<E>();
        c->mma_ok = jac_mma_env() != 0;
        if (c->mma_ok && (st = configure_compact_mma<E>(&c->grid_mma))) return st;
        if ((st = configure_compact<E, M_JVP>(&c->grid_jvp))) return st;
        if ((st = configure_compact<E, M_CSR>(&c->grid_csr))) return st;
        if ((st = configure_compact<E, M_DIAG>(&c->grid_diag))) return st;
    } else if (otf) {
        c->nstage_resid = c->nstage_jac = 0;
        st = configure_otf<E, M_RESID>(&c->grid_resid);
        if (st) return st;
        st = configure_otf<E, M_JAC>(&c->grid_jac);
        if (st) return st;
        st = configure_otf<E, M_JVP>(&c->grid_jvp);
        if (st) return st;
        st = configure_otf<E, M_CSR>(&c->grid_csr);
        if (st) return st;
        st = configure_otf<E, M_DIAG>(&c->grid_diag);
        if (st) return st;
        c->jac_mma = want_jac_mma<E>();
        c->mma_ok = jac_mma_env() != 0;
        if (c->mma_ok && (st = configure_otf_mma<E>(&c->grid_mma))) return st;
    } else {
        // ring depth: default per element, STOKESFO_STAGES_{RESID,JAC} override (2 or 3)
        c->nstage_resid = default_stages<E, false>();
        c->nstage_jac = default_stages<E, true>();
        if (const char *e = getenv("STOKESFO_STAGES_RESID")) c->nstage_resid = atoi(e) == 3 ? 3 : 2;
        if (const char *e = getenv("STOKESFO_STAGES_JAC")) c->nstage_jac = atoi(e) == 3 ? 3 : 2;
        st = c->nstage_resid == 3 ? configure_eval<E, M_RESID, 3>(&c->grid_resid)
                                  : configure_eval<E, M_RESID, 2>(&c->grid_resid);
        if (st) return st;
        st = c->nstage_jac == 3 ? configure_eval<E, M_JAC, 3>(&c->grid_jac)
                                : configure_eval<E, M_JAC, 2>(&c->grid_jac);
        if (st) return st;
        c->jac_mma = want_jac_mma<E>();
        c->mma_ok = jac_mma_env() != 0;
        if (c->mma_ok && (st = configure_mma<E>(&c->grid_mma))) return st;
        st = configure_eval<E, M_JVP, 2>(&c->grid_jvp);
        if (st) return st;
        st = configure_eval<E, M_CSR, 2>(&c->grid_csr);
        if (st) return st;
        st = configure_eval<E, M_DIAG, 2>(&c->grid_diag);
        if (st) return st;
    }
    if (cudaMemsetAsync(c->err, 0, sizeof(int), c->stream) != cudaSuccess) return cuda_status();
    if (c->ntiles > 0) {
        const int bs = 256;
        if (otf) {
            xyz4_kernel<<<(unsigned)((c->d.num_nodes + bs - 1) / bs), bs, 0, c->stream>>>(c->d.num_nodes, c->d.coords,
                                                                                          c->xyz4);
            const int64_t work = c->d.num_cells * E::Q;
            geometry_kernel<E, GEO_CHECK><<<(unsigned)((work + bs - 1) / bs), bs, 0, c->stream>>>(
                c->d.num_cells, c->d.num_nodes, c->d.conn, c->d.coords, nullptr, 0.0, nullptr, nullptr, nullptr,
                c->err);
        } else if (compact) {
            const int64_t work = c->ntiles * E::TC * E::Q;
            geometry_kernel<E, GEO_COMPACT><<<(unsigned)((work + bs - 1) / bs), bs, 0, c->stream>>>(
                c->d.num_cells, c->d.num_nodes, c->d.conn, c->d.coords, c->d.flow_factor, c->d.k, c->recs, nullptr,
                nullptr, c->err);
        } else {
            const int64_t work = c->ntiles * E::TC * E::Q;
            geometry_kernel<E, GEO_RECORDS><<<(unsigned)((work + bs - 1) / bs), bs, 0, c->stream>>>(
                c->d.num_cells, c->d.num_nodes, c->d.conn, c->d.coords, c->d.flow_factor, c->d.k, c->recs, nullptr,
                nullptr, c->err);
        }
    }
    return cuda_status();
}

// cuTensorMapEncodeTiled from the driver (no -lcuda link: fetched once through the runtime)
typedef CUresult (*encode_tiled_fn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                    const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
encode_tiled_fn tensor_map_encoder() {
    static encode_tiled_fn fn = [] {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            p = nullptr;
        cudaGetLastError();
        return reinterpret_cast<encode_tiled_fn>(p);
    }();
    return fn;
}

// J_cell as a 2-D tensor [C][NN] doubles, box (JPITCH x TC): one TMA store per
// tile writes the TC cells of a padded (odd-pitch) staging image; the padding
// columns and rows past C are outside the tensor.  STOKESFO_JMAP=0 disables it
// (per-cell 1-D bulk copies).
template <class E>
bool wedge_jmap(stokesfo_ctx *c, const double *J_cell) {
    constexpr int NN = 4 * E::N * E::N;
    if (E::JPITCH == NN || J_cell == nullptr) return false;
    if (const char *e = getenv("STOKESFO_JMAP"))
        if (atoi(e) == 0) return false;
    if (c->jmap_ptr == J_cell) return c->jmap_ok;
    c->jmap_ptr = J_cell;
    c->jmap_ok = false;
    encode_tiled_fn enc = tensor_map_encoder();
    if (!enc || c->d.num_cells > 0x7fffffff) return false;
    const cuuint64_t dims[2] = {(cuuint64_t)NN, (cuuint64_t)c->d.num_cells};
    const cuuint64_t strides[1] = {(cuuint64_t)NN * 8};
    const cuuint32_t box[2] = {(cuuint32_t)E::JPITCH, (cuuint32_t)E::TC};
    const cuuint32_t estr[2] = {1, 1};
    c->jmap_ok = enc(&c->jmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<double *>(J_cell), dims, strides, box,
                     estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                     CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
    return c->jmap_ok;
}

template <class E, int MODE>
int eval_impl(stokesfo_ctx *c, const double *U, double *mu_qp, double *R_cell, double *R, double *J_cell,
              const double *X = nullptr, double *Y = nullptr, double *csr_vals = nullptr, bool packed = false) {
    if (c->ntiles == 0) return STOKESFO_OK;
    EvalArgs a;
    a.recs = c->recs;
    a.xyz4 = c->xyz4;
    a.conn = c->d.conn;
    a.kc = c->d.flow_factor;
    a.kscal = c->d.k;
    a.err = c->err;
    a.ntiles = c->ntiles;
    a.ncells = c->d.num_cells;
    a.U = U;
    a.surface = c->d.surface;
    a.force_qp = c->d.force_qp;
    a.rho_g = c->d.rho_g;
    a.delta = c->d.delta;
    a.mu_qp = mu_qp;
    a.R_cell = R_cell;
    a.R = R;
    a.J_cell = J_cell;
    a.X = X;
    a.Y = Y;
    a.rem = c->rem;
    a.remtab = c->remtab;
    a.peers = c->peers;
    a.peers_y = c->peers_y;
    a.rowptr = c->rowptr;
    a.slots = c->slots;
    a.csr_vals = csr_vals;
    a.packed = packed ? 1 : 0;
    const int g = MODE == M_JAC ? c->grid_jac
                : MODE == M_JVP ? c->grid_jvp
                : MODE == M_CSR ? c->grid_csr
                : MODE == M_DIAG ? c->grid_diag : c->grid_resid;
    const bool otf = c->mode == STOKESFO_GEOMETRY_ON_THE_FLY;
    // the DMMA kernels store J with 32-B vector stores (16-B aligned J_cell: the vector kernels)
    const bool mma = MODE == M_JAC && c->mma_ok && (c->jac_mma || packed) && aligned(J_cell, 32);
    if (packed && !mma) return STOKESFO_EUNSUPPORTED;  // the packed form comes from the DMMA kernels only
    a.use_jmap = (!otf && !mma && MODE == M_JAC && wedge_jmap<E>(c, J_cell)) ? 1 : 0;
    const CUtensorMap jm = a.use_jmap ? c->jmap : CUtensorMap{};
    constexpr int WPC = warps_per_cta<E, MODE>();  // eval_kernel only (the on-the-fly kernel: 1)
    const int grid = (int)std::min<int64_t>(g, otf ? c->ntiles : (c->ntiles + WPC - 1) / WPC);
    const int ns = MODE == M_JAC ? c->nstage_jac : (MODE == M_RESID ? c->nstage_resid : 2);
    const int gm = (int)std::min<int64_t>(c->grid_mma, c->ntiles);
    if (mma && c->mode == STOKESFO_GEOMETRY_COMPACT)
        eval_compact_mma_kernel<E><<<gm, 32, CompactMmaSmem<E>::BYTES, c->stream>>>(a);
    else if (c->mode == STOKESFO_GEOMETRY_COMPACT)
        eval_compact_kernel<E, MODE><<<(int)std::min<int64_t>(g, c->ntiles), 32, CompactSmem<E, MODE>::BYTES,
                                        c->stream>>>(a, jm);
    else if (mma && otf)
        eval_otf_mma_kernel<E><<<gm, 32, OtfMmaSmem<E>::BYTES, c->stream>>>(a);
    else if (otf)
        eval_otf_kernel<E, MODE><<<grid, 32, OtfSmem<E, MODE>::BYTES, c->stream>>>(a);
    else if (mma)
        eval_mma_kernel<E, 2><<<gm, 32, MmaSmem<E, 2>::BYTES, c->stream>>>(a);
    else if (MODE != M_CSR && ns == 3)
        eval_kernel<E, MODE, 3><<<grid, 32 * WPC, eval_smem_bytes<E, MODE, 3>(), c->stream>>>(a, jm);
    else
        eval_kernel<E, MODE, 2><<<grid, 32 * WPC, eval_smem_bytes<E, MODE, 2>(), c->stream>>>(a, jm);
    return cuda_status();
}

#define DISPATCH(ctx, CALL)                                   \
    ((ctx)->d.elem == STOKESFO_HEX8 ? CALL(Hex8) : CALL(Wedge6))

}  // namespace

extern "C" {

const char *stokesfo_strerror(int s) {
    switch (s) {
        case STOKESFO_OK: return "ok";
        case STOKESFO_EINVAL: return "invalid argument (size, pointer or alignment)";
        case STOKESFO_EMESH: return "mesh error (det J <= 0, conn out of range or CSR entry missing)";
        case STOKESFO_ECUDA: return "CUDA runtime error";
        case STOKESFO_ENOMEM: return "workspace too small";
        case STOKESFO_EUNSUPPORTED:
            return "unsupported configuration (glen_n != 3, a node degree beyond the CSR kernels, or a packed "
                   "Jacobian without the tensor-core kernels)";
        case STOKESFO_ENONFINITE: return "non-finite value in an output (STOKESFO_CHECK_FINITE=1)";
        default: return "unknown status";
    }
}

int stokesfo_workspace_size(const stokesfo_desc_t *d, size_t *bytes) {
    SFO_RANGE("stokesfo_workspace_size");
    if (!d || !bytes || d->num_cells < 0) return STOKESFO_EINVAL;
    if (d->geometry_mode != STOKESFO_GEOMETRY_STORED && d->geometry_mode != STOKESFO_GEOMETRY_ON_THE_FLY &&
        d->geometry_mode != STOKESFO_GEOMETRY_COMPACT)
        return STOKESFO_EINVAL;
    if (d->elem == STOKESFO_HEX8) *bytes = (size_t)ws_bytes<Hex8>(d->num_cells, d->num_nodes, d->geometry_mode);
    else if (d->elem == STOKESFO_WEDGE6) *bytes = (size_t)ws_bytes<Wedge6>(d->num_cells, d->num_nodes, d->geometry_mode);
    else return STOKESFO_EINVAL;
    return STOKESFO_OK;
}

int stokesfo_create(const stokesfo_desc_t *d, stokesfo_ctx **out) {
    SFO_RANGE("stokesfo_create");
    if (!d || !out) return STOKESFO_EINVAL;
    *out = nullptr;
    if (d->abi_version != STOKESFO_ABI_VERSION) return STOKESFO_EINVAL;
    if (d->elem != STOKESFO_HEX8 && d->elem != STOKESFO_WEDGE6) return STOKESFO_EINVAL;
    if (d->num_cells < 0 || d->num_nodes < 0 || d->num_nodes > INT32_MAX) return STOKESFO_EINVAL;
    if (d->num_cells > 0 && (!d->conn || !d->coords || d->num_nodes == 0)) return STOKESFO_EINVAL;
    if (!(d->delta > 0.0)) return STOKESFO_EINVAL;
    if (d->glen_n != 3.0) return STOKESFO_EUNSUPPORTED;
    const void *ptrs[] = {d->conn, d->coords, d->surface, d->force_qp, d->flow_factor};
    for (const void *p : ptrs)
        if (p && !aligned(p, 16)) return STOKESFO_EINVAL;
    if (!d->workspace || !aligned(d->workspace, 256)) return STOKESFO_EINVAL;
    size_t need = 0;
    if (stokesfo_workspace_size(d, &need) != STOKESFO_OK) return STOKESFO_EINVAL;
    if (d->workspace_bytes < need) return STOKESFO_ENOMEM;
    stokesfo_ctx *c = new (std::nothrow) stokesfo_ctx();
    if (!c) return STOKESFO_ENOMEM;
    c->d = *d;
    c->stream = reinterpret_cast<cudaStream_t>(d->stream);
    if (const char *e = getenv("STOKESFO_CHECK_FINITE")) c->check_finite = atoi(e) == 1;
    c->err = reinterpret_cast<int *>(d->workspace);
    c->mode = d->geometry_mode;
    char *ws = reinterpret_cast<char *>(d->workspace);
    if (c->mode == STOKESFO_GEOMETRY_ON_THE_FLY) {
        c->xyz4 = reinterpret_cast<double4 *>(ws + WS_HEADER);
        c->recs = nullptr;
    } else {
        c->xyz4 = nullptr;
        c->recs = ws + WS_HEADER;
    }
    int st = (d->elem == STOKESFO_HEX8) ? create_impl<Hex8>(c) : create_impl<Wedge6>(c);
    // conn out of range is checked before any evaluation can use conn as an address (the on-the-fly
    // kernels and the side-set kernels read the caller's conn): one stream synchronisation at create
    if (st == STOKESFO_OK) {
        int h = 0;
        if (cudaMemcpyAsync(&h, c->err, sizeof(int), cudaMemcpyDeviceToHost, c->stream) != cudaSuccess ||
            cudaStreamSynchronize(c->stream) != cudaSuccess)
            st = cuda_status();
        else if (h & ERR_CONN)
            st = STOKESFO_EMESH;
    }
    if (st) {
        delete c;
        return st;
    }
    *out = c;
    return STOKESFO_OK;
}

void stokesfo_destroy(stokesfo_ctx *c) {
    SFO_RANGE("stokesfo_destroy"); delete c; }

int stokesfo_gather(stokesfo_ctx *c, const double *U, double *U_cell) {
    SFO_RANGE("stokesfo_gather");
    if (!c) return STOKESFO_EINVAL;
    if (c->d.num_cells == 0) return STOKESFO_OK;
    if (!U || !U_cell || !aligned(U, 16) || !aligned(U_cell, 16)) return STOKESFO_EINVAL;
    const int64_t work = c->d.num_cells * c->N;
    if (work == 0) return STOKESFO_OK;
    const int bs = 256;
    const unsigned g = (unsigned)((work + bs - 1) / bs);
    auto U2 = reinterpret_cast<const double2 *>(U);
    auto Uc = reinterpret_cast<double2 *>(U_cell);
    if (c->N == 8) gather_kernel<8><<<g, bs, 0, c->stream>>>(c->d.num_cells, c->d.conn, U2, Uc);
    else gather_kernel<6><<<g, bs, 0, c->stream>>>(c->d.num_cells, c->d.conn, U2, Uc);
    return cuda_status();
}

int stokesfo_viscosity_resid(stokesfo_ctx *c, const double *U, double *mu_qp, double *R_cell, double *R) {
    SFO_RANGE("stokesfo_viscosity_resid");
    if (!c) return STOKESFO_EINVAL;
    if (c->d.num_cells == 0) return STOKESFO_OK;
    if (!U || !aligned(U, 16)) return STOKESFO_EINVAL;
    const void *ps[] = {mu_qp, R_cell, R};
    for (const void *p : ps)
        if (p && !aligned(p, 16)) return STOKESFO_EINVAL;
#define CALL(E) eval_impl<E, M_RESID>(c, U, mu_qp, R_cell, R, nullptr)
    const int st = DISPATCH(c, CALL);
#undef CALL
    if (st == STOKESFO_OK) {
        check_finite(c, mu_qp, c->d.num_cells * c->Q);
        check_finite(c, R_cell, c->d.num_cells * c->N * 2);
        check_finite(c, R, c->d.num_nodes * 2);
    }
    return st == STOKESFO_OK ? cuda_status() : st;
}

int stokesfo_jacobian(stokesfo_ctx *c, const double *U, double *J_cell, double *R_cell, double *R) {
    SFO_RANGE("stokesfo_jacobian");
    if (!c) return STOKESFO_EINVAL;
    if (c->d.num_cells == 0) return STOKESFO_OK;  // nothing to evaluate (outputs may be NULL)
    if (!U || !J_cell || !aligned(U, 16) || !aligned(J_cell, 16)) return STOKESFO_EINVAL;
    const void *ps[] = {R_cell, R};
    for (const void *p : ps)
        if (p && !aligned(p, 16)) return STOKESFO_EINVAL;
#define CALL(E) eval_impl<E, M_JAC>(c, U, nullptr, R_cell, R, J_cell)
    const int st = DISPATCH(c, CALL);
#undef CALL
    if (st == STOKESFO_OK) {
        check_finite(c, J_cell, c->d.num_cells * 4 * c->N * c->N);
        check_finite(c, R_cell, c->d.num_cells * c->N * 2);
        check_finite(c, R, c->d.num_nodes * 2);
    }
    return st == STOKESFO_OK ? cuda_status() : st;
}

int stokesfo_jacobian_packed(stokesfo_ctx *c, const double *U, double *Jp, double *R_cell, double *R) {
    SFO_RANGE("stokesfo_jacobian_packed");
    if (!c) return STOKESFO_EINVAL;
    if (c->d.num_cells == 0) return STOKESFO_OK;
    if (!U || !Jp || !aligned(U, 16) || !aligned(Jp, 32)) return STOKESFO_EINVAL;
    const void *ps[] = {R_cell, R};
    for (const void *p : ps)
        if (p && !aligned(p, 16)) return STOKESFO_EINVAL;
#define CALL(E) eval_impl<E, M_JAC>(c, U, nullptr, R_cell, R, Jp, nullptr, nullptr, nullptr, true)
    const int st = DISPATCH(c, CALL);
#undef CALL
    if (st == STOKESFO_OK) {
        check_finite(c, Jp, c->d.num_cells * 2 * c->N * (c->N + 1));
        check_finite(c, R_cell, c->d.num_cells * c->N * 2);
        check_finite(c, R, c->d.num_nodes * 2);
    }
    return st == STOKESFO_OK ? cuda_status() : st;
}

int stokesfo_jacobian_csr(stokesfo_ctx *c, const double *U, double *csr_vals, double *R) {
    SFO_RANGE("stokesfo_jacobian_csr");
    if (!c) return STOKESFO_EINVAL;
    if (c->d.num_cells == 0) return STOKESFO_OK;
    if (!c->slots || !c->rowptr) return STOKESFO_EINVAL;  // needs stokesfo_csr_slots
    if (!U || !csr_vals || !aligned(U, 16) || !aligned(csr_vals, 16) || (R && !aligned(R, 16)))
        return STOKESFO_EINVAL;
#define CALL(E) eval_impl<E, M_CSR>(c, U, nullptr, nullptr, R, nullptr, nullptr, nullptr, csr_vals)
    return DISPATCH(c, CALL);
#undef CALL
}

// slots buffer: [slots C N uint64][inc_ptr (nodes+1) int64][inc C N int32]
static int64_t slots_off_incptr(const stokesfo_ctx *c) { return round_up(c->d.num_cells * c->N * 8, 16); }
static int64_t slots_off_inc(const stokesfo_ctx *c) {
    return slots_off_incptr(c) + round_up((c->d.num_nodes + 1) * 8, 16);
}
// + per-node pull records [nodes][PullCfg<N>::WORDS] uint64 (csr_gather_kernel)
static int64_t slots_off_nrec(const stokesfo_ctx *c) {
    return slots_off_inc(c) + round_up(c->d.num_cells * c->N * 4, 128);
}

int stokesfo_csr_slots_size(stokesfo_ctx *c, size_t *bytes) {
    SFO_RANGE("stokesfo_csr_slots_size");
    if (!c || !bytes) return STOKESFO_EINVAL;
    *bytes = (size_t)(slots_off_nrec(c) + c->d.num_nodes * (c->N == 8 ? pull_words<8>() : pull_words<6>()) * 8);
    return STOKESFO_OK;
}

int stokesfo_csr_slots(stokesfo_ctx *c, uint64_t *slots) {
    SFO_RANGE("stokesfo_csr_slots");
    if (!c || !slots || !aligned(slots, 16)) return STOKESFO_EINVAL;
    if (!c->rowptr || !c->colidx) return STOKESFO_EINVAL;  // needs the stokesfo_csr_pattern fill
    if (c->csr_maxdeg > 256) return STOKESFO_EUNSUPPORTED;
    const int64_t work = c->d.num_cells * c->N;
    if (work > 0) {
        const int bs = 256;
        const unsigned g = (unsigned)((work + bs - 1) / bs);
        if (c->N == 8)
            csr_slots_kernel<8><<<g, bs, 0, c->stream>>>(c->d.num_cells, c->d.conn, c->rowptr, c->colidx, slots, c->err);
        else
            csr_slots_kernel<6><<<g, bs, 0, c->stream>>>(c->d.num_cells, c->d.conn, c->rowptr, c->colidx, slots, c->err);
    }
    c->slots = slots;
    // node -> (cell, i) incidence for the atomic-free assembly kernel
    char *base = reinterpret_cast<char *>(slots);
    int64_t *ip = reinterpret_cast<int64_t *>(base + slots_off_incptr(c));
    int32_t *in = reinterpret_cast<int32_t *>(base + slots_off_inc(c));
    if ((int64_t)c->inc_ptr_h.size() == c->d.num_nodes + 1 && (int64_t)c->inc_h.size() == work) {
        if (cudaMemcpyAsync(ip, c->inc_ptr_h.data(), c->inc_ptr_h.size() * 8, cudaMemcpyHostToDevice, c->stream) !=
                cudaSuccess ||
            (work > 0 &&
             cudaMemcpyAsync(in, c->inc_h.data(), c->inc_h.size() * 4, cudaMemcpyHostToDevice, c->stream) != cudaSuccess) ||
            cudaStreamSynchronize(c->stream) != cudaSuccess)
            return cuda_status();
        c->inc_ptr = ip;
        c->inc = in;
        std::vector<int64_t>().swap(c->inc_ptr_h);
        std::vector<int32_t>().swap(c->inc_h);
    } else if (c->inc_ptr && c->inc && c->inc_ptr != ip) {
        // a second slot table for the same pattern: carry the incidence over from the previous buffer, so the
        // new table does not depend on the old buffer staying allocated
        if (cudaMemcpyAsync(ip, c->inc_ptr, (c->d.num_nodes + 1) * 8, cudaMemcpyDeviceToDevice, c->stream) !=
                cudaSuccess ||
            (work > 0 && cudaMemcpyAsync(in, c->inc, work * 4, cudaMemcpyDeviceToDevice, c->stream) != cudaSuccess))
            return cuda_status();
        c->inc_ptr = ip;
        c->inc = in;
    }
    if (c->inc_ptr && c->inc && c->d.num_nodes > 0) {  // per-node pull records
        uint64_t *nrec = reinterpret_cast<uint64_t *>(base + slots_off_nrec(c));
        const int bs = 256;
        const unsigned g = (unsigned)((c->d.num_nodes + bs - 1) / bs);
        if (c->N == 8)
            node_rec_kernel<8><<<g, bs, 0, c->stream>>>(c->d.num_nodes, c->rowptr, c->inc_ptr, c->inc, slots, nrec);
        else
            node_rec_kernel<6><<<g, bs, 0, c->stream>>>(c->d.num_nodes, c->rowptr, c->inc_ptr, c->inc, slots, nrec);
        c->nrec = nrec;
    }
    return cuda_status();
}

int stokesfo_jvp(stokesfo_ctx *c, const double *U, const double *X, double *Y, double *R) {
    SFO_RANGE("stokesfo_jvp");
    if (!c) return STOKESFO_EINVAL;
    if (c->d.num_cells == 0) return STOKESFO_OK;
    if (!U || !X || !Y || !aligned(U, 16) || !aligned(X, 16) || !aligned(Y, 16) || (R && !aligned(R, 16)))
        return STOKESFO_EINVAL;
    if (c->rem && !c->peers_y) return STOKESFO_EINVAL;  // Y would miss the peers' boundary contributions
#define CALL(E) eval_impl<E, M_JVP>(c, U, nullptr, nullptr, R, nullptr, X, Y)
    const int st = DISPATCH(c, CALL);
#undef CALL
    if (st == STOKESFO_OK) {
        check_finite(c, Y, c->d.num_nodes * 2);
        check_finite(c, R, c->d.num_nodes * 2);
    }
    return st == STOKESFO_OK ? cuda_status() : st;
}

int stokesfo_jacobian_diag(stokesfo_ctx *c, const double *U, double *diag, double *R) {
    SFO_RANGE("stokesfo_jacobian_diag");
    if (!c) return STOKESFO_EINVAL;
    if (c->d.num_cells == 0) return STOKESFO_OK;
    if (!U || !diag || !aligned(U, 16) || !aligned(diag, 16) || (R && !aligned(R, 16))) return STOKESFO_EINVAL;
    if (c->rem && !c->peers_y) return STOKESFO_EINVAL;  // diag would miss the peers' boundary contributions
#define CALL(E) eval_impl<E, M_DIAG>(c, U, nullptr, nullptr, R, nullptr, nullptr, diag)
    const int st = DISPATCH(c, CALL);
#undef CALL
    if (st == STOKESFO_OK) {
        check_finite(c, diag, c->d.num_nodes * 2);
        check_finite(c, R, c->d.num_nodes * 2);
    }
    return st == STOKESFO_OK ? cuda_status() : st;
}

int stokesfo_basal_friction(stokesfo_ctx *c, const int32_t *basal_cells, int64_t nfaces, const double *beta,
                            const double *U, double *R, double *J_face) {
    SFO_RANGE("stokesfo_basal_friction");
    if (!c || nfaces < 0) return STOKESFO_EINVAL;
    if (nfaces == 0) return STOKESFO_OK;
    if (!basal_cells || !beta || !U || !R || !aligned(U, 16) || !aligned(R, 16) || (J_face && !aligned(J_face, 16)))
        return STOKESFO_EINVAL;
    const int bs = 128;
    const unsigned g = (unsigned)((nfaces + bs - 1) / bs);
    if (c->N == 8)
        basal_friction_kernel<Hex8><<<g, bs, 0, c->stream>>>(nfaces, basal_cells, c->d.conn, c->d.coords, beta, U, R,
                                                              J_face);
    else
        basal_friction_kernel<Wedge6><<<g, bs, 0, c->stream>>>(nfaces, basal_cells, c->d.conn, c->d.coords, beta, U,
                                                                R, J_face);
    return cuda_status();
}

int stokesfo_lateral_pressure(stokesfo_ctx *c, const int32_t *faces, int64_t nfaces, const double *surface,
                              double rho_i_g, double rho_w_g, double sea_level, double *R) {
    SFO_RANGE("stokesfo_lateral_pressure");
    if (!c || nfaces < 0) return STOKESFO_EINVAL;
    if (nfaces == 0) return STOKESFO_OK;
    if (!faces || !surface || !R || !aligned(faces, 8) || !aligned(R, 16)) return STOKESFO_EINVAL;
    const int bs = 128;
    const unsigned g = (unsigned)((nfaces + bs - 1) / bs);
    const int64_t C = c->d.num_cells;
    if (c->N == 8)
        lateral_pressure_kernel<Hex8><<<g, bs, 0, c->stream>>>(nfaces, C, faces, c->d.conn, c->d.coords, surface,
                                                                rho_i_g, rho_w_g, sea_level, R, c->err);
    else
        lateral_pressure_kernel<Wedge6><<<g, bs, 0, c->stream>>>(nfaces, C, faces, c->d.conn, c->d.coords, surface,
                                                                  rho_i_g, rho_w_g, sea_level, R, c->err);
    return cuda_status();
}

int stokesfo_set_lateral(stokesfo_ctx *c, const int32_t *faces, int64_t nfaces, const double *surface,
                         double rho_i_g, double rho_w_g, double sea_level) {
    SFO_RANGE("stokesfo_set_lateral");
    if (!c || nfaces < 0) return STOKESFO_EINVAL;
    if (nfaces > 0 && (!faces || !surface || !aligned(faces, 8))) return STOKESFO_EINVAL;
    c->lat_faces = nfaces > 0 ? faces : nullptr;
    c->lat_n = nfaces > 0 ? nfaces : 0;
    c->lat_surface = surface;
    c->lat_rho_i_g = rho_i_g;
    c->lat_rho_w_g = rho_w_g;
    c->lat_sea = sea_level;
    return STOKESFO_OK;
}

int stokesfo_scatter_assemble(stokesfo_ctx *c, const double *R_cell, double *R, const double *J_cell,
                              double *csr_vals) {
    SFO_RANGE("stokesfo_scatter_assemble");
    if (!c) return STOKESFO_EINVAL;
    const void *ps[] = {R_cell, R, J_cell, csr_vals};
    for (const void *p : ps)
        if (p && !aligned(p, 16)) return STOKESFO_EINVAL;
    const int64_t C = c->d.num_cells;
    const int bs = 256;
    // STOKESFO_CSR_ATOMIC=1: slot-based atomic kernel instead of the pull kernel (A/B)
    static const bool pull = !(getenv("STOKESFO_CSR_ATOMIC") && atoi(getenv("STOKESFO_CSR_ATOMIC")) == 1);
    if (R_cell && R && C > 0) {
        const int64_t work = C * c->N;
        const unsigned g = (unsigned)((work + bs - 1) / bs);
        auto Rc = reinterpret_cast<const double2 *>(R_cell);
        if (c->N == 8) scatter_r_kernel<8><<<g, bs, 0, c->stream>>>(C, c->d.conn, Rc, R, c->rem, c->remtab, c->peers);
        else scatter_r_kernel<6><<<g, bs, 0, c->stream>>>(C, c->d.conn, Rc, R, c->rem, c->remtab, c->peers);
    }
    if (J_cell && csr_vals && C > 0) {
        if (!c->rowptr || !c->colidx) return STOKESFO_EINVAL;
        const int64_t work = C * 2 * c->N;
        const unsigned g = (unsigned)((work + bs - 1) / bs);
        if (c->slots && c->nrec && c->csr_maxdeg <= CSR_GATHER_MAXDEG && pull) {  // atomic-free, deterministic
            const int64_t NN = c->d.num_nodes;
            const int64_t per_block = (int64_t)CSR_GATHER_WARPS * (c->N == 8 ? pull_npw<8>() : pull_npw<6>());
            const unsigned gg = (unsigned)((NN + per_block - 1) / per_block);
            if (c->N == 8)
                csr_gather_kernel<8><<<gg, 32 * CSR_GATHER_WARPS, 0, c->stream>>>(NN, J_cell, c->nrec, c->inc,
                                                                                 c->slots, csr_vals);
            else
                csr_gather_kernel<6><<<gg, 32 * CSR_GATHER_WARPS, 0, c->stream>>>(NN, J_cell, c->nrec, c->inc,
                                                                                 c->slots, csr_vals);
        } else if (c->slots) {  // slot table attached: no per-entry search
            if (c->N == 8)
                scatter_csr_slots_kernel<8><<<g, bs, 0, c->stream>>>(C, c->d.conn, J_cell, c->rowptr, c->slots, csr_vals);
            else
                scatter_csr_slots_kernel<6><<<g, bs, 0, c->stream>>>(C, c->d.conn, J_cell, c->rowptr, c->slots, csr_vals);
        } else if (c->N == 8)
            scatter_csr_kernel<8><<<g, bs, 0, c->stream>>>(C, c->d.conn, J_cell, c->rowptr, c->colidx, csr_vals, c->err);
        else
            scatter_csr_kernel<6><<<g, bs, 0, c->stream>>>(C, c->d.conn, J_cell, c->rowptr, c->colidx, csr_vals, c->err);
    }
    return cuda_status();
}

}  // extern "C"
template <bool PACKED>
static int assemble_csr_impl(stokesfo_ctx *c, const double *J_cell, double *csr_vals, int accumulate) {
    if (!c || !J_cell || !csr_vals || !aligned(J_cell, 16) || !aligned(csr_vals, 16)) return STOKESFO_EINVAL;
    if (!c->slots || !c->nrec || !c->rowptr) return STOKESFO_EINVAL;  // needs stokesfo_csr_slots
    if (c->csr_maxdeg > CSR_GATHER_MAXDEG) return STOKESFO_EUNSUPPORTED;
    const int64_t NN = c->d.num_nodes;
    if (NN == 0) return STOKESFO_OK;
    const int64_t per_block = (int64_t)CSR_GATHER_WARPS * (c->N == 8 ? pull_npw<8>() : pull_npw<6>());
    const unsigned gg = (unsigned)((NN + per_block - 1) / per_block);
    const int bt = 32 * CSR_GATHER_WARPS;
#define PULL(NN_, ACC_)                                                                                       \
    csr_gather_kernel<NN_, ACC_, PACKED><<<gg, bt, 0, c->stream>>>(NN, J_cell, c->nrec, c->inc, c->slots, csr_vals)
    if (c->N == 8) {
        if (accumulate) PULL(8, true);
        else PULL(8, false);
    } else {
        if (accumulate) PULL(6, true);
        else PULL(6, false);
    }
#undef PULL
    return cuda_status();
}

extern "C" {

int stokesfo_assemble_csr(stokesfo_ctx *c, const double *J_cell, double *csr_vals, int accumulate) {
    SFO_RANGE("stokesfo_assemble_csr");
    return assemble_csr_impl<false>(c, J_cell, csr_vals, accumulate);
}

int stokesfo_assemble_csr_packed(stokesfo_ctx *c, const double *Jp, double *csr_vals, int accumulate) {
    SFO_RANGE("stokesfo_assemble_csr_packed");
    return assemble_csr_impl<true>(c, Jp, csr_vals, accumulate);
}

int stokesfo_geometry(stokesfo_ctx *c, double *grad_bf, double *w_measure) {
    SFO_RANGE("stokesfo_geometry");
    if (!c) return STOKESFO_EINVAL;
    if ((grad_bf && !aligned(grad_bf, 16)) || (w_measure && !aligned(w_measure, 16))) return STOKESFO_EINVAL;
    const int64_t work = c->d.num_cells * c->Q;
    if (work == 0) return STOKESFO_OK;
    const int bs = 256;
    const unsigned g = (unsigned)((work + bs - 1) / bs);
    if (c->mode == STOKESFO_GEOMETRY_ON_THE_FLY) {  // recompute with the same device code, canonical layout
        if (c->N == 8)
            geometry_kernel<Hex8, GEO_CANON><<<g, bs, 0, c->stream>>>(c->d.num_cells, c->d.num_nodes, c->d.conn,
                                                                      c->d.coords, nullptr, 0.0, nullptr, grad_bf,
                                                                      w_measure, c->err);
        else
            geometry_kernel<Wedge6, GEO_CANON><<<g, bs, 0, c->stream>>>(c->d.num_cells, c->d.num_nodes, c->d.conn,
                                                                        c->d.coords, nullptr, 0.0, nullptr, grad_bf,
                                                                        w_measure, c->err);
    } else if (c->mode == STOKESFO_GEOMETRY_COMPACT) {
        if (c->N == 8)
            geometry_export_compact_kernel<Hex8><<<g, bs, 0, c->stream>>>(c->d.num_cells, c->recs, grad_bf, w_measure);
        else
            geometry_export_compact_kernel<Wedge6><<<g, bs, 0, c->stream>>>(c->d.num_cells, c->recs, grad_bf,
                                                                            w_measure);
    } else if (c->N == 8) {
        geometry_export_kernel<Hex8><<<g, bs, 0, c->stream>>>(c->d.num_cells, c->recs, grad_bf, w_measure);
    } else {
        geometry_export_kernel<Wedge6><<<g, bs, 0, c->stream>>>(c->d.num_cells, c->recs, grad_bf, w_measure);
    }
    return cuda_status();
}

int stokesfo_halo_pack(stokesfo_ctx *c, const double *R, const int32_t *send_nodes, int64_t n, double *buf) {
    SFO_RANGE("stokesfo_halo_pack");
    if (!c || n < 0) return STOKESFO_EINVAL;
    if (n == 0) return STOKESFO_OK;
    if (!R || !send_nodes || !buf || !aligned(R, 16) || !aligned(buf, 16)) return STOKESFO_EINVAL;
    const int bs = 256;
    halo_pack_kernel<<<(unsigned)((n + bs - 1) / bs), bs, 0, c->stream>>>(
        n, send_nodes, reinterpret_cast<const double2 *>(R), reinterpret_cast<double2 *>(buf));
    return cuda_status();
}

int stokesfo_halo_unpack_add(stokesfo_ctx *c, const double *buf, const int32_t *recv_nodes, int64_t n, double *R) {
    SFO_RANGE("stokesfo_halo_unpack_add");
    if (!c || n < 0) return STOKESFO_EINVAL;
    if (n == 0) return STOKESFO_OK;
    if (!R || !recv_nodes || !buf || !aligned(R, 16) || !aligned(buf, 16)) return STOKESFO_EINVAL;
    const int bs = 256;
    halo_unpack_add_kernel<<<(unsigned)((n + bs - 1) / bs), bs, 0, c->stream>>>(
        n, recv_nodes, reinterpret_cast<const double2 *>(buf), reinterpret_cast<double2 *>(R));
    return cuda_status();
}

int stokesfo_set_remote(stokesfo_ctx *c, const int32_t *rem, const int32_t *remtab, double *const *peers) {
    SFO_RANGE("stokesfo_set_remote");
    if (!c) return STOKESFO_EINVAL;
    if (!rem) {  // detach
        c->rem = nullptr;
        c->remtab = nullptr;
        c->peers = nullptr;
        c->peers_y = nullptr;
        return STOKESFO_OK;
    }
    if (!remtab || !peers) return STOKESFO_EINVAL;
    c->rem = rem;
    c->remtab = remtab;
    c->peers = peers;
    return STOKESFO_OK;
}

int stokesfo_set_remote_jvp(stokesfo_ctx *c, double *const *peers_y) {
    SFO_RANGE("stokesfo_set_remote_jvp");
    if (!c) return STOKESFO_EINVAL;
    if (peers_y && !c->rem) return STOKESFO_EINVAL;  // needs the node table of stokesfo_set_remote
    c->peers_y = peers_y;
    return STOKESFO_OK;
}

int stokesfo_ipc_get_handle(const void *dev_ptr, void *handle, int64_t *offset) {
    SFO_RANGE("stokesfo_ipc_get_handle");
    if (!dev_ptr || !handle || !offset) return STOKESFO_EINVAL;
    cudaIpcMemHandle_t h;
    if (cudaIpcGetMemHandle(&h, const_cast<void *>(dev_ptr)) != cudaSuccess) return cuda_status();
    memcpy(handle, &h, sizeof(h));
    // the handle maps the whole allocation: report dev_ptr's offset from its base
    // (cuMemGetAddressRange through the runtime's driver entry point)
    typedef int (*GetRange)(unsigned long long *, size_t *, unsigned long long);
    void *fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn)
        return cuda_status() ? STOKESFO_ECUDA : STOKESFO_ECUDA;
    unsigned long long base = 0;
    size_t size = 0;
    if (reinterpret_cast<GetRange>(fn)(&base, &size, reinterpret_cast<unsigned long long>(dev_ptr)) != 0)
        return STOKESFO_ECUDA;
    *offset = (int64_t)(reinterpret_cast<unsigned long long>(dev_ptr) - base);
    return STOKESFO_OK;
}

int stokesfo_ipc_open_handle(const void *handle, void **dev_ptr) {
    SFO_RANGE("stokesfo_ipc_open_handle");
    if (!dev_ptr || !handle) return STOKESFO_EINVAL;
    cudaIpcMemHandle_t h;
    memcpy(&h, handle, sizeof(h));
    if (cudaIpcOpenMemHandle(dev_ptr, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) return cuda_status();
    return STOKESFO_OK;
}

int stokesfo_ipc_close(void *dev_ptr) {
    SFO_RANGE("stokesfo_ipc_close");
    if (!dev_ptr) return STOKESFO_EINVAL;
    if (cudaIpcCloseMemHandle(dev_ptr) != cudaSuccess) return cuda_status();
    return STOKESFO_OK;
}

int stokesfo_sync(stokesfo_ctx *c) {
    SFO_RANGE("stokesfo_sync");
    if (!c) return STOKESFO_EINVAL;
    if (cudaStreamSynchronize(c->stream) != cudaSuccess) return cuda_status();
    int h = 0;
    if (cudaMemcpy(&h, c->err, sizeof(int), cudaMemcpyDeviceToHost) != cudaSuccess) return cuda_status();
    if (h & (ERR_DETJ | ERR_CONN | ERR_CSR)) return STOKESFO_EMESH;
    return h ? STOKESFO_ENONFINITE : STOKESFO_OK;
}

int stokesfo_launch_info(stokesfo_ctx *c, int32_t *cells_per_tile, int32_t *grid_resid, int32_t *grid_jac,
                         int64_t *record_bytes_per_tile) {
    SFO_RANGE("stokesfo_launch_info");
    if (!c) return STOKESFO_EINVAL;
    if (cells_per_tile) *cells_per_tile = c->TC;
    if (grid_resid) *grid_resid = (int32_t)std::min<int64_t>(c->grid_resid, std::max<int64_t>(c->ntiles, 1));
    if (grid_jac) *grid_jac = (int32_t)std::min<int64_t>(c->grid_jac, std::max<int64_t>(c->ntiles, 1));
    if (record_bytes_per_tile) *record_bytes_per_tile = c->rec_bytes;
    return STOKESFO_OK;
}

}  // extern "C"

// ---------------------------------------------------------------------------
// NEXT-1: the paper's evaluator chain (sfo_albany.cuh)
// ---------------------------------------------------------------------------
namespace {
template <class E, int ND>
int albany_run(stokesfo_ctx *c, int stage, int variant, const double *U, double *S, double *R_cell, double *J_cell) {
    using namespace sfo::albany;
    const int64_t C = c->d.num_cells;
    if (C == 0) return STOKESFO_OK;
    const int bs = 128;
    const unsigned gc = (unsigned)((C + bs - 1) / bs);
    const unsigned gq = (unsigned)((C * E::Q + bs - 1) / bs);
    switch (stage) {
        case 0:  // setup: GradBF, wGradBF, wBF
            geometry_kernel<E, GEO_ALBANY><<<gq, bs, 0, c->stream>>>(C, c->d.num_nodes, c->d.conn, c->d.coords,
                                                                    nullptr, 0.0, nullptr, S, nullptr, c->err);
            break;
        case 1:  // evaluators
            gather_solution_kernel<E, ND><<<gc, bs, 0, c->stream>>>(C, c->d.conn, U, S);
            ugrad_kernel<E, ND><<<gq, bs, 0, c->stream>>>(C, S);
            viscosity_kernel<E, ND><<<gq, bs, 0, c->stream>>>(C, c->d.flow_factor, c->d.k, c->d.delta, S);
            bodyforce_kernel<E, ND><<<gq, bs, 0, c->stream>>>(C, c->d.conn, c->d.surface, c->d.rho_g, S);
            break;
        case 2: {  // StokesFOResid (Fig. 2), SFO_ALBANY_MAXT threads per block (its launch bound)
            const int bt = SFO_ALBANY_MAXT;
            const unsigned gt = (unsigned)((C + bt - 1) / bt);
            if (variant == STOKESFO_FIG2_BASELINE)
                stokesfo_resid_baseline_kernel<E, ND><<<gt, bt, 0, c->stream>>>(C, S);
            else
                stokesfo_resid_optimized_kernel<E, ND><<<gt, bt, 0, c->stream>>>(C, S);
            break;
        }
        case 3: {  // extract
            const unsigned gr = (unsigned)((C * 2 * E::N + bs - 1) / bs);
            extract_kernel<E, ND><<<gr, bs, 0, c->stream>>>(C, S, R_cell, J_cell);
            break;
        }
        default:
            return STOKESFO_EINVAL;
    }
    return cuda_status();
}

int albany_dispatch(stokesfo_ctx *c, int derivs, int stage, int variant, const double *U, double *S, double *R_cell,
                    double *J_cell) {
    if (!c || !S || (derivs != 0 && derivs != 1) || (variant != 0 && variant != 1)) return STOKESFO_EINVAL;
    if (c->d.force_qp) return STOKESFO_EUNSUPPORTED;  // the chain derives the force from the surface
    if (c->N == 8)
        return derivs ? albany_run<Hex8, 16>(c, stage, variant, U, S, R_cell, J_cell)
                      : albany_run<Hex8, 0>(c, stage, variant, U, S, R_cell, J_cell);
    return derivs ? albany_run<Wedge6, 12>(c, stage, variant, U, S, R_cell, J_cell)
                  : albany_run<Wedge6, 0>(c, stage, variant, U, S, R_cell, J_cell);
}
}  // namespace

extern "C" {

int stokesfo_albany_scratch_size(stokesfo_ctx *c, int derivs, size_t *bytes) {
    SFO_RANGE("stokesfo_albany_scratch_size");
    if (!c || !bytes || (derivs != 0 && derivs != 1)) return STOKESFO_EINVAL;
    int64_t per;
    if (c->N == 8) per = derivs ? sfo::albany::Scratch<Hex8, 16>::TOTAL : sfo::albany::Scratch<Hex8, 0>::TOTAL;
    else per = derivs ? sfo::albany::Scratch<Wedge6, 12>::TOTAL : sfo::albany::Scratch<Wedge6, 0>::TOTAL;
    *bytes = (size_t)(per * c->d.num_cells * 8);
    return STOKESFO_OK;
}
int stokesfo_albany_setup(stokesfo_ctx *c, int derivs, double *scratch) {
    SFO_RANGE("stokesfo_albany_setup");
    return albany_dispatch(c, derivs, 0, 0, nullptr, scratch, nullptr, nullptr);
}
int stokesfo_albany_evaluators(stokesfo_ctx *c, int derivs, const double *U, double *scratch) {
    SFO_RANGE("stokesfo_albany_evaluators");
    if (!U) return STOKESFO_EINVAL;
    return albany_dispatch(c, derivs, 1, 0, U, scratch, nullptr, nullptr);
}
int stokesfo_albany_resid(stokesfo_ctx *c, int derivs, int variant, double *scratch) {
    SFO_RANGE("stokesfo_albany_resid");
    return albany_dispatch(c, derivs, 2, variant, nullptr, scratch, nullptr, nullptr);
}
int stokesfo_albany_extract(stokesfo_ctx *c, int derivs, const double *scratch, double *R_cell, double *J_cell) {
    SFO_RANGE("stokesfo_albany_extract");
    return albany_dispatch(c, derivs, 3, 0, nullptr, const_cast<double *>(scratch), R_cell, J_cell);
}

// ---------------------------------------------------------------------------
// NEXT-3: damped Newton-Krylov driver (sfo_newton.cuh)
// ---------------------------------------------------------------------------
}  // extern "C"

namespace {
constexpr int CG_BLOCK = 8;  // CG iterations per graph replay (one host convergence check per block)
struct NewtonWork {
    double *F, *D, *Rr, *P, *AP, *Z, *Ut, *diag, *Jf, *scal, *hist;
    int64_t bytes;
};
NewtonWork newton_layout(const stokesfo_ctx *c, int64_t nbasal, char *base) {
    NewtonWork w{};
    const int64_t n = 2 * c->d.num_nodes, NFD = c->N;  // face matrix: 2*NB = N
    int64_t off = 0;
    auto take = [&](int64_t count) {
        double *p = reinterpret_cast<double *>(base + off);
        off += round_up(std::max<int64_t>(count, 1) * 8, 256);
        return p;
    };
    w.F = take(n); w.D = take(n); w.Rr = take(n); w.P = take(n); w.AP = take(n); w.Z = take(n); w.Ut = take(n);
    w.diag = take(n); w.Jf = take(nbasal * NFD * NFD); w.scal = take(32); w.hist = take(CG_BLOCK);
    w.bytes = off;
    return w;
}
}  // namespace

extern "C" {

int stokesfo_newton_work_size(stokesfo_ctx *c, int64_t nbasal, size_t *bytes) {
    SFO_RANGE("stokesfo_newton_work_size");
    if (!c || !bytes || nbasal < 0) return STOKESFO_EINVAL;
    *bytes = (size_t)newton_layout(c, nbasal, nullptr).bytes;
    return STOKESFO_OK;
}

int stokesfo_newton_solve(stokesfo_ctx *c, const int32_t *basal_cells, int64_t nbasal, const double *beta,
                          double *U, void *work, const stokesfo_newton_opts_t *o, double *hist_F, int32_t *hist_cg,
                          int32_t *iters) {
    SFO_RANGE("stokesfo_newton_solve");
    using namespace sfo::newton;
    if (!c || !U || !work || !o || !hist_F || !iters || nbasal < 0 || (nbasal > 0 && (!basal_cells || !beta)))
        return STOKESFO_EINVAL;
    if (!aligned(U, 16) || !aligned(work, 256)) return STOKESFO_EINVAL;
    if (c->rem) return STOKESFO_EINVAL;  // single-GPU driver: a peer table would add into other ranks' buffers
    NewtonWork w = newton_layout(c, nbasal, reinterpret_cast<char *>(work));
    const int64_t n = 2 * c->d.num_nodes;
    const size_t vb = (size_t)n * 8;
    const int bs = 256;
    const unsigned gv = (unsigned)std::min<int64_t>((n + bs - 1) / bs, 148 * 8);
    // the solve runs on a stream of its own (graph capture needs a non-legacy stream), ordered
    // after the caller's work on the ctx stream and before anything the caller enqueues next
    cudaStream_t user = c->stream, st = nullptr;
    cudaEvent_t ev = nullptr;
    cudaGraph_t graph = nullptr;
    cudaGraphExec_t gexec = nullptr;
    if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess || cudaEventRecord(ev, user) != cudaSuccess ||
        cudaStreamWaitEvent(st, ev, 0) != cudaSuccess) {
        if (st) cudaStreamDestroy(st);
        if (ev) cudaEventDestroy(ev);
        return cuda_status();
    }
    c->stream = st;
    int rc = STOKESFO_OK;
    double host_hist[CG_BLOCK];
#define CK(x)                            \
    do {                                 \
        rc = (x);                        \
        if (rc != STOKESFO_OK) goto done; \
    } while (0)
#define CU(x)                                   \
    do {                                        \
        if ((x) != cudaSuccess) {               \
            rc = cuda_status();                 \
            if (rc == STOKESFO_OK) rc = STOKESFO_ECUDA; \
            goto done;                          \
        }                                       \
    } while (0)
    {
        auto dot_dev = [&](const double *x, const double *y, double *slot) -> int {  // *slot = x . y (async)
            if (cudaMemsetAsync(slot, 0, 8, st) != cudaSuccess) return cuda_status();
            dot_kernel<<<gv, bs, 0, st>>>(n, x, y, slot);
            return cuda_status();
        };
        auto dot_host = [&](const double *x, const double *y, double &out) -> int {
            int r = dot_dev(x, y, w.scal + 16);
            if (r != STOKESFO_OK) return r;
            if (cudaMemcpyAsync(&out, w.scal + 16, 8, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
                cudaStreamSynchronize(st) != cudaSuccess)
                return cuda_status();
            return STOKESFO_OK;
        };
        auto eval_F = [&](const double *u, double *F) -> int {  // F = R_visc(u) + R_basal(u) + R_lateral
            if (cudaMemsetAsync(F, 0, vb, st) != cudaSuccess) return cuda_status();
            int r = stokesfo_viscosity_resid(c, u, nullptr, nullptr, F);
            if (r == STOKESFO_OK && nbasal > 0) r = stokesfo_basal_friction(c, basal_cells, nbasal, beta, u, F, nullptr);
            if (r == STOKESFO_OK && c->lat_n > 0)
                r = stokesfo_lateral_pressure(c, c->lat_faces, c->lat_n, c->lat_surface, c->lat_rho_i_g,
                                              c->lat_rho_w_g, c->lat_sea, F);
            return r;
        };
        // one CG iteration with device-side scalars (captured CG_BLOCK times into the graph)
        auto cg_iter = [&]() -> int {
            if (cudaMemsetAsync(w.AP, 0, vb, st) != cudaSuccess) return cuda_status();
            int r = stokesfo_jvp(c, U, w.P, w.AP, nullptr);                   // Ap = J(U) p
            if (r == STOKESFO_OK && nbasal > 0) r = stokesfo_basal_friction(c, basal_cells, nbasal, beta, w.P, w.AP, nullptr);
            if (r == STOKESFO_OK) r = dot_dev(w.P, w.AP, w.scal + S_PAP);
            if (r != STOKESFO_OK) return r;
            cg_alpha_kernel<<<1, 1, 0, st>>>(w.scal);
            axpy_dev_kernel<<<gv, bs, 0, st>>>(n, w.scal + S_ALPHA, 1.0, w.P, w.D);     // D += alpha p
            axpy_dev_kernel<<<gv, bs, 0, st>>>(n, w.scal + S_ALPHA, -1.0, w.AP, w.Rr);  // r -= alpha Ap
            r = dot_dev(w.Rr, w.Rr, w.scal + S_RR);
            if (r != STOKESFO_OK) return r;
            jacobi_kernel<<<gv, bs, 0, st>>>(n, w.Rr, w.diag, w.Z);                      // z = r / diag
            r = dot_dev(w.Rr, w.Z, w.scal + S_RZN);
            if (r != STOKESFO_OK) return r;
            cg_beta_kernel<<<1, 1, 0, st>>>(w.scal, w.hist);
            xpby_dev_kernel<<<gv, bs, 0, st>>>(n, w.Z, w.scal + S_BETA, w.P);           // p = z + beta p
            return cuda_status();
        };
        // the CG block graph: every pointer it touches is fixed for the whole solve (U is updated in place)
        CU(cudaStreamBeginCapture(st, cudaStreamCaptureModeRelaxed));
        {
            int r = STOKESFO_OK;
            for (int k = 0; k < CG_BLOCK && r == STOKESFO_OK; ++k) r = cg_iter();
            cudaGraph_t g = nullptr;
            const cudaError_t e = cudaStreamEndCapture(st, &g);
            graph = g;
            if (r != STOKESFO_OK) { rc = r; goto done; }
            CU(e);
        }
        CU(cudaGraphInstantiate(&gexec, graph, 0));

        double nF0 = 0.0;
        int k = 0;
        for (;; ++k) {
            CK(eval_F(U, w.F));
            double ff;
            CK(dot_host(w.F, w.F, ff));
            const double nF = sqrt(ff);
            hist_F[k] = nF;
            if (k == 0) nF0 = nF;
            if (nF <= std::max(o->atol_newton, o->rtol_newton * nF0) || k >= o->max_newton) break;
            // Jacobi diagonal of J(U) + J_basal: the diagonal-only evaluation (no element matrices)
            CU(cudaMemsetAsync(w.diag, 0, vb, st));
            CK(stokesfo_jacobian_diag(c, U, w.diag, nullptr));
            if (nbasal > 0) {
                CU(cudaMemsetAsync(w.Z, 0, vb, st));
                CK(stokesfo_basal_friction(c, basal_cells, nbasal, beta, U, w.Z, w.Jf));
                const unsigned g = (unsigned)((nbasal * c->N + bs - 1) / bs);
                if (c->N == 8) diag_faces_kernel<8><<<g, bs, 0, st>>>(nbasal, basal_cells, c->d.conn, w.Jf, w.diag);
                else diag_faces_kernel<6><<<g, bs, 0, st>>>(nbasal, basal_cells, c->d.conn, w.Jf, w.diag);
            }
            // CG on J D = -F: D = 0, r = -F, z = r / diag, p = z, r.z -> s[RZ]
            CU(cudaMemsetAsync(w.D, 0, vb, st));
            CU(cudaMemsetAsync(w.Rr, 0, vb, st));
            axpby_kernel<<<gv, bs, 0, st>>>(n, -1.0, w.F, 0.0, w.Rr);
            jacobi_kernel<<<gv, bs, 0, st>>>(n, w.Rr, w.diag, w.Z);
            CU(cudaMemcpyAsync(w.P, w.Z, vb, cudaMemcpyDeviceToDevice, st));
            CK(dot_dev(w.Rr, w.Z, w.scal + S_RZ));
            const double tol2 = (o->rtol_cg * nF) * (o->rtol_cg * nF);
            int j = 0, done_at = -1;
            while (j < o->max_cg && done_at < 0) {
                CU(cudaMemsetAsync(w.scal + S_IT, 0, 8, st));
                CU(cudaGraphLaunch(gexec, st));
                CU(cudaMemcpyAsync(host_hist, w.hist, sizeof(host_hist), cudaMemcpyDeviceToHost, st));
                CU(cudaStreamSynchronize(st));
                for (int t = 0; t < CG_BLOCK; ++t)
                    if (done_at < 0 && host_hist[t] <= tol2) done_at = j + t + 1;
                j += CG_BLOCK;
            }
            if (hist_cg) hist_cg[k] = done_at > 0 ? done_at : j;  // iterations to convergence (the block may run a few more)
            // Armijo backtracking on ||F||
            double a = 1.0;
            for (int ls = 0;; ++ls) {
                CU(cudaMemcpyAsync(w.Ut, U, vb, cudaMemcpyDeviceToDevice, st));
                axpby_kernel<<<gv, bs, 0, st>>>(n, a, w.D, 1.0, w.Ut);
                CK(eval_F(w.Ut, w.Rr));
                double ft;
                CK(dot_host(w.Rr, w.Rr, ft));
                if (sqrt(ft) <= (1.0 - o->ls_c * a) * nF || ls >= o->max_ls) break;
                a *= 0.5;
            }
            CU(cudaMemcpyAsync(U, w.Ut, vb, cudaMemcpyDeviceToDevice, st));
        }
        *iters = k;
    }
done:
#undef CK
#undef CU
    cudaStreamSynchronize(st);
    if (gexec) cudaGraphExecDestroy(gexec);
    if (graph) cudaGraphDestroy(graph);
    c->stream = user;
    cudaEventRecord(ev, st);
    cudaStreamWaitEvent(user, ev, 0);
    cudaEventDestroy(ev);
    cudaStreamDestroy(st);
    return rc != STOKESFO_OK ? rc : cuda_status();
}

// CSR pattern: host-side construction from a device->host copy of conn.
int stokesfo_csr_pattern(stokesfo_ctx *c, int64_t *nnz, int64_t *rowptr, int32_t *colidx) {
    SFO_RANGE("stokesfo_csr_pattern");
    if (!c || !nnz) return STOKESFO_EINVAL;
    const int64_t C = c->d.num_cells, NN = c->d.num_nodes;
    const int N = c->N;
    std::vector<int32_t> conn((size_t)(C * N));
    if (C > 0 &&
        cudaMemcpyAsync(conn.data(), c->d.conn, conn.size() * 4, cudaMemcpyDeviceToHost, c->stream) != cudaSuccess)
        return cuda_status();
    if (cudaStreamSynchronize(c->stream) != cudaSuccess) return cuda_status();
    // conn is used as a host index below: range-check it first (EMESH, as the header states)
    for (int64_t i = 0; i < C * N; ++i)
        if (conn[i] < 0 || conn[i] >= NN) return STOKESFO_EMESH;
    // node -> cells (CSR)
    std::vector<int64_t> nc(NN + 1, 0);
    for (int64_t i = 0; i < C * N; ++i) nc[conn[i] + 1]++;
    for (int64_t v = 0; v < NN; ++v) nc[v + 1] += nc[v];
    if (C * N > INT32_MAX) return STOKESFO_EUNSUPPORTED;
    std::vector<int32_t> ncell(C * N);  // node -> cell N + local index, ascending cell order
    {
        std::vector<int64_t> pos(nc.begin(), nc.end() - 1);
        for (int64_t i = 0; i < C * N; ++i) ncell[pos[conn[i]]++] = (int32_t)i;
    }
    // node -> sorted unique neighbour nodes
    std::vector<int64_t> rp(2 * NN + 1, 0);
    std::vector<int32_t> nb;
    std::vector<int32_t> all;
    std::vector<int64_t> nstart(NN + 1, 0);
    for (int64_t v = 0; v < NN; ++v) {
        nb.clear();
        for (int64_t k = nc[v]; k < nc[v + 1]; ++k) {
            const int64_t cell = ncell[k] / N;
            for (int n = 0; n < N; ++n) nb.push_back(conn[cell * N + n]);
        }
        std::sort(nb.begin(), nb.end());
        nb.erase(std::unique(nb.begin(), nb.end()), nb.end());
        all.insert(all.end(), nb.begin(), nb.end());
        nstart[v + 1] = (int64_t)all.size();
    }
    for (int64_t v = 0; v < NN; ++v) {
        const int64_t deg = 2 * (nstart[v + 1] - nstart[v]);
        rp[2 * v + 1] = rp[2 * v] + deg;
        rp[2 * v + 2] = rp[2 * v + 1] + deg;
    }
    *nnz = rp[2 * NN];
    int64_t maxdeg = 0;
    for (int64_t v = 0; v < NN; ++v) maxdeg = std::max(maxdeg, nstart[v + 1] - nstart[v]);
    if (!rowptr || !colidx) return STOKESFO_OK;
    if (!aligned(rowptr, 16)) return STOKESFO_EINVAL;  // (rowptr[2v], rowptr[2v+1]) pairs are loaded as 16 B
    if (!aligned(rowptr, 8) || !aligned(colidx, 4)) return STOKESFO_EINVAL;
    std::vector<int32_t> ci((size_t)*nnz);
    for (int64_t v = 0; v < NN; ++v)
        for (int a = 0; a < 2; ++a) {
            int64_t o = rp[2 * v + a];
            for (int64_t k = nstart[v]; k < nstart[v + 1]; ++k) {
                ci[o++] = 2 * all[k];
                ci[o++] = 2 * all[k] + 1;
            }
        }
    if (cudaMemcpyAsync(rowptr, rp.data(), rp.size() * 8, cudaMemcpyHostToDevice, c->stream) != cudaSuccess)
        return cuda_status();
    if (!ci.empty() &&
        cudaMemcpyAsync(colidx, ci.data(), ci.size() * 4, cudaMemcpyHostToDevice, c->stream) != cudaSuccess)
        return cuda_status();
    if (cudaStreamSynchronize(c->stream) != cudaSuccess) return cuda_status();
    c->rowptr = rowptr;
    c->colidx = colidx;
    c->csr_rows = 2 * NN;
    c->csr_maxdeg = maxdeg;
    c->slots = nullptr;  // a new pattern invalidates an attached slot table
    c->inc_ptr = nullptr;
    c->inc = nullptr;
    c->nrec = nullptr;
    c->inc_ptr_h = std::move(nc);
    c->inc_h = std::move(ncell);
    return STOKESFO_OK;
}

}  // extern "C"
