// sfo_mesh.cpp -- host-side mesh construction exported by libstokesfo.so:
// extrusion and numbering, column
// partition and halo lists.  Integer outputs are checked
// bit-exactly against the oracle's independent set-algebra versions.
#include <algorithm>
#include <cstdint>
#include <vector>

#include "../../include/stokesfo.h"

extern "C" {

int stokesfo_mesh_extrude(int32_t npoly, int64_t nv, const double *xy, int64_t nf, const int32_t *polys,
                          const double *b, const double *H, int32_t L, int32_t *conn, double *coords) {
    if ((npoly != 3 && npoly != 4) || nv < 0 || nf < 0 || L < 1) return STOKESFO_EINVAL;
    if (nv * (int64_t)(L + 1) > INT32_MAX) return STOKESFO_EINVAL;
    if ((nv > 0 && (!xy || !b || !H || !coords)) || (nf > 0 && (!polys || !conn))) return STOKESFO_EINVAL;
    const int64_t stride = L + 1;
    for (int64_t v = 0; v < nv; ++v)
        for (int32_t k = 0; k <= L; ++k) {
            double *x = coords + 3 * (v * stride + k);
            x[0] = xy[2 * v + 0];
            x[1] = xy[2 * v + 1];
            const double sigma = (double)k / (double)L;  // uniform sigma levels (reading Z10)
            x[2] = b[v] + H[v] * sigma;
        }
    const int npc = 2 * npoly;
    for (int64_t f = 0; f < nf; ++f) {
        for (int m = 0; m < npoly; ++m) {
            const int32_t v = polys[f * npoly + m];
            if (v < 0 || v >= nv) return STOKESFO_EINVAL;
        }
        for (int32_t k = 0; k < L; ++k) {
            int32_t *cc = conn + (f * L + k) * npc;
            for (int m = 0; m < npoly; ++m) {
                const int64_t base = (int64_t)polys[f * npoly + m] * stride + k;
                cc[m] = (int32_t)base;              // level k (bottom face)
                cc[npoly + m] = (int32_t)(base + 1); // level k+1 (top face)
            }
        }
    }
    return STOKESFO_OK;
}

int stokesfo_mesh_partition_columns(int64_t nf, int32_t nparts, int64_t *ranges) {
    if (nf < 0 || nparts < 1 || !ranges) return STOKESFO_EINVAL;
    for (int32_t r = 0; r <= nparts; ++r) ranges[r] = (nf * r) / nparts;
    return STOKESFO_OK;
}

int stokesfo_mesh_localize(int32_t npc, int64_t ncells, const int32_t *conn_global, int64_t *num_local_nodes,
                           int64_t *gids, int32_t *conn_local) {
    if (npc < 1 || ncells < 0 || !num_local_nodes || (ncells > 0 && !conn_global)) return STOKESFO_EINVAL;
    std::vector<int64_t> ids(conn_global, conn_global + ncells * npc);
    std::sort(ids.begin(), ids.end());
    ids.erase(std::unique(ids.begin(), ids.end()), ids.end());
    *num_local_nodes = (int64_t)ids.size();
    if (!gids) return STOKESFO_OK;
    std::copy(ids.begin(), ids.end(), gids);
    if (conn_local)
        for (int64_t i = 0; i < ncells * npc; ++i)
            conn_local[i] = (int32_t)(std::lower_bound(ids.begin(), ids.end(), (int64_t)conn_global[i]) - ids.begin());
    return STOKESFO_OK;
}

int stokesfo_mesh_halo_list(int64_t n_mine, const int64_t *gids_mine, int64_t n_other, const int64_t *gids_other,
                            int64_t *n_shared, int32_t *idx) {
    if (n_mine < 0 || n_other < 0 || !n_shared) return STOKESFO_EINVAL;
    int64_t i = 0, j = 0, k = 0;
    while (i < n_mine && j < n_other) {  // merge of two ascending lists
        if (gids_mine[i] < gids_other[j]) ++i;
        else if (gids_mine[i] > gids_other[j]) ++j;
        else {
            if (idx) idx[k] = (int32_t)i;
            ++k; ++i; ++j;
        }
    }
    *n_shared = k;
    return STOKESFO_OK;
}

int stokesfo_mesh_lateral_faces(int32_t npoly, int64_t nf, const int32_t *polys, int32_t L, int64_t *nfaces,
                                int32_t *faces) {
    if ((npoly != 3 && npoly != 4) || nf < 0 || L < 1 || !nfaces || (nf > 0 && !polys)) return STOKESFO_EINVAL;
    if (nf * (int64_t)L > INT32_MAX) return STOKESFO_EINVAL;
    // undirected edge key (min, max) of every polygon side; a boundary side is
    // one whose key occurs once.  Sort the keys, then look each side up.
    std::vector<std::pair<int64_t, int64_t>> keys;
    keys.reserve((size_t)(nf * npoly));
    auto key = [&](int64_t f, int m) {
        const int64_t a = polys[f * npoly + m], b = polys[f * npoly + (m + 1) % npoly];
        return std::make_pair(std::min(a, b), std::max(a, b));
    };
    for (int64_t f = 0; f < nf; ++f)
        for (int m = 0; m < npoly; ++m) keys.push_back(key(f, m));
    std::sort(keys.begin(), keys.end());
    int64_t n = 0;
    for (int64_t f = 0; f < nf; ++f)
        for (int m = 0; m < npoly; ++m) {
            const auto kk = key(f, m);
            const auto r = std::equal_range(keys.begin(), keys.end(), kk);
            if (r.second - r.first != 1) continue;
            if (faces)
                for (int32_t l = 0; l < L; ++l) {  // (f, side, layer) order; cell = f L + l (reading Z10)
                    faces[2 * (n + l) + 0] = (int32_t)(f * L + l);
                    faces[2 * (n + l) + 1] = m;
                }
            n += L;
        }
    *nfaces = n;
    return STOKESFO_OK;
}

}  // extern "C"
