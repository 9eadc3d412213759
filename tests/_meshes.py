"""Small seeded test meshes built with the ORACLE's extrusion (oracle.extrude)
from the shared input generators.  Used by both oracle pins and GPU parity
tests; never built from the CUDA path."""
from __future__ import annotations

import numpy as np

import oracle as O
from paper_conf_sc_antepara0cw24_b200 import synth


def tiny(elem: str = "hex8", n: int = 16, L: int = 5, jitter: float = 0.2, seed: int = 0):
    fp = synth.tiny_footprint(n=n, jitter=jitter, seed=seed)
    if elem == "wedge6":
        fp = synth.split_to_triangles(fp)
    conn, coords = O.extrude(fp.xy, fp.polys, fp.b, fp.H, L)
    return fp, conn, coords


def fields(fp, L, kind="random", seed=100):
    if kind == "random":
        U = synth.velocity_random(fp, L, seed=seed)
    else:
        U = synth.velocity_balance(fp, L, seed=seed)
    s = synth.surface_nodal(fp, L)
    kc = synth.flow_factor(fp, L)
    return U, s, kc


def box_cell(x0=(0.0, 0.0, 0.0), h=(2.0, 3.0, 0.5)):
    """One hex8 box cell in Shards order."""
    sx = [-1, 1, 1, -1, -1, 1, 1, -1]
    sy = [-1, -1, 1, 1, -1, -1, 1, 1]
    sz = [-1, -1, -1, -1, 1, 1, 1, 1]
    xyz = np.array([[x0[0] + 0.5 * h[0] * (1 + sx[n]), x0[1] + 0.5 * h[1] * (1 + sy[n]),
                     x0[2] + 0.5 * h[2] * (1 + sz[n])] for n in range(8)])
    return np.arange(8, dtype=np.int32)[None, :], xyz


def interior_nodes(fp, L, conn_nodes_count):
    """Nodes strictly inside the extruded block: not on the lateral boundary of
    the footprint, not on the bed (k=0) nor the surface (k=L)."""
    nv = fp.nv
    # lateral boundary vertices: edges used by exactly one polygon
    from collections import Counter
    cnt = Counter()
    npoly = fp.polys.shape[1]
    for poly in fp.polys:
        for m in range(npoly):
            a, b = int(poly[m]), int(poly[(m + 1) % npoly])
            cnt[(min(a, b), max(a, b))] += 1
    bnd = set()
    for (a, b), c in cnt.items():
        if c == 1:
            bnd.add(a)
            bnd.add(b)
    ids = []
    for v in range(nv):
        if v in bnd:
            continue
        for k in range(1, L):
            ids.append(v * (L + 1) + k)
    return np.array(ids, dtype=np.int64)


def rounding_scale_R(e, conn, G, wm, mu, U, s, rho_g):
    """A-priori rounding scale of R_cell[c][i][a] = sum_q wM_q (sigma_a(q) . G_i(q)
    + f_a(q) phi_i(q)): the sum of the absolute values of the terms that are added,
    with every Ugrad entry bounded by gbar_q = sum_n sum_a sum_d |U_n,a| |G_n[q][d]|
    (its value before cancellation) and |beta| <= 3 gbar:
        scale = sum_q wM_q (2 mu_q 3 gbar_q sum_d |G_i[q][d]|
                            + rho_g (sum_n |s_n| (|G_n0| + |G_n1|)) phi_i(q)).
    Two correct fp64 evaluations differ by O(eps) of it: on thin, wide cells (C4p:
    1 m x 16 km) the Ugrad sums cancel by up to 1e6 and the oracle itself moves by
    1e-11 of sum |R_cell| under a translation of the coordinates."""
    bf, _, _ = O.ref_element(e)               # [N][Q]
    Uc = np.abs(U[conn])                      # [C][N][2]
    aG = np.abs(G)                            # [C][N][Q][3]
    gbar = np.einsum("cna,cnqd->cq", Uc, aG)  # [C][Q]
    Gi = aG.sum(-1)                           # [C][N][Q]
    sc = np.einsum("cq,cnq->cn", wm * 2.0 * mu * 3.0 * gbar, Gi)
    if s is not None:
        fs = rho_g * np.einsum("cn,cnq->cq", np.abs(s[conn]), aG[..., 0] + aG[..., 1])
        sc = sc + np.einsum("cq,nq->cn", wm * fs, bf)
    return np.repeat(sc[:, :, None], 2, axis=2)
