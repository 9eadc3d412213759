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
