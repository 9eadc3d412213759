"""Seeded synthetic input generators (footprints and fields).

This module is shared by the CUDA path's tests/bench and by the oracle's tests.
It holds *none* of the method's arithmetic: no extrusion, numbering, basis,
geometry, viscosity, residual or Jacobian.  It only draws the inputs the paper's
workload is made of (Sec. III-B: an Antarctic footprint of
quadrilaterals, extruded by layers; L61: prisms from a triangulation), with the
shapes, sizes and value distributions restated in SURVEY.md Sec. 8(d1) and
DESIGN.md "Input recipe".

A footprint is a 2-D polygon mesh plus per-vertex bed ``b`` and thickness ``H``
(km).  Fields are returned per extruded node in the layout ``[nv][L+1][...]``;
reshaping to ``[nv*(L+1)][...]`` is the identity under the node numbering
v*(L+1)+k that both sides implement independently (reading Z10).
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np


@dataclasses.dataclass
class Footprint:
    """2-D footprint: xy [nv,2] km, polys [nf,npoly] int32 (CCW), b/H [nv] km."""

    name: str
    xy: np.ndarray
    polys: np.ndarray
    b: np.ndarray
    H: np.ndarray
    dist: np.ndarray | None = None      # distance to margin [nv] (km), for fields
    grid_ij: np.ndarray | None = None   # optional integer grid coords of columns

    @property
    def nv(self) -> int:
        return int(self.xy.shape[0])

    @property
    def nf(self) -> int:
        return int(self.polys.shape[0])

    @property
    def npoly(self) -> int:
        return int(self.polys.shape[1])


# ----------------------------------------------------------------------------
# Hilbert ordering (locality of columns; SURVEY 7 "Hilbert-order the columns")
# ----------------------------------------------------------------------------

def hilbert_index(ix: np.ndarray, iy: np.ndarray, order: int) -> np.ndarray:
    """Vectorised Hilbert-curve index of integer points in [0, 2**order)^2."""
    x = ix.astype(np.int64).copy()
    y = iy.astype(np.int64).copy()
    d = np.zeros_like(x)
    s = 1 << (order - 1)
    while s > 0:
        rx = ((x & s) > 0).astype(np.int64)
        ry = ((y & s) > 0).astype(np.int64)
        d += s * s * ((3 * rx) ^ ry)
        # rotate
        m = ry == 0
        flip = m & (rx == 1)
        x = np.where(flip, s - 1 - x, x)
        y = np.where(flip, s - 1 - y, y)
        xs = np.where(m, y, x)
        ys = np.where(m, x, y)
        x, y = xs, ys
        s >>= 1
    return d


def _renumber_vertices_by_first_use(polys: np.ndarray, nv_all: int):
    """Number vertices in order of first appearance in ``polys`` (row-major).

    Returns (new_polys, old_ids_of_new) so that locality follows column order.
    """
    flat = polys.reshape(-1)
    uniq, first = np.unique(flat, return_index=True)
    order = np.argsort(first, kind="stable")
    old_of_new = uniq[order]
    new_of_old = np.full(nv_all, -1, dtype=np.int64)
    new_of_old[old_of_new] = np.arange(old_of_new.size)
    return new_of_old[polys].astype(np.int32), old_of_new


# ----------------------------------------------------------------------------
# C1/C2: tiny structured footprint (BASELINE.json configs[0], configs[1])
# ----------------------------------------------------------------------------

def tiny_footprint(n: int = 16, h: float = 1.0, jitter: float = 0.2, seed: int = 0,
                   name: str = "C1") -> Footprint:
    """[0, n*h]^2 km of h-km quads; interior vertices jittered U(+-jitter) km.

    b = 0.1 sin(x/3) cos(y/4) km;  H = 1 + 0.5 sin(pi x/16) sin(pi y/16) km
    (SURVEY 8(d1) row C1).  Vertex v = j*(n+1)+i; quad f = j*n+i, CCW.
    """
    rng = np.random.default_rng(seed)
    i, j = np.meshgrid(np.arange(n + 1), np.arange(n + 1), indexing="xy")
    x = (i * h).astype(np.float64).reshape(-1)
    y = (j * h).astype(np.float64).reshape(-1)
    interior = ((i > 0) & (i < n) & (j > 0) & (j < n)).reshape(-1)
    if jitter > 0:
        jx = rng.uniform(-jitter, jitter, size=x.size)
        jy = rng.uniform(-jitter, jitter, size=y.size)
        x = np.where(interior, x + jx, x)
        y = np.where(interior, y + jy, y)
    L_ext = n * h
    b = 0.1 * np.sin(x / 3.0) * np.cos(y / 4.0)
    H = 1.0 + 0.5 * np.sin(math.pi * x / L_ext) * np.sin(math.pi * y / L_ext)
    fi, fj = np.meshgrid(np.arange(n), np.arange(n), indexing="xy")
    fi = fi.reshape(-1)
    fj = fj.reshape(-1)
    v00 = fj * (n + 1) + fi
    polys = np.stack([v00, v00 + 1, v00 + n + 2, v00 + n + 1], axis=1).astype(np.int32)
    # distance to the box boundary (for the balance-like field option)
    dist = np.minimum.reduce([x, y, L_ext - x, L_ext - y])
    return Footprint(name, np.stack([x, y], 1), polys, b, H, dist=dist,
                     grid_ij=np.stack([fi, fj], 1))


# ----------------------------------------------------------------------------
# C4: Antarctica-like union of ellipses (BASELINE.json configs[3])
# ----------------------------------------------------------------------------

def _in_ellipse(x, y, cx, cy, a, bb, th=0.0):
    c, s = math.cos(th), math.sin(th)
    xr = (x - cx) * c + (y - cy) * s
    yr = -(x - cx) * s + (y - cy) * c
    return (xr / a) ** 2 + (yr / bb) ** 2 < 1.0


def antarctica_mask(xc: np.ndarray, yc: np.ndarray) -> np.ndarray:
    """E(350,0;2250,1950) u W(-1250,300;1000,700;0.3)
    u Peninsula(-2050,1250;150,750;-0.6) minus embayments (-550,-750;450,350)
    and (-850,1150;450,320)."""
    m = _in_ellipse(xc, yc, 350.0, 0.0, 2250.0, 1950.0)
    m |= _in_ellipse(xc, yc, -1250.0, 300.0, 1000.0, 700.0, 0.3)
    m |= _in_ellipse(xc, yc, -2050.0, 1250.0, 150.0, 750.0, -0.6)
    m &= ~_in_ellipse(xc, yc, -550.0, -750.0, 450.0, 350.0)
    m &= ~_in_ellipse(xc, yc, -850.0, 1150.0, 450.0, 320.0)
    return m


def antarctica_footprint(h: float = 4.0, hmax: float = 4.0, radius: float = 900.0,
                         name: str = "C4") -> Footprint:
    """Uniform h-km grid masked on cell centres; columns in Hilbert order.

    Vertices sit at multiples of h; grid spans [-2700, 2700] x [-2400, 2400] km
    (covers every ellipse).  H = max(0.02, hmax*(1-(1-min(d/R,1))^(4/3))^(3/8))
    with d = distance to the margin (Vialov-type); b = 0.5 sin(2 pi x/800)
    cos(2 pi y/600) - 0.2.
    """
    from scipy import ndimage

    x0, x1, y0, y1 = -2700.0, 2700.0, -2400.0, 2400.0
    nx = int(round((x1 - x0) / h))
    ny = int(round((y1 - y0) / h))
    ci, cj = np.meshgrid(np.arange(nx), np.arange(ny), indexing="ij")
    xc = x0 + (ci + 0.5) * h
    yc = y0 + (cj + 0.5) * h
    mask = antarctica_mask(xc, yc)
    fi = ci[mask]
    fj = cj[mask]
    order_bits = int(math.ceil(math.log2(max(nx, ny))))
    hidx = hilbert_index(fi, fj, order_bits)
    perm = np.argsort(hidx, kind="stable")
    fi = fi[perm]
    fj = fj[perm]
    # vertex (i,j) global id on the (nx+1)x(ny+1) lattice
    vid = lambda i, j: i * (ny + 1) + j  # noqa: E731
    polys_all = np.stack([vid(fi, fj), vid(fi + 1, fj), vid(fi + 1, fj + 1), vid(fi, fj + 1)], 1)
    polys, old_of_new = _renumber_vertices_by_first_use(polys_all, (nx + 1) * (ny + 1))
    vi = old_of_new // (ny + 1)
    vj = old_of_new % (ny + 1)
    x = x0 + vi * h
    y = y0 + vj * h
    # distance to margin: lattice vertices that touch an outside cell are margin
    inside_cells = np.zeros((nx + 2, ny + 2), dtype=bool)
    inside_cells[1:-1, 1:-1] = mask
    # vertex (i,j) touches cells (i-1..i, j-1..j) -> padded index (i..i+1, j..j+1)
    all_in = (inside_cells[:-1, :-1] & inside_cells[1:, :-1]
              & inside_cells[:-1, 1:] & inside_cells[1:, 1:])
    dist_lat = ndimage.distance_transform_edt(all_in) * h
    dist = dist_lat[vi, vj]
    H = np.maximum(0.02, hmax * (1.0 - (1.0 - np.minimum(dist / radius, 1.0)) ** (4.0 / 3.0)) ** (3.0 / 8.0))
    b = 0.5 * np.sin(2 * math.pi * x / 800.0) * np.cos(2 * math.pi * y / 600.0) - 0.2
    return Footprint(name, np.stack([x, y], 1).astype(np.float64), polys, b, H, dist=dist,
                     grid_ij=np.stack([fi, fj], 1))


def split_to_triangles(fp: Footprint, name: str | None = None) -> Footprint:
    """C5: split each quad on the alternating diagonal (by (i+j) parity of the
    column's grid coordinates, else by index parity).  Both triangles CCW."""
    q = fp.polys
    if fp.grid_ij is not None:
        par = (fp.grid_ij[:, 0] + fp.grid_ij[:, 1]) % 2
    else:
        par = np.arange(q.shape[0]) % 2
    a, b_, c, d = q[:, 0], q[:, 1], q[:, 2], q[:, 3]
    # parity 0: diagonal a-c ; parity 1: diagonal b-d
    t1 = np.where(par[:, None] == 0, np.stack([a, b_, c], 1), np.stack([a, b_, d], 1))
    t2 = np.where(par[:, None] == 0, np.stack([a, c, d], 1), np.stack([b_, c, d], 1))
    tris = np.stack([t1, t2], 1).reshape(-1, 3).astype(np.int32)
    gij = None
    if fp.grid_ij is not None:
        gij = np.repeat(fp.grid_ij, 2, axis=0)
    return Footprint(name or fp.name + "-wedge", fp.xy, tris, fp.b, fp.H, dist=fp.dist,
                     grid_ij=gij)


# ----------------------------------------------------------------------------
# Fields on the extruded nodes / cells
# ----------------------------------------------------------------------------

def velocity_random(fp: Footprint, L: int, sigma: float = 100.0, seed: int = 100) -> np.ndarray:
    """U ~ N(0, sigma) m/yr per node and component; shape [nv*(L+1), 2]."""
    rng = np.random.default_rng(seed)
    return rng.normal(0.0, sigma, size=(fp.nv * (L + 1), 2))


def velocity_balance(fp: Footprint, L: int, seed: int = 12) -> np.ndarray:
    """Balance-like field: speed 10 + 990 exp(-d/100 km) m/yr along -grad d,
    vertical shear profile (1 - 0.8 (1-sigma)^4), 5% N(0,1) perturbation
    (SURVEY 8(d1) row C3).  Direction from the centroid-relative position when
    grad d is unavailable.  Shape [nv*(L+1), 2]."""
    rng = np.random.default_rng(seed)
    d = fp.dist if fp.dist is not None else np.zeros(fp.nv)
    speed = 10.0 + 990.0 * np.exp(-d / 100.0)
    # outward direction: away from the footprint's thickest region (proxy for -grad d)
    cx, cy = fp.xy[np.argmax(d)] if d.size else (0.0, 0.0)
    dx = fp.xy[:, 0] - cx
    dy = fp.xy[:, 1] - cy
    nrm = np.hypot(dx, dy) + 1e-9
    ux = speed * dx / nrm
    uy = speed * dy / nrm
    sig = np.arange(L + 1) / L
    prof = 1.0 - 0.8 * (1.0 - sig) ** 4
    U = np.empty((fp.nv, L + 1, 2))
    U[:, :, 0] = ux[:, None] * prof[None, :]
    U[:, :, 1] = uy[:, None] * prof[None, :]
    U *= 1.0 + 0.05 * rng.normal(size=U.shape)
    return U.reshape(-1, 2)


def surface_nodal(fp: Footprint, L: int) -> np.ndarray:
    """Surface height s = b + H of the node's column, repeated over levels."""
    s = fp.b + fp.H
    return np.repeat(s, L + 1)


def flow_factor(fp: Footprint, L: int, a0: float = 1e-4) -> np.ndarray:
    """Per-cell k_c for A_c = a0 * 10^(-sigma_c) (warm bed, cold surface), with
    sigma_c = (k+1/2)/L the cell's mid-layer fraction; k_c = A_c^(-1/3)/2 is
    the Glen prefactor the ABI consumes (reading Z1/Z4). [nf*L]."""
    sig = (np.arange(L) + 0.5) / L
    A = a0 * 10.0 ** (-sig)
    kc = 0.5 * A ** (-1.0 / 3.0)
    return np.tile(kc, fp.nf)


# ----------------------------------------------------------------------------
# Named configurations (BASELINE.json configs)
# ----------------------------------------------------------------------------

CONFIGS = {
    "C1": dict(desc="tiny 16x16 x 5 layers hex8, residual", layers=5, elem="hex8"),
    "C2": dict(desc="tiny 16x16 x 5 layers hex8, residual+Jacobian", layers=5, elem="hex8"),
    "C3": dict(desc="Greenland-like 1-10 km NVB footprint x 10 layers hex8, residual+Jacobian", layers=10,
               elem="hex8"),
    "C4": dict(desc="Antarctica-like 4 km x 10 layers hex8, residual+Jacobian", layers=10, elem="hex8"),
    "C4p": dict(desc="paper-shaped: Antarctica-like 16 km x 20 layers hex8 (~256K hex per GPU at 4 GPUs, "
                     "PAPER.md P:L74-82)", layers=20, elem="hex8"),
    "C5": dict(desc="Antarctica-like 4 km x 10 layers wedge6, residual+Jacobian", layers=10, elem="wedge6"),
}

PHYS_DEFAULTS = dict(k=10.77, glen_n=3.0, delta=1e-10, rho_g=8.927)


def make_config(name: str, h: float | None = None):
    """Return (footprint, L, elem) for a named configuration (C3 is defined
    below; the module is fully imported before this is called)."""
    cfg = CONFIGS[name]
    if name in ("C1", "C2"):
        fp = tiny_footprint()
    elif name == "C3":
        fp = greenland_footprint()
    elif name == "C4":
        fp = antarctica_footprint(h=h or 4.0)
    elif name == "C4p":
        fp = antarctica_footprint(h=h or 16.0, name="C4p")
    elif name == "C5":
        fp = split_to_triangles(antarctica_footprint(h=h or 4.0), name="C5")
    else:
        raise KeyError(name)
    return fp, cfg["layers"], cfg["elem"]


# ----------------------------------------------------------------------------
# C3: Greenland-like variable-resolution footprint (BASELINE.json configs[2])
# ----------------------------------------------------------------------------

def _greenland_halfwidth(y):
    c1 = np.clip((y - 200.0) / 1100.0, 0.0, 1.0)
    c2 = np.clip((-y - 550.0) / 550.0, 0.0, 1.0)
    return 480.0 * (1.0 - 0.45 * c1 ** 2) * (1.0 - 0.35 * c2)


def greenland_inside(x, y):
    """|x/w(y)|^2.5 + |y/1150|^2.5 < 1."""
    return np.abs(x / _greenland_halfwidth(y)) ** 2.5 + np.abs(y / 1150.0) ** 2.5 < 1.0


def greenland_footprint(h0: float = 20.0, hmin: float = 1.0, hmax: float = 10.0, ramp: float = 150.0,
                        raster: float = 1.0, name: str = "C3") -> Footprint:
    """Newest-vertex-bisection refinement (with conformity closure) of a
    criss-cross right-triangle background of h0-km squares until every
    hypotenuse <= 2 sqrt(2) h(d(centroid)), h(d) = min(hmax, hmin + (hmax-hmin) d/ramp),
    d = distance to the margin; keep triangles whose centroid is inside; split
    each triangle into 3 quads through its centroid and edge midpoints; columns
    in Hilbert order (SURVEY 8(d1) 'C3 footprint construction').

    H = max(0.02, 3.2 (1 - (1 - min(d/500, 1))^(4/3))^(3/8)) km;
    b = 0.3 sin(2 pi x/400) cos(2 pi y/300) km.
    """
    from scipy import ndimage
    x0, x1, y0, y1 = -560.0, 560.0, -1200.0, 1200.0
    nx, ny = int((x1 - x0) / h0), int((y1 - y0) / h0)
    # margin distance on a raster (outside and inside distances, unsigned)
    gx = np.arange(x0, x1 + raster, raster)
    gy = np.arange(y0, y1 + raster, raster)
    GX, GY = np.meshgrid(gx, gy, indexing="ij")
    ins = greenland_inside(GX, GY)
    d_in = ndimage.distance_transform_edt(ins) * raster
    d_out = ndimage.distance_transform_edt(~ins) * raster
    dist_r = np.where(ins, d_in, d_out)

    def dist_at(px, py):
        i = np.clip(np.rint((px - x0) / raster).astype(np.int64), 0, gx.size - 1)
        j = np.clip(np.rint((py - y0) / raster).astype(np.int64), 0, gy.size - 1)
        return dist_r[i, j]

    def hsize(d):
        return np.minimum(hmax, hmin + (hmax - hmin) * d / ramp)

    # --- background: vertices of the h0 lattice + square centres -------------
    verts = []
    vid = {}

    def vert(p):
        key = (round(p[0] * 1e6), round(p[1] * 1e6))
        if key not in vid:
            vid[key] = len(verts)
            verts.append((p[0], p[1]))
        return vid[key]

    # triangle = (e0, e1, apex): CCW, refinement edge e0-e1 (the hypotenuse)
    tris = {}
    tid = 0
    for i in range(nx):
        for j in range(ny):
            a = vert((x0 + i * h0, y0 + j * h0))
            b = vert((x0 + (i + 1) * h0, y0 + j * h0))
            c = vert((x0 + (i + 1) * h0, y0 + (j + 1) * h0))
            d = vert((x0 + i * h0, y0 + (j + 1) * h0))
            m = vert((x0 + (i + 0.5) * h0, y0 + (j + 0.5) * h0))
            for e0, e1 in ((a, b), (b, c), (c, d), (d, a)):
                tris[tid] = (e0, e1, m)
                tid += 1
    edge_tris = {}

    def ekey(u, v):
        return (u, v) if u < v else (v, u)

    def add_tri(t, tri):
        tris[t] = tri
        for u, v in ((tri[0], tri[1]), (tri[1], tri[2]), (tri[2], tri[0])):
            edge_tris.setdefault(ekey(u, v), set()).add(t)

    def del_tri(t):
        tri = tris.pop(t)
        for u, v in ((tri[0], tri[1]), (tri[1], tri[2]), (tri[2], tri[0])):
            edge_tris[ekey(u, v)].discard(t)

    for t, tri in list(tris.items()):
        add_tri(t, tri)
    next_id = [tid]
    mids = {}

    def midpoint(u, v):
        k = ekey(u, v)
        if k not in mids:
            pu, pv = verts[u], verts[v]
            mids[k] = vert((0.5 * (pu[0] + pv[0]), 0.5 * (pu[1] + pv[1])))
        return mids[k]

    def bisect(t):
        e0, e1, ap = tris[t]
        m = midpoint(e0, e1)
        del_tri(t)
        for tri in ((ap, e0, m), (e1, ap, m)):
            add_tri(next_id[0], tri)
            next_id[0] += 1

    def refine(t):
        if t not in tris:
            return
        e0, e1, _ = tris[t]
        nb = [s for s in edge_tris.get(ekey(e0, e1), ()) if s != t]
        if nb:
            s = nb[0]
            if ekey(*tris[s][:2]) != ekey(e0, e1):
                refine(s)
                nb = [s2 for s2 in edge_tris.get(ekey(e0, e1), ()) if s2 != t]
            bisect(t)
            for s in nb:
                if s in tris and ekey(*tris[s][:2]) == ekey(e0, e1):
                    bisect(s)
        else:
            bisect(t)

    import sys
    sys.setrecursionlimit(100000)
    while True:
        ids = np.fromiter(tris.keys(), dtype=np.int64)
        T = np.array([tris[t] for t in ids])
        V = np.asarray(verts)
        cen = V[T].mean(axis=1)
        hyp = np.hypot(*(V[T[:, 0]] - V[T[:, 1]]).T)
        mark = hyp > 2.0 * math.sqrt(2.0) * hsize(dist_at(cen[:, 0], cen[:, 1])) + 1e-9
        if not mark.any():
            break
        for t in ids[mark]:
            refine(int(t))
    ids = np.fromiter(tris.keys(), dtype=np.int64)
    T = np.array([tris[t] for t in ids], dtype=np.int64)
    V = np.asarray(verts)
    cen = V[T].mean(axis=1)
    T = T[greenland_inside(cen[:, 0], cen[:, 1])]
    # --- triangle -> 3 quads through centroid and edge midpoints -------------
    quads = []
    for a, b, c in T:
        g = vert(tuple(V[[a, b, c]].mean(axis=0)))
        mab, mbc, mca = midpoint(a, b), midpoint(b, c), midpoint(c, a)
        quads += [(a, mab, g, mca), (b, mbc, g, mab), (c, mca, g, mbc)]
    quads = np.array(quads, dtype=np.int64)
    V = np.asarray(verts)
    qc = V[quads].mean(axis=1)
    hi = np.floor((qc - np.array([x0, y0])) / 0.5).astype(np.int64)
    order = np.argsort(hilbert_index(hi[:, 0], hi[:, 1], 13), kind="stable")
    quads = quads[order]
    polys, old_of_new = _renumber_vertices_by_first_use(quads, V.shape[0])
    xy = V[old_of_new]
    d = dist_at(xy[:, 0], xy[:, 1]) * greenland_inside(xy[:, 0], xy[:, 1])
    H = np.maximum(0.02, 3.2 * (1.0 - (1.0 - np.minimum(d / 500.0, 1.0)) ** (4.0 / 3.0)) ** (3.0 / 8.0))
    b = 0.3 * np.sin(2 * math.pi * xy[:, 0] / 400.0) * np.cos(2 * math.pi * xy[:, 1] / 300.0)
    return Footprint(name, xy.astype(np.float64), polys, b, H, dist=d)
