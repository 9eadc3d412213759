"""Oracle for the lateral (calving-front / ocean) pressure side-set term
(NEXT-4; PAPER.md P:L59 -> ref [24]: "The full details of the model and the
boundary conditions ... are described in [24]").  TEST INFRASTRUCTURE ONLY
(see oracle/__init__.py).

Reading Z19: on the lateral boundary Gamma_l of the ice (the
vertical side faces over the footprint's boundary edges) the first-order
stress balances the hydrostatic ice overburden minus the ocean water pressure,
    2 mu eps_a . n = psi(z) n_a,   a = 0, 1,
    psi(z) = rho_i g (s - z) - rho_w g max(z_sl - z, 0),
so integrating eq. (1) against phi_i by parts (the volume residual of Fig. 2
is  int 2 mu eps_a . grad phi_i + rho g d_a s phi_i) adds
    R[i][a] -= int_{Gamma_l} psi(z) n_a phi_i dGamma.
Face of (cell, side k) = the quad over the footprint polygon's edge k -> k+1:
local nodes (k, k+1, k+1 + P, k + P) (P = 4 hex8 / 3 wedge6, indices mod P),
xi along the edge, eta upward; n dGamma = (dx/dxi x dx/deta) dxi deta, which
points outward for counter-clockwise footprint polygons.  Quadrature 2x2
Gauss (xi fastest, -1/sqrt(3) first), bilinear face basis in the Shards quad
order; z and s at a QP interpolated with the face basis (reading Z19).
The term does not depend on U: its Jacobian contribution is zero.
Plain numpy, one face at a time.
"""
from __future__ import annotations

import numpy as np


def boundary_sides(polys):
    """(f, k) of every footprint polygon side whose edge belongs to exactly one
    polygon (the footprint's boundary), ascending in (f, k).  Plain set algebra."""
    polys = np.asarray(polys)
    P = polys.shape[1]
    count = {}
    for f in range(polys.shape[0]):
        for k in range(P):
            a, b = int(polys[f, k]), int(polys[f, (k + 1) % P])
            key = (min(a, b), max(a, b))
            count[key] = count.get(key, 0) + 1
    out = []
    for f in range(polys.shape[0]):
        for k in range(P):
            a, b = int(polys[f, k]), int(polys[f, (k + 1) % P])
            if count[(min(a, b), max(a, b))] == 1:
                out.append((f, k))
    return np.array(out, dtype=np.int32).reshape(-1, 2)


def lateral_faces(polys, L: int):
    """Lateral faces [nfaces][2] = (cell, side) for every boundary side (f, k)
    and layer l = 0..L-1 (cell = f L + l, reading Z10), ordered by (f, k, l)."""
    sides = boundary_sides(polys)
    out = [(f * L + l, k) for f, k in sides for l in range(L)]
    return np.array(out, dtype=np.int32).reshape(-1, 2)


def face_nodes(P: int, k: int):
    """Local cell nodes of side k in face order (bottom k, bottom k+1, top k+1, top k)."""
    return [k, (k + 1) % P, (k + 1) % P + P, k + P]


def face_rule():
    """2x2 Gauss on [-1,1]^2 with the bilinear quad basis (Shards order)."""
    g = 1.0 / np.sqrt(3.0)
    pts = [(x, y) for y in (-g, g) for x in (-g, g)]
    sx = [-1.0, 1.0, 1.0, -1.0]
    sy = [-1.0, -1.0, 1.0, 1.0]
    phi = np.zeros((4, 4))
    dphi = np.zeros((4, 4, 2))
    for q, (x, y) in enumerate(pts):
        for n in range(4):
            phi[n, q] = 0.25 * (1 + sx[n] * x) * (1 + sy[n] * y)
            dphi[n, q, 0] = 0.25 * sx[n] * (1 + sy[n] * y)
            dphi[n, q, 1] = 0.25 * (1 + sx[n] * x) * sy[n]
    return np.ones(4), phi, dphi


def psi(z, s, rho_i_g, rho_w_g, z_sl):
    """Ice overburden minus ocean pressure at elevation z (reading Z19)."""
    return rho_i_g * (s - z) - rho_w_g * max(z_sl - z, 0.0)


def lateral_pressure(npc: int, conn, coords, faces, surface, rho_i_g, rho_w_g, z_sl):
    """Returns (R [nodes][2] contribution, force [nfaces][2] = -sum_i of the
    face's contributions = int psi n_a dGamma) for the listed (cell, side) faces."""
    P = npc // 2
    w, phi, dphi = face_rule()
    R = np.zeros((coords.shape[0], 2))
    force = np.zeros((len(faces), 2))
    for m, (c, k) in enumerate(faces):
        nodes = conn[c, face_nodes(P, int(k))]
        x = coords[nodes]
        xl = x - x[0]                        # face-local coordinates (reading Z17)
        for q in range(4):
            t0 = (xl * dphi[:, q, 0:1]).sum(0)
            t1 = (xl * dphi[:, q, 1:2]).sum(0)
            nd = np.cross(t0, t1) * w[q]     # n dGamma, outward for CCW polygons
            zq = float(x[:, 2] @ phi[:, q])
            sq = float(surface[nodes] @ phi[:, q])
            p = psi(zq, sq, rho_i_g, rho_w_g, z_sl)
            for a in range(2):
                force[m, a] += p * nd[a]
                for i in range(4):
                    R[nodes[i], a] -= p * nd[a] * phi[i, q]
    return R, force
