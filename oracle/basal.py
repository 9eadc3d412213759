"""Oracle for the basal-friction side-set term (NEXT-4; PAPER.md P:L59 -> ref
[24], Tezaur et al. 2015: basal sliding boundary condition 2 mu eps_1 . n +
beta u = 0 on the bed).  TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Weak form on the bed Gamma_b (reading Z18: linear friction law with
a nodal friction coefficient beta, interpolated with the face basis):
    R[i][a] += int_{Gamma_b} beta_h(x) u_{h,a}(x) phi_i(x) dGamma
    J[(i,a),(j,b)] = delta_ab int_{Gamma_b} beta_h phi_i phi_j dGamma
Face = bottom face of a basal cell (hex8 local nodes 0-3, wedge6 nodes 0-2).
Quadrature: 2x2 Gauss (quad face, xi fastest, -1/sqrt(3) first) or the
3-point interior triangle rule (1/6,1/6),(2/3,1/6),(1/6,2/3), w = 1/6.
Surface measure |dx/dxi x dx/deta| at each face QP, computed in face-local
coordinates (x_n - x_0, reading Z17).  Plain numpy, one face at a time.
"""
from __future__ import annotations

import numpy as np


def face_rule(nb: int):
    """(points [Qf][2], weights [Qf], phi [nb][Qf], dphi [nb][Qf][2]) of the face."""
    if nb == 4:
        g = 1.0 / np.sqrt(3.0)
        pts = np.array([(i and g or -g, j and g or -g) for j in (0, 1) for i in (0, 1)])
        w = np.ones(4)
        sx = np.array([-1.0, 1.0, 1.0, -1.0])
        sy = np.array([-1.0, -1.0, 1.0, 1.0])
        phi = np.zeros((4, 4))
        dphi = np.zeros((4, 4, 2))
        for n in range(4):
            for q, (x, y) in enumerate(pts):
                phi[n, q] = 0.25 * (1 + sx[n] * x) * (1 + sy[n] * y)
                dphi[n, q, 0] = 0.25 * sx[n] * (1 + sy[n] * y)
                dphi[n, q, 1] = 0.25 * (1 + sx[n] * x) * sy[n]
        return pts, w, phi, dphi
    pts = np.array([(1 / 6, 1 / 6), (2 / 3, 1 / 6), (1 / 6, 2 / 3)])
    w = np.full(3, 1.0 / 6.0)
    phi = np.zeros((3, 3))
    dphi = np.zeros((3, 3, 2))
    for q, (x, y) in enumerate(pts):
        phi[:, q] = (1 - x - y, x, y)
        dphi[:, q, :] = ((-1, -1), (1, 0), (0, 1))
    return pts, w, phi, dphi


def basal_friction(nb: int, conn, coords, cells, beta, U):
    """Returns (R [nodes][2] contribution, J_face [len(cells)][2nb][2nb],
    area [len(cells)]) for the bottom faces of `cells`."""
    pts, w, phi, dphi = face_rule(nb)
    R = np.zeros((coords.shape[0], 2))
    Jf = np.zeros((len(cells), 2 * nb, 2 * nb))
    area = np.zeros(len(cells))
    for k, c in enumerate(cells):
        nodes = conn[c, :nb]
        x = coords[nodes] - coords[nodes[0]]
        for q in range(len(w)):
            t0 = (x * dphi[:, q, 0:1]).sum(0)
            t1 = (x * dphi[:, q, 1:2]).sum(0)
            ds = np.linalg.norm(np.cross(t0, t1)) * w[q]
            area[k] += ds
            bq = float(beta[nodes] @ phi[:, q])
            for a in range(2):
                uq = float(U[nodes, a] @ phi[:, q])
                for i in range(nb):
                    R[nodes[i], a] += ds * bq * uq * phi[i, q]
            for i in range(nb):
                for j in range(nb):
                    m = ds * bq * phi[i, q] * phi[j, q]
                    Jf[k, 2 * i, 2 * j] += m
                    Jf[k, 2 * i + 1, 2 * j + 1] += m
    return R, Jf, area
