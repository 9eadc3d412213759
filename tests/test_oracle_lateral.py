"""Pins of the lateral-pressure oracle (NEXT-4, oracle/lateral.py; PAPER.md
P:L59 -> [24]; reading Z19) against what mechanics and geometry fix:
the 1/2 rho g H^2 spreading force of a grounded front, the
1/2 rho_i g H^2 (1 - rho_i/rho_w) force of a floating front, per-node closed
forms on a vertical rectangle, an independent adaptive quadrature of the
integral on a sloped face (above and below sea level), cancellation around a
closed column, rotation covariance, outward normals, and the boundary-edge set
by brute force."""
import numpy as np
import pytest

import oracle as O
from oracle import lateral as LT
from paper_conf_sc_antepara0cw24_b200 import synth

RIG = 8.927          # rho_i g (kPa/km-ish units, reading Z4)
RWG = 10.05          # rho_w g
NO_OCEAN = -1e30     # sea level far below the bed: no ocean pressure


def _column(xy, b, H, L):
    """One footprint polygon (CCW) extruded by L layers with the oracle's extrusion."""
    xy = np.asarray(xy, dtype=np.float64)
    P = xy.shape[0]
    polys = np.arange(P, dtype=np.int32)[None]
    conn, coords = O.extrude(xy, polys, np.asarray(b, float), np.asarray(H, float), L)
    s = np.repeat(np.asarray(b, float) + np.asarray(H, float), L + 1)   # s per node, v(L+1)+k numbering
    return polys, conn, coords, s


def test_boundary_sides_brute_force():
    for elem in ("hex8", "wedge6"):
        n = 5
        fp = synth.tiny_footprint(n=n, jitter=0.2, seed=1)
        if elem == "wedge6":
            fp = synth.split_to_triangles(fp)
        sides = LT.boundary_sides(fp.polys)
        assert len(sides) == 4 * n
        P = fp.polys.shape[1]
        for f, k in sides:   # both end vertices on the box boundary (interior vertices are jittered off it)
            for v in (fp.polys[f, k], fp.polys[f, (k + 1) % P]):
                x, y = fp.xy[v]
                assert min(x, y, n - x, n - y) == 0.0
        faces = LT.lateral_faces(fp.polys, 3)
        assert faces.shape == (3 * 4 * n, 2)
        assert (faces[:, 0] // 3 == np.repeat(sides[:, 0], 3)).all()
        assert (faces[:, 1] == np.repeat(sides[:, 1], 3)).all()


@pytest.mark.parametrize("L", [1, 4, 7])
def test_grounded_front_spreading_force(L):
    """Box column [0,a]x[0,w], no ocean: the x = a side pushes +x with
    rho_i g w H^2 / 2 (the textbook spreading force), exact for any L."""
    a, w, H = 2.0, 3.0, 1.3
    polys, conn, coords, s = _column([(0, 0), (a, 0), (a, w), (0, w)], [0.2] * 4, [H] * 4, L)
    faces = LT.lateral_faces(polys, L)
    R, F = LT.lateral_pressure(8, conn, coords, faces, s, RIG, RWG, NO_OCEAN)
    side = faces[:, 1]
    tot = {k: F[side == k].sum(0) for k in range(4)}
    ref = RIG * w * H * H / 2
    assert abs(tot[1][0] - ref) <= 1e-13 * ref and abs(tot[1][1]) <= 1e-13 * ref
    assert abs(tot[3][0] + ref) <= 1e-13 * ref
    refy = RIG * a * H * H / 2
    assert abs(tot[2][1] - refy) <= 1e-13 * refy and abs(tot[0][1] + refy) <= 1e-13 * refy
    # closed column: forces cancel; the residual is minus the face forces
    assert np.abs(F.sum(0)).max() <= 1e-13 * ref
    assert np.abs(R.sum(0) + F.sum(0)).max() <= 1e-13 * ref


def test_floating_front_force():
    """Shelf at flotation (draft rho_i/rho_w H, sea level on a layer interface):
    net push rho_i g H^2 / 2 (1 - rho_i / rho_w) per unit width."""
    H, L, a, w = 0.5, 10, 1.0, 2.0
    ratio = 0.9
    b = -ratio * H
    polys, conn, coords, s = _column([(0, 0), (a, 0), (a, w), (0, w)], [b] * 4, [H] * 4, L)
    faces = LT.lateral_faces(polys, L)
    R, F = LT.lateral_pressure(8, conn, coords, faces, s, RIG, RIG / ratio, 0.0)
    Fx = F[faces[:, 1] == 1].sum(0)[0]
    ref = RIG * w * H * H / 2 * (1 - ratio)
    assert abs(Fx - ref) <= 1e-12 * RIG * w * H * H


def test_vertical_rectangle_node_closed_form():
    """One layer, x = a face of width w between z0 and z1, psi linear in z:
    bottom nodes get -w/2 h (2 psi0 + psi1) / 6, top nodes -w/2 h (psi0 + 2 psi1) / 6."""
    a, w, z0, H = 1.5, 2.5, 0.3, 0.8
    polys, conn, coords, s = _column([(0, 0), (a, 0), (a, w), (0, w)], [z0] * 4, [H] * 4, 1)
    faces = np.array([[0, 1]], dtype=np.int32)
    R, F = LT.lateral_pressure(8, conn, coords, faces, s, RIG, RWG, NO_OCEAN)
    z1 = z0 + H
    p0, p1 = RIG * (z1 - z0), 0.0
    bot = -w / 2 * H * (2 * p0 + p1) / 6
    top = -w / 2 * H * (p0 + 2 * p1) / 6
    # local nodes of side 1: bottom 1, 2; top 6, 5
    for loc, ref in ((1, bot), (2, bot), (6, top), (5, top)):
        assert abs(R[conn[0, loc], 0] - ref) <= 1e-14 * abs(bot)
        assert abs(R[conn[0, loc], 1]) <= 1e-14 * abs(bot)
    untouched = [conn[0, m] for m in (0, 3, 4, 7)]
    assert np.abs(R[untouched]).max() == 0.0


@pytest.mark.parametrize("zsl", [NO_OCEAN, 50.0])
def test_sloped_face_vs_adaptive_quadrature(zsl):
    """Face over a slanted edge with different bed / thickness at its two ends
    (entirely above or entirely below sea level, so psi is smooth on the face):
    the 2x2 Gauss rule equals the exact integral, checked against scipy's
    adaptive dblquad of psi n_a phi_i on the bilinear face map."""
    from scipy import integrate
    xy = [(0.0, 0.0), (2.0, 0.4), (2.3, 1.9), (-0.2, 1.6)]
    b = [0.1, 0.35, 0.2, 0.05]
    H = [1.0, 0.6, 0.9, 1.2]
    polys, conn, coords, s = _column(xy, b, H, 2)
    for k in range(4):
        faces = np.array([[1, k]], dtype=np.int32)      # upper layer
        R, F = LT.lateral_pressure(8, conn, coords, faces, s, RIG, RWG, zsl)
        nodes = conn[1, LT.face_nodes(4, k)]
        X = coords[nodes]
        S = s[nodes]
        sx = np.array([-1.0, 1.0, 1.0, -1.0])
        sy = np.array([-1.0, -1.0, 1.0, 1.0])

        def phi(xi, et):
            return 0.25 * (1 + sx * xi) * (1 + sy * et)

        def integrand(et, xi, i, a):
            p = phi(xi, et)
            t0 = (0.25 * sx * (1 + sy * et)) @ X
            t1 = (0.25 * (1 + sx * xi) * sy) @ X
            nd = np.cross(t0, t1)
            z = p @ X[:, 2]
            ps = RIG * (p @ S - z) - RWG * max(zsl - z, 0.0)
            return -ps * nd[a] * p[i]

        for i in range(4):
            for a in range(2):
                ref, _ = integrate.dblquad(integrand, -1, 1, -1, 1, args=(i, a), epsabs=1e-15, epsrel=1e-13)
                assert abs(R[nodes[i], a] - ref) <= 1e-12 * max(abs(ref), np.abs(F).max())


def test_rotation_covariance_and_outward_normals():
    fp = synth.tiny_footprint(n=4, jitter=0.2, seed=3)
    L = 3
    conn, coords = O.extrude(fp.xy, fp.polys, fp.b, fp.H, L)
    s = synth.surface_nodal(fp, L)
    faces = LT.lateral_faces(fp.polys, L)
    R, F = LT.lateral_pressure(8, conn, coords, faces, s, RIG, RWG, -5.0)
    # outward: the force of every boundary face points away from the box centre
    ctr = np.array([2.0, 2.0])
    for m, (c, k) in enumerate(faces):
        mid = coords[conn[c, LT.face_nodes(4, int(k))], :2].mean(0)
        assert F[m] @ (mid - ctr) > 0
    th = 0.7
    Rm = np.array([[np.cos(th), -np.sin(th)], [np.sin(th), np.cos(th)]])
    coords2 = coords.copy()
    coords2[:, :2] = coords[:, :2] @ Rm.T
    R2, F2 = LT.lateral_pressure(8, conn, coords2, faces, s, RIG, RWG, -5.0)
    assert np.abs(F2 - F @ Rm.T).max() <= 1e-13 * np.abs(F).max()
    assert np.abs(R2 - R @ Rm.T).max() <= 1e-13 * np.abs(R).max()


def test_wedge_column_spreading_force():
    """Triangular column, no ocean: each side pushes rho_i g |edge| H^2 / 2 along its outward normal."""
    xy = np.array([(0.0, 0.0), (3.0, 0.5), (1.0, 2.0)])
    H, L = 0.9, 5
    polys, conn, coords, s = _column(xy, [0.0] * 3, [H] * 3, L)
    faces = LT.lateral_faces(polys, L)
    R, F = LT.lateral_pressure(6, conn, coords, faces, s, RIG, RWG, NO_OCEAN)
    for k in range(3):
        e = xy[(k + 1) % 3] - xy[k]
        nrm = np.array([e[1], -e[0]])   # |e| times the outward unit normal of a CCW triangle
        ref = RIG * H * H / 2 * nrm
        got = F[faces[:, 1] == k].sum(0)
        assert np.abs(got - ref).max() <= 1e-13 * np.abs(ref).max()
