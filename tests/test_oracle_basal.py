"""Pins of the basal-friction oracle (NEXT-4, oracle/basal.py; PAPER.md P:L59
-> [24]; reading Z18) against closed forms: face areas (shoelace,
slope factor), constant-field integrals, exact linear-field integral,
linearity R = J U, symmetric positive-definite face matrices."""
import numpy as np
import pytest

from oracle import basal as B


def _quad_cell(xy, z):
    """A one-cell 'column' whose bottom face is the quad xy at heights z."""
    coords = np.array([(x, y, zz) for (x, y), zz in zip(xy, z)] + [(x, y, zz + 1.0) for (x, y), zz in zip(xy, z)])
    return np.arange(8, dtype=np.int32)[None], coords


def test_rectangle_constant_fields():
    a, b = 2.0, 3.0
    conn, coords = _quad_cell([(0, 0), (a, 0), (a, b), (0, b)], [0.5] * 4)
    beta = np.full(8, 1.7)
    U = np.tile([3.0, -2.0], (8, 1))
    R, J, area = B.basal_friction(4, conn, coords, [0], beta, U)
    assert abs(area[0] - a * b) < 1e-14
    assert np.allclose(R[:4, 0], 1.7 * 3.0 * a * b / 4, rtol=1e-14)
    assert np.allclose(R[:4, 1], 1.7 * -2.0 * a * b / 4, rtol=1e-14)
    assert np.abs(R[4:]).max() == 0.0  # top nodes untouched


def test_sloped_planar_quad_area_and_linear_field():
    xy = [(0.0, 0.0), (3.0, 0.4), (3.5, 2.9), (-0.3, 2.5)]
    al, be = 0.2, -0.15
    z = [al * x + be * y + 1.0 for x, y in xy]
    conn, coords = _quad_cell(xy, z)
    P = np.array(xy)
    shoelace = 0.5 * abs(np.sum(P[:, 0] * np.roll(P[:, 1], -1) - np.roll(P[:, 0], -1) * P[:, 1]))
    beta = np.full(8, 2.0)
    U = np.zeros((8, 2))
    R, J, area = B.basal_friction(4, conn, coords, [0], beta, U)
    assert abs(area[0] - shoelace * np.sqrt(1 + al**2 + be**2)) < 1e-13
    # linear field u = g x on a rectangle: sum_i R_i = beta * int g x dA (exact)
    a, b, g = 2.0, 3.0, 0.7
    conn, coords = _quad_cell([(0, 0), (a, 0), (a, b), (0, b)], [0.0] * 4)
    U = np.stack([g * coords[:, 0], np.zeros(8)], 1)
    R, J, _ = B.basal_friction(4, conn, coords, [0], beta, U)
    assert abs(R[:, 0].sum() - 2.0 * g * a * a / 2 * b) < 1e-13


def test_triangle_area_and_constant_fields():
    xy = [(0.0, 0.0), (2.0, 0.3), (0.4, 1.7)]
    coords = np.array([(x, y, 0.2) for x, y in xy] + [(x, y, 1.2) for x, y in xy])
    conn = np.arange(6, dtype=np.int32)[None]
    P = np.array(xy)
    A = 0.5 * abs((P[1, 0] - P[0, 0]) * (P[2, 1] - P[0, 1]) - (P[2, 0] - P[0, 0]) * (P[1, 1] - P[0, 1]))
    beta = np.full(6, 0.9)
    U = np.tile([1.5, 4.0], (6, 1))
    R, J, area = B.basal_friction(3, conn, coords, [0], beta, U)
    assert abs(area[0] - A) < 1e-14
    assert np.allclose(R[:3, 1], 0.9 * 4.0 * A / 3, rtol=1e-14)


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_linearity_and_spd(elem):
    from tests import _meshes as M
    fp, conn, coords = M.tiny(elem, n=4, L=2)
    nb = 4 if elem == "hex8" else 3
    cells = np.arange(0, conn.shape[0], 2)   # k = 0 cells (L = 2)
    rng = np.random.default_rng(3)
    beta = rng.uniform(0.5, 2.0, coords.shape[0])
    U = rng.normal(0, 10, (coords.shape[0], 2))
    R, J, area = B.basal_friction(nb, conn, coords, cells, beta, U)
    RJ = np.zeros_like(R)
    for k, c in enumerate(cells):
        nodes = conn[c, :nb]
        RJ[nodes] += (J[k] @ U[nodes].reshape(-1)).reshape(nb, 2)
    assert np.abs(R - RJ).max() < 1e-13 * np.abs(R).max()
    for k in range(len(cells)):
        assert np.abs(J[k] - J[k].T).max() <= 1e-15 * np.abs(J[k]).max()
        assert np.linalg.eigvalsh(0.5 * (J[k] + J[k].T)).min() > 0
    # the bed area is at least the footprint area (shoelace) and only slightly larger (gentle bed slopes)
    P = fp.xy[fp.polys]
    flat = 0.5 * np.abs(np.sum(P[:, :, 0] * np.roll(P[:, :, 1], -1, 1) - np.roll(P[:, :, 0], -1, 1) * P[:, :, 1], 1)).sum()
    assert flat * (1 - 1e-14) <= area.sum() <= flat * 1.01
