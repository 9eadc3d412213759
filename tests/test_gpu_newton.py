"""NEXT-3: the damped Newton-Krylov driver (stokesfo_newton_solve) on the
fused evaluators + basal friction must converge (quadratically at the end,
PAPER.md P:L68) to the same velocity field as a Newton iteration on the
oracle's assembled F and J (dense solve)."""
import numpy as np
import pytest

import oracle as O
from oracle import basal as B
from oracle import lateral as LT
from tests import _meshes as M

pytestmark = pytest.mark.gpu


def _oracle_newton(elem, conn, coords, G, wm, s, kc, cells, beta, U0, iters=12, lateral=None):
    e = O.ELEM[elem]
    N = conn.shape[1]
    nb = N // 2
    nn = coords.shape[0]
    dofs = (2 * conn[:, :, None] + np.arange(2)).reshape(conn.shape[0], 2 * N)
    bd = (2 * conn[cells][:, :nb, None] + np.arange(2)).reshape(len(cells), 2 * nb)

    def F_J(U, need_J=True):
        out = O.evaluate(e, conn, G, wm, U, surface=s, kc=kc, mode="jac" if need_J else "resid")
        Rb, Jb, _ = B.basal_friction(nb, conn, coords, cells, beta, U)
        F = O.scatter(e, conn, out["R_cell"], nn) + Rb
        if lateral is not None:   # (faces, rho_i_g, rho_w_g, sea level): U-independent, F only
            F = F + LT.lateral_pressure(N, conn, coords, lateral[0], s, *lateral[1:])[0]
        F = F.reshape(-1)
        if not need_J:
            return F, None
        J = np.zeros((2 * nn, 2 * nn))
        for c in range(conn.shape[0]):
            J[np.ix_(dofs[c], dofs[c])] += out["J_cell"][c]
        for k in range(len(cells)):
            J[np.ix_(bd[k], bd[k])] += Jb[k]
        return F, J

    U = U0.copy()
    for _ in range(iters):
        F, J = F_J(U)
        d = np.linalg.solve(J, -F).reshape(nn, 2)
        a = 1.0
        nF = np.linalg.norm(F)
        for _ in range(30):
            Ft, _ = F_J(U + a * d, need_J=False)
            if np.linalg.norm(Ft) <= (1 - 1e-4 * a) * nF:
                break
            a *= 0.5
        U = U + a * d
    return U, np.linalg.norm(F_J(U, need_J=False)[0])


@pytest.mark.parametrize("lateral", [False, True])
@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_newton_krylov_matches_oracle_newton(elem, lateral):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    L = 3
    fp, conn, coords = M.tiny(elem, n=8, L=L)
    U0, s, kc = M.fields(fp, L)
    U0 = np.full_like(U0, 1.0)
    e = O.ELEM[elem]
    G, wm, _ = O.geometry(e, conn, coords)
    cells = np.arange(0, conn.shape[0], L, dtype=np.int32)
    beta = np.full(coords.shape[0], 5.0)
    lat = None
    if lateral:   # NEXT-4 lateral (ocean) pressure on every footprint-boundary face (reading Z19)
        z = coords[:, 2]
        lat = (LT.lateral_faces(fp.polys, L), 8.927, 10.05, 0.5 * (z.min() + z.max()))
    Uo, nFo = _oracle_newton(elem, conn, coords, G, wm, s, kc, cells, beta, U0, lateral=lat)
    ctx = StokesFO(elem, torch.from_numpy(conn).cuda(), torch.from_numpy(coords).cuda(),
                   surface=torch.from_numpy(s).cuda(), flow_factor=torch.from_numpy(kc).cuda())
    if lat is not None:
        ctx.set_lateral(torch.from_numpy(lat[0]).cuda(), torch.from_numpy(s).cuda(), *lat[1:])
    Ud = torch.from_numpy(U0).cuda()
    h = ctx.newton_solve(torch.from_numpy(cells).cuda(), torch.from_numpy(beta).cuda(), Ud, max_newton=12,
                         max_cg=2000, rtol_newton=1e-11, rtol_cg=1e-10)
    F = h["F"]
    assert F[-1] <= 1e-9 * F[0], F
    # quadratic tail of an inexact Newton: once below 1e-3 of the start, each step
    # squares the relative residual up to the linear-solve tolerance (rtol_cg 1e-10)
    rel = [f / F[0] for f in F]
    tail = [(a, b) for a, b in zip(rel, rel[1:]) if a < 1e-3 and b > 1e-13]
    assert all(b <= 10 * a * a + 1e-8 * a + 1e-14 for a, b in tail), rel
    Ug = Ud.cpu().numpy()
    assert np.abs(Ug - Uo).max() <= 1e-8 * np.abs(Uo).max()
