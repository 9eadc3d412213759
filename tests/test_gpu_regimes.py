"""GPU parity in the regularisation regime of Glen's law (§III-A;
readings Z1-Z3: mu = k_c (eps_e^2 + delta)^(-1/3)) and on the special fields
whose results the mathematics fixes.

The kernels evaluate mu = k_c rcbrt(eps_e^2 + delta) and the tangent weight
gamma = wM 2 mu p r^3 (r^3 standing in for 1/(eps_e^2 + delta)); the oracle
uses pow.  These tests compare the two element by element exactly where delta
dominates or matches eps_e^2:

  field    U                                   eps_e^2 vs delta
  zero     U = 0                               0 (mu = k_c delta^(-1/3) exactly)
  rigid    U = t + omega (-y, x)               rounding only
  linear   U = G_lin (x - x_mean) + c          closed form, Ugrad = G_lin
  scaled   random U scaled so median eps^2 = delta   comparable (the gamma term is O(1))

for delta in {1e-10, 1e-6, 1}, hex8 and wedge6, stored and on-the-fly geometry,
through the C ABI.  Besides oracle parity, the CUDA results are pinned directly:
mu = k_c delta^(-1/3) (zero / rigid), the closed-form mu of the linear field,
R_cell == 0 bitwise for U = 0 without body force, R_visc ~ 0 for rigid motion,
the patch test on the CUDA-assembled R at interior nodes, J symmetric with the
x-translation in its null space, and golden cell A.

Tolerances.  mu and J are well conditioned here: per cell 1e-12 relative (the
north_star bound).  R_cell and R in these fields are sums with heavy
cancellation (rigid motion: the viscous part is pure rounding), so their
bound is 1e-12 times the a-priori rounding scale of the sum -- the sum of the
absolute values of the terms that are added (SURVEY 8(c) 'Assembled R' uses the
same idea, sum |contributions|):
  scale[c][i][a] = sum_q wM_q (2 mu_q 3 gbar_q sum_d |G_i[q][d]|
                               + rho_g (sum_n |s_n| (|G_n0| + |G_n1|)) phi_i(q)),
  gbar_q = sum_n sum_a sum_d |U_n,a| |G_n[q][d]|  (>= |every Ugrad entry| before cancellation)
(tests/_meshes.py rounding_scale_R).
"""
import numpy as np
import pytest

import oracle as O
from tests import _meshes as M

pytestmark = pytest.mark.gpu

TOL = 1e-12
RHO_G = 8.927
DELTAS = [1e-10, 1e-6, 1.0]
FIELDS = ["zero", "rigid", "linear", "scaled"]
GEOMS = ["stored", "on_the_fly", "compact"]


@pytest.fixture(scope="module")
def torch():
    import torch as _t
    if not _t.cuda.is_available():
        pytest.skip("no CUDA device")
    return _t


def _t(torch, a):
    return torch.from_numpy(np.ascontiguousarray(a)).to("cuda")


def _field(kind, fp, L, conn, coords, G, wm, kc, delta, e):
    if kind == "zero":
        return np.zeros((coords.shape[0], 2))
    if kind == "rigid":
        om = 0.37
        return np.stack([5.0 - om * coords[:, 1], -2.0 + om * coords[:, 0]], 1)
    if kind == "linear":
        Gl = np.array([[0.3, -1.2, 4.0], [0.7, 0.25, -2.5]])
        return (coords - coords.mean(0)) @ Gl.T + np.array([3.0, -1.0])
    # scaled: a random field whose median eps_e^2 equals delta (the gamma term of the
    # tangent is then as large as the B term); eps^2 from the oracle's mu at tiny delta
    U = np.random.default_rng(41).normal(0.0, 50.0, (coords.shape[0], 2))
    mu = O.evaluate(e, conn, G, wm, U, kc=kc, delta=1e-300)["mu_qp"]
    e2 = (mu / kc[:, None]) ** -3.0
    return U * np.sqrt(delta / np.median(e2))


def _run(torch, elem, geometry, conn, coords, U, s, kc, delta):
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    ctx = StokesFO(elem, _t(torch, conn), _t(torch, coords), surface=None if s is None else _t(torch, s),
                   flow_factor=_t(torch, kc), delta=delta, rho_g=RHO_G, geometry=geometry)
    C, N, Q = conn.shape[0], ctx.N, ctx.Q
    J = torch.full((C, 2 * N, 2 * N), float("nan"), dtype=torch.float64, device="cuda")
    Rc = torch.full((C, N, 2), float("nan"), dtype=torch.float64, device="cuda")
    R = torch.zeros((coords.shape[0], 2), dtype=torch.float64, device="cuda")
    mu = torch.empty((C, Q), dtype=torch.float64, device="cuda")
    Rc2 = torch.empty((C, N, 2), dtype=torch.float64, device="cuda")
    Ud = _t(torch, U)
    ctx.jacobian(Ud, J, R_cell=Rc, R=R)
    ctx.viscosity_resid(Ud, mu_qp=mu, R_cell=Rc2)
    ctx.sync()
    return (J.cpu().numpy(), Rc.cpu().numpy(), R.cpu().numpy(), mu.cpu().numpy(), Rc2.cpu().numpy())


@pytest.mark.parametrize("geometry", GEOMS)
@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
@pytest.mark.parametrize("delta", DELTAS)
@pytest.mark.parametrize("kind", FIELDS)
def test_regime_parity(torch, kind, delta, elem, geometry):
    L = 5
    fp, conn, coords = M.tiny(elem, n=16, L=L)
    _, s, kc = M.fields(fp, L)
    e = O.ELEM[elem]
    G, wm, bad = O.geometry(e, conn, coords)
    assert bad == 0
    U = _field(kind, fp, L, conn, coords, G, wm, kc, delta, e)
    C, N = conn.shape
    nn = coords.shape[0]
    # with body force and per-cell k_c (parity), then without force and with a constant
    # k_c (the invariants: zero / rigid residuals, and the patch test, which needs a
    # constant stress, i.e. a constant mu)
    kc_const = np.full_like(kc, 10.77)
    for surf, kcv in ((s, kc), (None, kc_const)):
        kc = kcv
        Jg, Rcg, Rg, mug, Rc2g = _run(torch, elem, geometry, conn, coords, U, surf, kc, delta)
        ref = O.evaluate(e, conn, G, wm, U, surface=surf, kc=kc, delta=delta, rho_g=RHO_G, mode="jac")
        # --- mu: vs the oracle, and vs the closed forms the field fixes
        assert np.abs(mug / ref["mu_qp"] - 1.0).max() <= TOL
        if kind in ("zero", "rigid"):
            closed = kc[:, None] * delta ** (-1.0 / 3.0)
            mtol = 1e-14 if kind == "zero" else TOL   # zero: eps^2 = 0 exactly; rigid: rounding-size eps^2
            assert np.abs(mug / closed - 1.0).max() <= mtol
        if kind == "linear":
            ux, uy, uz, vx, vy, vz = 0.3, -1.2, 4.0, 0.7, 0.25, -2.5
            e2 = ux * ux + vy * vy + ux * vy + 0.25 * (uy + vx) ** 2 + 0.25 * uz * uz + 0.25 * vz * vz
            assert np.abs(mug / (kc[:, None] * (e2 + delta) ** (-1.0 / 3.0)) - 1.0).max() <= TOL
        # --- J: element by element, per cell relative to max |J_c|
        assert np.isfinite(Jg).all()
        jsc = np.abs(ref["J_cell"]).reshape(C, -1).max(1)
        assert (np.abs(Jg - ref["J_cell"]).reshape(C, -1).max(1) <= TOL * jsc).all()
        # J is a Hessian (symmetric) and annihilates the x- and y-translations
        assert (np.abs(Jg - Jg.transpose(0, 2, 1)).reshape(C, -1).max(1) <= 1e-13 * jsc).all()
        for a in (0, 1):
            t = np.zeros(2 * N)
            t[a::2] = 1.0
            assert (np.abs(Jg @ t).max(1) <= 1e-12 * jsc * N).all()
        # --- R_cell (both kernels) and assembled R against the rounding scale of the sum
        scale = M.rounding_scale_R(e, conn, G, wm, ref["mu_qp"], U, surf, RHO_G)
        assert np.isfinite(Rcg).all()
        assert (np.abs(Rcg - ref["R_cell"]) <= TOL * scale).all()
        assert (np.abs(Rc2g - ref["R_cell"]) <= TOL * scale).all()
        Rref = O.scatter(e, conn, ref["R_cell"], nn)
        Rsc = O.scatter(e, conn, scale, nn)
        assert (np.abs(Rg - Rref) <= TOL * Rsc).all()
        # --- invariants of the CUDA results themselves (no body force)
        if surf is None:
            if kind == "zero":
                assert not Rcg.any() and not Rc2g.any() and not Rg.any()   # bitwise zero
            elif kind == "rigid":
                assert (np.abs(Rcg) <= 1e-13 * scale).all()
            elif kind == "linear":
                absR = O.scatter(e, conn, np.abs(ref["R_cell"]), nn)
                inner = M.interior_nodes(fp, L, nn)
                assert inner.size > 100
                assert (np.abs(Rg[inner]) <= 1e-13 * absR[inner]).all()
                assert np.abs(Rg).max() > 1e-3 * absR.max()   # boundary nodes: the test is not vacuous


@pytest.mark.parametrize("geometry", GEOMS)
def test_golden_cell_A_gpu(torch, golden, geometry):
    """SURVEY 8(c4) cell A: hex8 box [0,2]x[0,3]x[0,0.5], linear field, k = 1,
    delta = 1e-10, no force: eps^2 = 10.3125 and mu = 10.3125^(-1/3) at every QP,
    R_cell by hand (-8.125 mu for n0's x entry), antisymmetry n4..n7 = -(n2, n3, n0, n1)."""
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    g = golden["A"]
    tol = golden["tolerance_gpu"]
    conn, xyz = M.box_cell((0, 0, 0), (2.0, 3.0, 0.5))
    U = np.stack([1 + 2 * xyz[:, 0] - xyz[:, 1] + 3 * xyz[:, 2],
                  -1 + 0.5 * xyz[:, 0] + xyz[:, 1] - 2 * xyz[:, 2]], 1)
    ctx = StokesFO("hex8", _t(torch, conn), _t(torch, xyz), k=g["k"], delta=g["delta"], rho_g=g["rho_g"],
                   geometry=geometry)
    J = torch.empty((1, 16, 16), dtype=torch.float64, device="cuda")
    Rc = torch.empty((1, 8, 2), dtype=torch.float64, device="cuda")
    mu = torch.empty((1, 8), dtype=torch.float64, device="cuda")
    Ud = _t(torch, U)
    ctx.jacobian(Ud, J, R_cell=Rc)
    ctx.viscosity_resid(Ud, mu_qp=mu)
    G, wm = ctx.geometry()
    ctx.sync()
    J, R, mu = J.cpu().numpy()[0], Rc.cpu().numpy()[0], mu.cpu().numpy()[0]
    assert abs(wm.cpu().numpy().sum() / g["volume"] - 1) <= tol
    assert np.abs(mu / g["mu"] - 1).max() <= tol
    assert np.abs(R[:4] - np.array(g["R_cell_0_4"])).max() <= tol * np.abs(R).max()
    assert abs(R[0, 0] / (-8.125 * g["mu"]) - 1) <= tol
    for n, m in enumerate(g["R_cell_4_8_is_minus"]):
        assert np.abs(R[4 + n] + R[m]).max() <= tol * np.abs(R).max()
    assert np.abs(R.sum(0)).max() <= tol * np.abs(R).max()
    assert abs(np.trace(J) / g["J_trace"] - 1) <= tol
    assert abs(np.linalg.norm(J) / g["J_fro"] - 1) <= tol
