"""Pins of the CPU oracle against what the paper and the mathematics fix
(closed forms, invariants, golden cells, complex step, finite differences).
None of these re-types the oracle's formula; each would fail on a plausible
mistake (dropped term, wrong sign/index, transposed operand).
Cited: PAPER.md eq. (1), eq. (3), Fig. 2 P:L131-213,
Sacado AD P:L215-221; SURVEY.md 8(c3) pin table."""
import math

import numpy as np
import pytest

import oracle as O
from tests import _meshes as M

HEX, WED = O.HEX8, O.WEDGE6


# --------------------------------------------------------------------------
# O2 reference elements
# --------------------------------------------------------------------------

@pytest.mark.parametrize("elem", [HEX, WED])
def test_reference_partition_of_unity_and_weights(elem):
    bf, dbf, w = O.ref_element(elem)
    assert abs(w.sum() - (8.0 if elem == HEX else 1.0)) < 1e-15   # reference volumes
    assert np.allclose(bf.sum(0), 1.0, atol=1e-15, rtol=0)
    assert np.allclose(dbf.sum(0), 0.0, atol=1e-15, rtol=0)
    rng = np.random.default_rng(1)
    for _ in range(20):
        p = rng.uniform(-1, 1, 3) if elem == HEX else np.array([*(rng.dirichlet([1, 1, 1])[:2]), rng.uniform(-1, 1)])
        phi, dphi = O.basis_at(elem, p)
        assert abs(phi.sum() - 1) < 1e-15
        assert np.abs(dphi.sum(0)).max() < 1e-15
        # gradient == finite difference of the values (pins the derivative formulas)
        for d in range(3):
            e = np.zeros(3)
            e[d] = 1e-6
            fd = (O.basis_at(elem, p + e)[0] - O.basis_at(elem, p - e)[0]) / 2e-6
            assert np.abs(fd - dphi[:, d]).max() < 1e-9


@pytest.mark.parametrize("elem", [HEX, WED])
def test_reference_kronecker_at_nodes(elem):
    if elem == HEX:
        nodes = [(-1, -1, -1), (1, -1, -1), (1, 1, -1), (-1, 1, -1),
                 (-1, -1, 1), (1, -1, 1), (1, 1, 1), (-1, 1, 1)]     # Shards order (Z9)
    else:
        nodes = [(0, 0, -1), (1, 0, -1), (0, 1, -1), (0, 0, 1), (1, 0, 1), (0, 1, 1)]
    for j, p in enumerate(nodes):
        phi, _ = O.basis_at(elem, np.array(p, float))
        e = np.zeros(len(nodes))
        e[j] = 1
        assert np.abs(phi - e).max() < 1e-15


def test_hex_gauss_exactness():
    """2-point Gauss per direction integrates xi^a eta^b zeta^c exactly for a,b,c <= 3."""
    xq, w = O.quadrature(HEX)
    for a in range(4):
        for b in range(4):
            for c in range(4):
                exact = 1.0
                for e in (a, b, c):
                    exact *= 0.0 if e % 2 else 2.0 / (e + 1)
                got = np.sum(w * xq[:, 0] ** a * xq[:, 1] ** b * xq[:, 2] ** c)
                assert abs(got - exact) < 1e-14


def test_wedge_rule_exactness():
    """Triangle rule exact to degree 2 (int xi^a eta^b = a! b!/(a+b+2)!), x Gauss in zeta to degree 3."""
    xq, w = O.quadrature(WED)
    for a in range(3):
        for b in range(3 - a):
            for c in range(4):
                tri = math.factorial(a) * math.factorial(b) / math.factorial(a + b + 2)
                zeta = 0.0 if c % 2 else 2.0 / (c + 1)
                got = np.sum(w * xq[:, 0] ** a * xq[:, 1] ** b * xq[:, 2] ** c)
                assert abs(got - tri * zeta) < 1e-15


# --------------------------------------------------------------------------
# O3 geometry
# --------------------------------------------------------------------------

def test_geometry_box_closed_form():
    conn, xyz = M.box_cell((1.0, -2.0, 0.3), (2.0, 3.0, 0.5))
    G, wm, bad = O.geometry(HEX, conn, xyz)
    _, dbf, _ = O.ref_element(HEX)
    assert bad == 0
    assert np.allclose(wm, 2.0 * 3.0 * 0.5 / 8.0, rtol=1e-15, atol=0)
    expect = dbf * np.array([2 / 2.0, 2 / 3.0, 2 / 0.5])
    assert np.abs(G[0] - expect).max() < 1e-15
    # integral of grad phi_0 over the box = -(face area)/4 per direction
    ig = np.einsum("nqd,q->nd", G[0], wm[0])
    assert np.allclose(ig[0], [-3.0 * 0.5 / 4, -2.0 * 0.5 / 4, -2.0 * 3.0 / 4], atol=1e-15)


def test_geometry_affine_map():
    """x = A xi + x0 on the reference hex: GradBF = A^-T grad_xi phi, det = det A."""
    rng = np.random.default_rng(3)
    A = np.eye(3) + 0.3 * rng.normal(size=(3, 3))
    x0 = rng.normal(size=3)
    ref = np.array([(-1, -1, -1), (1, -1, -1), (1, 1, -1), (-1, 1, -1),
                    (-1, -1, 1), (1, -1, 1), (1, 1, 1), (-1, 1, 1)], float)
    xyz = ref @ A.T + x0
    G, wm, bad = O.geometry(HEX, np.arange(8, dtype=np.int32)[None], xyz)
    _, dbf, _ = O.ref_element(HEX)
    assert bad == 0
    assert np.allclose(wm, np.linalg.det(A), rtol=1e-13)
    exp = np.einsum("rs,nqs->nqr", np.linalg.inv(A).T, dbf)
    assert np.abs(G[0] - exp).max() < 1e-13


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_geometry_column_volume(elem):
    """Constant thickness on a jittered footprint: each column's volume = H x
    polygon area (shoelace), independent of the bed shape."""
    from paper_conf_sc_antepara0cw24_b200 import synth
    fp = synth.tiny_footprint(jitter=0.2, seed=4)
    if elem == "wedge6":
        fp = synth.split_to_triangles(fp)
    H = np.full(fp.nv, 0.7)
    L = 5
    conn, coords = O.extrude(fp.xy, fp.polys, fp.b, H, L)
    G, wm, bad = O.geometry(O.ELEM[elem], conn, coords)
    assert bad == 0
    colvol = wm.sum(1).reshape(fp.nf, L).sum(1)
    xy = fp.xy[fp.polys]
    area = 0.5 * np.abs(np.sum(xy[:, :, 0] * np.roll(xy[:, :, 1], -1, 1) - np.roll(xy[:, :, 0], -1, 1) * xy[:, :, 1], 1))
    assert np.abs(colvol - 0.7 * area).max() < 1e-13


def test_geometry_flags_inverted_cells():
    conn, xyz = M.box_cell()
    xyz = xyz[[4, 5, 6, 7, 0, 1, 2, 3]]  # top and bottom swapped -> det J < 0
    _, _, bad = O.geometry(HEX, conn, xyz)
    assert bad == 8


# --------------------------------------------------------------------------
# O4-O6 residual invariants
# --------------------------------------------------------------------------

@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_linear_field_closed_form_mu(elem):
    """U = Gx + c  =>  Ugrad = G at every QP on distorted cells, so mu is the
    closed form k (eps^2(G) + delta)^(-1/3) (SURVEY 8(c3) 'Ugrad')."""
    fp, conn, coords = M.tiny(elem)
    Gm = np.array([[0.3, -1.2, 4.0], [0.7, 0.25, -2.5]])
    U = coords @ Gm.T + np.array([3.0, -1.0])
    G, wm, _ = O.geometry(O.ELEM[elem], conn, coords)
    out = O.evaluate(O.ELEM[elem], conn, G, wm, U, k=2.0, delta=1e-10, rho_g=0.0)
    ux, uy, uz = Gm[0]
    vx, vy, vz = Gm[1]
    e2 = ux**2 + vy**2 + ux * vy + 0.25 * (uy + vx) ** 2 + 0.25 * uz**2 + 0.25 * vz**2
    assert np.abs(out["mu_qp"] / (2.0 * (e2 + 1e-10) ** (-1 / 3)) - 1).max() < 1e-13


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_rigid_motion_zero_viscous_residual(elem):
    fp, conn, coords = M.tiny(elem)
    G, wm, _ = O.geometry(O.ELEM[elem], conn, coords)
    om = 0.37
    U = np.stack([5.0 - om * coords[:, 1], -2.0 + om * coords[:, 0]], 1)
    out = O.evaluate(O.ELEM[elem], conn, G, wm, U, k=3.0, delta=1e-6, rho_g=0.0)
    assert np.allclose(out["mu_qp"], 3.0 * 1e-6 ** (-1 / 3), rtol=1e-12)
    # scale: the same cells under a random field of similar magnitude
    Ur = np.random.default_rng(0).normal(0, 5.0, U.shape)
    scale = np.abs(O.evaluate(O.ELEM[elem], conn, G, wm, Ur, k=3.0, delta=1e-6, rho_g=0.0)["R_cell"]).max()
    assert np.abs(out["R_cell"]).max() < 1e-13 * scale


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_patch_test_interior_nodes(elem):
    """Linear field => constant stress => assembled R = 0 at interior nodes
    (exact quadrature of int grad phi_i; P:L61 low-order FE)."""
    fp, conn, coords = M.tiny(elem)
    L = 5
    e = O.ELEM[elem]
    G, wm, _ = O.geometry(e, conn, coords)
    Gm = np.array([[0.3, -1.2, 4.0], [0.7, 0.25, -2.5]])
    U = coords @ Gm.T
    out = O.evaluate(e, conn, G, wm, U, k=2.0, rho_g=0.0)
    R = O.scatter(e, conn, out["R_cell"], coords.shape[0])
    absR = O.scatter(e, conn, np.abs(out["R_cell"]), coords.shape[0])
    inner = M.interior_nodes(fp, L, coords.shape[0])
    assert inner.size > 100
    assert np.abs(R[inner]).max() < 1e-13 * absR.max()
    # and the boundary nodes are not all zero (the test is not vacuous)
    assert np.abs(R).max() > 1e-3 * absR.max()


def test_force_only_box_closed_form():
    """U = 0: R = force term only. s = alpha x + beta y: on a box each node gets
    rho g (alpha, beta) vol/8 (eq. (1): + rho g ds/dx)."""
    conn, xyz = M.box_cell((0.0, 0.0, 0.0), (2.0, 3.0, 0.5))
    G, wm, _ = O.geometry(HEX, conn, xyz)
    al, be = 0.013, -0.021
    s = al * xyz[:, 0] + be * xyz[:, 1] + 1.0
    out = O.evaluate(HEX, conn, G, wm, np.zeros((8, 2)), surface=s, k=1.0, rho_g=8.927)
    vol = 3.0
    assert np.allclose(out["R_cell"][0, :, 0], 8.927 * al * vol / 8, rtol=1e-13, atol=0)
    assert np.allclose(out["R_cell"][0, :, 1], 8.927 * be * vol / 8, rtol=1e-13, atol=0)


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_force_only_sum_distorted(elem):
    """Sum over nodes of the force term = rho g (alpha, beta) x cell volume for a
    linear s, on distorted cells (partition of unity)."""
    fp, conn, coords = M.tiny(elem)
    e = O.ELEM[elem]
    G, wm, _ = O.geometry(e, conn, coords)
    al, be = 0.013, -0.021
    s = al * coords[:, 0] + be * coords[:, 1]
    out = O.evaluate(e, conn, G, wm, np.zeros((coords.shape[0], 2)), surface=s, rho_g=8.927)
    vol = wm.sum(1)
    got = out["R_cell"].sum(1)
    assert np.abs(got[:, 0] - 8.927 * al * vol).max() < 1e-14 * np.abs(8.927 * al * vol).max() * 10
    assert np.abs(got[:, 1] - 8.927 * be * vol).max() < 1e-14 * np.abs(8.927 * be * vol).max() * 10


def test_force_qp_override_equals_surface_force():
    fp, conn, coords = M.tiny("hex8", n=4, L=2)
    G, wm, _ = O.geometry(HEX, conn, coords)
    U, s, kc = M.fields(fp, 2)
    a = O.evaluate(HEX, conn, G, wm, U, surface=s, kc=kc)
    # force at QPs computed here independently from the definition rho g grad s_h
    sc = s[conn]
    f = 8.927 * np.einsum("cn,cnqd->cqd", sc, G[..., 0:2])
    b = O.evaluate(HEX, conn, G, wm, U, force_qp=f, kc=kc)
    assert np.abs(a["R_cell"] - b["R_cell"]).max() < 1e-12 * np.abs(a["R_cell"]).max()


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_fig2_baseline_equals_optimized(elem):
    """Fig. 2: the baseline and optimized loop structures compute the same
    residual up to reassociation."""
    fp, conn, coords = M.tiny(elem)
    e = O.ELEM[elem]
    G, wm, _ = O.geometry(e, conn, coords)
    U, s, kc = M.fields(fp, 5)
    a = O.evaluate(e, conn, G, wm, U, surface=s, kc=kc, mode="resid")["R_cell"]
    b = O.evaluate(e, conn, G, wm, U, surface=s, kc=kc, mode="resid_baseline")["R_cell"]
    scale = np.abs(a).max(axis=(1, 2), keepdims=True)
    assert np.abs(a - b).max() / scale.min() < 1e-13


def test_linear_stokes_n1_residual_is_J_times_U():
    """Glen n = 1 => mu = k constant => the viscous residual is linear and
    homogeneous in U, so R(U) = J U exactly (pins every J term)."""
    fp, conn, coords = M.tiny("hex8", n=4, L=2)
    G, wm, _ = O.geometry(HEX, conn, coords)
    U = np.random.default_rng(5).normal(0, 10, (coords.shape[0], 2))
    out = O.evaluate(HEX, conn, G, wm, U, k=1.7, glen_n=1.0, rho_g=0.0, mode="jac")
    Uc = U[conn].reshape(conn.shape[0], -1)
    JU = np.einsum("ckl,cl->ck", out["J_cell"], Uc)
    R = out["R_cell"].reshape(conn.shape[0], -1)
    assert np.abs(JU - R).max() < 1e-13 * np.abs(R).max()


# --------------------------------------------------------------------------
# O7 Jacobian
# --------------------------------------------------------------------------

def _jac_setup(elem, n=6, L=3):
    fp, conn, coords = M.tiny(elem, n=n, L=L)
    e = O.ELEM[elem]
    G, wm, _ = O.geometry(e, conn, coords)
    U, s, kc = M.fields(fp, L)
    out = O.evaluate(e, conn, G, wm, U, surface=s, kc=kc, mode="jac")
    return e, conn, G, wm, U, s, kc, out


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_ad_jacobian_equals_closed_form_tangent(elem):
    e, conn, G, wm, U, s, kc, out = _jac_setup(elem)
    ana = O.evaluate(e, conn, G, wm, U, surface=s, kc=kc, mode="jac_analytic")["J_cell"]
    J = out["J_cell"]
    scale = np.abs(J).max(axis=(1, 2))
    assert (np.abs(J - ana).max(axis=(1, 2)) / scale).max() < 1e-13


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_ad_jacobian_equals_complex_step(elem):
    e, conn, G, wm, U, s, kc, out = _jac_setup(elem)
    bf, _, _ = O.ref_element(e)
    Jcs = O.jac_complex_step(e, G, wm, U[conn], s[conn], kc, bf=bf)
    J = out["J_cell"]
    scale = np.abs(J).max(axis=(1, 2))
    assert (np.abs(J - Jcs).max(axis=(1, 2)) / scale).max() < 1e-13
    # the numpy residual (independent implementation) also matches the C residual
    Rn = O.resid_numpy(e, G, wm, U[conn], s[conn], kc, bf=bf)
    assert np.abs(Rn - out["R_cell"]).max() < 1e-13 * np.abs(out["R_cell"]).max()


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_ad_jacobian_matches_central_fd(elem):
    """north_star: 'Jacobian columns matching central finite differences'."""
    e, conn, G, wm, U, s, kc, out = _jac_setup(elem)
    bf, _, _ = O.ref_element(e)
    Jfd = O.jac_central_fd(e, G, wm, U[conn], s[conn], kc, bf=bf)
    J = out["J_cell"]
    scale = np.abs(J).max(axis=(1, 2))
    assert (np.abs(J - Jfd).max(axis=(1, 2)) / scale).max() < 1e-6


@pytest.mark.parametrize("elem,rank", [("hex8", 13), ("wedge6", 9)])
def test_jacobian_symmetric_psd_nullspace(elem, rank):
    """J is the Hessian of the convex quadrature energy sum wM W(g): symmetric,
    PSD, null space {x-translation, y-translation, z-rotation}."""
    e, conn, G, wm, U, s, kc, out = _jac_setup(elem, n=4, L=2)
    N = 8 if elem == "hex8" else 6
    from paper_conf_sc_antepara0cw24_b200 import synth  # noqa: F401
    fp, conn2, coords = M.tiny(elem, n=4, L=2)
    for c in range(conn.shape[0]):
        J = out["J_cell"][c]
        sc = np.abs(J).max()
        assert np.abs(J - J.T).max() < 1e-13 * sc
        ev = np.linalg.eigvalsh(0.5 * (J + J.T))
        assert ev.min() > -1e-12 * sc
        assert int(np.sum(ev > 1e-9 * sc)) == rank
        x = coords[conn[c]]
        tx = np.zeros((N, 2)); tx[:, 0] = 1
        ty = np.zeros((N, 2)); ty[:, 1] = 1
        rz = np.stack([-x[:, 1], x[:, 0]], 1)
        for v in (tx, ty, rz):
            assert np.abs(J @ v.reshape(-1)).max() < 1e-11 * sc * max(1.0, np.abs(v).max())


# --------------------------------------------------------------------------
# Golden worked cells (tests/golden/cells.json)
# --------------------------------------------------------------------------

def _rel(a, b):
    a = np.asarray(a, float)
    b = np.asarray(b, float)
    return np.abs(a - b).max() / max(np.abs(b).max(), 1e-300)


@pytest.mark.parametrize("name", ["B", "W"])
def test_golden_cells(golden, name):
    g = golden[name]
    tol = golden["tolerance_oracle"]
    e = O.ELEM[g["elem"]]
    N = 8 if e == HEX else 6
    xyz = np.array(g["coords"], float)
    U = np.array(g["U"], float)
    conn = np.arange(N, dtype=np.int32)[None]
    G, wm, bad = O.geometry(e, conn, xyz)
    assert bad == 0
    assert _rel(wm.sum(), g["volume"]) < tol
    out = O.evaluate(e, conn, G, wm, U, surface=np.array(g["s"]), k=g["k"], delta=g["delta"],
                     rho_g=g["rho_g"], mode="jac")
    assert _rel(out["mu_qp"][0], g["mu_q"]) < tol
    assert _rel(out["R_cell"][0], g["R_cell"]) < tol
    assert _rel(out["R_cell"][0].sum(0), g["sum_R"]) < 1e-12
    J = out["J_cell"][0]
    assert _rel(J[0], g["J_row0"]) < tol
    assert _rel(np.diag(J), g["J_diag"]) < tol
    assert _rel(np.trace(J), g["J_trace"]) < tol
    assert _rel(np.linalg.norm(J), g["J_fro"]) < tol
    assert _rel((J @ U.reshape(-1))[:4], g["JU_0_4"]) < tol


def test_golden_box_A(golden):
    g = golden["A"]
    tol = golden["tolerance_oracle"]
    conn, xyz = M.box_cell((0, 0, 0), (2.0, 3.0, 0.5))
    U = np.stack([1 + 2 * xyz[:, 0] - xyz[:, 1] + 3 * xyz[:, 2],
                  -1 + 0.5 * xyz[:, 0] + xyz[:, 1] - 2 * xyz[:, 2]], 1)
    G, wm, _ = O.geometry(HEX, conn, xyz)
    out = O.evaluate(HEX, conn, G, wm, U, k=g["k"], delta=g["delta"], rho_g=g["rho_g"], mode="jac")
    assert _rel(wm.sum(), g["volume"]) < tol
    assert _rel(out["mu_qp"][0], np.full(8, g["mu"])) < 1e-14
    R = out["R_cell"][0]
    assert _rel(R[:4], g["R_cell_0_4"]) < tol
    for n, m in enumerate(g["R_cell_4_8_is_minus"]):
        assert np.abs(R[4 + n] + R[m]).max() < 1e-14 * np.abs(R).max()
    assert np.abs(R.sum(0)).max() < 1e-14 * np.abs(R).max()
    J = out["J_cell"][0]
    assert _rel(np.trace(J), g["J_trace"]) < tol
    assert _rel(np.linalg.norm(J), g["J_fro"]) < tol


# --------------------------------------------------------------------------
# O1 extrusion, O8 scatter, O9 CSR (integer structures)
# --------------------------------------------------------------------------

def test_extrusion_counts_and_numbering():
    fp, conn, coords = M.tiny("hex8")
    assert conn.shape == (1280, 8) and coords.shape == (1734, 3)
    L = 5
    f, k = 37, 3
    c = f * L + k
    poly = fp.polys[f]
    assert list(conn[c]) == [int(v) * (L + 1) + k for v in poly] + [int(v) * (L + 1) + k + 1 for v in poly]
    v = int(poly[2])
    assert coords[v * (L + 1) + L, 2] == fp.b[v] + fp.H[v]  # surface node: z = b + H exactly


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_gather_node_id_probe(elem):
    """O-gather (eq. (3): the element sees U at its own nodes, interleaved dof
    2 node + comp, reading Z9): with the probe field U[v] = (v, -v - 1/2) the
    gathered block must be exactly (conn, -conn - 1/2) -- integers and halves are
    exact in fp64, so any wrong index, swapped component or node-order slip in
    the oracle's gather shows up as a bit difference.  A ragged subset of cells
    (every 7th, reversed) pins that gather is per cell, not a prefix copy."""
    e = O.ELEM[elem]
    fp, conn, coords = M.tiny(elem)
    nn = coords.shape[0]
    v = np.arange(nn, dtype=np.float64)
    U = np.stack([v, -v - 0.5], 1)
    got = O.gather(e, conn, U)
    assert got.shape == (conn.shape[0], O.NODES[e], 2)
    assert np.array_equal(got[..., 0], conn.astype(np.float64))
    assert np.array_equal(got[..., 1], -conn.astype(np.float64) - 0.5)
    sub = np.ascontiguousarray(conn[::-7])
    got2 = O.gather(e, sub, U)
    assert np.array_equal(got2[..., 0], sub.astype(np.float64))
    # empty mesh: nothing gathered
    assert O.gather(e, conn[:0], U).shape == (0, O.NODES[e], 2)


def test_scatter_valence_probe():
    fp, conn, coords = M.tiny("hex8")
    R = O.scatter(HEX, conn, np.ones((conn.shape[0], 8, 2)), coords.shape[0])
    val = np.bincount(conn.reshape(-1), minlength=coords.shape[0]).astype(float)
    assert np.array_equal(R[:, 0], val) and np.array_equal(R[:, 1], val)
    assert val.max() == 8 and val.min() == 1


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_csr_pattern_closed_forms(elem):
    fp, conn, coords = M.tiny(elem, n=6, L=3)
    rowptr, colidx = O.csr_pattern(conn, coords.shape[0])
    nnz_row = np.diff(rowptr)
    inner = M.interior_nodes(fp, 3, coords.shape[0])
    counts = set(int(nnz_row[2 * i]) for i in inner)
    if elem == "hex8":
        assert counts == {54}            # 27 neighbour nodes x 2 comps
    else:
        assert counts <= {54, 30} and len(counts) == 2
    assert rowptr[-1] == colidx.size
    # symmetric pattern
    rows = np.repeat(np.arange(rowptr.size - 1), nnz_row)
    S = set(zip(rows.tolist(), colidx.tolist()))
    assert all((c, r) in S for (r, c) in list(S)[:5000])


def test_csr_scatter_equals_dense_assembly():
    fp, conn, coords = M.tiny("hex8", n=3, L=2)
    G, wm, _ = O.geometry(HEX, conn, coords)
    U, s, kc = M.fields(fp, 2)
    J = O.evaluate(HEX, conn, G, wm, U, surface=s, kc=kc, mode="jac")["J_cell"]
    rowptr, colidx = O.csr_pattern(conn, coords.shape[0])
    vals, miss = O.scatter_csr(HEX, conn, J, rowptr, colidx)
    assert miss == 0
    nd = 2 * coords.shape[0]
    D = np.zeros((nd, nd))
    dofs = (2 * conn[:, :, None] + np.arange(2)).reshape(conn.shape[0], 16)
    for c in range(conn.shape[0]):
        D[np.ix_(dofs[c], dofs[c])] += J[c]
    rows = np.repeat(np.arange(nd), np.diff(rowptr))
    S = np.zeros((nd, nd))
    S[rows, colidx] = vals
    assert np.abs(S - D).max() < 1e-12 * np.abs(D).max()


def test_partition_and_halo_sum_equals_serial():
    """Column partition + halo sum of shared-node partial residuals equals the
    serial assembled residual; pure set algebra, no GPU."""
    fp, conn, coords = M.tiny("hex8", n=8, L=3)
    L = 3
    G, wm, _ = O.geometry(HEX, conn, coords)
    U, s, kc = M.fields(fp, L)
    Rc = O.evaluate(HEX, conn, G, wm, U, surface=s, kc=kc)["R_cell"]
    Rser = O.scatter(HEX, conn, Rc, coords.shape[0])
    P = 3
    cuts = O.partition_columns(fp.nf, P)
    parts = []
    for r in range(P):
        lconn, gids = O.local_mesh(conn, L, cuts[r], cuts[r + 1])
        Rl = O.scatter(HEX, lconn, Rc[cuts[r] * L:cuts[r + 1] * L], gids.size)
        parts.append((lconn, gids, Rl))
    halo = O.halo_lists([p[1] for p in parts])
    sent = {key: parts[key[0]][2][idx].copy() for key, idx in halo.items()}   # pack all first
    for (r, s_), idx in halo.items():
        parts[s_][2][halo[(s_, r)]] += sent[(r, s_)]                           # then unpack-add
    for lconn, gids, Rl in parts:
        assert np.abs(Rl - Rser[gids]).max() < 1e-12 * np.abs(Rser).max()


def test_geometry_translation_invariant_and_exact_on_offset_thin_cell():
    """Reading Z17: GradBF and det J depend only on relative node positions.
    A metre-thick, sloped cell 800 km from the origin must give the same
    geometry as the same cell at the origin, and det J must match an exact
    rational evaluation of the cofactor expansion (pins the cancellation fix)."""
    from fractions import Fraction
    xyz = np.array([(0, 0, 0), (1.25, 0.1, 0.006), (1.3, 1.2, 0.004), (-0.05, 1.25, -0.002),
                    (0, 0, 0.002), (1.25, 0.1, 0.0085), (1.3, 1.2, 0.0061), (-0.05, 1.25, 0.0003)], float)
    conn = np.arange(8, dtype=np.int32)[None]
    G0, wm0, bad0 = O.geometry(HEX, conn, xyz)
    off = xyz + np.array([812.345678, -655.4321, 1.7])
    G1, wm1, bad1 = O.geometry(HEX, conn, off)
    assert bad0 == 0 and bad1 == 0
    assert np.abs(wm1 / wm0 - 1).max() < 1e-13
    assert np.abs(G1 - G0).max() < 1e-13 * np.abs(G0).max()
    _, dbf, w = O.ref_element(HEX)
    X = [[Fraction(float(v)) for v in p] for p in off]
    for q in range(8):
        Jm = [[sum(X[n][r] * Fraction(float(dbf[n, q, s])) for n in range(8)) for s in range(3)] for r in range(3)]
        det = (Jm[0][0] * (Jm[1][1] * Jm[2][2] - Jm[1][2] * Jm[2][1])
               - Jm[0][1] * (Jm[1][0] * Jm[2][2] - Jm[1][2] * Jm[2][0])
               + Jm[0][2] * (Jm[1][0] * Jm[2][1] - Jm[1][1] * Jm[2][0]))
        assert abs(wm1[0, q] / float(det) - 1) < 1e-14
