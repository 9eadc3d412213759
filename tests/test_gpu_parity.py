"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by
element on the same seeded inputs.  Tolerances (SURVEY 8(c) 'Tolerances';
BASELINE.json north_star '1e-12 relative'):
  element outputs  per cell ||X_gpu - X_orc||_max <= 1e-12 ||X_orc||_max
  assembled R      per entry |dR| <= 1e-12 sum|contributions|
  geometry         per (c,q) ||dGradBF|| <= 1e-12 sum_n ||GradBF||
  gather, integer structures, valence probe: bit-exact."""
import numpy as np
import pytest

import oracle as O
from tests import _meshes as M

pytestmark = pytest.mark.gpu

TOL = 1e-12


@pytest.fixture(scope="module")
def torch():
    import torch as _t
    if not _t.cuda.is_available():
        pytest.skip("no CUDA device")
    return _t


def _t(torch, a, dtype=None):
    a = np.ascontiguousarray(a)
    return torch.from_numpy(a).to("cuda") if dtype is None else torch.from_numpy(a).to("cuda", dtype)


GEOMS = ["stored", "on_the_fly", "compact"]


def _setup(torch, elem="hex8", n=16, L=5, drop=0, kind="random", scalar_k=False, surface=True, geometry="stored"):
    fp, conn, coords = M.tiny(elem, n=n, L=L)
    if drop:
        conn = conn[:conn.shape[0] - drop]
    U, s, kc = M.fields(fp, L, kind=kind)
    kc = kc[:conn.shape[0]]
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    ctx = StokesFO(elem, _t(torch, conn), _t(torch, coords), surface=_t(torch, s) if surface else None,
                   flow_factor=None if scalar_k else _t(torch, kc), k=10.77, geometry=geometry)
    e = O.ELEM[elem]
    G, wm, bad = O.geometry(e, conn, coords)
    assert bad == 0
    orc = dict(G=G, wm=wm, conn=conn, coords=coords, U=U, s=s if surface else None,
               kc=None if scalar_k else kc, e=e)
    return ctx, orc


def _cell_rel(a, b):
    a = a.reshape(a.shape[0], -1)
    b = b.reshape(b.shape[0], -1)
    sc = np.maximum(np.abs(b).max(1), 1e-300)
    return float((np.abs(a - b).max(1) / sc).max())


def _assembled_check(R_gpu, orc, R_cell_orc):
    e = orc["e"]
    Rref = O.scatter(e, orc["conn"], R_cell_orc, orc["coords"].shape[0])
    absR = O.scatter(e, orc["conn"], np.abs(R_cell_orc), orc["coords"].shape[0])
    err = np.abs(R_gpu - Rref)
    assert (err <= TOL * absR + 1e-300).all(), float((err / np.maximum(absR, 1e-300)).max())


@pytest.mark.parametrize("geometry", GEOMS)
@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_geometry_parity(torch, elem, geometry):
    ctx, orc = _setup(torch, elem, geometry=geometry)
    G, wm = ctx.geometry()
    ctx.sync()
    G = G.cpu().numpy()
    wm = wm.cpu().numpy()
    scale = np.abs(orc["G"]).sum(axis=(1, 3))  # [C][Q]: sum over n, d
    err = np.abs(G - orc["G"]).max(axis=(1, 3))
    assert (err <= TOL * scale).all()
    assert (np.abs(wm - orc["wm"]) <= TOL * np.abs(orc["wm"])).all()


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_gather_bit_exact(torch, elem):
    ctx, orc = _setup(torch, elem)
    Uc = ctx.gather(_t(torch, orc["U"]))
    ctx.sync()
    assert np.array_equal(Uc.cpu().numpy(), O.gather(orc["e"], orc["conn"], orc["U"]))


@pytest.mark.parametrize("geometry", GEOMS)
@pytest.mark.parametrize("elem,drop,kind", [("hex8", 0, "random"), ("hex8", 5, "balance"),
                                            ("wedge6", 0, "random"), ("wedge6", 7, "balance")])
def test_viscosity_resid_parity(torch, elem, drop, kind, geometry):
    ctx, orc = _setup(torch, elem, drop=drop, kind=kind, geometry=geometry)
    C, N, Q = ctx.num_cells, ctx.N, ctx.Q
    mu = torch.empty((C, Q), dtype=torch.float64, device="cuda")
    Rc = torch.empty((C, N, 2), dtype=torch.float64, device="cuda")
    R = torch.zeros((ctx.num_nodes, 2), dtype=torch.float64, device="cuda")
    ctx.viscosity_resid(_t(torch, orc["U"]), mu_qp=mu, R_cell=Rc, R=R)
    ctx.sync()
    ref = O.evaluate(orc["e"], orc["conn"], orc["G"], orc["wm"], orc["U"], surface=orc["s"], kc=orc["kc"])
    assert np.abs(mu.cpu().numpy() / ref["mu_qp"] - 1).max() <= TOL
    assert _cell_rel(Rc.cpu().numpy(), ref["R_cell"]) <= TOL
    _assembled_check(R.cpu().numpy(), orc, ref["R_cell"])


@pytest.mark.parametrize("geometry", GEOMS)
@pytest.mark.parametrize("elem,drop", [("hex8", 0), ("hex8", 3), ("wedge6", 0), ("wedge6", 11)])
def test_jacobian_parity(torch, elem, drop, geometry):
    ctx, orc = _setup(torch, elem, drop=drop, geometry=geometry)
    C, N = ctx.num_cells, ctx.N
    J = torch.full((C, 2 * N, 2 * N), float("nan"), dtype=torch.float64, device="cuda")
    Rc = torch.empty((C, N, 2), dtype=torch.float64, device="cuda")
    R = torch.zeros((ctx.num_nodes, 2), dtype=torch.float64, device="cuda")
    ctx.jacobian(_t(torch, orc["U"]), J, R_cell=Rc, R=R)
    ctx.sync()
    ref = O.evaluate(orc["e"], orc["conn"], orc["G"], orc["wm"], orc["U"], surface=orc["s"], kc=orc["kc"],
                     mode="jac")
    Jg = J.cpu().numpy()
    assert np.isfinite(Jg).all()
    assert _cell_rel(Jg, ref["J_cell"]) <= TOL
    assert _cell_rel(Rc.cpu().numpy(), ref["R_cell"]) <= TOL
    _assembled_check(R.cpu().numpy(), orc, ref["R_cell"])


@pytest.mark.parametrize("geometry", GEOMS)
def test_jacobian_residual_equals_viscosity_resid(torch, geometry):
    ctx, orc = _setup(torch, "hex8", geometry=geometry)
    C, N = ctx.num_cells, ctx.N
    J = torch.empty((C, 16, 16), dtype=torch.float64, device="cuda")
    R1 = torch.empty((C, N, 2), dtype=torch.float64, device="cuda")
    R2 = torch.empty((C, N, 2), dtype=torch.float64, device="cuda")
    U = _t(torch, orc["U"])
    ctx.jacobian(U, J, R_cell=R1)
    ctx.viscosity_resid(U, R_cell=R2)
    ctx.sync()
    # same residual up to reassociation (reading Z12): the stored-geometry residual-only
    # kernel sums per-QP partial contributions G_n . (wmu2 beta) in a rotated order
    assert _cell_rel(R1.cpu().numpy(), R2.cpu().numpy()) <= 1e-13


@pytest.mark.parametrize("geometry", GEOMS)
@pytest.mark.parametrize("scalar_k,surface", [(True, True), (False, False), (True, False)])
def test_optional_inputs(torch, scalar_k, surface, geometry):
    ctx, orc = _setup(torch, "hex8", n=6, L=3, scalar_k=scalar_k, surface=surface, geometry=geometry)
    C = ctx.num_cells
    J = torch.empty((C, 16, 16), dtype=torch.float64, device="cuda")
    Rc = torch.empty((C, 8, 2), dtype=torch.float64, device="cuda")
    ctx.jacobian(_t(torch, orc["U"]), J, R_cell=Rc)
    ctx.sync()
    ref = O.evaluate(orc["e"], orc["conn"], orc["G"], orc["wm"], orc["U"], surface=orc["s"], kc=orc["kc"],
                     k=10.77, mode="jac")
    assert _cell_rel(J.cpu().numpy(), ref["J_cell"]) <= TOL
    assert _cell_rel(Rc.cpu().numpy(), ref["R_cell"]) <= TOL


@pytest.mark.parametrize("geometry", GEOMS)
def test_force_qp_input(torch, geometry):
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    fp, conn, coords = M.tiny("hex8", n=6, L=3)
    U, s, kc = M.fields(fp, 3)
    f = np.random.default_rng(9).normal(0, 1, (conn.shape[0], 8, 2))
    ctx = StokesFO("hex8", _t(torch, conn), _t(torch, coords), surface=_t(torch, s), force_qp=_t(torch, f),
                   flow_factor=_t(torch, kc), geometry=geometry)
    Rc = torch.empty((conn.shape[0], 8, 2), dtype=torch.float64, device="cuda")
    ctx.viscosity_resid(_t(torch, U), R_cell=Rc)
    ctx.sync()
    G, wm, _ = O.geometry(0, conn, coords)
    ref = O.evaluate(0, conn, G, wm, U, force_qp=f, kc=kc)
    assert _cell_rel(Rc.cpu().numpy(), ref["R_cell"]) <= TOL


@pytest.mark.parametrize("geometry", GEOMS)
@pytest.mark.parametrize("name", ["B", "W"])
def test_golden_cells_gpu(torch, golden, name, geometry):
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    g = golden[name]
    N = 8 if g["elem"] == "hex8" else 6
    conn = np.arange(N, dtype=np.int32)[None]
    ctx = StokesFO(g["elem"], _t(torch, conn), _t(torch, np.array(g["coords"], float)),
                   surface=_t(torch, np.array(g["s"], float)), k=g["k"], delta=g["delta"], rho_g=g["rho_g"],
                   geometry=geometry)
    J = torch.empty((1, 2 * N, 2 * N), dtype=torch.float64, device="cuda")
    Rc = torch.empty((1, N, 2), dtype=torch.float64, device="cuda")
    mu = torch.empty((1, N), dtype=torch.float64, device="cuda")
    U = _t(torch, np.array(g["U"], float))
    ctx.jacobian(U, J, R_cell=Rc)
    ctx.viscosity_resid(U, mu_qp=mu)
    ctx.sync()
    tol = golden["tolerance_gpu"]
    J = J.cpu().numpy()[0]
    assert np.abs(mu.cpu().numpy()[0] - g["mu_q"]).max() <= tol * max(g["mu_q"])
    assert np.abs(Rc.cpu().numpy()[0] - np.array(g["R_cell"])).max() <= tol * np.abs(g["R_cell"]).max()
    assert np.abs(J[0] - g["J_row0"]).max() <= tol * np.abs(J).max()
    assert np.abs(np.diag(J) - g["J_diag"]).max() <= tol * np.abs(J).max()


def test_valence_probe_bit_exact(torch):
    ctx, orc = _setup(torch, "hex8")
    ones = torch.ones((ctx.num_cells, 8, 2), dtype=torch.float64, device="cuda")
    R = torch.zeros((ctx.num_nodes, 2), dtype=torch.float64, device="cuda")
    ctx.scatter_assemble(R_cell=ones, R=R)
    ctx.sync()
    val = np.bincount(orc["conn"].reshape(-1), minlength=ctx.num_nodes).astype(float)
    Rh = R.cpu().numpy()
    assert np.array_equal(Rh[:, 0], val) and np.array_equal(Rh[:, 1], val)


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_csr_pattern_and_assembly(torch, elem):
    ctx, orc = _setup(torch, elem, n=5, L=3)
    rowptr, colidx = ctx.csr_pattern()
    rp2, ci2 = O.csr_pattern(orc["conn"], ctx.num_nodes)
    assert np.array_equal(rowptr.cpu().numpy(), rp2) and np.array_equal(colidx.cpu().numpy(), ci2)
    C, N = ctx.num_cells, ctx.N
    J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device="cuda")
    ctx.jacobian(_t(torch, orc["U"]), J)
    vals = torch.zeros(colidx.numel(), dtype=torch.float64, device="cuda")
    ctx.scatter_assemble(J_cell=J, csr_vals=vals)
    ctx.sync()
    ref = O.evaluate(orc["e"], orc["conn"], orc["G"], orc["wm"], orc["U"], surface=orc["s"], kc=orc["kc"],
                     mode="jac")["J_cell"]
    v2, miss = O.scatter_csr(orc["e"], orc["conn"], ref, rp2, ci2)
    # per-entry bound consistent with the element tolerance (per cell
    # ||dJ||_max <= 1e-12 ||J||_max): sum over contributing cells of max|J_cell|
    cell_scale = np.abs(ref).reshape(C, -1).max(1)[:, None, None] * np.ones_like(ref)
    a2, _ = O.scatter_csr(orc["e"], orc["conn"], cell_scale, rp2, ci2)
    assert miss == 0
    assert (np.abs(vals.cpu().numpy() - v2) <= TOL * a2).all()


def test_halo_pack_unpack(torch):
    ctx, orc = _setup(torch, "hex8", n=4, L=2)
    R = torch.from_numpy(np.random.default_rng(3).normal(size=(ctx.num_nodes, 2))).cuda()
    nodes = torch.tensor([5, 0, 17, 3], dtype=torch.int32, device="cuda")
    buf = torch.empty((4, 2), dtype=torch.float64, device="cuda")
    ctx.halo_pack(R, nodes, buf)
    R2 = R.clone()
    ctx.halo_unpack_add(buf, nodes, R2)
    ctx.sync()
    assert torch.equal(buf, R[nodes.long()])
    assert torch.equal(R2[nodes.long()], R[nodes.long()] * 2)


@pytest.mark.parametrize("geometry", GEOMS)
def test_edge_cases_and_errors(torch, geometry):
    from paper_conf_sc_antepara0cw24_b200 import StokesFO, StokesFOError
    fp, conn, coords = M.tiny("hex8", n=2, L=1)
    # empty mesh: every call is a no-op
    ctx0 = StokesFO("hex8", _t(torch, conn[:0]), _t(torch, coords), geometry=geometry)
    J0 = torch.empty((0, 16, 16), dtype=torch.float64, device="cuda")
    ctx0.jacobian(torch.zeros((coords.shape[0], 2), dtype=torch.float64, device="cuda"), J0)
    ctx0.sync()
    # one cell
    ctx1 = StokesFO("hex8", _t(torch, conn[:1]), _t(torch, coords), geometry=geometry)
    J1 = torch.empty((1, 16, 16), dtype=torch.float64, device="cuda")
    U = np.random.default_rng(0).normal(0, 50, (coords.shape[0], 2))
    ctx1.jacobian(_t(torch, U), J1)
    ctx1.sync()
    G, wm, _ = O.geometry(0, conn[:1], coords)
    ref = O.evaluate(0, conn[:1], G, wm, U, k=10.77, mode="jac")
    assert _cell_rel(J1.cpu().numpy(), ref["J_cell"]) <= TOL
    # glen_n != 3
    with pytest.raises(StokesFOError, match="EUNSUPPORTED"):
        StokesFO("hex8", _t(torch, conn), _t(torch, coords), glen_n=2.0, geometry=geometry)
    # inverted cell -> EMESH at sync
    bad = conn.copy()
    bad[0] = bad[0][[4, 5, 6, 7, 0, 1, 2, 3]]
    ctxb = StokesFO("hex8", _t(torch, bad), _t(torch, coords), geometry=geometry)
    with pytest.raises(StokesFOError, match="EMESH"):
        ctxb.sync()
    # conn out of range (past the end, or negative) -> EMESH from create itself: no ctx
    # exists that could use it as an address (on-the-fly and side-set kernels)
    for v in (coords.shape[0] + 5, -1):
        bad2 = conn.copy()
        bad2[1, 3] = v
        with pytest.raises(StokesFOError, match="EMESH"):
            StokesFO("hex8", _t(torch, bad2), _t(torch, coords), geometry=geometry)
    # csr_pattern range-checks conn on the host before indexing with it (a caller
    # that corrupts conn after create gets EMESH, not a heap overwrite)
    connd = _t(torch, conn)
    ctxd = StokesFO("hex8", connd, _t(torch, coords), geometry=geometry)
    ctxd.sync()
    connd[0, 0] = coords.shape[0] + 1
    with pytest.raises(StokesFOError, match="EMESH"):
        ctxd.csr_pattern()
    # a peer table without the peers' Y -> jvp refuses (Y would miss boundary
    # contributions); the single-GPU Newton driver refuses any peer table
    nn = coords.shape[0]
    rem = torch.full((nn,), -1, dtype=torch.int32, device="cuda")
    remtab = torch.zeros((1, 15), dtype=torch.int32, device="cuda")
    peers = torch.zeros(2, dtype=torch.int64, device="cuda")
    ctx1.set_remote(rem, remtab, peers)
    Z = torch.zeros((nn, 2), dtype=torch.float64, device="cuda")
    with pytest.raises(StokesFOError, match="EINVAL"):
        ctx1.jvp(Z, Z, Z.clone())
    with pytest.raises(StokesFOError, match="EINVAL"):
        ctx1.newton_solve(None, None, Z.clone(), max_newton=1)
    ctx1.set_remote_jvp(peers)
    ctx1.jvp(Z, Z, Z.clone())
    ctx1.set_remote(None, None, None)
    ctx1.sync()
    # misaligned output pointer -> EINVAL
    big = torch.empty(2 * 16 * 16 + 1, dtype=torch.float64, device="cuda")
    lib = __import__("paper_conf_sc_antepara0cw24_b200.stokesfo", fromlist=["_lib"])._lib()
    import ctypes
    st = lib.stokesfo_jacobian(ctx1._h, ctypes.c_void_p(_t(torch, U).data_ptr()),
                               ctypes.c_void_p(big.data_ptr() + 8), None, None)
    assert st == 1


@pytest.mark.parametrize("geometry", GEOMS)
@pytest.mark.parametrize("elem,drop", [("hex8", 0), ("hex8", 3), ("wedge6", 7)])
def test_jvp_matrix_free_parity(torch, elem, drop, geometry):
    """NEXT-3: Y += J(U) X computed matrix-free (directional derivative of the
    fused chain) equals the oracle's assembled AD Jacobian applied to X; the
    residual of the same pass equals the oracle residual."""
    ctx, orc = _setup(torch, elem, drop=drop, geometry=geometry)
    nn = ctx.num_nodes
    X = np.random.default_rng(77).normal(0, 30.0, (nn, 2))
    Y = torch.zeros((nn, 2), dtype=torch.float64, device="cuda")
    R = torch.zeros((nn, 2), dtype=torch.float64, device="cuda")
    ctx.jvp(_t(torch, orc["U"]), _t(torch, X), Y, R=R)
    ctx.sync()
    ref = O.evaluate(orc["e"], orc["conn"], orc["G"], orc["wm"], orc["U"], surface=orc["s"], kc=orc["kc"],
                     mode="jac")
    C, N = orc["conn"].shape
    Xc = X[orc["conn"]].reshape(C, 2 * N)
    JX = np.einsum("ckl,cl->ck", ref["J_cell"], Xc).reshape(C, N, 2)
    # per-entry bound: element tolerance (1e-12 of max|J_c| |X_c|) summed over contributing cells
    scale_c = (np.abs(ref["J_cell"]).reshape(C, -1).max(1) * np.abs(Xc).sum(1))[:, None, None] * np.ones((C, N, 2))
    Yref = O.scatter(orc["e"], orc["conn"], JX, nn)
    Yscale = O.scatter(orc["e"], orc["conn"], scale_c, nn)
    assert (np.abs(Y.cpu().numpy() - Yref) <= TOL * Yscale).all()
    _assembled_check(R.cpu().numpy(), orc, ref["R_cell"])
    # linearity in X: J(U)(2X) = 2 J(U) X (bitwise up to the atomics' order -> 1e-15)
    Y2 = torch.zeros((nn, 2), dtype=torch.float64, device="cuda")
    ctx.jvp(_t(torch, orc["U"]), _t(torch, 2 * X), Y2)
    ctx.sync()
    assert torch.allclose(Y2, 2 * Y, rtol=1e-14, atol=1e-14 * float(Y.abs().max()))


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_basal_friction_parity(torch, elem):
    """NEXT-4 (reading Z18): GPU basal-friction side-set term vs the numpy oracle."""
    from oracle import basal as B
    L = 5
    ctx, orc = _setup(torch, elem, n=8, L=L)
    nb = 4 if elem == "hex8" else 3
    cells = np.arange(0, ctx.num_cells, L, dtype=np.int32)    # k = 0: bed cells
    beta = np.random.default_rng(8).uniform(0.1, 3.0, ctx.num_nodes)
    R = torch.zeros((ctx.num_nodes, 2), dtype=torch.float64, device="cuda")
    Jf = torch.empty((cells.size, 2 * nb, 2 * nb), dtype=torch.float64, device="cuda")
    ctx.basal_friction(_t(torch, cells), _t(torch, beta), _t(torch, orc["U"]), R, J_face=Jf)
    ctx.sync()
    Rr, Jr, _ = B.basal_friction(nb, orc["conn"], orc["coords"], cells, beta, orc["U"])
    Jg = Jf.cpu().numpy()
    sc = np.abs(Jr).reshape(cells.size, -1).max(1)
    assert (np.abs(Jg - Jr).reshape(cells.size, -1).max(1) <= TOL * sc).all()
    assert np.abs(R.cpu().numpy() - Rr).max() <= TOL * np.abs(Rr).max()


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_lateral_pressure_parity(torch, elem):
    """NEXT-4 (reading Z19): GPU lateral (calving-front) pressure term vs the numpy
    oracle on every footprint-boundary face; sea level cuts through the faces of
    some columns (above-, below- and straddling-water faces all occur)."""
    from oracle import lateral as LT
    L = 5
    ctx, orc = _setup(torch, elem, n=8, L=L)
    faces = LT.lateral_faces(M.tiny(elem, n=8, L=L)[0].polys, L)
    z = orc["coords"][:, 2]
    zsl = 0.5 * (z.min() + z.max())
    assert (z < zsl).any() and (z > zsl).any()
    R = torch.zeros((ctx.num_nodes, 2), dtype=torch.float64, device="cuda")
    ctx.lateral_pressure(_t(torch, faces), _t(torch, orc["s"]), R, rho_i_g=8.927, rho_w_g=10.05, sea_level=zsl)
    ctx.sync()
    Rr, F = LT.lateral_pressure(ctx.N, orc["conn"], orc["coords"], faces, orc["s"],
                                8.927, 10.05, zsl)
    assert np.abs(Rr).max() > 0
    assert np.abs(R.cpu().numpy() - Rr).max() <= TOL * np.abs(Rr).max()
    # a side index outside [0, P) raises the sticky EMESH flag
    bad = faces[:1].copy()
    bad[0, 1] = ctx.N // 2
    ctx.lateral_pressure(_t(torch, bad), _t(torch, orc["s"]), R)
    from paper_conf_sc_antepara0cw24_b200.stokesfo import StokesFOError
    with pytest.raises(StokesFOError):
        ctx.sync()


@pytest.mark.parametrize("geometry", GEOMS)
@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_csr_slots_and_fused_assembly(torch, elem, geometry):
    """NEXT-2: per-cell CSR slots bit-exact vs the oracle's pattern (searchsorted),
    slot-based scatter_assemble and the fused jacobian_csr (no element matrices)
    vs the oracle's CSR scatter of its element Jacobians; ragged last tile."""
    ctx, orc = _setup(torch, elem, n=5, L=3, drop=3, geometry=geometry)
    C, N = ctx.num_cells, ctx.N
    rowptr, colidx = ctx.csr_pattern()
    rp2, ci2 = O.csr_pattern(orc["conn"], ctx.num_nodes)
    slots = ctx.csr_slots().cpu().numpy().view(np.uint8).reshape(C, N, 8)[:, :, :N]
    conn = orc["conn"]
    want = np.zeros((C, N, N), dtype=np.uint8)
    for c in range(C):
        for i in range(N):
            row = 2 * conn[c, i]
            cols = ci2[rp2[row]:rp2[row + 1]]
            for j in range(N):
                k = int(np.searchsorted(cols, 2 * conn[c, j]))
                assert cols[k] == 2 * conn[c, j]
                want[c, i, j] = k // 2
    assert np.array_equal(slots, want)
    ref = O.evaluate(orc["e"], conn, orc["G"], orc["wm"], orc["U"], surface=orc["s"], kc=orc["kc"], mode="jac")
    v2, miss = O.scatter_csr(orc["e"], conn, ref["J_cell"], rp2, ci2)
    cell_scale = np.abs(ref["J_cell"]).reshape(C, -1).max(1)[:, None, None] * np.ones_like(ref["J_cell"])
    a2, _ = O.scatter_csr(orc["e"], conn, cell_scale, rp2, ci2)
    assert miss == 0
    U = _t(torch, orc["U"])
    # slot-based assembly of element matrices
    J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device="cuda")
    ctx.jacobian(U, J)
    vals = torch.zeros(colidx.numel(), dtype=torch.float64, device="cuda")
    ctx.scatter_assemble(J_cell=J, csr_vals=vals)
    ctx.sync()
    assert (np.abs(vals.cpu().numpy() - v2) <= TOL * a2).all()
    # the slot-based assembly is atomic-free (one warp owns a node's two rows): bitwise reproducible
    vals2 = torch.zeros_like(vals)
    ctx.scatter_assemble(J_cell=J, csr_vals=vals2)
    ctx.sync()
    assert torch.equal(vals, vals2)
    # overwrite mode (stokesfo_assemble_csr, accumulate = 0): every entry of the pattern is written
    # (a NaN prefill must disappear) and equals the accumulated assembly bitwise; accumulate = 1 adds
    vals3 = torch.full_like(vals, float("nan"))
    ctx.assemble_csr(J, vals3, accumulate=False)
    ctx.sync()
    assert torch.equal(vals3, vals)
    ctx.assemble_csr(J, vals3, accumulate=True)
    ctx.sync()
    assert torch.equal(vals3, 2 * vals)
    # fused: residual + Jacobian straight into CSR
    vals.zero_()
    R = torch.zeros((ctx.num_nodes, 2), dtype=torch.float64, device="cuda")
    ctx.jacobian_csr(U, vals, R=R)
    ctx.sync()
    assert (np.abs(vals.cpu().numpy() - v2) <= TOL * a2).all()
    _assembled_check(R.cpu().numpy(), orc, ref["R_cell"])


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_second_slot_table_is_self_contained(torch, elem):
    """A second stokesfo_csr_slots call into a new buffer (same pattern) carries the node incidence and
    rebuilds the per-node pull records in that buffer: overwriting the first buffer afterwards must not change
    the pull assembly (it matches the oracle's CSR scatter)."""
    ctx, orc = _setup(torch, elem, n=5, L=3, drop=2)
    C, N = ctx.num_cells, ctx.N
    conn = orc["conn"]
    rowptr, colidx = ctx.csr_pattern()
    rp2, ci2 = O.csr_pattern(conn, ctx.num_nodes)
    ctx.csr_slots()
    first = ctx.slots
    ctx.csr_slots()
    assert ctx.slots.data_ptr() != first.data_ptr()
    first.fill_(-1)  # garbage where the first table, incidence and records were
    ref = O.evaluate(orc["e"], conn, orc["G"], orc["wm"], orc["U"], surface=orc["s"], kc=orc["kc"], mode="jac")
    v2, _ = O.scatter_csr(orc["e"], conn, ref["J_cell"], rp2, ci2)
    cell_scale = np.abs(ref["J_cell"]).reshape(C, -1).max(1)[:, None, None] * np.ones_like(ref["J_cell"])
    a2, _ = O.scatter_csr(orc["e"], conn, cell_scale, rp2, ci2)
    J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device="cuda")
    ctx.jacobian(_t(torch, orc["U"]), J)
    vals = torch.full((colidx.numel(),), float("nan"), dtype=torch.float64, device="cuda")
    ctx.assemble_csr(J, vals, accumulate=False)
    ctx.sync()
    assert (np.abs(vals.cpu().numpy() - v2) <= TOL * a2).all()


def _unpack_blocks(Jp, N):
    """Full [C][2N][2N] element matrices from the symmetric block-packed form (header: block (i, j >= i) at
    index i N - i (i - 1) / 2 + (j - i), entries [a][b] = J[(i,a),(j,b)]; block (j, i) = block (i, j)^T)."""
    C = Jp.shape[0]
    J = np.empty((C, 2 * N, 2 * N))
    k = 0
    for i in range(N):
        for j in range(i, N):
            J[:, 2 * i:2 * i + 2, 2 * j:2 * j + 2] = Jp[:, k]
            J[:, 2 * j:2 * j + 2, 2 * i:2 * i + 2] = np.transpose(Jp[:, k], (0, 2, 1))
            k += 1
    return J


@pytest.mark.parametrize("geometry", GEOMS)
@pytest.mark.parametrize("elem,drop", [("hex8", 0), ("hex8", 3), ("wedge6", 0), ("wedge6", 11)])
def test_jacobian_packed_and_assembly(torch, elem, drop, geometry):
    """NEXT-2 symmetric block-packed element matrices (stokesfo_jacobian_packed): unpacked, they match the
    oracle's dual-number J at 1e-12 (the oracle's J is symmetric to rounding: a transposed operand or a
    wrong block index in the packing fails this), R_cell / R as the full path; no write past the last
    cell; the pull assembly from the packed form (stokesfo_assemble_csr_packed) matches the oracle's CSR
    scatter, overwrites every entry and is bitwise reproducible."""
    ctx, orc = _setup(torch, elem, n=6, L=3, drop=drop, geometry=geometry)
    C, N = ctx.num_cells, ctx.N
    NB = N * (N + 1) // 2
    conn = orc["conn"]
    ref = O.evaluate(orc["e"], conn, orc["G"], orc["wm"], orc["U"], surface=orc["s"], kc=orc["kc"], mode="jac")
    U = _t(torch, orc["U"])
    buf = torch.full(((C + 2) * NB * 4,), 7.0, dtype=torch.float64, device="cuda")
    Jp = buf[:C * NB * 4].view(C, NB, 2, 2)
    Rc = torch.empty((C, N, 2), dtype=torch.float64, device="cuda")
    R = torch.zeros((ctx.num_nodes, 2), dtype=torch.float64, device="cuda")
    ctx.jacobian_packed(U, Jp, R_cell=Rc, R=R)
    ctx.sync()
    assert (buf[C * NB * 4:] == 7.0).all()
    Jpn = Jp.cpu().numpy()
    assert np.isfinite(Jpn).all()
    assert _cell_rel(_unpack_blocks(Jpn, N), ref["J_cell"]) <= TOL
    assert _cell_rel(Rc.cpu().numpy(), ref["R_cell"]) <= TOL
    _assembled_check(R.cpu().numpy(), orc, ref["R_cell"])
    # pull assembly from the packed form
    rowptr, colidx = ctx.csr_pattern()
    rp2, ci2 = O.csr_pattern(conn, ctx.num_nodes)
    ctx.csr_slots()
    v2, miss = O.scatter_csr(orc["e"], conn, ref["J_cell"], rp2, ci2)
    cell_scale = np.abs(ref["J_cell"]).reshape(C, -1).max(1)[:, None, None] * np.ones_like(ref["J_cell"])
    a2, _ = O.scatter_csr(orc["e"], conn, cell_scale, rp2, ci2)
    assert miss == 0
    vals = torch.full((colidx.numel(),), float("nan"), dtype=torch.float64, device="cuda")
    ctx.assemble_csr_packed(Jp, vals, accumulate=False)
    ctx.sync()
    assert (np.abs(vals.cpu().numpy() - v2) <= TOL * a2).all()
    vals2 = torch.zeros_like(vals)
    ctx.assemble_csr_packed(Jp, vals2, accumulate=True)
    ctx.sync()
    assert torch.equal(vals, vals2)


def test_jacobian_packed_unsupported(torch, monkeypatch):
    """The packed form comes from the tensor-core kernels only: STOKESFO_JAC_MMA=0 at create returns
    EUNSUPPORTED in every geometry mode (a loud error, no silent fallback)."""
    from paper_conf_sc_antepara0cw24_b200.stokesfo import StokesFOError
    for geometry, mma in (("on_the_fly", "0"), ("stored", "0"), ("compact", "0")):
        monkeypatch.setenv("STOKESFO_JAC_MMA", mma)
        ctx, orc = _setup(torch, "hex8", n=4, L=2, geometry=geometry)
        C, N = ctx.num_cells, ctx.N
        Jp = torch.empty((C, N * (N + 1) // 2, 2, 2), dtype=torch.float64, device="cuda")
        with pytest.raises(StokesFOError, match="unsupported|EUNSUPPORTED"):
            ctx.jacobian_packed(_t(torch, orc["U"]), Jp)


@pytest.mark.parametrize("drop", [0, 11])
def test_wedge_tensor_map_store(torch, drop, monkeypatch):
    """wedge6 J tiles leave the kernel as ONE 2-D TMA tensor store of the padded
    (146-double pitch) staging image per tile (csrc/sfo_kernels.cuh store_J): the
    result must be bitwise the per-cell bulk-copy path's (STOKESFO_JMAP=0), and
    neither the padding columns nor the box rows past the last cell may land in
    memory: a sentinel after J[C-1] (ragged last tile for drop=11) stays intact."""
    monkeypatch.setenv("STOKESFO_JAC_MMA", "0")  # the vector kernel (the DMMA kernel stores J directly)
    ctx, orc = _setup(torch, "wedge6", drop=drop)
    C, N = ctx.num_cells, ctx.N
    U = _t(torch, orc["U"])
    outs = []
    for jmap in ("1", "0"):
        monkeypatch.setenv("STOKESFO_JMAP", jmap)
        buf = torch.full((C + 3, 2 * N, 2 * N), 7.0, dtype=torch.float64, device="cuda")
        ctx.jacobian(U, buf[:C])
        ctx.sync()
        outs.append(buf.cpu().numpy())
    a, b = outs
    assert (a[C:] == 7.0).all() and (b[C:] == 7.0).all()
    assert np.array_equal(a[:C], b[:C])
    ref = O.evaluate(orc["e"], orc["conn"], orc["G"], orc["wm"], orc["U"], surface=orc["s"], kc=orc["kc"],
                     mode="jac")
    assert _cell_rel(a[:C], ref["J_cell"]) <= TOL


@pytest.mark.parametrize("geometry", GEOMS)
@pytest.mark.parametrize("elem,drop", [("hex8", 0), ("hex8", 3), ("wedge6", 0), ("wedge6", 11)])
def test_jacobian_tensor_core_vs_vector(torch, elem, drop, geometry, monkeypatch):
    """The element Jacobians on the fp64 tensor cores (eval_mma_kernel / eval_compact_mma_kernel; default for
    hex8, STOKESFO_JAC_MMA=1 forces them for wedge6 too) and on the vector pipes (STOKESFO_JAC_MMA=0) both
    match the oracle at 1e-12; a J_cell that is only
    16-B aligned (the ABI's requirement) takes the vector kernel on a DMMA context; the DMMA kernels write
    no byte past the last cell (ragged last tile: sentinel cells after J[C-1] stay intact)."""
    outs = {}
    for mma in ("1", "0"):
        monkeypatch.setenv("STOKESFO_JAC_MMA", mma)
        ctx, orc = _setup(torch, elem, drop=drop, geometry=geometry)
        C, N = ctx.num_cells, ctx.N
        U = _t(torch, orc["U"])
        buf = torch.full(((C + 3) * 4 * N * N + 2,), 7.0, dtype=torch.float64, device="cuda")
        for off in (0, 2):  # 32-B aligned, then 16-B aligned only
            J = buf[off:off + C * 4 * N * N].view(C, 2 * N, 2 * N)
            Rc = torch.empty((C, N, 2), dtype=torch.float64, device="cuda")
            R = torch.zeros((ctx.num_nodes, 2), dtype=torch.float64, device="cuda")
            ctx.jacobian(U, J, R_cell=Rc, R=R)
            ctx.sync()
            b = buf.cpu().numpy()
            assert (b[off + C * 4 * N * N:] == 7.0).all()
            outs[(mma, off)] = (J.cpu().numpy().copy(), Rc.cpu().numpy(), R.cpu().numpy())
            buf.fill_(7.0)
    ref = O.evaluate(orc["e"], orc["conn"], orc["G"], orc["wm"], orc["U"], surface=orc["s"], kc=orc["kc"],
                     mode="jac")
    for key, (J, Rc, R) in outs.items():
        assert np.isfinite(J).all(), key
        assert _cell_rel(J, ref["J_cell"]) <= TOL, key
        assert _cell_rel(Rc, ref["R_cell"]) <= TOL, key
        _assembled_check(R, orc, ref["R_cell"])
    # the misaligned call on the DMMA context ran the vector kernel: bitwise the JAC_MMA=0 result
    assert np.array_equal(outs[("1", 2)][0], outs[("0", 0)][0])


@pytest.mark.parametrize("geometry", GEOMS)
@pytest.mark.parametrize("elem,drop", [("hex8", 0), ("hex8", 3), ("wedge6", 7)])
def test_jacobian_diag_parity(torch, elem, drop, geometry):
    """NEXT-3 Jacobi preconditioner: stokesfo_jacobian_diag adds the diagonal of
    the assembled Jacobian without forming element matrices; it must equal the
    oracle's AD element Jacobians' diagonals scattered to the nodes (every cell's
    J is PSD, so the diagonal sums have no cancellation: per-entry 1e-12 relative),
    and the residual of the same pass the oracle residual."""
    ctx, orc = _setup(torch, elem, drop=drop, geometry=geometry)
    nn = ctx.num_nodes
    diag = torch.zeros((nn, 2), dtype=torch.float64, device="cuda")
    R = torch.zeros((nn, 2), dtype=torch.float64, device="cuda")
    ctx.jacobian_diag(_t(torch, orc["U"]), diag, R=R)
    ctx.sync()
    ref = O.evaluate(orc["e"], orc["conn"], orc["G"], orc["wm"], orc["U"], surface=orc["s"], kc=orc["kc"],
                     mode="jac")
    C, N = orc["conn"].shape
    dcell = np.diagonal(ref["J_cell"], axis1=1, axis2=2).reshape(C, N, 2)
    assert (dcell > 0).all()
    dref = O.scatter(orc["e"], orc["conn"], dcell, nn)
    used = np.bincount(orc["conn"].reshape(-1), minlength=nn) > 0
    assert (np.abs(diag.cpu().numpy() - dref) <= TOL * dref).all()
    assert not diag.cpu().numpy()[~used].any()
    _assembled_check(R.cpu().numpy(), orc, ref["R_cell"])


@pytest.mark.parametrize("geometry", GEOMS)
def test_check_finite_flags_nan_outputs(torch, geometry, monkeypatch):
    """Failure detection: with STOKESFO_CHECK_FINITE=1 at create, a NaN
    in U propagates to R / J and stokesfo_sync reports ENONFINITE; finite inputs stay OK,
    and without the switch nothing is scanned."""
    from paper_conf_sc_antepara0cw24_b200 import StokesFOError
    monkeypatch.setenv("STOKESFO_CHECK_FINITE", "1")
    ctx, orc = _setup(torch, "hex8", n=6, L=3, geometry=geometry)
    C, nn = ctx.num_cells, ctx.num_nodes
    J = torch.empty((C, 16, 16), dtype=torch.float64, device="cuda")
    R = torch.zeros((nn, 2), dtype=torch.float64, device="cuda")
    U = _t(torch, orc["U"])
    ctx.jacobian(U, J, R=R)
    ctx.sync()   # finite: OK
    Ubad = U.clone()
    Ubad[nn // 2, 0] = float("nan")
    ctx.jacobian(Ubad, J, R=R)
    with pytest.raises(StokesFOError, match="ENONFINITE"):
        ctx.sync()
    monkeypatch.setenv("STOKESFO_CHECK_FINITE", "0")
    ctx2, _ = _setup(torch, "hex8", n=6, L=3, geometry=geometry)
    ctx2.jacobian(Ubad, J, R=R)
    ctx2.sync()   # not scanned
