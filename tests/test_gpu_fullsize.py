"""Full-size parity at BASELINE.json's sizes, in the launch configuration
bench.py times (stokesfo_jacobian with J_cell and assembled R, R zeroed
first): sampled cells and sampled nodes are recomputed one by one by the
oracle.  C4 = configs[3] (8,431,650 hex8), C5 = configs[4] (16,863,300 wedge6)."""
import numpy as np
import pytest

import oracle as O
from paper_conf_sc_antepara0cw24_b200 import synth

pytestmark = pytest.mark.gpu
TOL = 1e-12


@pytest.mark.parametrize("geometry", ["stored", "on_the_fly", "compact"])
@pytest.mark.parametrize("cfg", ["C3", "C4", "C5"])
def test_fullsize_sampled_parity(cfg, geometry):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    fp, L, elem = synth.make_config(cfg)
    conn, coords = O.extrude(fp.xy, fp.polys, fp.b, fp.H, L)
    U = synth.velocity_balance(fp, L, seed=11 if cfg == "C3" else 12)
    s = synth.surface_nodal(fp, L)
    kc = synth.flow_factor(fp, L)
    C, N = conn.shape
    ctx = StokesFO(elem, torch.from_numpy(conn).cuda(), torch.from_numpy(coords).cuda(),
                   surface=torch.from_numpy(s).cuda(), flow_factor=torch.from_numpy(kc).cuda(), geometry=geometry)
    J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device="cuda")
    R = torch.zeros((coords.shape[0], 2), dtype=torch.float64, device="cuda")
    Ud = torch.from_numpy(U).cuda()
    ctx.jacobian(Ud, J, R=R)
    ctx.sync()
    rng = np.random.default_rng(2024)
    cells = np.unique(np.concatenate([rng.integers(0, C, 1500), [0, C - 1], np.arange(C - 40, C)]))
    e = O.ELEM[elem]
    G, wm, bad = O.geometry(e, conn[cells], coords)
    assert bad == 0
    ref = O.evaluate(e, conn[cells], G, wm, U, surface=s, kc=kc[cells], mode="jac")
    Jg = J[torch.from_numpy(cells).cuda()].cpu().numpy()
    sc = np.abs(ref["J_cell"]).reshape(len(cells), -1).max(1)
    err = np.abs(Jg - ref["J_cell"]).reshape(len(cells), -1).max(1)
    assert (err <= TOL * sc).all(), float((err / sc).max())
    # assembled R at sampled nodes: sum over every cell containing the node
    nodes = np.unique(rng.integers(0, coords.shape[0], 200))
    hit = np.isin(conn, nodes)
    rows = np.nonzero(hit.any(1))[0]
    G2, wm2, _ = O.geometry(e, conn[rows], coords)
    Rc = O.evaluate(e, conn[rows], G2, wm2, U, surface=s, kc=kc[rows])["R_cell"]
    Rref = np.zeros((coords.shape[0], 2))
    Aref = np.zeros((coords.shape[0], 2))
    np.add.at(Rref, conn[rows].reshape(-1), Rc.reshape(-1, 2))
    np.add.at(Aref, conn[rows].reshape(-1), np.abs(Rc).reshape(-1, 2))
    Rg = R[torch.from_numpy(nodes).cuda()].cpu().numpy()
    assert (np.abs(Rg - Rref[nodes]) <= TOL * Aref[nodes] + 1e-300).all()


def _sample_nodes_expect(e, conn, coords, U, s, kc, nodes, need_j):
    """Oracle residual (and element Jacobians) of every cell incident to the sampled nodes."""
    hit = np.isin(conn, nodes)
    rows = np.nonzero(hit.any(1))[0]
    G, wm, _ = O.geometry(e, conn[rows], coords)
    out = O.evaluate(e, conn[rows], G, wm, U, surface=s, kc=kc[rows], mode="jac" if need_j else "resid")
    return rows, out


@pytest.mark.parametrize("cfg", ["C4", "C5"])
def test_fullsize_residual_only_sampled(cfg):
    """stokesfo_viscosity_resid (partial-sum kernel) at full size, sampled assembled nodes."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    fp, L, elem = synth.make_config(cfg)
    conn, coords = O.extrude(fp.xy, fp.polys, fp.b, fp.H, L)
    U = synth.velocity_balance(fp, L, seed=12)
    s = synth.surface_nodal(fp, L)
    kc = synth.flow_factor(fp, L)
    ctx = StokesFO(elem, torch.from_numpy(conn).cuda(), torch.from_numpy(coords).cuda(),
                   surface=torch.from_numpy(s).cuda(), flow_factor=torch.from_numpy(kc).cuda())
    R = torch.zeros((coords.shape[0], 2), dtype=torch.float64, device="cuda")
    ctx.viscosity_resid(torch.from_numpy(U).cuda(), R=R)
    ctx.sync()
    rng = np.random.default_rng(7)
    nodes = np.unique(np.concatenate([rng.integers(0, coords.shape[0], 300), [coords.shape[0] - 1]]))
    e = O.ELEM[elem]
    rows, out = _sample_nodes_expect(e, conn, coords, U, s, kc, nodes, False)
    Rref = np.zeros((coords.shape[0], 2))
    Aref = np.zeros((coords.shape[0], 2))
    np.add.at(Rref, conn[rows].reshape(-1), out["R_cell"].reshape(-1, 2))
    np.add.at(Aref, conn[rows].reshape(-1), np.abs(out["R_cell"]).reshape(-1, 2))
    Rg = R[torch.from_numpy(nodes).cuda()].cpu().numpy()
    assert (np.abs(Rg - Rref[nodes]) <= TOL * Aref[nodes] + 1e-300).all()


@pytest.mark.parametrize("cfg", ["C3", "C5"])
def test_fullsize_csr_assembly_sampled_rows(cfg):
    """NEXT-2 at full size: CSR pattern rows (bit-exact vs the incident cells' node sets),
    pull assembly of stokesfo_jacobian's element matrices, the fused jacobian_csr and the
    packed path (jacobian_packed + assemble_csr_packed), on sampled rows recomputed by the oracle."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    fp, L, elem = synth.make_config(cfg)
    conn, coords = O.extrude(fp.xy, fp.polys, fp.b, fp.H, L)
    U = synth.velocity_balance(fp, L, seed=11 if cfg == "C3" else 12)
    s = synth.surface_nodal(fp, L)
    kc = synth.flow_factor(fp, L)
    C, N = conn.shape
    ctx = StokesFO(elem, torch.from_numpy(conn).cuda(), torch.from_numpy(coords).cuda(),
                   surface=torch.from_numpy(s).cuda(), flow_factor=torch.from_numpy(kc).cuda())
    rowptr, colidx = ctx.csr_pattern()
    ctx.csr_slots()
    Ud = torch.from_numpy(U).cuda()
    rng = np.random.default_rng(11)
    nodes = np.unique(np.concatenate([rng.integers(0, coords.shape[0], 120), [0, coords.shape[0] - 1]]))
    e = O.ELEM[elem]
    rows, out = _sample_nodes_expect(e, conn, coords, U, s, kc, nodes, True)
    rp = rowptr.cpu().numpy()
    want = {}
    for v in nodes:
        nb = np.unique(conn[np.nonzero((conn == v).any(1))[0]])
        cols = np.stack([2 * nb, 2 * nb + 1], 1).reshape(-1)
        for a in range(2):
            got = colidx[int(rp[2 * v + a]):int(rp[2 * v + a + 1])].cpu().numpy()
            assert np.array_equal(got, cols)
            want[(v, a)] = (cols, np.zeros(cols.size), np.zeros(cols.size))
    for r, c in enumerate(rows):
        for i in range(N):
            v = conn[c, i]
            for a in range(2):
                if (v, a) not in want:
                    continue
                cols, val, absv = want[(v, a)]
                pos = np.searchsorted(cols, (2 * conn[c][:, None] + np.arange(2)).reshape(-1))
                np.add.at(val, pos, out["J_cell"][r, 2 * i + a])
                # bound consistent with the per-cell element tolerance: sum of max|J_cell| of contributing cells
                np.add.at(absv, pos, np.full(2 * N, np.abs(out["J_cell"][r]).max()))
    nnz = colidx.numel()
    for how in ("pull", "fused", "packed"):
        vals = torch.zeros(nnz, dtype=torch.float64, device="cuda")
        if how == "fused":
            ctx.jacobian_csr(Ud, vals)
        elif how == "pull":
            J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device="cuda")
            ctx.jacobian(Ud, J)
            ctx.scatter_assemble(J_cell=J, csr_vals=vals)
            del J
        else:  # symmetric block-packed element matrices (tensor cores) + their pull assembly, overwriting
            Jp = torch.empty((C, ctx.packed_blocks, 2, 2), dtype=torch.float64, device="cuda")
            ctx.jacobian_packed(Ud, Jp)
            vals.fill_(float("nan"))
            ctx.assemble_csr_packed(Jp, vals, accumulate=False)
            del Jp
        ctx.sync()
        for (v, a), (cols, val, absv) in want.items():
            got = vals[int(rp[2 * v + a]):int(rp[2 * v + a + 1])].cpu().numpy()
            assert (np.abs(got - val) <= TOL * absv + 1e-300).all(), (how, v, a)
        del vals
        torch.cuda.empty_cache()


@pytest.mark.parametrize("cfg", ["C4", "C5"])
def test_fullsize_jvp_sampled(cfg):
    """NEXT-3 at full size, in the launch bench.py --op jvp times (Y += J(U) X with
    R += R(U) in the same pass): Y and R at sampled nodes equal the oracle's element
    AD Jacobians of every incident cell applied to X, and the oracle residual."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    fp, L, elem = synth.make_config(cfg)
    conn, coords = O.extrude(fp.xy, fp.polys, fp.b, fp.H, L)
    U = synth.velocity_balance(fp, L, seed=12)
    s = synth.surface_nodal(fp, L)
    kc = synth.flow_factor(fp, L)
    C, N = conn.shape
    nn = coords.shape[0]
    X = np.random.default_rng(5).normal(0, 10.0, (nn, 2))
    ctx = StokesFO(elem, torch.from_numpy(conn).cuda(), torch.from_numpy(coords).cuda(),
                   surface=torch.from_numpy(s).cuda(), flow_factor=torch.from_numpy(kc).cuda())
    Y = torch.zeros((nn, 2), dtype=torch.float64, device="cuda")
    R = torch.zeros((nn, 2), dtype=torch.float64, device="cuda")
    ctx.jvp(torch.from_numpy(U).cuda(), torch.from_numpy(X).cuda(), Y, R=R)
    ctx.sync()
    rng = np.random.default_rng(13)
    nodes = np.unique(np.concatenate([rng.integers(0, nn, 150), [0, nn - 1]]))
    e = O.ELEM[elem]
    rows, out = _sample_nodes_expect(e, conn, coords, U, s, kc, nodes, True)
    nr = len(rows)
    Xc = X[conn[rows]].reshape(nr, 2 * N)
    JX = np.einsum("ckl,cl->ck", out["J_cell"], Xc).reshape(nr, N, 2)
    # per-entry bound as in test_jvp_matrix_free_parity: 1e-12 of max|J_c| |X_c| per contributing cell
    scale_c = (np.abs(out["J_cell"]).reshape(nr, -1).max(1) * np.abs(Xc).sum(1))[:, None, None] * np.ones((nr, N, 2))
    Yref = np.zeros((nn, 2))
    Yscale = np.zeros((nn, 2))
    Rref = np.zeros((nn, 2))
    Aref = np.zeros((nn, 2))
    np.add.at(Yref, conn[rows].reshape(-1), JX.reshape(-1, 2))
    np.add.at(Yscale, conn[rows].reshape(-1), scale_c.reshape(-1, 2))
    np.add.at(Rref, conn[rows].reshape(-1), out["R_cell"].reshape(-1, 2))
    np.add.at(Aref, conn[rows].reshape(-1), np.abs(out["R_cell"]).reshape(-1, 2))
    idx = torch.from_numpy(nodes).cuda()
    Yg = Y[idx].cpu().numpy()
    Rg = R[idx].cpu().numpy()
    assert (np.abs(Yg - Yref[nodes]) <= TOL * Yscale[nodes]).all()
    assert (np.abs(Rg - Rref[nodes]) <= TOL * Aref[nodes] + 1e-300).all()
