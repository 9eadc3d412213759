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


@pytest.mark.parametrize("geometry", ["stored", "on_the_fly"])
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
