"""NEXT-1 parity: the paper's evaluator chain on B200 (separate gather, Ugrad,
muLandIce, force kernels with HBM intermediates + StokesFOResid in Fig. 2's
baseline and optimized loop structures; Jacobian with 2N SFad
lanes) must reproduce the oracle's R_cell and J_cell (1e-12 per
cell max-norm), like the fused path."""
import numpy as np
import pytest

import oracle as O
from tests import _meshes as M

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("variant", ["baseline", "optimized"])
@pytest.mark.parametrize("derivs", [False, True])
@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_fig2_chain_parity(elem, derivs, variant):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    L = 4
    fp, conn, coords = M.tiny(elem, n=9, L=L)
    conn = conn[:conn.shape[0] - 3]                 # ragged size
    U, s, kc = M.fields(fp, L)
    kc = kc[:conn.shape[0]]
    e = O.ELEM[elem]
    N = conn.shape[1]
    C = conn.shape[0]
    ctx = StokesFO(elem, torch.from_numpy(conn).cuda(), torch.from_numpy(coords).cuda(),
                   surface=torch.from_numpy(s).cuda(), flow_factor=torch.from_numpy(kc).cuda())
    S = ctx.albany_scratch(derivs)
    ctx.albany_setup(derivs, S)
    ctx.albany_evaluators(derivs, torch.from_numpy(U).cuda(), S)
    ctx.albany_resid(derivs, variant, S)
    Rc = torch.empty((C, N, 2), dtype=torch.float64, device="cuda")
    J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device="cuda") if derivs else None
    ctx.albany_extract(derivs, S, R_cell=Rc, J_cell=J)
    ctx.sync()
    G, wm, _ = O.geometry(e, conn, coords)
    ref = O.evaluate(e, conn, G, wm, U, surface=s, kc=kc, mode="jac" if derivs else "resid")

    def rel(a, b):
        a = a.reshape(C, -1)
        b = b.reshape(C, -1)
        return float((np.abs(a - b).max(1) / np.abs(b).max(1)).max())
    assert rel(Rc.cpu().numpy(), ref["R_cell"]) <= 1e-12
    if derivs:
        assert rel(J.cpu().numpy(), ref["J_cell"]) <= 1e-12
