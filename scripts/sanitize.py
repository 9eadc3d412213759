"""Small runs of every eval kernel variant for compute-sanitizer (memcheck /
racecheck / synccheck / initcheck): hex8 + wedge6, stored + on-the-fly,
residual + Jacobian, ragged tiles, plus the NEXT-1 chain and assembly kernels."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle as O
from tests import _meshes as M
from paper_conf_sc_antepara0cw24_b200 import StokesFO

for elem in ("hex8", "wedge6"):
    fp, conn, coords = M.tiny(elem, n=5, L=3)
    conn = conn[:conn.shape[0] - 3]
    U, s, kc = M.fields(fp, 3)
    kc = kc[:conn.shape[0]]
    C, N = conn.shape
    for geo in ("stored", "on_the_fly"):
        ctx = StokesFO(elem, torch.from_numpy(conn).cuda(), torch.from_numpy(coords).cuda(),
                       surface=torch.from_numpy(s).cuda(), flow_factor=torch.from_numpy(kc).cuda(), geometry=geo)
        Ud = torch.from_numpy(U).cuda()
        J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device="cuda")
        Rc = torch.empty((C, N, 2), dtype=torch.float64, device="cuda")
        R = torch.zeros((coords.shape[0], 2), dtype=torch.float64, device="cuda")
        mu = torch.empty((C, N), dtype=torch.float64, device="cuda")
        ctx.jacobian(Ud, J, R_cell=Rc, R=R)
        ctx.viscosity_resid(Ud, mu_qp=mu, R_cell=Rc, R=R)
        ctx.gather(Ud)
        G, wm = ctx.geometry()
        rp, ci = ctx.csr_pattern()
        vals = torch.zeros(ci.numel(), dtype=torch.float64, device="cuda")
        ctx.scatter_assemble(R_cell=Rc, R=R, J_cell=J, csr_vals=vals)
        ctx.sync()
    for derivs in (False, True):
        S = ctx.albany_scratch(derivs)
        ctx.albany_setup(derivs, S)
        ctx.albany_evaluators(derivs, Ud, S)
        for v in ("baseline", "optimized"):
            ctx.albany_resid(derivs, v, S)
        ctx.albany_extract(derivs, S, R_cell=Rc, J_cell=J if derivs else None)
    ctx.sync()
print("sanitize workload done")
