"""Runs of every kernel variant for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck): hex8 + wedge6, stored + on-the-fly + compact geometry, residual
(partial-sum exchange), Jacobian (vector and tensor-core kernels, packed form), J.v, diagonal, fused CSR,
slot table + pull assembly (full and packed),
ragged tiles, side sets, the NEXT-1 chain and a short Newton solve.  A second,
larger mesh (more tiles than resident warps) exercises the persistent tile
loop: record ring refills, next-tile gathers and the partial-sum overlay of a
stage that is refilled right after."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from oracle import lateral as LT
from tests import _meshes as M
from paper_conf_sc_antepara0cw24_b200 import StokesFO


def run(elem, n, L, drop, full):
    fp, conn, coords = M.tiny(elem, n=n, L=L)
    conn = conn[:conn.shape[0] - drop]
    U, s, kc = M.fields(fp, L)
    kc = kc[:conn.shape[0]]
    C, N = conn.shape
    for geo in ("stored", "on_the_fly", "compact"):
        ctx = StokesFO(elem, torch.from_numpy(conn).cuda(), torch.from_numpy(coords).cuda(),
                       surface=torch.from_numpy(s).cuda(), flow_factor=torch.from_numpy(kc).cuda(), geometry=geo)
        Ud = torch.from_numpy(U).cuda()
        J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device="cuda")
        Rc = torch.empty((C, N, 2), dtype=torch.float64, device="cuda")
        R = torch.zeros((coords.shape[0], 2), dtype=torch.float64, device="cuda")
        Y = torch.zeros_like(R)
        mu = torch.empty((C, N), dtype=torch.float64, device="cuda")
        ctx.jacobian(Ud, J, R_cell=Rc, R=R)
        ctx.viscosity_resid(Ud, mu_qp=mu, R_cell=Rc, R=R)
        ctx.jvp(Ud, Ud, Y, R=R)
        ctx.jacobian_diag(Ud, Y, R=R)
        rp, ci = ctx.csr_pattern()
        ctx.csr_slots()
        vals = torch.zeros(ci.numel(), dtype=torch.float64, device="cuda")
        ctx.jacobian_csr(Ud, vals, R=R)
        ctx.scatter_assemble(R_cell=Rc, R=R, J_cell=J, csr_vals=vals)
        ctx.assemble_csr(J, vals, accumulate=False)
        if True:  # tensor-core kernels: packed element matrices + their pull assembly
            Jp = torch.empty((C, N * (N + 1) // 2, 2, 2), dtype=torch.float64, device="cuda")
            ctx.jacobian_packed(Ud, Jp, R_cell=Rc, R=R)
            ctx.assemble_csr_packed(Jp, vals, accumulate=True)
            Jm = torch.empty((C * 4 * N * N + 2,), dtype=torch.float64, device="cuda")[2:].view(C, 2 * N, 2 * N)
            ctx.jacobian(Ud, Jm, R=R)  # 16-B aligned only: the vector kernel
            if elem == "wedge6":  # the wedge6 DMMA kernel (opt-in)
                os.environ["STOKESFO_JAC_MMA"] = "1"
                c2 = StokesFO(elem, torch.from_numpy(conn).cuda(), torch.from_numpy(coords).cuda(),
                              surface=torch.from_numpy(s).cuda(), flow_factor=torch.from_numpy(kc).cuda(),
                              geometry=geo)
                del os.environ["STOKESFO_JAC_MMA"]
                c2.jacobian(Ud, J, R_cell=Rc, R=R)
                c2.sync()
        ctx.sync()
        if not full:
            continue
        ctx.gather(Ud)
        G, wm = ctx.geometry()
        cells = torch.arange(0, C, L, dtype=torch.int32, device="cuda")
        beta = torch.full((coords.shape[0],), 2.0, dtype=torch.float64, device="cuda")
        ctx.basal_friction(cells, beta, Ud, R, J_face=torch.empty((cells.numel(), N, N), dtype=torch.float64,
                                                                    device="cuda"))
        lf = LT.lateral_faces(fp.polys, L)
        faces = torch.from_numpy(np.ascontiguousarray(lf[lf[:, 0] < C])).cuda()  # faces of dropped cells: EMESH
        sd = torch.from_numpy(s).cuda()
        ctx.lateral_pressure(faces, sd, R)
        ctx.sync()
        if geo in ("stored", "compact"):
            ctx.set_lateral(faces, sd)
            Un = torch.ones_like(Ud)
            ctx.newton_solve(cells, beta, Un, max_newton=2, max_cg=20)
            for derivs in (False, True):
                S = ctx.albany_scratch(derivs)
                ctx.albany_setup(derivs, S)
                ctx.albany_evaluators(derivs, Ud, S)
                for v in ("baseline", "optimized"):
                    ctx.albany_resid(derivs, v, S)
                ctx.albany_extract(derivs, S, R_cell=Rc, J_cell=J if derivs else None)
            ctx.sync()


for elem in ("hex8", "wedge6"):
    run(elem, 5, 3, 3, True)          # every kernel, ragged last tile
    run(elem, 48, 8, 1, False)        # more tiles than resident warps: the persistent pipelines
print("sanitize workload done")
