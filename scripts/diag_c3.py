"""Dump the worst-parity C3 cells (GPU vs oracle) for offline analysis."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle as O
from paper_conf_sc_antepara0cw24_b200 import synth, StokesFO
fp, L, elem = synth.make_config("C3")
conn, coords = O.extrude(fp.xy, fp.polys, fp.b, fp.H, L)
U = synth.velocity_balance(fp, L, seed=11); s = synth.surface_nodal(fp, L); kc = synth.flow_factor(fp, L)
C = conn.shape[0]
ctx = StokesFO(elem, torch.from_numpy(conn).cuda(), torch.from_numpy(coords).cuda(),
               surface=torch.from_numpy(s).cuda(), flow_factor=torch.from_numpy(kc).cuda())
J = torch.empty((C, 16, 16), dtype=torch.float64, device="cuda")
mu = torch.empty((C, 8), dtype=torch.float64, device="cuda")
Ud = torch.from_numpy(U).cuda()
ctx.jacobian(Ud, J)
ctx.viscosity_resid(Ud, mu_qp=mu)
Gg, wmg = ctx.geometry()
ctx.sync()
rng = np.random.default_rng(2024)
cells = np.unique(np.concatenate([rng.integers(0, C, 20000), [0, C - 1], np.arange(C - 40, C)]))
G, wm, bad = O.geometry(0, conn[cells], coords)
ref = O.evaluate(0, conn[cells], G, wm, U, surface=s, kc=kc[cells], mode="jac")
tc = torch.from_numpy(cells).cuda()
Jg = J[tc].cpu().numpy(); mug = mu[tc].cpu().numpy(); Gg = Gg[tc].cpu().numpy(); wmg = wmg[tc].cpu().numpy()
sc = np.abs(ref["J_cell"]).reshape(len(cells), -1).max(1)
rel = np.abs(Jg - ref["J_cell"]).reshape(len(cells), -1).max(1) / sc
order = np.argsort(-rel)[:50]
print("worst rel", rel[order[:10]])
np.savez_compressed("gpurun_out/diag_c3.npz", cells=cells[order], rel=rel[order], Jg=Jg[order], Jo=ref["J_cell"][order],
                    mug=mug[order], muo=ref["mu_qp"][order], Gg=Gg[order], Go=G[order], wmg=wmg[order], wmo=wm[order])
