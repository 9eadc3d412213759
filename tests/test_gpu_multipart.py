"""The N>1 path on one GPU: P column partitions (halo.LocalPart), one
StokesFO context per part, partial residuals assembled by each part's
jacobian kernel, then the halo exchange emulated with device copies between
the parts' pack/unpack buffers (stokesfo_halo_pack / _unpack_add kernels) in
the same pack-all-then-unpack order as halo.Halo over NCCL.  Every part must
end with the serial oracle residual on all of its local nodes (1e-12 of
sum|contributions|), and the valence probe must be bit-exact."""
import numpy as np
import pytest

import oracle as O
from tests import _meshes as M

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("elem,P", [("hex8", 2), ("hex8", 3), ("wedge6", 4)])
def test_partitioned_evaluation_with_halo_sum(elem, P):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    from paper_conf_sc_antepara0cw24_b200.halo import LocalPart
    L = 3
    fp, conn, coords = M.tiny(elem, n=12, L=L)
    U, s, kc = M.fields(fp, L)
    e = O.ELEM[elem]
    N = conn.shape[1]
    G, wm, _ = O.geometry(e, conn, coords)
    Rc = O.evaluate(e, conn, G, wm, U, surface=s, kc=kc)["R_cell"]
    Rser = O.scatter(e, conn, Rc, coords.shape[0])
    Aser = O.scatter(e, conn, np.abs(Rc), coords.shape[0])
    val = np.bincount(conn.reshape(-1), minlength=coords.shape[0]).astype(float)

    parts, ctxs, Rs, Vs = [], [], [], []
    for r in range(P):
        part = LocalPart(conn, L, fp.nf, r, P)
        g = part.gids
        ctx = StokesFO(elem, torch.from_numpy(part.conn).cuda(), torch.from_numpy(coords[g]).cuda(),
                       surface=torch.from_numpy(s[g]).cuda(),
                       flow_factor=torch.from_numpy(kc[part.cell_lo:part.cell_hi]).cuda())
        C = part.conn.shape[0]
        J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device="cuda")
        R = torch.zeros((g.size, 2), dtype=torch.float64, device="cuda")
        ctx.jacobian(torch.from_numpy(U[g]).cuda(), J, R=R)
        V = torch.zeros((g.size, 2), dtype=torch.float64, device="cuda")
        ctx.scatter_assemble(R_cell=torch.ones((C, N, 2), dtype=torch.float64, device="cuda"), R=V)
        parts.append(part)
        ctxs.append(ctx)
        Rs.append(R)
        Vs.append(V)
    for X in (Rs, Vs):
        bufs = {}
        for r, part in enumerate(parts):          # pack everything first
            for nb, idx in part.neighbors.items():
                ti = torch.from_numpy(idx).cuda()
                b = torch.empty((idx.size, 2), dtype=torch.float64, device="cuda")
                ctxs[r].halo_pack(X[r], ti, b)
                bufs[(r, nb)] = b
        for r, part in enumerate(parts):          # then unpack-add what the neighbours sent
            for nb, idx in part.neighbors.items():
                ctxs[r].halo_unpack_add(bufs[(nb, r)], torch.from_numpy(idx).cuda(), X[r])
    for r, part in enumerate(parts):
        ctxs[r].sync()
        g = part.gids
        err = np.abs(Rs[r].cpu().numpy() - Rser[g])
        assert (err <= 1e-12 * Aser[g]).all(), (r, float((err / Aser[g]).max()))
        v = Vs[r].cpu().numpy()
        assert np.array_equal(v[:, 0], val[g]) and np.array_equal(v[:, 1], val[g])
    assert sum(len(p.neighbors) for p in parts) >= 2


@pytest.mark.parametrize("elem,P", [("hex8", 3), ("wedge6", 4)])
def test_fused_peer_halo_single_process(elem, P):
    """The fused halo (stokesfo_set_remote): each part's evaluation kernel adds
    boundary-node contributions straight into the other parts' R through
    device pointers.  Here the 'peers' are the other parts' buffers on the same
    GPU (the kernel path is identical to NVLink-mapped peers); every part must
    hold the serial residual afterwards, with no pack/exchange/unpack."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    from paper_conf_sc_antepara0cw24_b200.halo import LocalPart
    L = 3
    fp, conn, coords = M.tiny(elem, n=12, L=L)
    U, s, kc = M.fields(fp, L)
    e = O.ELEM[elem]
    N = conn.shape[1]
    G, wm, _ = O.geometry(e, conn, coords)
    Rc = O.evaluate(e, conn, G, wm, U, surface=s, kc=kc)["R_cell"]
    Rser = O.scatter(e, conn, Rc, coords.shape[0])
    Aser = O.scatter(e, conn, np.abs(Rc), coords.shape[0])
    parts = [LocalPart(conn, L, fp.nf, r, P) for r in range(P)]
    Rs = [torch.zeros((p.gids.size, 2), dtype=torch.float64, device="cuda") for p in parts]
    peers = torch.tensor([R.data_ptr() for R in Rs], dtype=torch.int64, device="cuda")
    keep = []
    for r, part in enumerate(parts):
        g = part.gids
        ctx = StokesFO(elem, torch.from_numpy(part.conn).cuda(), torch.from_numpy(coords[g]).cuda(),
                       surface=torch.from_numpy(s[g]).cuda(),
                       flow_factor=torch.from_numpy(kc[part.cell_lo:part.cell_hi]).cuda())
        rem, remtab = part.remote_table()
        ctx.set_remote(torch.from_numpy(rem).cuda(), torch.from_numpy(remtab).cuda(), peers)
        C = part.conn.shape[0]
        J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device="cuda")
        ctx.jacobian(torch.from_numpy(U[g]).cuda(), J, R=Rs[r])
        keep.append(ctx)
    torch.cuda.synchronize()
    for r, part in enumerate(parts):
        keep[r].sync()
        g = part.gids
        err = np.abs(Rs[r].cpu().numpy() - Rser[g])
        assert (err <= 1e-12 * Aser[g]).all(), (r, float((err / Aser[g]).max()))
