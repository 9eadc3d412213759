"""Multi-process (gloo, CPU) test of the N>1 path: column partition, local
numbering, halo lists and the grouped send/recv halo sum.
Each rank evaluates its own cells with the oracle (CPU), exchanges shared-node
partial sums through paper_conf_sc_antepara0cw24_b200.halo.Halo over gloo,
and must end with the serial assembled residual on all its local nodes."""
import os
import socket

import numpy as np
import pytest


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, elem, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        import sys
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        sys.path.insert(0, root)
        import torch
        import torch.distributed as dist

        import oracle as O
        from paper_conf_sc_antepara0cw24_b200.halo import Halo, LocalPart
        from tests import _meshes as M
        dist.init_process_group("gloo", rank=rank, world_size=world)
        L = 3
        fp, conn, coords = M.tiny(elem, n=8, L=L)
        U, s, kc = M.fields(fp, L)
        e = O.ELEM[elem]
        part = LocalPart(conn, L, fp.nf, rank, world)
        lc = part.conn
        lx = coords[part.gids]
        G, wm, _ = O.geometry(e, lc, lx)
        Rc = O.evaluate(e, lc, G, wm, U[part.gids], surface=s[part.gids], kc=kc[part.cell_lo:part.cell_hi])["R_cell"]
        R = torch.from_numpy(O.scatter(e, lc, Rc, part.gids.size))
        halo = Halo(part.neighbors, "cpu")
        halo.exchange(R)
        # serial reference
        Gs, wms, _ = O.geometry(e, conn, coords)
        Rcs = O.evaluate(e, conn, Gs, wms, U, surface=s, kc=kc)["R_cell"]
        Rs = O.scatter(e, conn, Rcs, coords.shape[0])
        As = O.scatter(e, conn, np.abs(Rcs), coords.shape[0])
        err = np.abs(R.numpy() - Rs[part.gids])
        ok = bool((err <= 1e-12 * As[part.gids] + 1e-300).all())
        # valence probe through the same exchange: bit-exact integers
        ones = torch.from_numpy(O.scatter(e, lc, np.ones_like(Rc), part.gids.size))
        halo.exchange(ones)
        val = np.bincount(conn.reshape(-1), minlength=coords.shape[0]).astype(float)[part.gids]
        ok2 = bool(np.array_equal(ones.numpy()[:, 0], val))
        dist.barrier()
        dist.destroy_process_group()
        q.put((rank, ok, ok2, len(part.neighbors)))
    except Exception as ex:  # pragma: no cover
        import traceback
        q.put((rank, False, False, traceback.format_exc()))


@pytest.mark.parametrize("world,elem", [(2, "hex8"), (3, "hex8"), (2, "wedge6")])
def test_halo_sum_gloo(world, elem):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, elem, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, ok, ok2, info in res:
        assert ok and ok2, (rank, info)
        assert isinstance(info, int) and info >= 1
