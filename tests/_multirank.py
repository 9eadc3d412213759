"""Multi-rank parity of the partitioned evaluation and its halo sum (SURVEY 8(e)
and §4 'Multi-GPU parity'; one rank per GPU).  Launched by
tests/test_gpu_multigpu.py under torch.distributed.run; not a test module.

Every rank evaluates its column partition (contiguous Hilbert column ranges,
halo.LocalPart) through the C ABI and sums shared-node contributions with the
fused peer-memory halo (p2p: red.global.add.f64 into the peers' buffers) or
the pack / NCCL send-recv / unpack-add schedule (nccl).  Each rank then checks
its own nodes against the CPU ORACLE (not against another GPU run):

  R (jacobian and jvp passes)  |dR| <= 1e-12 x the rounding scale of the summed terms, per entry
  Y = J(U) X (jvp, halo-summed) |dY| <= 1e-12 sum_c max|J_c| |X_c|  per entry
  valence probe                scatter of all-ones R_cell == node valence, bit-exact

The oracle runs only over the cells touching this rank's nodes, so every
shared node gets its complete serial sum.  With fewer GPUs than ranks the
ranks share GPU 0 over gloo (CUDA IPC between processes still maps the peers'
buffers; the nccl schedule stages its buffers through host memory).
Rank 0 prints one JSON line: {"world", "backend", "results": [...]}.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

TOL = 1e-12


def meshes(name):
    import oracle as O
    from paper_conf_sc_antepara0cw24_b200 import synth
    if name == "C1":
        fp, L, elem = synth.tiny_footprint(), 5, "hex8"
    elif name == "C1w":
        fp, L, elem = synth.split_to_triangles(synth.tiny_footprint()), 5, "wedge6"
    elif name == "C4p":
        fp, L, elem = synth.antarctica_footprint(h=16.0, name="C4p"), 20, "hex8"
    elif name == "C5p":
        fp, L, elem = synth.split_to_triangles(synth.antarctica_footprint(h=16.0), name="C5p"), 20, "wedge6"
    else:
        raise KeyError(name)
    conn, coords = O.extrude(fp.xy, fp.polys, fp.b, fp.H, L)   # the oracle's extrusion
    U = synth.velocity_balance(fp, L, seed=12)
    s = synth.surface_nodal(fp, L)
    kc = synth.flow_factor(fp, L)
    return fp, L, elem, conn, coords, U, s, kc


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C1,C1w,C4p")
    ap.add_argument("--halos", default="p2p,nccl")
    ap.add_argument("--geometry", default="stored")
    args = ap.parse_args()
    import numpy as np
    import torch
    import torch.distributed as dist

    import oracle as O
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    from paper_conf_sc_antepara0cw24_b200.halo import Halo, LocalPart, P2PHalo
    from tests._meshes import rounding_scale_R

    rank = int(os.environ["RANK"])
    world = int(os.environ["WORLD_SIZE"])
    local = int(os.environ.get("LOCAL_RANK", rank))
    ngpu = torch.cuda.device_count()
    backend = "nccl" if ngpu >= world else "gloo"
    gpu = local if backend == "nccl" else 0
    torch.cuda.set_device(gpu)
    dev = torch.device("cuda", gpu)
    if backend == "nccl":
        dist.init_process_group("nccl", device_id=dev)
    else:
        dist.init_process_group("gloo")

    results = []
    for cfg in args.configs.split(","):
        fp, L, elem, conn_g, coords_g, U_g, s_g, kc_g = meshes(cfg)
        e = O.ELEM[elem]
        part = LocalPart(conn_g, L, fp.nf, rank, world)
        gids = part.gids
        NN = gids.size
        # oracle over the cells touching this rank's nodes: complete sums on every local node
        touch = np.isin(conn_g, gids).any(axis=1)
        csub = np.ascontiguousarray(conn_g[touch])
        G, wm, bad = O.geometry(e, csub, coords_g)
        assert bad == 0
        ref = O.evaluate(e, csub, G, wm, U_g, surface=s_g, kc=kc_g[touch], mode="jac")
        nn_g = coords_g.shape[0]
        R_ref = O.scatter(e, csub, ref["R_cell"], nn_g)[gids]
        # per-entry scale: the rounding scale of the summed terms (tests/_meshes.py
        # rounding_scale_R); C4p's 1 m x 16 km cells cancel by up to 1e6 inside Ugrad
        R_sc = O.scatter(e, csub, rounding_scale_R(e, csub, G, wm, ref["mu_qp"], U_g, s_g, 8.927), nn_g)[gids]
        X_g = np.random.default_rng(5).normal(0, 10.0, (nn_g, 2))
        C, N = csub.shape
        Xc = X_g[csub].reshape(C, 2 * N)
        JX = np.einsum("ckl,cl->ck", ref["J_cell"], Xc).reshape(C, N, 2)
        jsc = (np.abs(ref["J_cell"]).reshape(C, -1).max(1) * np.abs(Xc).sum(1))[:, None, None] * np.ones((C, N, 2))
        Y_ref = O.scatter(e, csub, JX, nn_g)[gids]
        Y_sc = O.scatter(e, csub, jsc, nn_g)[gids]
        valence = np.bincount(conn_g.reshape(-1), minlength=nn_g)[gids].astype(np.float64)

        def T(a):
            return torch.from_numpy(np.ascontiguousarray(a)).to(dev)

        conn = T(part.conn)
        ctx = StokesFO(elem, conn, T(coords_g[gids]), surface=T(s_g[gids]),
                       flow_factor=T(kc_g[part.cell_lo:part.cell_hi]), geometry=args.geometry)
        U, X = T(U_g[gids]), T(X_g[gids])
        Cl = part.conn.shape[0]
        J = torch.empty((Cl, 2 * N, 2 * N), dtype=torch.float64, device=dev)
        ones = torch.ones((Cl, N, 2), dtype=torch.float64, device=dev)
        for halo_kind in args.halos.split(","):
            out = {"config": cfg, "elem": elem, "halo": halo_kind, "rank_cells": int(Cl), "rank_nodes": int(NN),
                   "neighbors": sorted(int(r) for r in part.neighbors)}
            if halo_kind == "p2p":
                h = P2PHalo(ctx, part, dev, gloo_debug=(backend != "nccl"), fields=2)
                assert h.ok, "peer mapping failed"

                def run(fn):
                    Rb, Yb = h.begin()
                    fn(Rb, Yb)
                    return h.end()
            else:
                h = Halo(part.neighbors, dev, pack=ctx.halo_pack, unpack_add=ctx.halo_unpack_add,
                         host_staging=(backend != "nccl"))
                Rb = torch.zeros((NN, 2), dtype=torch.float64, device=dev)
                Yb = torch.zeros_like(Rb)

                def run(fn):
                    Rb.zero_()
                    Yb.zero_()
                    fn(Rb, Yb)
                    h.exchange(Rb)
                    h.exchange(Yb)
                    return Rb, Yb
            # residual + Jacobian pass
            R1, _ = run(lambda Rb, Yb: ctx.jacobian(U, J, R=Rb))
            torch.cuda.synchronize(dev)
            R1 = R1.cpu().numpy()
            # matrix-free J.v pass (Y halo-summed too)
            R2, Y2 = run(lambda Rb, Yb: ctx.jvp(U, X, Yb, R=Rb))
            torch.cuda.synchronize(dev)
            R2, Y2 = R2.cpu().numpy(), Y2.cpu().numpy()
            # valence probe through the same halo
            V, _ = run(lambda Rb, Yb: ctx.scatter_assemble(R_cell=ones, R=Rb))
            torch.cuda.synchronize(dev)
            V = V.cpu().numpy()
            ctx.sync()
            if halo_kind == "p2p":
                h.close()
            out["R_jac_err_over_scale"] = float((np.abs(R1 - R_ref) / np.maximum(R_sc, 1e-300)).max())
            out["R_jvp_err_over_scale"] = float((np.abs(R2 - R_ref) / np.maximum(R_sc, 1e-300)).max())
            out["Y_err_over_scale"] = float((np.abs(Y2 - Y_ref) / np.maximum(Y_sc, 1e-300)).max())
            out["valence_bit_exact"] = bool(np.array_equal(V[:, 0], valence) and np.array_equal(V[:, 1], valence))
            out["ok"] = (out["R_jac_err_over_scale"] <= TOL and out["R_jvp_err_over_scale"] <= TOL
                         and out["Y_err_over_scale"] <= TOL and out["valence_bit_exact"])
            allr = [None] * world
            dist.all_gather_object(allr, out)
            if rank == 0:
                results.append({"config": cfg, "halo": halo_kind, "ok": all(r["ok"] for r in allr), "ranks": allr})
        ctx.destroy()
    if rank == 0:
        print(json.dumps({"world": world, "backend": backend, "gpus": ngpu, "results": results}), flush=True)
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
