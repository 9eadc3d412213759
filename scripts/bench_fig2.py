#!/usr/bin/env python
"""NEXT-1: the paper's baseline-vs-optimized experiment (Table III / IV,
PAPER.md P:L266-319) re-run on B200 with the Albany-structured evaluator chain
(stokesfo_albany_*), next to the fused B200 kernels on the same mesh.

    python scripts/bench_fig2.py [--config C4p] [--reps 20] [--out gpurun_out/fig2.json] [--ncu]

Times per call (CUDA events, median over reps after warm-up) of StokesFOResid
(Fig. 2 baseline / optimized) for the Residual (double) and the Jacobian
(SFad lanes), of the whole chain, and of stokesfo_viscosity_resid /
stokesfo_jacobian.  Theoretical minimum bytes of StokesFOResid follow the
paper's definition (sizes of the arrays it reads and writes).
With --ncu each kernel runs once (for an ncu --metrics dram__bytes pass).
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4p")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "fig2.json"))
    ap.add_argument("--ncu", action="store_true")
    a = ap.parse_args()
    import torch
    from paper_conf_sc_antepara0cw24_b200 import StokesFO, mesh_extrude, synth
    fp, L, elem = synth.make_config(a.config)
    conn, coords = mesh_extrude(fp.xy, fp.polys, fp.b, fp.H, L)
    U = synth.velocity_balance(fp, L, seed=12)
    s = synth.surface_nodal(fp, L)
    kc = synth.flow_factor(fp, L)
    C, N = conn.shape
    Q = N
    dev = torch.device("cuda", 0)
    ctx = StokesFO(elem, torch.from_numpy(conn).to(dev), torch.from_numpy(coords).to(dev),
                   surface=torch.from_numpy(s).to(dev), flow_factor=torch.from_numpy(kc).to(dev))
    Ud = torch.from_numpy(U).to(dev)
    stream = torch.cuda.current_stream(dev)
    reps = 1 if a.ncu else a.reps
    warm = 0 if a.ncu else 3

    def timeit(fn):
        for _ in range(warm):
            fn()
        ts = []
        for _ in range(reps):
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fn()
            e1.record(stream)
            torch.cuda.synchronize(dev)
            ts.append(e0.elapsed_time(e1))
        ts.sort()
        return ts[len(ts) // 2] * 1e-3

    res = {"config": a.config, "cells": C, "nodes": int(coords.shape[0]), "elem": elem, "reps": reps}
    for derivs in (False, True):
        K = (2 * N + 1) if derivs else 1
        # paper's theoretical minimum for StokesFOResid: mu, Ugrad, force (ScalarT, K comps),
        # wGradBF, wBF (MeshScalarT), Residual (ScalarT, written once)
        min_bytes = 8 * C * ((Q + 6 * Q + 2 * Q + 2 * N) * K + 3 * N * Q + N * Q)
        S = ctx.albany_scratch(derivs)
        ctx.albany_setup(derivs, S)
        ctx.albany_evaluators(derivs, Ud, S)
        key = "jacobian" if derivs else "residual"
        r = {"min_bytes_stokesfo_resid": min_bytes}
        for variant in ("baseline", "optimized"):
            r[f"stokesfo_resid_{variant}_s"] = timeit(lambda: ctx.albany_resid(derivs, variant, S))
        r["evaluators_s"] = timeit(lambda: ctx.albany_evaluators(derivs, Ud, S))
        del S
        torch.cuda.empty_cache()
        if derivs:
            J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device=dev)
            R = torch.zeros((coords.shape[0], 2), dtype=torch.float64, device=dev)
            r["fused_s"] = timeit(lambda: ctx.jacobian(Ud, J, R=R))
            del J
        else:
            R = torch.zeros((coords.shape[0], 2), dtype=torch.float64, device=dev)
            r["fused_s"] = timeit(lambda: ctx.viscosity_resid(Ud, R=R))
        res[key] = r
    ctx.sync()
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    if not a.ncu:
        with open(a.out, "w") as f:
            json.dump(res, f, indent=1)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
