"""Measurement of the auxiliary (NEXT-row) kernels on a full-size config, one
JSON line per op: NEXT-2 assembly (stokesfo_scatter_assemble: R and CSR
values), NEXT-4 side sets (stokesfo_basal_friction over every bed face,
stokesfo_lateral_pressure over every lateral face), NEXT-3 jvp for context.

Times each op with CUDA events on the launching stream (warm-up first), and
reports algorithmic bytes per launch / time against the HBM peak:
  scatter R      per cell conn 4N + R_cell 16N;  per node R read+write 32
  scatter CSR    per cell conn 4N + J_cell 8 (2N)^2; per dof row rowptr 8;
                 colidx 4 nnz (binary searches) + vals read+write 16 nnz
  basal          per face cell id 4 + conn 4 NB (+ J_face 8 (2NB)^2);
                 per bed node beta 8 + U 16 + coords 24 + R 32
  lateral        per face (cell, side) 8 + conn 16;
                 per lateral node s 8 + coords 24 + R 32
(unique nodes counted once: the node arrays are L2-resident between faces).

    python scripts/bench_aux.py --config C3 [--ops scatter_r,csr,basal,lateral]
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def timed(fn, stream, iters=10, warmup=3, pre=None):
    import torch
    for _ in range(warmup):
        if pre:
            pre()
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(iters):
        if pre:
            pre()
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        fn()
        b.record(stream)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--ops", default="scatter_r,csr,basal,lateral")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    import numpy as np
    import torch
    from paper_conf_sc_antepara0cw24_b200 import StokesFO, mesh_lateral_faces

    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    fp, L, elem, conn_np, coords_np, U_np, s_np, kc_np = bench.build_mesh(args.config)
    peak, peak_src = bench.load_peaks()
    conn = torch.from_numpy(conn_np).to(dev)
    coords = torch.from_numpy(coords_np).to(dev)
    s = torch.from_numpy(s_np).to(dev)
    U = torch.from_numpy(U_np).to(dev)
    kc = torch.from_numpy(kc_np).to(dev)
    C, NN, N = conn.shape[0], coords.shape[0], conn.shape[1]
    NB = N // 2
    stream = torch.cuda.current_stream(dev)
    ctx = StokesFO(elem, conn, coords, surface=s, flow_factor=kc, stream=stream)
    R = torch.zeros((NN, 2), dtype=torch.float64, device=dev)
    ops = args.ops.split(",")
    lines = []

    def emit(op, ms, nbytes, units, unit_name, extra=None):
        gbs = nbytes / (ms * 1e-3) / 1e9
        line = {"op": op, "config": args.config, "elem": elem, unit_name: units, "ms": ms,
                f"{unit_name}_per_s": units / (ms * 1e-3), "algorithmic_bytes": nbytes, "achieved_gbs": gbs,
                "peak_gbs": peak, "peak_source": peak_src, "frac": gbs / peak}
        if extra:
            line.update(extra)
        print(json.dumps(line), flush=True)
        lines.append(line)

    if "scatter_r" in ops or "csr" in ops:
        Rc = torch.empty((C, N, 2), dtype=torch.float64, device=dev)
        J = torch.empty((C, 2 * N, 2 * N), dtype=torch.float64, device=dev)
        ctx.jacobian(U, J, R_cell=Rc)
        ctx.sync()
        if "scatter_r" in ops:
            ms = timed(lambda: ctx.scatter_assemble(R_cell=Rc, R=R), stream, pre=R.zero_)
            emit("scatter_assemble:R", ms, C * (4 * N + 16 * N) + NN * 32, C, "cells")
        if "csr" in ops:
            t0 = time.perf_counter()
            rowptr, colidx = ctx.csr_pattern()
            t_pat = time.perf_counter() - t0
            nnz = int(colidx.numel())
            vals = torch.zeros(nnz, dtype=torch.float64, device=dev)
            ms = timed(lambda: ctx.scatter_assemble(J_cell=J, csr_vals=vals), stream, pre=vals.zero_)
            ctx.sync()
            nb = C * (4 * N + 8 * (2 * N) ** 2) + 2 * NN * 8 + nnz * (4 + 16)
            emit("scatter_assemble:CSR", ms, nb, C, "cells",
                 {"nnz": nnz, "atomics_per_s": C * (2 * N) ** 2 / (ms * 1e-3),
                  "pattern_host_s": t_pat})
            t0 = time.perf_counter()
            ctx.csr_slots()
            ctx.sync()
            t_slots = time.perf_counter() - t0
            ms = timed(lambda: ctx.scatter_assemble(J_cell=J, csr_vals=vals), stream, pre=vals.zero_)
            ctx.sync()
            nb = C * (4 * N + 8 * (2 * N) ** 2 + 8 * N) + 2 * NN * 8 + nnz * 16
            emit("scatter_assemble:CSR(slots, atomics)" if os.environ.get("STOKESFO_CSR_ATOMIC") == "1"
                 else "scatter_assemble:CSR(slots, pull: warp per node, no atomics)", ms, nb, C, "cells",
                 {"nnz": nnz, "atomics_per_s": C * (2 * N) ** 2 / (ms * 1e-3), "slots_setup_s": t_slots})
            del vals, rowptr, colidx
            ctx.rowptr = ctx.colidx = ctx.slots = None
        del J, Rc
        torch.cuda.empty_cache()
    if "basal" in ops:
        cells = torch.arange(0, C, L, dtype=torch.int32, device=dev)   # k = 0: one bed face per column
        beta = torch.from_numpy(np.random.default_rng(8).uniform(0.1, 3.0, NN)).to(dev)
        nf = int(cells.numel())
        bed_nodes = fp.nv
        ms = timed(lambda: ctx.basal_friction(cells, beta, U, R), stream)
        emit("basal_friction", ms, nf * (4 + 4 * NB) + bed_nodes * 80, nf, "faces")
        Jf = torch.empty((nf, 2 * NB, 2 * NB), dtype=torch.float64, device=dev)
        ms = timed(lambda: ctx.basal_friction(cells, beta, U, R, J_face=Jf), stream)
        emit("basal_friction+J_face", ms, nf * (4 + 4 * NB + 8 * (2 * NB) ** 2) + bed_nodes * 80, nf, "faces")
        del Jf
    if "lateral" in ops:
        faces_np = mesh_lateral_faces(fp.polys, L)
        faces = torch.from_numpy(faces_np).to(dev)
        nf = int(faces.shape[0])
        lat_nodes = len(np.unique(conn_np[faces_np[:, 0]][:, :]))  # upper bound proxy: nodes of lateral cells
        ms = timed(lambda: ctx.lateral_pressure(faces, s, R, sea_level=0.0), stream)
        nside = nf // L
        emit("lateral_pressure", ms, nf * (8 + 16) + 2 * nside * (L + 1) * 64, nf, "faces",
             {"lateral_cells_nodes_upper_bound": int(lat_nodes)})
    ctx.sync()
    if args.out:
        with open(args.out, "w") as f:
            for ln in lines:
                f.write(json.dumps(ln) + "\n")


if __name__ == "__main__":
    main()
