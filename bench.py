#!/usr/bin/env python
"""Benchmark: fused Stokes-FO residual + forward-AD Jacobian evaluation on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C4|C5|C1] [--impl ours|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...   (N > 1: NCCL halo exchange)

One step = one pass of the whole hot path over the
configuration's mesh: R <- 0; stokesfo_jacobian (gather -> Ugrad -> Glen mu ->
stress -> QP sum -> scatter-add R, plus the element Jacobians J_cell); at N > 1
the NCCL halo sum of shared-node residuals.  Inputs are resident in HBM
(C4: ~31 GB, far larger than the 126 MB L2, so no L2 flush is needed).
Prints ONE JSON line on rank 0 (the driver's bench contract, DESIGN.md
"Measurement").
"""
from __future__ import annotations

import argparse
import datetime
import json
import os
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "Stokes-FO Jacobian+residual cells/s and achieved HBM GB/s at 1/2/4/8 B200"
WORKLOADS = {
    "C4": "C4 Antarctica-like 4 km footprint x 10 layers, hex8, 8 QPs, residual+Jacobian (BASELINE.json configs[3])",
    "C5": "C5 Antarctica-like wedge6 (quads split), 10 layers, 6 QPs, residual+Jacobian (BASELINE.json configs[4])",
    "C1": "C1/C2 tiny 16x16 footprint x 5 layers, hex8, residual+Jacobian (BASELINE.json configs[1])",
    "C3": "C3 Greenland-like 1-10 km NVB footprint x 10 layers, hex8, residual+Jacobian (BASELINE.json configs[2])",
    "C4p": "C4p paper-shaped Antarctica-like 16 km x 20 layers, hex8 (~1.05M cells; the paper's ~256K/GPU at 4 GPUs)",
}


def jac_mma(elem: str, geometry: str, packed: bool = False) -> bool:
    """The element Jacobians run on the fp64 tensor cores (eval_mma_kernel / eval_compact_mma_kernel /
    eval_otf_mma_kernel, one per geometry mode); STOKESFO_JAC_MMA (read by stokesfo_create) unset: hex8 only, 1: both elements, 0:
    neither. The packed form (stokesfo_jacobian_packed) always comes from them unless STOKESFO_JAC_MMA=0."""
    v = os.environ.get("STOKESFO_JAC_MMA")
    if v == "0":
        return False
    return packed or v == "1" or elem == "hex8"


def kernel_name(elem: str, geometry: str, op: str, packed: bool = False) -> str:
    E = "Hex8" if elem == "hex8" else "Wedge6"
    if op in ("jacobian", "jac_global", "jac_packed") and (packed or jac_mma(elem, geometry)):
        k = {"compact": "eval_compact_mma_kernel<", "on_the_fly": "eval_otf_mma_kernel<"}.get(geometry,
                                                                                            "eval_mma_kernel<") + E + ">"
        if op == "jacobian":
            return k + " (stokesfo_jacobian)"
        if op == "jac_packed":
            return k + " (stokesfo_jacobian_packed)"
        if packed:
            return k + " (stokesfo_jacobian_packed) + csr_gather_kernel<packed> (stokesfo_assemble_csr_packed " \
                       "overwriting, both timed)"
        return k + " (stokesfo_jacobian) + csr_gather_kernel (stokesfo_assemble_csr overwriting, both timed)"
    k = {"on_the_fly": "eval_otf_kernel", "compact": "eval_compact_kernel", "stored": "eval_kernel"}[geometry]
    k += "<" + E + "," + {"jacobian": "M_JAC>", "resid": "M_RESID>", "jvp": "M_JVP>", "jvp_y": "M_JVP>",
                         "jac_csr": "M_CSR>", "jac_global": "M_JAC> + csr_gather_kernel"}[op]
    return k + {"jacobian": " (stokesfo_jacobian)", "resid": " (stokesfo_viscosity_resid)",
                "jvp": " (stokesfo_jvp)", "jvp_y": " (stokesfo_jvp, R = NULL)", "jac_csr": " (stokesfo_jacobian_csr)",
                "jac_global": " (stokesfo_jacobian + stokesfo_assemble_csr overwriting, both timed)"}[op]


def bytes_per_launch(elem: str, cells: int, nodes: int, geometry: str = "stored", op: str = "jacobian",
                     nnz: int = 0, packed: bool = False) -> int:
    """Algorithmic (compulsory) HBM bytes of one stokesfo_jacobian launch with
    assembled R.
    stored:     per cell conn 4N + GradBF 24NQ + wMeasure 8Q + k_c 8 + J_cell 8(2N)^2;
                per node U 16 + s 8 + R read+write 32.
    on_the_fly: per cell conn 4N + k_c 8 + J_cell 8(2N)^2;
                per node U 16 + s 8 + R 32 + coordinates 32 (x, y, z, pad)."""
    N = 8 if elem == "hex8" else 6
    Q = N
    J = 8 * (2 * N) ** 2 if op == "jacobian" else (8 * 4 * N * (N + 1) // 2 if op == "jac_packed" else 0)
    xy = (16 + 32) if op in ("jvp", "jvp_y") else 0  # X gather, Y read+write
    rb = 0 if op == "jvp_y" else 32                   # R read + write (jvp_y: the Krylov apply, no residual)
    if op == "jac_csr":
        # NEXT-2 fused CSR: no J_cell; per cell the slot row 8N, per node the
        # rowptr pair 16, and every CSR value read + written once (16 nnz)
        J = 8 * N
        xy = 16
    if op == "jac_global":
        # jacobian (J_cell written) + pull assembly overwriting the CSR values (DESIGN §6 NEXT-2): J_cell read
        # again, per cell the slot row 8N and incidence 4N, per node rowptr pair 16 + incidence pointer 8,
        # every CSR value written once (8 nnz)
        # packed: the N(N+1)/2 upper 2 x 2 node blocks (symmetric J) written and read instead of (2N)^2 entries
        J = 2 * 8 * (4 * N * (N + 1) // 2 if packed else (2 * N) ** 2) + 8 * N + 4 * N
        xy = 24
    vals = {"jac_csr": 16 * nnz, "jac_global": 8 * nnz}.get(op, 0)
    if geometry == "on_the_fly":
        return cells * (4 * N + 8 + J) + nodes * (16 + 8 + rb + 32 + xy) + vals
    if geometry == "compact":   # A_q = J_q^-T (9 doubles) + wM per QP instead of GradBF
        return cells * (4 * N + 72 * Q + 8 * Q + 8 + J) + nodes * (16 + 8 + rb + xy) + vals
    per_cell = 4 * N + 24 * N * Q + 8 * Q + 8 + J
    return cells * per_cell + nodes * (16 + 8 + rb + xy) + vals


MESH_SIZES = {"C4": (8431650, 9313304), "C5": (16863300, 9313304), "C3": (2033100, 2274459),
              "C4p": (1053660, 1124697), "C1": (1280, 1734)}


def units_per_launch(key: str) -> int:
    """Tiles of one evaluation launch for a traffic key 'CFG:elem:op:geometry'
    (hex8 4 cells per tile, wedge6 5): the unit of the per-tile ncu breakdowns."""
    cfg, elem = key.split(":")[:2]
    tc = 4 if elem == "hex8" else 5
    return (MESH_SIZES[cfg][0] + tc - 1) // tc


def lookup_traffic(config: str, elem: str, op: str, geometry: str, world: int):
    """(dram bytes per launch, source) from profiles/traffic.json when an ncu
    capture of THIS build's kernel exists (entries are keyed by workload and
    carry the source revision they were measured with), else (None, why)."""
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    key = f"{config}:{elem}:{op}:{geometry}"
    if world != 1 or os.environ.get("STOKESFO_LIB") or not os.path.exists(tpath):
        return None, "no ncu capture for this launch configuration"
    from paper_conf_sc_antepara0cw24_b200 import build as B
    with open(tpath) as f:
        tr = json.load(f)
    e = tr.get(key)
    if e is None or e.get("rev") != B.source_rev():
        return None, "no ncu capture of this build (profiles/traffic.json is keyed by source revision)"
    return e["dram_bytes_per_launch"], f"profiles/{e['tag']}_ncu_summary.md (ncu --set full, rev {e['rev']})"


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks / power / throttle reasons sampled every 20 ms; only the
    samples whose nvidia-smi timestamp falls inside the timed region (host wall
    clock, set by mark_start / mark_stop) are reported."""
    Q = ("timestamp,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.proc = None
        self.file = None
        self.t0 = self.t1 = None

    def start(self):
        try:
            self.file = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.idx}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "20"],
                                         stdout=self.file, stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def mark_start(self):
        self.t0 = time.time()

    def mark_stop(self):
        self.t1 = time.time()

    def stop(self):
        if self.proc is None:
            return None
        time.sleep(0.1)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.file.flush()
        self.file.seek(0)
        rows = [r.split(", ") for r in self.file.read().strip().splitlines() if r.strip()]
        os.unlink(self.file.name)
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        parsed = []
        for r in rows:
            try:
                ts = datetime.datetime.strptime(r[0].strip(), "%Y/%m/%d %H:%M:%S.%f").timestamp()
                rs = {n for n, v in zip(names, r[5:9]) if v.strip().lower().startswith("active")}
                parsed.append((ts, float(r[1]), float(r[2]), float(r[3]), rs))
            except Exception:
                continue
        if not parsed:
            return None
        win = [p for p in parsed if self.t0 is not None and self.t0 <= p[0] <= (self.t1 or p[0])]
        if not win:   # timed region shorter than the sampling period: the first sample after its start
            after = [p for p in parsed if self.t0 is not None and p[0] >= self.t0]
            win = after[:1] or parsed[-1:]
        sm = sorted(p[1] for p in win)
        pw = sorted(p[3] for p in win)
        return {"sm_mhz": sm[len(sm) // 2], "sm_min_mhz": sm[0], "sm_max_mhz": max(p[2] for p in parsed),
                "power_w": pw[len(pw) // 2], "reasons": sorted(set().union(*(p[4] for p in win))),
                "samples": len(win), "window": "nvidia-smi every 20 ms, samples inside the timed region"}


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def build_mesh(cfg: str, oracle_side: bool = False):
    """Seeded synthetic mesh + fields of a config.  The GPU arm extrudes with the
    product's C ABI (stokesfo_mesh_extrude); the oracle arm (--impl reference)
    with the oracle's own extrusion (bit-exact equal, tests/test_abi_mesh.py), so
    that arm loads nothing from the product."""
    from paper_conf_sc_antepara0cw24_b200 import synth
    fp, L, elem = synth.make_config(cfg)
    if oracle_side:
        import oracle as O
        conn, coords = O.extrude(fp.xy, fp.polys, fp.b, fp.H, L)
    else:
        from paper_conf_sc_antepara0cw24_b200 import mesh_extrude
        conn, coords = mesh_extrude(fp.xy, fp.polys, fp.b, fp.H, L)
    U = synth.velocity_balance(fp, L, seed=11 if cfg == "C3" else 12)
    s = synth.surface_nodal(fp, L)
    kc = synth.flow_factor(fp, L)
    return fp, L, elem, conn, coords, U, s, kc


# ---------------------------------------------------------------------------
# CPU oracle leg (cpu_baseline and --impl reference)
# ---------------------------------------------------------------------------

def host_cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or "unknown"


def oracle_sample_rate(elem, conn, coords, U, s, kc, target_s=12.0, start_cell=0, mode="jac"):
    """Time the oracle (as it stands) on a bounded contiguous sample of cells;
    geometry precomputed untimed (the GPU contract).  Returns (cells/s, cells, s)."""
    import numpy as np
    import oracle as O
    e = O.ELEM[elem]

    def run(n):
        cs = slice(start_cell, start_cell + n)
        G, wm, _ = O.geometry(e, conn[cs], coords)
        t0 = time.perf_counter()
        O.evaluate(e, conn[cs], G, wm, U, surface=s, kc=kc[cs], mode=mode)
        return time.perf_counter() - t0

    n = 4096
    dt = run(n)
    n2 = int(min(conn.shape[0] - start_cell, max(n, n * target_s / max(dt, 1e-6))))
    dt2 = run(n2)
    return n2 / dt2, n2, dt2


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle timed on this host's cores (rank 0 only)."""
    if rank != 0:
        return 0
    import oracle as O
    cfg = args.config
    fp, L, elem, conn, coords, U, s, kc = build_mesh(cfg, oracle_side=True)
    import numpy as np
    e = O.ELEM[elem]
    # calibrate a per-step sample so that warmup + steps end within a few minutes
    rate, _, _ = oracle_sample_rate(elem, conn, coords, U, s, kc, target_s=2.0)
    per_step_s = min(8.0, 120.0 / max(1, args.steps + args.warmup))
    n = int(max(1024, min(conn.shape[0], rate * per_step_s)))
    G, wm, _ = O.geometry(e, conn[:n], coords)
    for _ in range(args.warmup):
        O.evaluate(e, conn[:n], G, wm, U, surface=s, kc=kc[:n], mode="jac")
    t0 = time.perf_counter()
    for _ in range(args.steps):
        O.evaluate(e, conn[:n], G, wm, U, surface=s, kc=kc[:n], mode="jac")
    dt = (time.perf_counter() - t0) / args.steps
    value = n / dt
    sample = f"first {n} of {conn.shape[0]} cells per step (contiguous columns), geometry precomputed untimed"
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "cells/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": WORKLOADS[cfg], "cells": int(conn.shape[0]), "sampled_cells_per_step": n},
        "cpu_baseline": {"value": value, "unit": "cells/s", "cores": O.num_threads(), "kind": "oracle",
                         "sample": sample, "host_cpu": host_cpu_model()},
        "e2e": {"value": value, "unit": "cells/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "gpu_launches": 0,
    }
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------------------
# GPU leg
# ---------------------------------------------------------------------------

def relaunch(n: int) -> int:
    """`python bench.py --gpus N` without a torchrun environment: start N ranks
    (one process per GPU) with torch.distributed.run on 127.0.0.1 and return
    their exit status; rank 0 prints the JSON line."""
    import socket
    if os.environ.get("STOKESFO_BENCH_BACKEND", "nccl") == "nccl":
        import torch
        have = torch.cuda.device_count()
        if have < n:
            sys.stderr.write(f"bench.py: --gpus {n} needs {n} visible GPUs, found {have} "
                             "(STOKESFO_BENCH_BACKEND=gloo shares one GPU for debugging)\n")
            return 2
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="C4", choices=sorted(WORKLOADS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--geometry", default="stored", choices=["stored", "on_the_fly", "compact"])
    ap.add_argument("--global-format", default="full", choices=["packed", "full"],
                    help="--op jac_global: element matrices in symmetric block-packed form (tensor-core kernels) "
                         "or full [C][2N][2N]")
    ap.add_argument("--op", default="jacobian", choices=["jacobian", "jac_packed", "resid", "jvp", "jvp_y", "jac_csr",
                                                         "jac_global"],
                    help="jacobian: residual + element Jacobians (the headline); resid: stokesfo_viscosity_resid "
                         "only; jvp: matrix-free J(U) X + residual (stokesfo_jvp)")
    ap.add_argument("--halo", default="p2p", choices=["p2p", "nccl"],
                    help="N>1 halo sum: p2p = fused into the evaluation kernel over NVLink-mapped peer memory "
                         "(falls back to nccl if peer mapping fails); nccl = pack / grouped send-recv / unpack-add")
    ap.add_argument("--check", action="store_true",
                    help="N>1: compare every rank's halo-summed R with a one-GPU evaluation of the whole mesh")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--sustain", type=float, default=2.0,
                    help="seconds of back-to-back steps after the timed region (0 = off): the 'sustained' "
                         "sub-object, i.e. the throughput once the board's power controller has settled")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ and args.impl == "ours":
        return relaunch(args.gpus)
    rank, world, local = dist_env()
    if args.impl == "reference":
        return run_reference(args, rank, world)
    if world != args.gpus:
        sys.stderr.write(f"bench.py: --gpus {args.gpus} but WORLD_SIZE = {world}\n")
        return 2

    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_sc_antepara0cw24_b200 import StokesFO
    from paper_conf_sc_antepara0cw24_b200.halo import Halo, LocalPart, P2PHalo

    # STOKESFO_BENCH_BACKEND=gloo (debug only): ranks may share a GPU and the
    # halo buffers are staged through host memory; the timed product path is NCCL.
    backend = os.environ.get("STOKESFO_BENCH_BACKEND", "nccl")
    gpu = local % max(1, torch.cuda.device_count()) if backend == "gloo" else local
    torch.cuda.set_device(gpu)
    dev = torch.device("cuda", gpu)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")

    fp, L, elem, conn_g, coords_g, U_g, s_g, kc_g = build_mesh(args.config)
    part = LocalPart(conn_g, L, fp.nf, rank, world)
    gids = part.gids
    conn = torch.from_numpy(part.conn).to(dev)
    coords = torch.from_numpy(np.ascontiguousarray(coords_g[gids])).to(dev)
    surface = torch.from_numpy(np.ascontiguousarray(s_g[gids])).to(dev)
    kc = torch.from_numpy(np.ascontiguousarray(kc_g[part.cell_lo:part.cell_hi])).to(dev)
    U_host = torch.from_numpy(np.ascontiguousarray(U_g[gids])).pin_memory()
    U = U_host.to(dev)
    C, NN = conn.shape[0], coords.shape[0]
    N = conn.shape[1]
    stream = torch.cuda.current_stream(dev)
    ctx = StokesFO(elem, conn, coords, surface=surface, flow_factor=kc, stream=stream, geometry=args.geometry)
    if world > 1 and args.op in ("jac_csr", "jac_global", "jvp_y"):
        sys.stderr.write("bench.py: --op jac_csr / jac_global / jvp_y are single-GPU lines\n")
        return 2
    packed = (args.op == "jac_packed" or
              (args.op == "jac_global" and args.global_format == "packed")) and jac_mma(elem, args.geometry, True)
    if args.op == "jac_packed" and not packed:
        sys.stderr.write("bench.py: --op jac_packed needs the tensor-core kernels (STOKESFO_JAC_MMA not 0)\n")
        return 2
    J = torch.empty((C, N * (N + 1) // 2, 2, 2) if packed else
                    ((C, 2 * N, 2 * N) if args.op in ("jacobian", "jac_global") else (0,)), dtype=torch.float64,
                    device=dev)
    # J.v direction: one global seeded field, restricted to this rank's nodes (consistent across ranks)
    JV = args.op in ("jvp", "jvp_y")
    x_global = np.random.default_rng(5).normal(0, 10.0, (coords_g.shape[0], 2)) if JV else None
    Xd = torch.from_numpy(np.ascontiguousarray(x_global[gids])).to(dev) if JV else None
    Yd = torch.zeros((NN, 2), dtype=torch.float64, device=dev) if JV else None
    R = torch.zeros((NN, 2), dtype=torch.float64, device=dev)
    nnz, vals = 0, None
    if args.op in ("jac_csr", "jac_global"):   # NEXT-2: pattern + slot table once per mesh (untimed)
        _, colidx = ctx.csr_pattern()
        ctx.csr_slots()
        nnz = int(colidx.numel())
        vals = torch.zeros(nnz, dtype=torch.float64, device=dev)
    halo = None
    p2p = None
    halo_mode = "none"
    if world > 1:
        if args.halo == "p2p":
            p2p = P2PHalo(ctx, part, dev, gloo_debug=(backend != "nccl"), fields=2 if args.op == "jvp" else 1)
            if not p2p.ok:
                p2p.close()
                p2p = None
        if p2p is None:
            halo = Halo(part.neighbors, dev, pack=ctx.halo_pack, unpack_add=ctx.halo_unpack_add,
                        host_staging=(backend != "nccl"))
            halo_mode = "nccl pack/send-recv/unpack"
        else:
            halo_mode = "fused: peer-memory atomics in the evaluation kernel + 1 barrier"
    ctx.sync()
    torch.cuda.synchronize(dev)

    k0 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    k1 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    R_last = [R, Yd]

    def begin():
        """This step's (R, Y) output buffers, zeroed (Y only for --op jvp)."""
        if p2p is not None:
            out = p2p.begin()
            return out if args.op == "jvp" else (out, None)
        R.zero_()
        if Yd is not None:
            Yd.zero_()
        return R, Yd

    def finish(Rc, Yc):
        if p2p is not None:
            p2p.end()
        elif halo is not None:
            halo.exchange(Rc)
            if Yc is not None:
                halo.exchange(Yc)
        R_last[0], R_last[1] = Rc, Yc

    def evaluate(Uc, Rc, Yc):
        if args.op == "jacobian":
            ctx.jacobian(Uc, J, R=Rc)
        elif args.op == "jac_packed":   # symmetric block-packed element matrices (N(N+1)/2 upper node blocks)
            ctx.jacobian_packed(Uc, J, R=Rc)
        elif args.op == "jac_csr":
            ctx.jacobian_csr(Uc, vals, R=Rc)
        elif args.op == "jac_global" and packed:   # packed element matrices, then the pull assembly
            ctx.jacobian_packed(Uc, J, R=Rc)
            ctx.assemble_csr_packed(J, vals, accumulate=False)
        elif args.op == "jac_global":   # element matrices, then the atomic-free pull assembly overwriting CSR
            ctx.jacobian(Uc, J, R=Rc)
            ctx.assemble_csr(J, vals, accumulate=False)
        elif args.op == "jvp":
            ctx.jvp(Uc, Xd, Yc, R=Rc)
        elif args.op == "jvp_y":   # the Krylov operator apply: Y += J(U) X only
            ctx.jvp(Uc, Xd, Yc)
        else:
            ctx.viscosity_resid(Uc, R=Rc)

    def step(i=None):
        Rc, Yc = begin()
        if vals is not None and args.op == "jac_csr":   # jac_global overwrites every CSR value
            vals.zero_()
        if i is not None:
            k0[i].record(stream)
        evaluate(U, Rc, Yc)
        if i is not None:
            k1[i].record(stream)
        finish(Rc, Yc)

    for _ in range(args.warmup):
        step()
    ctx.sync()

    # live context for the peak: a plain device-to-device copy on this box right now
    live_copy = None
    if rank == 0:
        try:
            nb = 1 << 31
            src = torch.empty(nb // 8, dtype=torch.float64, device=dev)
            dst = torch.empty_like(src)
            for _ in range(2):
                dst.copy_(src)
            c0 = torch.cuda.Event(enable_timing=True)
            c1 = torch.cuda.Event(enable_timing=True)
            c0.record(stream)
            for _ in range(5):
                dst.copy_(src)
            c1.record(stream)
            torch.cuda.synchronize(dev)
            live_copy = 2 * nb * 5 / (c0.elapsed_time(c1) * 1e-3) / 1e9
            del src, dst
        except Exception:
            live_copy = None

    clocks = ClockSampler(local)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    clocks.start()
    time.sleep(0.3)
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    clocks.mark_start()
    t0.record(stream)
    for i in range(args.steps):
        step(i)
    t1.record(stream)
    torch.cuda.synchronize(dev)
    clocks.mark_stop()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    ms_total = t0.elapsed_time(t1)
    kern_ms = sum(a.elapsed_time(b) for a, b in zip(k0, k1)) / args.steps
    ctx.sync()

    # ---- sustained: back-to-back steps for --sustain seconds (power controller settled) ----
    sustained = None
    if args.sustain > 0:
        n_sus = max(1, int(args.sustain * 1e3 / max(ms_total / args.steps, 1e-3)) + 1)
        if world > 1:
            nt = torch.tensor([n_sus], dtype=torch.int64, device="cpu" if backend != "nccl" else dev)
            dist.all_reduce(nt, op=dist.ReduceOp.MAX)
            n_sus = int(nt.item())
        ks0 = [torch.cuda.Event(enable_timing=True) for _ in range(n_sus)]
        ks1 = [torch.cuda.Event(enable_timing=True) for _ in range(n_sus)]
        clk_s = ClockSampler(local)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)
        clk_s.start()
        time.sleep(0.3)
        s0 = torch.cuda.Event(enable_timing=True)
        s1 = torch.cuda.Event(enable_timing=True)
        clk_s.mark_start()
        s0.record(stream)
        for i in range(n_sus):
            Rc, Yc = begin()
            if vals is not None and args.op == "jac_csr":
                vals.zero_()
            ks0[i].record(stream)
            evaluate(U, Rc, Yc)
            ks1[i].record(stream)
            finish(Rc, Yc)
        s1.record(stream)
        torch.cuda.synchronize(dev)
        clk_s.mark_stop()
        if world > 1:
            dist.barrier()
        ck = clk_s.stop()
        kms = [a.elapsed_time(b) for a, b in zip(ks0, ks1)]
        q = max(1, n_sus // 4)
        sustained = {"seconds": s0.elapsed_time(s1) * 1e-3, "steps": n_sus,
                     "ms_per_step": s0.elapsed_time(s1) / n_sus, "kernel_ms": sum(kms) / n_sus,
                     "kernel_ms_last_quarter": sum(kms[-q:]) / q, "clocks": ck}

    # ---- end-to-end through the public API with host buffers ----
    # Every step uploads that step's U from pinned host memory and downloads its R;
    # the copies run on their own streams, double-buffered, so step t's compute
    # overlaps step t+1's upload and step t-1's download (J stays on the device).
    e2e = None
    if not args.no_e2e:
        s_h2d = torch.cuda.Stream(dev)
        s_d2h = torch.cuda.Stream(dev)
        Ub = [U, torch.empty_like(U)]
        Rb = [R, torch.zeros_like(R)]
        Yb = [Yd, None if Yd is None else torch.zeros_like(Yd)]
        R_host = [torch.empty((NN, 2), dtype=torch.float64).pin_memory() for _ in range(2)]
        ev_h2d = [torch.cuda.Event() for _ in range(2)]
        ev_comp = [torch.cuda.Event() for _ in range(2)]
        ev_d2h = [torch.cuda.Event() for _ in range(2)]

        def e2e_step(t):
            b = t % 2
            with torch.cuda.stream(s_h2d):
                if t >= 2:
                    s_h2d.wait_event(ev_comp[b])        # U[b] no longer read by step t-2
                Ub[b].copy_(U_host, non_blocking=True)
                ev_h2d[b].record(s_h2d)
            stream.wait_event(ev_h2d[b])
            if p2p is not None:
                if t >= 1:
                    stream.wait_event(ev_d2h[(t - 1) % 2])  # begin() clears the other buffer
                out = p2p.begin()
                Rc, Yc = out if args.op == "jvp" else (out, None)
            else:
                if t >= 2:
                    stream.wait_event(ev_d2h[b])        # R[b] of step t-2 has been downloaded
                Rc, Yc = Rb[b], Yb[b]
                Rc.zero_()
                if Yc is not None:
                    Yc.zero_()
            if vals is not None and args.op == "jac_csr":
                vals.zero_()
            evaluate(Ub[b], Rc, Yc)
            finish(Rc, Yc)
            ev_comp[b].record(stream)
            with torch.cuda.stream(s_d2h):
                s_d2h.wait_event(ev_comp[b])
                R_host[b].copy_(Rc, non_blocking=True)
                ev_d2h[b].record(s_d2h)

        for t in range(3):
            e2e_step(t)
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        s_h2d.wait_stream(stream)
        s_d2h.wait_stream(stream)
        for t in range(args.steps):
            e2e_step(t)
        stream.wait_stream(s_d2h)
        stream.wait_stream(s_h2d)
        e1.record(stream)
        torch.cuda.synchronize(dev)
        e2e_ms = e0.elapsed_time(e1) / args.steps
        e2e = [e2e_ms, U_host.numel() * 8, R_host[0].numel() * 8]

    # ---- optional correctness check of the N>1 halo sum ----
    check = None
    if args.check and world > 1:
        step()
        torch.cuda.synchronize(dev)
        mine = [R_last[0].cpu().numpy()] + ([R_last[1].cpu().numpy()] if args.op == "jvp" else [])
        full = StokesFO(elem, torch.from_numpy(conn_g).to(dev), torch.from_numpy(coords_g).to(dev),
                        surface=torch.from_numpy(s_g).to(dev), flow_factor=torch.from_numpy(kc_g).to(dev),
                        geometry=args.geometry)
        Rf = torch.zeros((coords_g.shape[0], 2), dtype=torch.float64, device=dev)
        if args.op == "jvp":
            Yf = torch.zeros_like(Rf)
            full.jvp(torch.from_numpy(U_g).to(dev), torch.from_numpy(x_global).to(dev), Yf, R=Rf)
            refs = [Rf, Yf]
        else:
            Jf = torch.empty((conn_g.shape[0], 2 * N, 2 * N), dtype=torch.float64, device=dev)
            full.jacobian(torch.from_numpy(U_g).to(dev), Jf, R=Rf)
            refs = [Rf]
        full.sync()
        e = 0.0
        for m, r in zip(mine, refs):
            rr = r.cpu().numpy()[gids]
            e = max(e, float(np.abs(m - rr).max() / max(np.abs(rr).max(), 1e-300)))
        err = torch.tensor([e], dtype=torch.float64, device="cpu" if backend != "nccl" else dev)
        dist.all_reduce(err, op=dist.ReduceOp.MAX)
        check = float(err.item())

    # ---- reduce over ranks (max time) ----
    mine_stats = [ms_total / args.steps, kern_ms, e2e[0] if e2e else 0.0, float(C),
                  sustained["ms_per_step"] if sustained else 0.0, sustained["kernel_ms"] if sustained else 0.0,
                  sustained["kernel_ms_last_quarter"] if sustained else 0.0]
    if world > 1:
        allst = [None] * world
        dist.all_gather_object(allst, mine_stats)
    else:
        allst = [mine_stats]
    ms_step = max(a[0] for a in allst)
    kern_ms_max = max(a[1] for a in allst)
    e2e_ms = max(a[2] for a in allst)
    total_cells = int(sum(a[3] for a in allst))

    if rank == 0:
        peak, peak_src = load_peaks()
        bpl = bytes_per_launch(elem, C, NN, args.geometry, args.op, nnz, packed)
        achieved = bpl / (kern_ms_max * 1e-3) / 1e9
        traffic, traffic_src = lookup_traffic(args.config, elem, args.op, args.geometry, world)
        l2_bytes = 126 * 2 ** 20
        line = {
            "metric": {"jacobian": METRIC,
                       "jac_packed": "Stokes-FO residual + Jacobian with symmetric block-packed element matrices "
                                     "(stokesfo_jacobian_packed) cells/s and achieved HBM GB/s",
                       "resid": "Stokes-FO residual-only (stokesfo_viscosity_resid) cells/s and achieved HBM GB/s",
                       "jvp": "Stokes-FO matrix-free J(U)X + residual (stokesfo_jvp) cells/s and achieved HBM GB/s",
                       "jvp_y": "Stokes-FO matrix-free J(U)X only (stokesfo_jvp, the Krylov operator apply) cells/s "
                                "and achieved HBM GB/s",
                       "jac_csr": "Stokes-FO residual + Jacobian assembled into global CSR (stokesfo_jacobian_csr) "
                                  "cells/s and achieved HBM GB/s",
                       "jac_global": "Stokes-FO residual + Jacobian assembled into global CSR (element matrices + "
                                     "pull assembly) cells/s and achieved HBM GB/s"}[args.op],
            "value": total_cells / (ms_step * 1e-3),
            "unit": "cells/s",
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": ms_step,
            "higher_is_better": True,
            "scaling": "strong",
            "vs_baseline": None,
            "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": WORKLOADS[args.config], "cells": total_cells, "elem": elem, "layers": L,
                       "geometry": args.geometry, "op": args.op,
                       "cells_rank0": C, "nodes_rank0": NN, "parallelism": f"column-partition x{world}",
                       "l2": "inputs exceed L2 (no flush needed)" if bpl > 4 * l2_bytes
                       else "inputs fit in L2 (not flushed; small-config line)",
                       "launch": ctx.launch_info()},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "traffic_source": traffic_src,
                         "kernel": kernel_name(elem, args.geometry, args.op, packed),
                         "kernel_ms": kern_ms_max, "algorithmic_bytes_per_launch": bpl, "peak_source": peak_src,
                         "live_copy_gbs": live_copy,
                         "note": "live_copy_gbs: torch device-to-device copy of 2 GiB on this box before the timed "
                                 "region (context for box-to-box variance; not the denominator)"},
            "achieved_hbm_gbs": achieved,
            "gpu_launches": args.steps * ((2 if args.op == "jac_global" else 1)
                                          + (halo.launches_per_exchange * (2 if args.op == "jvp" else 1)
                                             if halo else 0)),
            "halo": halo_mode,
            "clocks": clk,
        }
        if world > 1:
            line["per_rank"] = [{"rank": r, "cells": int(a[3]), "ms_per_step": a[0], "kernel_ms": a[1]}
                                for r, a in enumerate(allst)]
        if sustained:
            sms = max(a[4] for a in allst)
            skm = max(a[5] for a in allst)
            skq = max(a[6] for a in allst)
            sach = bpl / (skq * 1e-3) / 1e9
            line["sustained"] = {
                "value": total_cells / (sms * 1e-3), "unit": "cells/s", "seconds": sustained["seconds"],
                "steps": sustained["steps"], "ms_per_step": sms, "kernel_ms": skm, "kernel_ms_last_quarter": skq,
                "roofline_frac_last_quarter": sach / peak, "clocks": sustained["clocks"],
                "note": "back-to-back steps for --sustain seconds right after the timed region (the burst value "
                        "above is the first ~0.1 s, before the 1000 W power controller reacts); "
                        "roofline_frac_last_quarter = algorithmic bytes / mean kernel time of the last quarter / peak"}
        if check is not None:
            line["halo_check_max_rel_err"] = check
        if nnz:
            line["config"]["csr_nnz"] = nnz
        if e2e:
            line["e2e"] = {"value": total_cells / (e2e_ms * 1e-3), "unit": "cells/s",
                           "h2d_bytes_per_step": e2e[1], "d2h_bytes_per_step": e2e[2],
                           "note": "every step: pinned-host U H2D + evaluation + R D2H, copies on their own streams "
                                   "overlapping the neighbouring steps' compute; J_cell stays on device"}
        if world == 1 and not args.no_cpu_baseline:
            import oracle as O
            rate, n, dt = oracle_sample_rate(elem, conn_g, coords_g, U_g, s_g, kc_g, target_s=12.0,
                                             mode="resid" if args.op == "resid" else "jac")
            what = "residual" if args.op == "resid" else "residual+AD Jacobian"
            cores = O.num_threads()
            O.set_num_threads(1)
            rate1, n1, dt1 = oracle_sample_rate(elem, conn_g, coords_g, U_g, s_g, kc_g, target_s=3.0,
                                                mode="resid" if args.op == "resid" else "jac")
            O.set_num_threads(cores)
            line["cpu_baseline"] = {"value": rate, "unit": "cells/s", "cores": cores, "kind": "oracle",
                                    "sample": f"first {n} cells of {args.config} ({what}, "
                                              f"geometry precomputed untimed), {dt:.1f} s",
                                    "value_1_thread": rate1,
                                    "sample_1_thread": f"first {n1} cells, {dt1:.1f} s, OpenMP 1 thread",
                                    "host_cpu": host_cpu_model()}
        print(json.dumps(line), flush=True)
    if world > 1:
        if p2p is not None:
            torch.cuda.synchronize(dev)
            dist.barrier()
            p2p.close()
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
