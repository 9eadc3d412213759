#!/usr/bin/env python
"""Per-launch kernel time vs SM clock / power over a long run of back-to-back
evaluations (is the bench's kernel time set by the power cap?).

    python scripts/diag_power.py [--config C4] [--op jacobian] [--launches 200]
"""
import argparse
import json
import os
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--op", default="jacobian", choices=["jacobian", "resid"])
    ap.add_argument("--launches", type=int, default=200)
    ap.add_argument("--gap-ms", type=float, default=0.0, help="host sleep between launches (cool-down probe)")
    args = ap.parse_args()
    import numpy as np
    import torch
    import bench
    from paper_conf_sc_antepara0cw24_b200 import StokesFO

    fp, L, elem, conn_g, coords_g, U_g, s_g, kc_g = bench.build_mesh(args.config)
    dev = torch.device("cuda", 0)
    conn = torch.from_numpy(conn_g).to(dev)
    ctx = StokesFO(elem, conn, torch.from_numpy(coords_g).to(dev), surface=torch.from_numpy(s_g).to(dev),
                   flow_factor=torch.from_numpy(kc_g).to(dev))
    C, N = conn.shape
    U = torch.from_numpy(U_g).to(dev)
    J = torch.empty((C, 2 * N, 2 * N) if args.op == "jacobian" else (0,), dtype=torch.float64, device=dev)
    R = torch.zeros_like(U)
    stream = torch.cuda.current_stream(dev)
    for _ in range(3):
        ctx.jacobian(U, J, R=R) if args.op == "jacobian" else ctx.viscosity_resid(U, R=R)
    torch.cuda.synchronize()
    f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
    p = subprocess.Popen(["nvidia-smi", "--id=0", "--query-gpu=timestamp,clocks.sm,power.draw,temperature.gpu,"
                          "clocks_event_reasons.sw_power_cap,clocks_event_reasons.hw_slowdown",
                          "--format=csv,noheader,nounits", "-lms", "20"], stdout=f, stderr=subprocess.DEVNULL)
    time.sleep(0.5)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.launches)]
    t_host = []
    for a, b in ev:
        R.zero_()
        a.record(stream)
        ctx.jacobian(U, J, R=R) if args.op == "jacobian" else ctx.viscosity_resid(U, R=R)
        b.record(stream)
        if args.gap_ms > 0:
            torch.cuda.synchronize()
            time.sleep(args.gap_ms * 1e-3)
    torch.cuda.synchronize()
    time.sleep(0.3)
    p.terminate()
    p.wait()
    f.seek(0)
    rows = [r.split(", ") for r in f.read().strip().splitlines()]
    ms = [a.elapsed_time(b) for a, b in ev]
    chunk = max(1, args.launches // 10)
    out = {"config": args.config, "op": args.op, "gap_ms": args.gap_ms,
           "kernel_ms_by_chunk": [round(float(np.mean(ms[i:i + chunk])), 4) for i in range(0, len(ms), chunk)],
           "kernel_ms_min": round(min(ms), 4), "kernel_ms_median": round(float(np.median(ms)), 4)}
    smp = []
    for r in rows:
        try:
            smp.append((float(r[1]), float(r[2]), float(r[3]), r[4].strip()))
        except Exception:
            pass
    if smp:
        busy = [s for s in smp if s[1] > 300]
        out["samples"] = len(smp)
        out["busy_samples"] = len(busy)
        if busy:
            out["sm_mhz_busy"] = sorted(s[0] for s in busy)[len(busy) // 2]
            out["sm_mhz_busy_min"] = min(s[0] for s in busy)
            out["power_w_busy_median"] = sorted(s[1] for s in busy)[len(busy) // 2]
            out["power_w_max"] = max(s[1] for s in busy)
            out["temp_max"] = max(s[2] for s in busy)
            out["power_cap_active_frac"] = round(sum(1 for s in busy if s[3].lower().startswith("active")) / len(busy), 3)
        out["trace"] = [[s[0], s[1]] for s in smp[::max(1, len(smp) // 40)]]
    print(json.dumps(out))


if __name__ == "__main__":
    main()
