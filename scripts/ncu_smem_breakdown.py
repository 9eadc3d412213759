#!/usr/bin/env python
"""Shared-memory wavefronts and stall samples per SASS instruction class (opcode, measured
wavefronts per execution, ideal) from an ncu report's source page, per unit of work.

    python scripts/ncu_smem_breakdown.py REP.ncu-rep UNITS   (e.g. UNITS = tiles per launch)
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

rep, units = sys.argv[1], float(sys.argv[2])
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = next(r for r in rows if r and r[0] == "Address")
ix = {h: i for i, h in enumerate(hdr)}
st = "Warp Stall Sampling (All Samples)"
data = [r for r in rows[rows.index(hdr) + 1:] if len(r) >= len(hdr)]
tot_st = sum(int(r[ix[st]] or 0) for r in data)
agg = defaultdict(lambda: [0.0, 0.0, 0.0])
tot_wf = 0.0
for r in data:
    src = r[ix["Source"]].strip()
    if not ("LDS" in src or "STS" in src):
        continue
    toks = src.split()
    op = toks[1] if toks[0].startswith("@") else toks[0]
    e = int(r[ix["Instructions Executed"]] or 0)
    if not e:
        continue
    w = int(r[ix["L1 Wavefronts Shared"]] or 0)
    wi = int(r[ix["L1 Wavefronts Shared Ideal"]] or 0)
    k = (op, round(w / e, 2), round(wi / e, 2))
    agg[k][0] += e / units
    agg[k][1] += w / units
    agg[k][2] += int(r[ix[st]] or 0)
    tot_wf += w / units
print(f"shared wavefronts per unit {tot_wf:.1f}; stall samples {tot_st}")
print(f"{'op':10s} {'wf/exec':>8s} {'ideal':>6s} {'exec/unit':>10s} {'wf/unit':>8s} {'stall%':>7s}")
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{k[0]:10s} {k[1]:8.2f} {k[2]:6.2f} {v[0]:10.1f} {v[1]:8.1f} {100 * v[2] / tot_st:7.2f}")
