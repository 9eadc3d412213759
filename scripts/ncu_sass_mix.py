#!/usr/bin/env python
"""Dynamic instruction mix and stall samples by opcode from an ncu report's SASS source page.

    python scripts/ncu_sass_mix.py REP.ncu-rep [top]
"""
import csv
import io
import re
import subprocess
import sys
from collections import defaultdict

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = next(r for r in rows if r and r[0] == "Address")
ix = {h: i for i, h in enumerate(hdr)}
ex, st, wf = defaultdict(int), defaultdict(int), defaultdict(int)
tot_ex = tot_st = 0
for r in rows[rows.index(hdr) + 1:]:
    if len(r) < len(hdr):
        continue
    src = re.sub(r"^\s*@!?U?P[0-9T]+\s+", "", r[ix["Source"]].strip())
    op = src.split(" ")[0].split(".")[0].rstrip(";")
    e = int(r[ix["Instructions Executed"]] or 0)
    s = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    w = int(r[ix["L1 Wavefronts Shared"]] or 0) if "L1 Wavefronts Shared" in ix else 0
    ex[op] += e; st[op] += s; wf[op] += w
    tot_ex += e; tot_st += s
print(f"total warp instructions executed {tot_ex:.4e}, stall samples {tot_st}")
print(f"{'op':10s} {'executed':>12s} {'share':>7s} {'stall%':>7s} {'smem wavefronts':>16s}")
for op in sorted(ex, key=lambda o: -ex[o])[:top]:
    print(f"{op:10s} {ex[op]:12d} {ex[op] / tot_ex:7.3f} {100 * st[op] / max(1, tot_st):7.1f} {wf[op]:16d}")
