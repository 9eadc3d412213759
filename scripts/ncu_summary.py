#!/usr/bin/env python
"""Summarise an ncu capture + launch list into profiles/<tag>_*.{md,csv} and
update profiles/traffic.json (dram bytes per launch of the profiled kernel).

    python scripts/ncu_summary.py --tag r01 --rep gpurun_out/prof_r01.ncu-rep \
        --launches gpurun_out/launches_r01.csv --key C4:hex8:jacobian
"""
import argparse
import csv
import io
import json
import os
import subprocess
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__shared_mem_per_block_dynamic", "launch__occupancy_limit_shared_mem", "launch__occupancy_limit_registers",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "smsp__inst_executed.sum", "sm__cycles_elapsed.avg.per_second", "lts__t_bytes.sum",
]


def ncu_csv(args):
    out = subprocess.run(["ncu", *args], capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(out)))


def raw_metrics(rep):
    rows = ncu_csv(["-i", rep, "--page", "raw", "--csv"])
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {}
        for m in METRICS + ["Kernel Name"]:
            if m in hdr:
                d[m] = (vals[hdr.index(m)], units[hdr.index(m)])
        res.append(d)
    return res


UNIT = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
        "KB": 1e3, "MB": 1e6, "GB": 1e9, "KiB": 1024.0, "MiB": 1024.0 ** 2, "GiB": 1024.0 ** 3}


def to_bytes(value: str, unit: str) -> float:
    """One ncu raw-page value in bytes, with ITS OWN unit (ncu scales every
    metric independently: reads may print in Gbyte while writes print in Mbyte)."""
    if unit not in UNIT:
        raise ValueError(f"unknown byte unit {unit!r}")
    return float(value.replace(",", "")) * UNIT[unit]


def dram_bytes(d) -> float:
    """dram__bytes_read.sum + dram__bytes_write.sum of one kernel row, in bytes."""
    return to_bytes(*d["dram__bytes_read.sum"]) + to_bytes(*d["dram__bytes_write.sum"])


def stall_summary(rep):
    rows = ncu_csv(["-i", rep, "--page", "source", "--csv", "--print-source", "sass"])
    if len(rows) < 3:
        return {}
    hdr = rows[1]
    tot = defaultdict(float)
    for r in rows[2:]:
        for k, v in zip(hdr, r):
            if k.startswith("stall_") and "Not Issued" not in k:
                try:
                    tot[k[6:]] += float(v.replace(",", "") or 0)
                except ValueError:
                    pass
    s = sum(tot.values()) or 1.0
    return {k: round(100 * v / s, 1) for k, v in sorted(tot.items(), key=lambda x: -x[1])[:8]}


def launch_shares(path):
    rows = list(csv.reader(open(path)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    ix = {k: j for j, k in enumerate(hdr)}
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[start + 1:]:
        if len(r) < len(hdr) or r[ix["Metric Name"]] != "gpu__time_duration.sum":
            continue
        scale = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "nsecond": 1e-3}.get(
            r[ix["Metric Unit"]], 1.0)
        k = r[ix["Kernel Name"]].split("(")[0][:90]
        agg[k][0] += 1
        agg[k][1] += float(r[ix["Metric Value"]].replace(",", "")) * scale
    return agg


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", required=True)
    ap.add_argument("--rep")
    ap.add_argument("--launches")
    ap.add_argument("--key", default="C4:hex8:jacobian:stored")
    ap.add_argument("--note", default="")
    ap.add_argument("--rev", default=None,
                    help="source revision the capture was made with (build.source_rev() of that build); "
                         "default: the current tree's")
    a = ap.parse_args()
    if a.rev is None:
        import sys
        sys.path.insert(0, ROOT)
        from paper_conf_sc_antepara0cw24_b200 import build as B
        a.rev = B.source_rev()
    prof = os.path.join(ROOT, "profiles")
    os.makedirs(prof, exist_ok=True)
    md = [f"# ncu summary {a.tag} ({a.key})", "", a.note, ""]
    if a.launches:
        agg = launch_shares(a.launches)
        tot = sum(v[1] for v in agg.values())
        md += ["## Launch list (ncu --metrics gpu__time_duration.sum --clock-control none; cold-cache, serialised)",
               "", "| kernel | launches | total us | mean us | share |", "|---|---|---|---|---|"]
        for k, (n, v) in sorted(agg.items(), key=lambda x: -x[1][1]):
            md.append(f"| `{k}` | {n} | {v:.1f} | {v / n:.1f} | {100 * v / tot:.1f}% |")
        md.append("")
        # keep the raw launch list too
        with open(a.launches) as f, open(os.path.join(prof, f"{a.tag}_launches.csv"), "w") as g:
            g.write(f.read())
    if a.rep:
        for d in raw_metrics(a.rep):
            md += [f"## `{d.get('Kernel Name', ('?', ''))[0][:100]}` (ncu --set full)", "",
                   "| metric | value | unit |", "|---|---|---|"]
            for m in METRICS:
                if m in d:
                    md.append(f"| {m} | {d[m][0]} | {d[m][1]} |")
            traffic = dram_bytes(d)
            md += ["", f"DRAM traffic per launch: {traffic:.4e} B", ""]
            tp = os.path.join(prof, "traffic.json")
            tr = json.load(open(tp)) if os.path.exists(tp) else {}
            tr[a.key] = {"dram_bytes_per_launch": traffic, "tag": a.tag, "rev": a.rev,
                         "kernel": d.get("Kernel Name", ("?", ""))[0][:100]}
            json.dump(tr, open(tp, "w"), indent=1)
        st = stall_summary(a.rep)
        md += ["## Warp stall samples (share of all samples)", "", json.dumps(st), ""]
    with open(os.path.join(prof, f"{a.tag}_ncu_summary.md"), "w") as f:
        f.write("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main()
