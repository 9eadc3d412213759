"""Markdown table of bench lines (BASELINE.md "Measured on B200"): python scripts/bench_table.py FILE..."""
import json
import sys

OPS = {"jacobian": "residual + Jacobian", "jac_packed": "residual + Jacobian (symmetric block-packed J)", "resid": "residual", "jvp": "J·v + residual", "jvp_y": "J·v only (Krylov apply)",
       "jac_csr": "Jacobian into global CSR (fused, atomics)", "jac_global": "Jacobian into global CSR (element matrices + pull assembly)"}
print("| config | elem | op | geometry | kernel | cells/s | ms/step | HBM frac | traffic / algorithmic | sustained cells/s | e2e cells/s |")
print("|---|---|---|---|---|---|---|---|---|---|---|")
for f in sys.argv[1:]:
    for ln in open(f):
        if not ln.startswith("{"):
            continue
        d = json.loads(ln)
        if d.get("impl") == "reference":
            continue
        c, r = d["config"], d["roofline"]
        wl = c["workload"].split()[0]
        tr = r.get("traffic")
        ratio = f"{tr / r['algorithmic_bytes_per_launch']:.3f}" if tr else "—"
        op = OPS.get(c["op"], c["op"])
        if c["op"] == "jac_global":
            op += " (packed J)" if "packed" in r["kernel"] else " (full J)"
        print(f"| {wl} | {c['elem']} | {op} | {c['geometry']} | `{r['kernel'].split(' ')[0]}` | {d['value']:.4g} | "
              f"{d['ms_per_step']:.3f} | {r['frac']:.3f} | {ratio} | {d.get('sustained', {}).get('value', 0):.4g} | "
              f"{d.get('e2e', {}).get('value', 0):.4g} |")
