#!/usr/bin/env python
"""Static SASS instruction mix of the eval kernels in a built library (A/B before GPU time).

    python scripts/sass_stats.py [LIB] [name-regex]
"""
import re
import subprocess
import sys

lib = sys.argv[1] if len(sys.argv) > 1 else "paper_conf_sc_antepara0cw24_b200/libstokesfo.so"
pat = re.compile(sys.argv[2] if len(sys.argv) > 2 else r"eval_kernel.*ELi[0-3]ELi2E")
txt = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
for fn in re.split(r"\n\s+Function : ", txt)[1:]:
    name = fn.split("\n", 1)[0].strip()
    if not pat.search(name):
        continue
    ins = [l for l in fn.split("\n") if re.match(r"\s+/\*[0-9a-f]{4}\*/", l)]
    c = lambda k: sum(1 for l in ins if re.search(k, l))
    print(f"{name[:56]:56s} n={len(ins):5d} DFMA={c(r'DFMA'):4d} DMUL={c(r'DMUL'):4d} DADD={c(r'DADD'):4d} "
          f"LDS={c(r"LDS"):4d} LDS128={c(r"LDS\.128"):3d} STS={c(r'STS'):4d} SEL={c(r' F?SEL'):4d} SHFL={c(r'SHFL'):3d}")
