#!/bin/bash
# Registers / spills per kernel of libstokesfo (ptxas -v), demangled.  Usage: bash scripts/ptxas_regs.sh [regex]
cd "$(dirname "$0")/.."
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Xptxas -v -I include \
  -c paper_conf_sc_antepara0cw24_b200/csrc/sfo_capi.cu -o /tmp/ptxas_regs.o 2>&1 | python3 -c "
import re, sys, subprocess
cur = None; out = []
for line in sys.stdin:
    m = re.search(r\"Compiling entry function '(\S+)'\", line)
    if m: cur = m.group(1); continue
    m = re.search(r'(\d+) bytes spill stores', line)
    if m and cur: spill = m.group(1)
    m = re.search(r'Used (\d+) registers', line)
    if m and cur:
        out.append((cur, m.group(1), spill)); cur = None
names = subprocess.run(['c++filt'], input='\n'.join(o[0] for o in out), capture_output=True, text=True).stdout.split('\n')
pat = sys.argv[1] if len(sys.argv) > 1 else ''
for (m, r, sp), n in zip(out, names):
    if re.search(pat, n): print(f'{r:>4} regs  {sp:>4} B spill  {n[:110]}')
" "$1"
