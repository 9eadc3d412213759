python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for D in 1 0; do
 STOKESFO_GLOBAL_DISCARD=$D timeout 600 python bench.py --op jac_global --geometry compact --no-cpu-baseline --sustain 0 --no-e2e --steps 5 > gpurun_out/glob_c$D.json 2> gpurun_out/glob_c$D.err
 python -c "
import json; d=json.loads(open('gpurun_out/glob_c$D.json').read())
print('discard=$D', round(d['value']/1e9,4), 'e9 cells/s', round(d['ms_per_step'],3), 'ms/step')" || tail -3 gpurun_out/glob_c$D.err
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval -s 1 -c 1 -o /tmp/glob python bench.py --op jac_global --geometry compact --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --sustain 0 > gpurun_out/glob_ncu.log 2>&1
ncu -i /tmp/glob.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null | gzip > gpurun_out/glob_src.csv.gz
ncu -i /tmp/glob.ncu-rep --page raw --csv 2>/dev/null > gpurun_out/glob_raw.csv
