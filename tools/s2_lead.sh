#!/bin/bash
# lead-mode sweep on the current kernels: bench ms/step for GMPSVM_LEAD / GMPSVM_LEAD_RESERVE
out=gpurun_out/${1:-lead}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for cfg in "GMPSVM_LEAD=1 GMPSVM_LEAD_RESERVE=8" "GMPSVM_LEAD=2 GMPSVM_LEAD_RESERVE=8" "GMPSVM_LEAD=2 GMPSVM_LEAD_RESERVE=12" "GMPSVM_LEAD=3 GMPSVM_LEAD_RESERVE=12" "GMPSVM_LEAD=4 GMPSVM_LEAD_RESERVE=16" "GMPSVM_LEAD=6 GMPSVM_LEAD_RESERVE=16" "GMPSVM_LEAD=2 GMPSVM_LEAD_RESERVE=16"; do
env $cfg timeout 300 python bench.py --steps 15 --warmup 3 --no-cpu-baseline > $out/b.json 2> $out/b.err
echo "$cfg: $(python -c "
import json,statistics as S;d=json.load(open('$out/b.json'));s=d['step_ms'];print(round(d['ms_per_step'],2), 'med', round(S.median(s),2), 'kv', round(d['phases_ms']['kernel_values'],2), 'train', round(d['phases_ms']['train_total'],2))" 2>&1 | tail -1)"
done
