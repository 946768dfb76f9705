#!/bin/bash
out=gpurun_out/${1:-lp}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for cfg in "GMPSVM_LEAD=1" "GMPSVM_LEAD=1 GMPSVM_GROUPS=2" "GMPSVM_LEAD=1 GMPSVM_GROUPS=3" "GMPSVM_LEAD=1 GMPSVM_GROUPS=2 GMPSVM_LEAD_RESERVE=16" "GMPSVM_LEAD=1 GMPSVM_GROUPS=3 GMPSVM_LEAD_RESERVE=24" "GMPSVM_LEAD=2 GMPSVM_GROUPS=2 GMPSVM_LEAD_RESERVE=16"; do
echo "== $cfg"
env $cfg GMPSVM_LEAD_DEBUG=1 python tools/lead_probe.py > $out/p.log 2>&1
grep "dev_ms\|timeline\|lead ms" $out/p.log | tail -3 | cut -c1-250
env $cfg timeout 600 python bench.py --steps 30 --warmup 3 --no-cpu-baseline > $out/b.json 2> $out/b.err
python -c "
import json,statistics as S;d=json.load(open('$out/b.json'));s=d['step_ms'];print('BENCH', round(d['ms_per_step'],2), 'median', round(S.median(s),2), 'max', round(max(s),2), 'e2e', round(d['e2e']['value']*1e3,2), d['phases_ms']['train_total'])"
done
