#!/bin/bash
# lead-mode sweep: bench ms/step for GMPSVM_LEAD / GMPSVM_LEAD_RESERVE settings
out=gpurun_out/${1:-lead}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
run() { tag=$1; shift; env "$@" timeout 600 python bench.py --steps 30 --warmup 3 --no-cpu-baseline > $out/b_$tag.json 2> $out/b_$tag.err
  python -c "
import json,statistics as S;d=json.load(open('$out/b_$tag.json'));s=d['step_ms'];print('$tag', round(d['ms_per_step'],2), 'median', round(S.median(s),2), 'min', round(min(s),2), 'kern', d.get('phases_ms',{}).get('kernel') if isinstance(d.get('phases_ms'),dict) else '', 'e2e', round(d['e2e']['value']*1e3,2))" 2>&1 | tail -1; }
run l0 GMPSVM_LEAD=0
run l1r8 GMPSVM_LEAD=1 GMPSVM_LEAD_RESERVE=8
run l1r4 GMPSVM_LEAD=1 GMPSVM_LEAD_RESERVE=4
run l1r16 GMPSVM_LEAD=1 GMPSVM_LEAD_RESERVE=16
run l2r8 GMPSVM_LEAD=2 GMPSVM_LEAD_RESERVE=8
run l3r8 GMPSVM_LEAD=3 GMPSVM_LEAD_RESERVE=12
run l0b GMPSVM_LEAD=0
