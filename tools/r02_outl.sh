#!/bin/bash
out=gpurun_out/${1:-outl}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for i in 1 2; do
timeout 600 python bench.py --steps 60 --warmup 3 --no-cpu-baseline > $out/on_$i.json 2> $out/on_$i.err
GMPSVM_BENCH_CLOCKS=off timeout 600 python bench.py --steps 60 --warmup 3 --no-cpu-baseline > $out/off_$i.json 2> $out/off_$i.err
done
GMPSVM_HOST_TIMING=1 timeout 600 python bench.py --steps 60 --warmup 3 --no-cpu-baseline > $out/ht.json 2> $out/ht.err
for f in $out/*.json; do python -c "
import json,sys;d=json.load(open('$f'));s=d['step_ms'];print('$f', round(d['ms_per_step'],2), 'e2e', d['e2e']['value'] if isinstance(d.get('e2e'),dict) else None, 'max', round(max(s),1), 'n>42:', sum(x>42 for x in s), [round(x,1) for x in s if x>42])"; done
