#!/bin/bash
out=gpurun_out/${1:-slow}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for i in 1 2; do
GMPSVM_SLOW_API=2 timeout 600 python bench.py --steps 60 --warmup 3 --no-cpu-baseline > $out/s_$i.json 2> $out/s_$i.err
done
for f in $out/s_*.json; do python -c "
import json,sys;d=json.load(open('$f'));s=d['step_ms'];print('$f', round(d['ms_per_step'],2), 'max', round(max(s),1), [(i,round(x,1)) for i,x in enumerate(s) if x>42])"; done
grep "slow api" $out/s_*.err | sed 's/([^)]*engine.cu/(engine.cu/' | awk '{print $0}' | cut -c1-200 | sort | uniq -c | sort -rn | head -40
