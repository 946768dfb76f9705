#!/bin/bash
out=gpurun_out/${1:-ptrace}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for cfg in "GMPSVM_LEAD=0 GMPSVM_TRACE=0" "GMPSVM_LEAD=0 GMPSVM_TRACE=7" "GMPSVM_TRACE=7" "GMPSVM_LEAD=0 GMPSVM_PERSIST=0 GMPSVM_TRACE=0"; do
env $cfg timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $out/t.json 2> $out/t.err
echo "$cfg: $(python -c "import json;d=json.load(open('$out/t.json'));print(round(d['ms_per_step'],2), d['phases_ms']['train_total'])")"
grep "gmpsvm trace\] pair (" $out/t.err | tail -1 | cut -c1-900
done
