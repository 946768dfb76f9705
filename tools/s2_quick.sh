#!/bin/bash
# quick: bench 20 steps (+ optional env) and a hardest-pair trace
out=gpurun_out/${1:-quick}; shift; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
env "$@" timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $out/b.json 2> $out/b.err
python -c "
import json,statistics as S;d=json.load(open('$out/b.json'));s=d['step_ms'];print(round(d['ms_per_step'],2), 'med', round(S.median(s),2), 'kv', round(d['phases_ms']['kernel_values'],2), 'train', round(d['phases_ms']['train_total'],2), 'e2e', round(d['e2e']['value']*1e3,2), d['counters'])" 2>&1 | tail -1
env "$@" GMPSVM_TRACE=0 timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $out/t.json 2> $out/t.err
grep "gmpsvm trace\] pair (" $out/t.err | tail -1 | cut -c1-420
