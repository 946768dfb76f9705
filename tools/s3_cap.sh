#!/bin/bash
# local SMO step cap per outer iteration (inner_iter_cap) sweep
out=gpurun_out/${1:-cap}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for c in ${CAPS:-0 48 64 96 128 192 0}; do
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --inner-cap $c > $out/b.json 2> $out/b.err
echo "cap=$c: $(python -c "
import json,statistics as S;d=json.load(open('$out/b.json'));s=d['step_ms'];print(round(d['ms_per_step'],2), 'med', round(S.median(s),2), 'train', round(d['phases_ms']['train_total'],2), d['counters']['outer_iters_max'], d['counters']['inner_iters_sum'], d['checks']['test_accuracy'])" 2>&1 | tail -1)"
done
