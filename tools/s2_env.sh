#!/bin/bash
# bench (15 steps) under several env settings: tools/s2_env.sh <tag> "<env1>" "<env2>" ...
out=gpurun_out/$1; shift; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for cfg in "$@"; do
env $cfg timeout 300 python bench.py --steps 15 --warmup 3 --no-cpu-baseline > $out/b.json 2> $out/b.err
echo "$cfg: $(python -c "
import json,statistics as S;d=json.load(open('$out/b.json'));s=d['step_ms'];print(round(d['ms_per_step'],2), 'med', round(S.median(s),2), 'kv', round(d['phases_ms']['kernel_values'],2), 'train', round(d['phases_ms']['train_total'],2), d['counters']['outer_iters_max'], d['counters']['inner_iters_sum'], round(d['counters']['smo_cycles_per_step']))" 2>&1 | tail -1)"
done
