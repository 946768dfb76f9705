#!/bin/bash
# q (new rows per outer iteration) sweep at B = 192 / 208 / 224
out=gpurun_out/${1:-q}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for a in "192 96" "192 64" "192 80" "192 112" "192 128" "208 128" "224 144" "224 160" "256 160"; do
set -- $a
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --ws-size $1 --q $2 > $out/b.json 2> $out/b.err
echo "B=$1 q=$2: $(python -c "
import json,statistics as S;d=json.load(open('$out/b.json'));s=d['step_ms'];print(round(d['ms_per_step'],2), 'med', round(S.median(s),2), 'train', round(d['phases_ms']['train_total'],2), d['counters']['outer_iters_max'], d['counters']['inner_iters_sum'], round(d['counters']['smo_cycles_per_step']))" 2>&1 | tail -1)"
done
