#!/bin/bash
# working-set size sweep on the current kernels (q = B / 2)
out=gpurun_out/${1:-ws}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for B in 160 176 192 208 224 128; do
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --ws-size $B > $out/b.json 2> $out/b.err
echo "B=$B: $(python -c "
import json,statistics as S;d=json.load(open('$out/b.json'));s=d['step_ms'];print(round(d['ms_per_step'],2), 'med', round(S.median(s),2), 'train', round(d['phases_ms']['train_total'],2), d['counters'])" 2>&1 | tail -1)"
done
