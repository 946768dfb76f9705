#!/bin/bash
# f-update CTA width sweep (GMPSVM_FU_CHUNKS: 128-column chunks per CTA): bench ms/step + hardest-pair trace
out=gpurun_out/${1:-fu}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for C in 1 2 4 8 1; do
GMPSVM_FU_CHUNKS=$C timeout 600 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $out/b_$C.json 2> $out/b_$C.err
python -c "
import json,statistics as S;d=json.load(open('$out/b_$C.json'));s=d['step_ms'];print('chunks $C', round(d['ms_per_step'],2), 'median', round(S.median(s),2), 'min', round(min(s),2), d['counters'])"
GMPSVM_FU_CHUNKS=$C GMPSVM_TRACE=0 timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $out/t_$C.json 2> $out/t_$C.err
grep "gmpsvm trace\] pair (" $out/t_$C.err | tail -1 | cut -c1-700
done
