#!/bin/bash
# Persistent solver vs per-kernel graphs: bench, trace, schedule/parity tests.
out=gpurun_out/${1:-persist}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.log 2>&1; tail -2 $out/smoke.log
for P in 1 0; do
GMPSVM_PERSIST=$P timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $out/b_$P.json 2> $out/b_$P.err
python -c "
import json,statistics as S;d=json.load(open('$out/b_$P.json'));s=d['step_ms'];print('persist $P', round(d['ms_per_step'],2), 'median', round(S.median(s),2), 'min', round(min(s),2), d['counters'], d['phases_ms']['train_total'], d['checks'])" || tail -5 $out/b_$P.err
done
GMPSVM_TRACE=0 timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $out/t.json 2> $out/t.err
grep "gmpsvm trace\]" $out/t.err | tail -2 | cut -c1-900
timeout 900 python -m pytest tests/test_gpu_schedule.py tests/test_gpu_parity.py -x -q > $out/pytest.log 2>&1; tail -3 $out/pytest.log
