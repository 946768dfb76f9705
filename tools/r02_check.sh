#!/bin/bash
# GPU suite + smoke + default bench
out=gpurun_out/${1:-check}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log; tail -4 $out/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.log 2>&1; tail -1 $out/smoke.log
timeout 900 python bench.py > $out/bench_default.json 2> $out/bench_default.err
python -c "
import json,statistics as S;d=json.load(open('$out/bench_default.json'));s=d['step_ms'];print('BENCH', round(d['ms_per_step'],2), 'median', round(S.median(s),2), 'max', round(max(s),2), 'e2e', d['e2e'], d['checks'], d['cpu_baseline'])"
