#!/bin/bash
# full GPU suite + smoke + bench (20 steps)
out=gpurun_out/${1:-check}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log; tail -3 $out/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.log 2>&1; tail -1 $out/smoke.log
timeout 600 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $out/bench_20.json 2> $out/bench_20.err
python -c "
import json,statistics as S;d=json.load(open('$out/bench_20.json'));s=d['step_ms'];print(round(d['ms_per_step'],2), 'med', round(S.median(s),2), 'kv', round(d['phases_ms']['kernel_values'],3), 'train', round(d['phases_ms']['train_total'],2), 'pred', round(d['phases_ms']['predict_total'],2), 'frac', round(d['roofline']['frac'],3), 'e2e', round(d['e2e']['value']*1e3,2), d['counters'])"
