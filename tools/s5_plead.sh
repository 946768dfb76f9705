#!/bin/bash
# hybrid persistent lead group (GMPSVM_PERSIST=lead) vs the default graphs: schedule test, 20-step benches, lead-pair traces
out=gpurun_out/${1:-s5pl}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_schedule.py -m gpu -q -x > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log; tail -2 $out/pytest.log
for cfg in "X=0" "GMPSVM_PERSIST=lead" "GMPSVM_PERSIST=lead GMPSVM_LEAD_RESERVE=16" "GMPSVM_PERSIST=lead GMPSVM_LEAD_RESERVE=24" "X=1"; do
env $cfg timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $out/b.json 2> $out/b.err
echo "$cfg: $(python -c "import json,statistics as S;d=json.load(open('$out/b.json'));print(round(d['ms_per_step'],2), 'med', round(S.median(d['step_ms']),2), 'train', round(d['phases_ms']['train_total'],2), d['counters']['outer_iters_max'], d['gpu_launches'])")"
env $cfg GMPSVM_TRACE=0 timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $out/t.json 2> $out/t.err
grep "gmpsvm trace\] pair (" $out/t.err | tail -1 | cut -c1-900
done
