#!/bin/bash
# krow cluster-multicast: tests + bench with / without, lead on / off
out=gpurun_out/${1:-mc}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for cfg in "GMPSVM_KROW_MC=1" "GMPSVM_KROW_MC=0" "GMPSVM_KROW_MC=1 GMPSVM_LEAD=0" "GMPSVM_KROW_MC=0 GMPSVM_LEAD=0"; do
env $cfg timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $out/b.json 2> $out/b.err
echo "$cfg: $(python -c "
import json,statistics as S;d=json.load(open('$out/b.json'));s=d['step_ms'];print(round(d['ms_per_step'],2), 'med', round(S.median(s),2), 'kv', round(d['phases_ms']['kernel_values'],3), 'train', round(d['phases_ms']['train_total'],2), 'frac', round(d['roofline']['frac'],3), d['counters']['outer_iters_max'], d['counters']['inner_iters_sum'])" 2>&1 | tail -1)"
done
timeout 1200 python -m pytest tests/test_gpu_schedule.py tests/test_gpu_parity.py tests/test_gpu_full.py -x -q > $out/pytest.log 2>&1; tail -3 $out/pytest.log
