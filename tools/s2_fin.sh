#!/bin/bash
out=gpurun_out/${1:-fin}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_schedule.py tests/test_gpu_parity.py -x -q > $out/pytest.log 2>&1; tail -2 $out/pytest.log
for cfg in "GMPSVM_GROUPS=1" "GMPSVM_GROUPS=2" "GMPSVM_GROUPS=3" "GMPSVM_GROUPS=2 GMPSVM_LEAD_RESERVE=16"; do
env $cfg timeout 300 python bench.py --steps 15 --warmup 3 --no-cpu-baseline > $out/b.json 2> $out/b.err
echo "$cfg: $(python -c "
import json,statistics as S;d=json.load(open('$out/b.json'));s=d['step_ms'];print(round(d['ms_per_step'],2), 'med', round(S.median(s),2), 'kv', round(d['phases_ms']['kernel_values'],2), 'train', round(d['phases_ms']['train_total'],2), 'fin', round(d['phases_ms']['finalize'],2), d['gpu_launches'])" 2>&1 | tail -1)"
done
