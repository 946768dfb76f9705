#!/bin/bash
# local SMO with FP32 working-set f (GMPSVM_SMO_F32=1) vs FP64: bench + parity under F32
out=gpurun_out/${1:-f32}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for cfg in "GMPSVM_SMO_F32=1" "GMPSVM_SMO_F32=0" "GMPSVM_SMO_F32=1 GMPSVM_LEAD=0"; do
env $cfg timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $out/b.json 2> $out/b.err
echo "$cfg: $(python -c "
import json,statistics as S;d=json.load(open('$out/b.json'));s=d['step_ms'];print(round(d['ms_per_step'],2), 'med', round(S.median(s),2), 'train', round(d['phases_ms']['train_total'],2), d['counters'], d['checks']['test_accuracy'])" 2>&1 | tail -1)"
done
GMPSVM_SMO_F32=1 GMPSVM_TRACE=0 timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $out/t.json 2> $out/t.err
grep "gmpsvm trace\] pair (" $out/t.err | tail -1 | cut -c1-500
GMPSVM_SMO_F32=1 timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full.py tests/test_gpu_edge.py -x -q > $out/pytest.log 2>&1; tail -3 $out/pytest.log
