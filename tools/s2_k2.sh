#!/bin/bash
# 2-CTA (cta_group::2) kernel values vs single-CTA (+cluster multicast), lead off
out=gpurun_out/${1:-k2}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for cfg in "GMPSVM_KROW_CTA=2 GMPSVM_LEAD=0" "GMPSVM_LEAD=0" "GMPSVM_KROW_CTA=2 GMPSVM_LEAD=0 GMPSVM_KROW_DIAG=64" "GMPSVM_KROW_CTA=2 GMPSVM_LEAD=0 GMPSVM_KROW_DIAG=1" "GMPSVM_KROW_CTA=2 GMPSVM_LEAD=0 GMPSVM_KROW_DIAG=2"; do
env $cfg timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $out/b.json 2> $out/b.err
echo "$cfg: $(python -c "
import json,statistics as S;d=json.load(open('$out/b.json'));s=d['step_ms'];print(round(d['ms_per_step'],2), 'kv', round(d['phases_ms']['kernel_values'],3), 'frac', round(d['roofline']['frac'],3), d['counters']['outer_iters_max'], d['counters']['inner_iters_sum'])" 2>&1 | tail -1)"
done
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "cta" > $out/pytest.log 2>&1; tail -3 $out/pytest.log
