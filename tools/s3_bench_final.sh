#!/bin/bash
# final bench lines (default run with the CPU baseline, 20 steps, reference arm), launch list, smoke
out=gpurun_out/${1:-bfinal}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.log 2>&1; tail -1 $out/smoke.log
timeout 900 python bench.py > $out/bench_default.json 2> $out/bench_default.err
timeout 900 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $out/bench_20.json 2> $out/bench_20.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > $out/bench_reference.json 2> $out/bench_reference.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $out/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > $out/b_ncu.log 2>&1
python tools/launch_sum.py $out/launches.csv > $out/launches_sum.txt 2>&1
for f in bench_default bench_20; do python -c "
import json;d=json.load(open('$out/$f.json'));print('$f', round(d['ms_per_step'],2), 'e2e', round(d['e2e']['value']*1e3,2), 'frac', round(d['roofline']['frac'],3), round(d['roofline']['frac_of_launch_sms'],3), d['phases_ms']['kernel_values'], d['phases_ms']['train_total'], d['phases_ms']['predict_total'], d['clocks'], d['counters'])"; done
