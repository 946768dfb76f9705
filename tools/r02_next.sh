#!/bin/bash
out=gpurun_out/${1:-next}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for i in 1 2; do timeout 900 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $out/bench20_$i.json 2> $out/bench20_$i.err
python -c "import json;d=json.load(open('$out/bench20_$i.json'));print('BENCH', round(d['ms_per_step'],2), [round(x,1) for x in d['step_ms']], d['host_ms_train_predict'], d['phases_ms']['decision_values'])"; done
timeout 900 python -m pytest tests -m gpu -x -q -k "int8 or full_size or letter or hyperparameter or mnist_shaped or fp64 or forced" > $out/focus.log 2>&1; echo "focus rc=$?" >> $out/focus.log; tail -3 $out/focus.log
timeout 300 python tools/prof_dec.py --reps 5 > $out/dec.jsonl 2>> $out/dec.err; cat $out/dec.jsonl
GMPSVM_TRACE=0 timeout 300 python tools/prof_step.py --ws-size 192 > $out/trace_cfg3.log 2>&1; grep "gmpsvm trace\] pair (" $out/trace_cfg3.log
GMPSVM_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline > $out/bench_torchrun2_gloo.json 2> $out/bench_torchrun2_gloo.err; head -c 400 $out/bench_torchrun2_gloo.json; echo
