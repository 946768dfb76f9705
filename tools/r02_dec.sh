#!/bin/bash
out=gpurun_out/${1:-dec}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "int8 or hyperparameter or forced" > $out/focus.log 2>&1; tail -3 $out/focus.log
for env in "GMPSVM_I8_COLLECT=1" ${EXTRA_ENVS}; do
  env $env timeout 300 python tools/prof_dec.py --reps 5 >> $out/dec.jsonl 2>> $out/dec.err
done
if [ -n "$NCU" ]; then timeout 600 ncu --set full --clock-control none --import-source on -k regex:dec_i8 -c 1 -f -o $out/dec_i8 python tools/prof_dec.py --reps 1 > $out/ncu.log 2>&1; fi
cat $out/dec.jsonl; tail -2 $out/ncu.log 2>/dev/null
