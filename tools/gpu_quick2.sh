#!/bin/bash
# Tests + bench + hardest-pair solver trace (GMPSVM_TRACE=1) in one gpurun call.
#   gpurun -- 'bash tools/gpu_quick2.sh <tag>'
tag=${1:-q2}; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $out/bench.json 2> $out/bench.err
GMPSVM_TRACE=1 timeout 300 python tools/prof_step.py --ws-size 192 --reps 2 2>&1 | grep "outer 232\|t_solver" > $out/trace.log
tail -2 $out/pytest.log; cat $out/trace.log; head -c 300 $out/bench.json; echo
python -c "import json;d=json.load(open('$out/bench.json'));print(d['value'],d['roofline']['frac'],d['e2e']['value'],d['phases_ms'],d['clocks'])"
