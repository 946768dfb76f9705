#!/bin/bash
# Quick iteration on the GPU: tests + bench (+ optional ncu of one kernel regex).
#   gpurun -- 'bash tools/gpu_quick.sh <tag> [kernel-regex]'
tag=${1:-q}; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log
timeout 300 python tools/krow_check.py > $out/krow_check.log 2>&1
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $out/bench.json 2> $out/bench.err
if [ -n "$2" ]; then
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$2 -c 1 -f -o $out/k \
      python tools/prof_step.py --ws-size 192 > $out/ncu.log 2>&1
fi
tail -3 $out/pytest.log; tail -3 $out/krow_check.log; head -c 400 $out/bench.json
