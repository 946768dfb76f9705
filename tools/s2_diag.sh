#!/bin/bash
# Solver diagnostics: primitive latencies, hardest-pair chain trace, local-SMO / selection phase cycles.
out=gpurun_out/${1:-diag}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/lat tools/micro/lat.cu && /tmp/lat > $out/lat.txt 2>&1; cat $out/lat.txt
GMPSVM_TRACE=0 timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $out/trace.json 2> $out/trace.err
grep "gmpsvm trace\] pair (" $out/trace.err | tail -1 | cut -c1-400
grep "gmpsvm trace\] pair windows" $out/trace.err | tail -1 > $out/windows.txt
GMPSVM_SMO_PHASES=1 timeout 600 python tools/prof_step.py --ws-size 192 > $out/phases.log 2>&1
grep "cycles" $out/phases.log
