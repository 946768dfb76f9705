#!/bin/bash
# Solver / finalize diagnostics on the GPU (host phase times, per-pair iterations, kernel timeline).
tag=${1:-d}; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
GMPSVM_HOST_TIMING=1 timeout 300 python tools/prof_step.py --ws-size 192 --reps 3 > $out/host_timing.log 2>&1
GMPSVM_SMO_PHASES=1 timeout 300 python tools/prof_step.py --ws-size 192 --reps 2 > $out/phases.log 2>&1
for p in 0 1 2; do GMPSVM_TRACE=$p timeout 300 python tools/prof_step.py --ws-size 192 --reps 2 > $out/trace$p.log 2>&1; done
tail -n 4 $out/host_timing.log
