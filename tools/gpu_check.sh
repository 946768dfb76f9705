#!/bin/bash
# One gpurun call: GPU tests, bench line, ncu launch lists and full captures of the top kernels.
#   gpurun --timeout 2400 -- 'bash tools/gpu_check.sh [tag]'
tag=${1:-chk}
out=gpurun_out/$tag
mkdir -p $out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > $out/smi.txt
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log
timeout 900 python bench.py --steps 5 --warmup 3 > $out/bench.json 2> $out/bench.err
# launch list of one train + predict: the solver graph as one entry (its share of the step) ...
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --graph-profiling graph --csv \
    --log-file $out/launches_graph.csv python tools/prof_step.py --ws-size 192 > $out/launches_graph.log 2>&1
# ... and every kernel (solver launched on streams, not in a graph, so ncu sees each kernel; serialised)
GMPSVM_SOLVER=streams timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $out/launches.csv python tools/prof_step.py --ws-size 192 > $out/launches.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:krow_tc -c 1 -f -o $out/krow_tc \
    python tools/prof_step.py --ws-size 192 > $out/ncu_krow.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dec_tc -c 1 -f -o $out/dec_tc \
    python tools/prof_step.py --ws-size 192 > $out/ncu_dec.log 2>&1
tail -2 $out/pytest.log; head -c 600 $out/bench.json
