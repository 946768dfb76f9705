out=gpurun_out/$1; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log
GMPSVM_SMO_PHASES=1 timeout 300 python tools/prof_step.py --ws-size 192 --reps 2 > $out/phases.log 2>&1
GMPSVM_TRACE=1 timeout 300 python tools/prof_step.py --ws-size 192 --reps 2 > $out/trace1.log 2>&1
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $out/bench.json 2> $out/bench.err
