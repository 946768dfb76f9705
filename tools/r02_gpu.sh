#!/bin/bash
# Round-2 GPU iteration: build, focused tests, full gpu suite, bench (+ variants).
#   gpurun -- 'bash tools/r02_gpu.sh <tag> [pytest -k expr] [nofull]'   (BENCH_ENVS="A=1 B=2": extra bench runs)
tag=${1:-g}; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
if [ -n "$2" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q -k "$2" > $out/focus.log 2>&1; echo "focus rc=$?" >> $out/focus.log
  tail -5 $out/focus.log
fi
if [ "$3" != "nofull" ]; then
  timeout 2400 python -m pytest tests -m gpu -q > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log
  tail -15 $out/pytest.log
fi
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $out/bench.json 2> $out/bench.err
python -c "import json;d=json.load(open('$out/bench.json'));print('BENCH', d['ms_per_step'], d['phases_ms'], d['counters'])"
for ev in $BENCH_ENVS; do
  env ${ev//,/ } timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $out/bench_$ev.json 2> $out/bench_$ev.err
  python -c "import json;d=json.load(open('$out/bench_$ev.json'));print('BENCH $ev', d['ms_per_step'], d['phases_ms'], d['counters'])"
done
if [ -n "$TRACE" ]; then
  GMPSVM_TRACE=0 timeout 300 python tools/prof_step.py --ws-size 192 > $out/trace.log 2>&1; grep "gmpsvm trace" $out/trace.log | tail -2
fi
