#!/bin/bash
# Round-2 GPU iteration: build, focused tests, full gpu suite, bench.  gpurun -- 'bash tools/r02_gpu.sh <tag> [pytest -k expr]'
tag=${1:-g}; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
if [ -n "$2" ]; then
  timeout 600 python -m pytest tests -m gpu -x -q -k "$2" > $out/focus.log 2>&1; echo "focus rc=$?" >> $out/focus.log
  tail -5 $out/focus.log
fi
if [ "$3" != "nofull" ]; then
  timeout 1800 python -m pytest tests -m gpu -q > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log
  tail -15 $out/pytest.log
fi
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $out/bench.json 2> $out/bench.err
head -c 600 $out/bench.json
