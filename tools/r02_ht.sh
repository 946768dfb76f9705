#!/bin/bash
out=gpurun_out/${1:-ht}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
GMPSVM_HOST_TIMING=1 timeout 900 python bench.py --steps 30 --warmup 3 --no-cpu-baseline > $out/bench_ht.json 2> $out/bench_ht.err
python -c "import json;d=json.load(open('$out/bench_ht.json'));print('BENCH', round(d['ms_per_step'],2), [round(x,1) for x in d['step_ms']])"
grep "host ms" $out/bench_ht.err | head -40 | cut -c1-400
