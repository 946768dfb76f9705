#!/bin/bash
out=gpurun_out/${1:-trace}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for L in 0 1; do
GMPSVM_LEAD=$L GMPSVM_TRACE=0 timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $out/t_$L.json 2> $out/t_$L.err
grep "gmpsvm trace\] pair windows" $out/t_$L.err | tail -1 | cut -c1-1500
grep "gmpsvm trace\] pair (" $out/t_$L.err | tail -1 | cut -c1-300
done
