#!/bin/bash
# Hardest-pair chain with handoff records (f-update grid end -> selection release), lead on/off.
out=gpurun_out/${1:-trace}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for L in 1 0; do
GMPSVM_LEAD=$L GMPSVM_TRACE=0 timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $out/t_$L.json 2> $out/t_$L.err
echo "LEAD=$L"; grep "gmpsvm trace\] pair (" $out/t_$L.err | tail -1 | cut -c1-700
done
GMPSVM_TRACE=7 timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $out/t_p7.json 2> $out/t_p7.err
echo "pos 7"; grep "gmpsvm trace\] pair (" $out/t_p7.err | tail -1 | cut -c1-700
