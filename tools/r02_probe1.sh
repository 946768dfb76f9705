#!/bin/bash
out=gpurun_out/r02a; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 900 python tests/probe_parity.py $out/parity_tc.json > $out/parity_tc.log 2>&1
GMPSVM_DEC=f64 timeout 900 python tests/probe_parity.py $out/parity_f64.json > $out/parity_f64.log 2>&1
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $out/bench.json 2> $out/bench.err
nproc > $out/host.txt; lscpu | grep -i "model name" >> $out/host.txt; free -g >> $out/host.txt
tail -2 $out/parity_tc.log; head -c 300 $out/bench.json
