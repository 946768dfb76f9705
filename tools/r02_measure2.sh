#!/bin/bash
out=gpurun_out/${1:-meas2}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "shard or dist" > $out/focus.log 2>&1; echo "focus rc=$?" >> $out/focus.log; tail -3 $out/focus.log
timeout 1800 python tools/shard_probe_intra.py mnist8m 1000000 > $out/intra_1m.log 2>&1; tail -5 $out/intra_1m.log
timeout 1500 ncu --graph-profiling node --metrics gpu__time_duration.sum --clock-control none -c 20000 --csv --log-file $out/m8m_1m_launches.csv python tools/scale_probe.py mnist8m 1000000 10000 > $out/m8m_ncu.log 2>&1
python tools/launch_sum.py $out/m8m_1m_launches.csv | head -16
timeout 3000 python tools/scale_probe.py mnist8m 8100000 10000 > $out/m8m_8100k.log 2>&1; echo "rc=$?" >> $out/m8m_8100k.log; tail -3 $out/m8m_8100k.log
