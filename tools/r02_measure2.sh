#!/bin/bash
out=gpurun_out/${1:-meas2}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "shard or dist" > $out/focus.log 2>&1; echo "focus rc=$?" >> $out/focus.log; tail -3 $out/focus.log
timeout 1800 python tools/shard_probe_intra.py mnist8m 1000000 > $out/intra_1m.log 2>&1; tail -5 $out/intra_1m.log
timeout 3000 python tools/scale_probe.py mnist8m 8100000 10000 > $out/m8m_8100k.log 2>&1; echo "rc=$?" >> $out/m8m_8100k.log; tail -3 $out/m8m_8100k.log
