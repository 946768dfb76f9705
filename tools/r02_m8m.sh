#!/bin/bash
out=gpurun_out/${1:-m8m}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
./tools/micro/i8_mma_rate > $out/i8_mma_rate.log 2>&1; cat $out/i8_mma_rate.log
timeout 3000 python tools/scale_probe.py mnist8m 8100000 10000 > $out/m8m_8100k.log 2>&1; echo "rc=$?" >> $out/m8m_8100k.log; tail -2 $out/m8m_8100k.log | cut -c1-900
