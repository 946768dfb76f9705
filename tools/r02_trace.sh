#!/bin/bash
out=gpurun_out/${1:-trace}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for pos in 0; do
GMPSVM_TRACE=$pos timeout 900 python tools/scale_probe.py mnist8m ${2:-2000000} 10000 > $out/m8m_trace_$pos.log 2>&1; grep "gmpsvm trace\] pair (" $out/m8m_trace_$pos.log; tail -1 $out/m8m_trace_$pos.log | cut -c1-300
done
