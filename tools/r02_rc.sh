#!/bin/bash
out=gpurun_out/${1:-rc}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q -k "rowcache or large" > $out/focus.log 2>&1; echo "focus rc=$?" >> $out/focus.log; tail -4 $out/focus.log
timeout 900 python tools/scale_probe.py mnist8m 1000000 10000 > $out/m8m_1m.log 2>&1; tail -1 $out/m8m_1m.log | cut -c1-700
timeout 900 python tools/scale_probe.py covtype 581012 58101 > $out/covtype.log 2>&1; tail -1 $out/covtype.log | cut -c1-500
