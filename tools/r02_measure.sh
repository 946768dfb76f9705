#!/bin/bash
# Round-2 measurement batch: full CPU baseline (config 3), letter full, MNIST8M-shaped probes.
out=gpurun_out/${1:-meas}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
(timeout 2400 python tools/cpu_full.py mnist 1e-3 $out/cpu_full_mnist.json > $out/cpu_full.log 2>&1 &)
timeout 600 python tools/scale_probe.py letter 20000 5000 > $out/letter.log 2>&1; tail -1 $out/letter.log
GMPSVM_TRACE=0 timeout 1200 python tools/scale_probe.py mnist8m 1000000 10000 > $out/m8m_1m.log 2>&1; grep -v "^generated" $out/m8m_1m.log | tail -3
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv --log-file $out/m8m_1m_launches.csv python tools/scale_probe.py mnist8m 1000000 10000 > $out/m8m_ncu.log 2>&1
python tools/launch_sum.py $out/m8m_1m_launches.csv | head -20
while pgrep -f cpu_full.py > /dev/null; do sleep 10; done
cat $out/cpu_full.log
