#!/bin/bash
# class-means staging change: parity + schedule tests, a quick bench, the launch list
out=gpurun_out/${1:-s5cm}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_schedule.py -m gpu -q -x > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log; tail -2 $out/pytest.log
bash tools/s2_quick.sh ${1:-s5cm}_q
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $out/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > $out/b_ncu.log 2>&1
python tools/launch_sum.py $out/launches.csv > $out/launches_sum.txt 2>&1; grep -i class_means $out/launches_sum.txt; head -12 $out/launches_sum.txt
