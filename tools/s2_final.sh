#!/bin/bash
# Round-2 evidence (session 2): full GPU suite, smoke, bench (default + 20 steps), reference arm,
# launch list, ncu captures of krow / dec_i8 and of the solver kernels (host-driven loop)
out=gpurun_out/${1:-final}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log; tail -3 $out/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.log 2>&1; tail -1 $out/smoke.log
timeout 900 python bench.py > $out/bench_default.json 2> $out/bench_default.err; head -c 300 $out/bench_default.json; echo
timeout 900 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $out/bench_20.json 2> $out/bench_20.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > $out/bench_reference.json 2> $out/bench_reference.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $out/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > $out/b_ncu.log 2>&1
python tools/launch_sum.py $out/launches.csv > $out/launches_sum.txt 2>&1; head -14 $out/launches_sum.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:krow_tc_kernel -s 1 -c 1 -f -o $out/krow_tc python tools/prof_step.py --ws-size 192 > $out/ncu_krow.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dec_i8_kernel -c 1 -f -o $out/dec_i8 python tools/prof_dec.py --reps 1 > $out/ncu_dec.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:krow_csr_kernel -c 1 -f -o $out/krow_csr python tools/sparse_probe.py --n 20000 --reps 1 > $out/ncu_csr.log 2>&1
for k in ws_select_kernel ws_smo_kernel ws_fupdate_kernel ws_gather_kernel; do
GMPSVM_NOGRAPH=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 100 -c 1 -f -o $out/$k python tools/prof_step.py --ws-size 192 > $out/ncu_$k.log 2>&1
done
ls -la $out
