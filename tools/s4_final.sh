#!/bin/bash
# end-of-round evidence: full GPU suite, smoke, bench lines, reference arm, launch list, ncu of the top kernels
out=gpurun_out/${1:-final4}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log; tail -3 $out/pytest.log
bash tools/s3_bench_final.sh ${1:-final4}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:krow_tc_kernel -s 1 -c 1 -f -o $out/krow_tc python tools/prof_step.py --ws-size 192 > $out/ncu_krow.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dec_i8_kernel -c 1 -f -o $out/dec_i8 python tools/prof_dec.py --reps 1 > $out/ncu_dec.log 2>&1
for k in ws_select_kernel ws_smo_kernel ws_fupdate_kernel ws_gather_kernel; do
GMPSVM_NOGRAPH=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 100 -c 1 -f -o $out/$k python tools/prof_step.py --ws-size 192 > $out/ncu_$k.log 2>&1
done
ls $out
