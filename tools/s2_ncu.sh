#!/bin/bash
# ncu captures of the solver kernels (host-driven loop, GMPSVM_NOGRAPH=1) and of krow / dec_i8 in the default step
out=gpurun_out/${1:-ncu}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
GMPSVM_NOGRAPH=1 timeout 300 python tools/prof_step.py --ws-size 192 > $out/nograph.log 2>&1; tail -2 $out/nograph.log
for k in ws_select_kernel ws_smo_kernel ws_fupdate_kernel ws_gather_kernel; do
GMPSVM_NOGRAPH=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 100 -c 1 -f -o $out/$k python tools/prof_step.py --ws-size 192 > $out/ncu_$k.log 2>&1; tail -1 $out/ncu_$k.log
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:krow_tc_kernel -s 1 -c 1 -f -o $out/krow_tc python tools/prof_step.py --ws-size 192 > $out/ncu_krow.log 2>&1; tail -1 $out/ncu_krow.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dec_i8_kernel -c 1 -f -o $out/dec_i8 python tools/prof_dec.py --reps 1 > $out/ncu_dec.log 2>&1; tail -1 $out/ncu_dec.log
ls -la $out
