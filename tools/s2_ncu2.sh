#!/bin/bash
out=gpurun_out/${1:-ncu2}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for k in ws_select_kernel ws_smo_kernel ws_fupdate_kernel ws_gather_kernel; do
GMPSVM_NOGRAPH=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 100 -c 1 -f -o $out/$k python tools/prof_step.py --ws-size 192 > $out/ncu_$k.log 2>&1; tail -1 $out/ncu_$k.log
done
