out=gpurun_out/$1; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q > $out/pytest.log 2>&1; echo "rc=$?" >> $out/pytest.log
echo base >> $out/ov.log; timeout 300 python tools/sweep.py "ws_size=192" >> $out/ov.log 2>&1
for r in 0 8 16 32; do echo "overlap reserve $r" >> $out/ov.log; GMPSVM_OVERLAP=1 GMPSVM_KROW_RESERVE=$r timeout 300 python tools/sweep.py "ws_size=192" >> $out/ov.log 2>&1; done
GMPSVM_SMO_PHASES=1 timeout 300 python tools/prof_step.py --ws-size 192 --reps 2 2>&1 | grep -i sigmoid >> $out/ov.log
tail -2 $out/pytest.log; cat $out/ov.log | cut -c1-190
