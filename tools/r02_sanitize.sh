#!/bin/bash
# compute-sanitizer on the T1-shaped workload (tools/sanitize.py).  racecheck / synccheck instrument
# shared memory and barriers and do not run the tcgen05 / TMA kernels, so those two (and initcheck,
# which does not see TMA bulk stores) run with the SIMT kernel values / per-thread K stores / FP64
# decision values; memcheck runs the default path.
out=gpurun_out/${1:-san}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 900 compute-sanitizer --tool memcheck --print-limit 50 python tools/sanitize.py > $out/memcheck.log 2>&1; echo "memcheck rc=$?" >> $out/memcheck.log
GMPSVM_KROW_STORE=st GMPSVM_DEC=f64 timeout 900 compute-sanitizer --tool initcheck --print-limit 50 python tools/sanitize.py > $out/initcheck.log 2>&1; echo "initcheck rc=$?" >> $out/initcheck.log
for tool in racecheck synccheck; do
  env GMPSVM_KROW=simt GMPSVM_DEC=f64 $RC_ENV timeout 1200 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize.py > $out/$tool.log 2>&1
  echo "$tool rc=$?" >> $out/$tool.log
done
for f in memcheck initcheck racecheck synccheck; do echo "== $f"; grep -E "SUMMARY|rc=|Error|error" $out/$f.log | head -6; done
