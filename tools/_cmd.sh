out=gpurun_out/$1; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
echo "1cta+hints" >> $out/diag.log; GMPSVM_KROW_CTA=1 timeout 120 python tools/krow_check.py 2>&1 | grep krow | tail -1 >> $out/diag.log
for dg in 4 68 69 5; do echo "diag $dg" >> $out/diag.log; GMPSVM_KROW_DIAG=$dg timeout 120 python tools/krow_check.py 2>&1 | grep krow | tail -1 >> $out/diag.log; done
cat $out/diag.log
