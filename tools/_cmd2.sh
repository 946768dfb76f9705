out=gpurun_out/$1; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > $out/pytest.log 2>&1; echo "pytest rc=$?" >> $out/pytest.log
timeout 600 python tools/sweep.py "ws_size=0" > $out/sweep.log 2>&1
timeout 900 python tools/scale_probe.py covtype 581012 58101 > $out/cov.log 2>&1
timeout 900 python tools/scale_probe.py mnist8m 1000000 10000 > $out/m8m1m.log 2>&1
timeout 900 python tools/scale_probe.py mnist 200000 10000 > $out/mn200k.log 2>&1
tail -2 $out/pytest.log; cut -c1-200 $out/sweep.log
for f in $out/cov.log $out/m8m1m.log $out/mn200k.log; do echo $f; grep -o '"train_s[^,]*\|"predict_s[^,]*\|"outer_iters_max[^,]*\|"t_solver_ms[^,]*\|"test_acc[^,]*\|"n_sv[^,]*' $f | tr '\n' ' '; echo; done
