out=gpurun_out/$1; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_edge.py -x -q > $out/pytest.log 2>&1; echo "rc=$?" >> $out/pytest.log
timeout 900 python tools/shard_probe.py mnist 3 > $out/shard.log 2>&1
tail -2 $out/pytest.log; cat $out/shard.log | cut -c1-3000
