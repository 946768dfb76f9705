python tools/sweep.py "" "ws_size=160" "ws_size=176" "ws_size=208" 2>&1 | grep total
for r in 0.05 0.15 0.2; do echo ratio $r; GMPSVM_LOCAL_RATIO=$r python tools/sweep.py "" 2>&1 | grep total; done
python bench.py --steps 5 --warmup 3 > gpurun_out/bench2.json 2> gpurun_out/bench2.err; cat gpurun_out/bench2.json
