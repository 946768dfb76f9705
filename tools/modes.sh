python tools/sweep.py "" 2>&1 | grep total
python bench.py --steps 5 --warmup 3 > gpurun_out/bench3.json 2> gpurun_out/bench3.err; cat gpurun_out/bench3.json
