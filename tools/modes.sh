python -m pytest tests -m gpu -x -q 2>&1 | tail -3
python tools/sweep.py "" "ws_size=192" 2>&1 | grep total
GMPSVM_UNROLL=1 python tools/sweep.py "" 2>&1 | grep total
GMPSVM_UNROLL=4 python tools/sweep.py "" 2>&1 | grep total
GMPSVM_SOLVER=streams python tools/sweep.py "" 2>&1 | grep total
GMPSVM_TRACE=32 python tools/sweep.py "" 2>&1 | grep trace | tail -1
