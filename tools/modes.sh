python -m pytest tests -m gpu -x -q 2>&1 | tail -3
python tools/sweep.py "" "ws_size=192" "ws_size=160" 2>&1 | grep total
GMPSVM_SMO_PHASES=1 python tools/sweep.py "" 2>&1 | grep -v "^$" | head -3
GMPSVM_TRACE=32 python tools/sweep.py "" 2>&1 | grep trace | tail -1
