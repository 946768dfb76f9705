python -m pytest tests -m gpu -x -q 2>&1 | tail -3
python tools/krow_check.py 2>&1 | tail -3
GMPSVM_SPLIT=tf32 python tools/krow_check.py 2>&1 | tail -3
python tools/sweep.py "" 2>&1 | grep total
python tools/prof_step.py 2>&1 | tail -1
