#!/bin/bash
out=gpurun_out/${1:-dec2}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for D in 0 4 6 5 3; do
GMPSVM_I8_DIAG=$D python tools/prof_dec.py --reps 3 > $out/d$D.log 2>&1; echo "DIAG=$D $(tail -1 $out/d$D.log | grep -o '"dec_ms": [0-9.]*')"
done
