#!/bin/bash
# parity on the generalised k_quad, then the calibration sweep (calib29)
O=gpurun_out/exp29; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; rc=$?; echo "pytest rc=$rc" >> $O/pytest_gpu.log
[ $rc -ne 0 ] && exit 1
timeout 1200 python tools/calib_sweep.py --group c2 --max-cand 200 --reps 5 > $O/calib29_c2.jsonl 2> $O/c2.err
timeout 900 python tools/calib_sweep.py --group c4 --max-cand 200 --reps 5 > $O/calib29_c4.jsonl 2> $O/c4.err
timeout 900 python tools/calib_sweep.py --group c3 --max-cand 120 --reps 5 > $O/calib29_c3.jsonl 2> $O/c3.err
timeout 1500 python tools/calib_sweep.py --recipe 160 --seed 11 --max-cand 120 --reps 5 > $O/calib29_recipe.jsonl 2> $O/recipe.err
