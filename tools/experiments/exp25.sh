#!/bin/bash
# calibration sweep on the lean k_pipe kernels (calib25)
O=gpurun_out/exp25; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python tools/calib_sweep.py --group c2 --max-cand 200 --reps 5 > $O/calib25_c2.jsonl 2> $O/c2.err
timeout 900 python tools/calib_sweep.py --group c4 --max-cand 200 --reps 5 > $O/calib25_c4.jsonl 2> $O/c4.err
timeout 900 python tools/calib_sweep.py --group c3 --max-cand 120 --reps 5 > $O/calib25_c3.jsonl 2> $O/c3.err
timeout 1500 python tools/calib_sweep.py --recipe 160 --seed 11 --max-cand 120 --reps 5 > $O/calib25_recipe.jsonl 2> $O/recipe.err
