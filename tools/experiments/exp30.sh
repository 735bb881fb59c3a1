#!/bin/bash
# calibration sweep on the final k_quad / padding code (calib30): spread + top of the linear screen
O=gpurun_out/exp30; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python tools/calib_sweep.py --group c2 --max-cand 200 --reps 5 > $O/calib30_c2.jsonl 2> $O/c2.err
timeout 900 python tools/calib_sweep.py --group c2 --max-cand 40 --top --reps 5 > $O/calib30_c2top.jsonl 2> $O/c2top.err
timeout 900 python tools/calib_sweep.py --group c4 --max-cand 200 --reps 5 > $O/calib30_c4.jsonl 2> $O/c4.err
timeout 900 python tools/calib_sweep.py --group c3 --max-cand 120 --reps 5 > $O/calib30_c3.jsonl 2> $O/c3.err
timeout 1500 python tools/calib_sweep.py --recipe 160 --seed 12 --max-cand 120 --reps 5 > $O/calib30_recipe.jsonl 2> $O/recipe.err
timeout 900 python tools/calib_sweep.py --recipe 80 --seed 13 --max-cand 40 --top --reps 5 > $O/calib30_recipetop.jsonl 2> $O/recipetop.err
