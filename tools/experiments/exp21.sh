#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python tools/calib_sweep.py --group c2 --max-cand 40 --top --reps 7 > gpurun_out/calib21_c2.jsonl 2> gpurun_out/calib21_c2.err
timeout 900 python tools/calib_sweep.py --group c4 --max-cand 40 --top --reps 7 > gpurun_out/calib21_c4.jsonl 2> gpurun_out/calib21_c4.err
timeout 1500 python tools/calib_sweep.py --recipe 200 --seed 7 --max-cand 40 --top --reps 7 > gpurun_out/calib21_recipe.jsonl 2> gpurun_out/calib21_recipe.err
timeout 900 python tools/calib_sweep.py --group c3 --max-cand 40 --top --reps 5 > gpurun_out/calib21_c3.jsonl 2> gpurun_out/calib21_c3.err
