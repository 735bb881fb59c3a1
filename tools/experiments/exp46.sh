#!/bin/bash
# calib31: the linear screen's top candidates on the current kernels (ranking-stage data)
O=gpurun_out/exp46; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python tools/calib_sweep.py --group c3 --max-cand 60 --top --reps 5 > $O/calib31_c3top.jsonl 2> $O/c3.err
timeout 900 python tools/calib_sweep.py --group c2 --max-cand 40 --top --reps 5 > $O/calib31_c2top.jsonl 2> $O/c2.err
timeout 900 python tools/calib_sweep.py --group c4 --max-cand 60 --top --reps 5 > $O/calib31_c4top.jsonl 2> $O/c4.err
timeout 1200 python tools/calib_sweep.py --recipe 100 --seed 14 --max-cand 48 --top --reps 5 > $O/calib31_recipetop.jsonl 2> $O/recipetop.err
