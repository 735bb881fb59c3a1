#!/bin/bash
# calib32: the linear screen's top candidates with the deep input-run tiles (ranking-stage data)
O=gpurun_out/exp52; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python tools/calib_sweep.py --group c3 --max-cand 48 --top --reps 5 > $O/calib32_c3top.jsonl 2> $O/c3.err
timeout 900 python tools/calib_sweep.py --group c2 --max-cand 40 --top --reps 5 > $O/calib32_c2top.jsonl 2> $O/c2.err
timeout 900 python tools/calib_sweep.py --group c4 --max-cand 40 --top --reps 5 > $O/calib32_c4top.jsonl 2> $O/c4.err
timeout 1200 python tools/calib_sweep.py --recipe 100 --seed 15 --max-cand 48 --top --reps 5 > $O/calib32_recipetop.jsonl 2> $O/recipetop.err
