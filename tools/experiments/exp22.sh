#!/bin/bash
# focused candidate sweep on representative TTC cases (new k_pipe mappings)
O=gpurun_out/exp22; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 900 python tools/calib_sweep.py --group c2 --ids 2001,2016,2019,2024,2034,2035,2046,2047,2053 --max-cand 400 --reps 5 > $O/sweep.jsonl 2> $O/sweep.err
./tools/copybench > $O/copybench.txt 2>&1
