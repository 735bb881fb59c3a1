#!/bin/bash
# focused candidate sweep on representative TTC cases (new k_pipe mappings)
O=gpurun_out/exp24; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 900 python tools/calib_sweep.py --group c2 --ids 2001,2016,2019,2024,2034,2035,2046,2047,2053 --max-cand 400 --reps 5 > $O/sweep.jsonl 2> $O/sweep.err
TTLG_BENCH_CASES=1 timeout 900 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench.json 2> $O/bench.err
