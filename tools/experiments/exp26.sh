#!/bin/bash
# parity (incl. k_quad), bench, focused sweeps (c2 subset + c4) on the k_quad build
O=gpurun_out/exp26; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
TTLG_BENCH_CASES=1 timeout 900 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench.json 2> $O/bench.err
TTLG_BENCH_CASES=1 timeout 900 python bench.py --workload smallfvi --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_smallfvi.json 2> $O/bench_smallfvi.err
timeout 900 python tools/calib_sweep.py --group c2 --ids 2001,2016,2019,2024,2034,2035,2046,2047,2053 --max-cand 400 --reps 5 > $O/sweep.jsonl 2> $O/sweep.err
timeout 900 python tools/calib_sweep.py --group c4 --max-cand 400 --reps 5 > $O/sweep_c4.jsonl 2> $O/sweep_c4.err
