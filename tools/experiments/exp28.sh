#!/bin/bash
# parity (incl. k_quad), bench, focused sweeps (c2 subset + c4) on the k_quad build
O=gpurun_out/exp28; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
TTLG_BENCH_CASES=1 timeout 900 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench.json 2> $O/bench.err
TTLG_BENCH_CASES=1 timeout 900 python bench.py --workload smallfvi --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_smallfvi.json 2> $O/bench_smallfvi.err
timeout 900 python tools/calib_sweep.py --group c2 --ids 2001,2016,2019,2024,2034,2035,2046,2047,2053 --max-cand 400 --reps 5 > $O/sweep.jsonl 2> $O/sweep.err
timeout 900 python tools/calib_sweep.py --group c4 --max-cand 400 --reps 5 > $O/sweep_c4.jsonl 2> $O/sweep_c4.err
for v in 1 3; do python tools/sweep.py --case 5120,5120:1,0:8 --case 4,4096,4096:1,2,0:4 --case 8,4096,4096:2,1,0:4 --hints "{\"variant\": $v}" --reps 20 >> $O/t.log 2>&1; done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_ -s 3 -c 1 -o $O/p2 \
    python tools/sweep.py --case 5120,5120:1,0:8 --hints '{"schema": "OD", "in_dim": 0, "in_block": 64, "out_dim": 0, "out_block": 32, "threads": 256, "variant": 3}' --reps 2 > $O/p2.log 2>&1
