#!/bin/bash
# exchange choice + strided parity (full GPU suite), sharded bench, TTC short-list sweep (model regret study)
O=gpurun_out/exp41
mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 900 python -m pytest tests/test_strided.py tests/test_sharded.py -m gpu -q > $O/pytest_new.log 2>&1; echo "rc=$?" >> $O/pytest_new.log
timeout 600 python bench.py --workload sharded --steps 5 --warmup 3 > $O/bench_sharded.json 2> $O/bench_sharded.err
timeout 900 python tools/calib_sweep.py --group c2 --max-cand 24 --top > $O/c2_top.jsonl 2> $O/c2_top.err
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
