#!/bin/bash
# strided sub-tensor plans + fused p2p exchange: GPU parity, 2-process IPC test, sharded bench
O=gpurun_out/exp40
mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 900 python -m pytest tests/test_strided.py tests/test_sharded.py -m gpu -x -q > $O/pytest_new.log 2>&1; echo "rc=$?" >> $O/pytest_new.log
timeout 600 python bench.py --workload sharded --steps 5 --warmup 3 > $O/bench_sharded.json 2> $O/bench_sharded.err
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
