#!/bin/bash
# round check s4f (all GPU tests incl. k_inter) + config-3 suite + sharded + N3 sweeps
bash tools/round_check.sh s4f
O=gpurun_out/s4f
timeout 900 python tools/suite.py --groups c3 --out $O/suite_c3.jsonl > $O/suite_c3.log 2>&1
timeout 600 python bench.py --workload sharded --steps 5 --warmup 3 > $O/bench_sharded.json 2> $O/bench_sharded.err
timeout 600 python tools/fig5.py > $O/fig5.jsonl 2> $O/fig5.err
