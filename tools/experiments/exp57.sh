#!/bin/bash
# round check s4e (all GPU tests incl. strided torch views) + config-3 suite + sharded
bash tools/round_check.sh s4e
O=gpurun_out/s4e
timeout 900 python tools/suite.py --groups c3 --out $O/suite_c3.jsonl > $O/suite_c3.log 2>&1
timeout 600 python bench.py --workload sharded --steps 5 --warmup 3 > $O/bench_sharded.json 2> $O/bench_sharded.err
