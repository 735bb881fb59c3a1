#!/bin/bash
# final round check s4g: GPU tests, smoke, bench (+ reference arm, ncu), suites, sharded, k_inter at n1 = 7, 8
bash tools/round_check.sh s4g
O=gpurun_out/s4g
timeout 900 python tools/suite.py --groups c3 --out $O/suite_c3.jsonl > $O/suite_c3.log 2>&1
timeout 600 python bench.py --workload sharded --steps 5 --warmup 3 > $O/bench_sharded.json 2> $O/bench_sharded.err
for n1 in 7 8; do
  python tools/sweep.py --case 16777216,$n1:1,0:4 --reps 10 >> $O/inter.jsonl 2>> $O/inter.err
  python tools/sweep.py --case 16777216,$n1:1,0:4 --reps 10 --hints '{"variant": 2}' >> $O/inter_pipe.jsonl 2>> $O/inter.err
done
