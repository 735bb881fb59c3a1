#!/bin/bash
# A/B: tile digits ordered by stride (TTLG_GRID_ORDER=1, new default) vs input order (0)
O=gpurun_out/exp43
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for go in 0 1; do
  for w in ttc57 ccsdt smallfvi; do
    TTLG_GRID_ORDER=$go TTLG_BENCH_CASES=1 timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_${w}_go$go.json 2> $O/bench_${w}_go$go.err
  done
  TTLG_GRID_ORDER=$go timeout 600 python bench.py --workload sharded --steps 5 --warmup 3 --no-emulate > $O/bench_sharded_go$go.json 2> $O/bench_sharded_go$go.err
done
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
