#!/bin/bash
# Parity + bench on 1 B200 (under gpurun): bash tools/quick_check.sh TAG [extra bench workloads...]
T=${1:-q}; shift
O=gpurun_out/$T
mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
TTLG_BENCH_CASES=1 timeout 900 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench.json 2> $O/bench.err
for w in "$@"; do
  TTLG_BENCH_CASES=1 timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_$w.json 2> $O/bench_$w.err
done
