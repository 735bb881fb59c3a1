#!/bin/bash
# round 2, call 51: sanity on the final commit -- smoke, the full GPU suite, the headline bench line
O=gpurun_out/r2e51
mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
TTLG_BENCH_CASES=1 timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
timeout 2400 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -2 $O/pytest_gpu.log; tail -1 $O/smoke.log
