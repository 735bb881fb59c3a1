#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
TTLG_BENCH_CASES=1 timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 1500 python tools/suite.py --groups c1,c2,c3,c4,c5,fig13,fig5 --out gpurun_out/suite.jsonl > gpurun_out/suite.err 2>&1
