#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python tools/sweep.py --group c2 --reps 10 --hints '{}' --hints '{"variant":1}' > gpurun_out/sweep2_c2.jsonl 2> gpurun_out/sweep2_c2.err
timeout 1500 python tools/calib_sweep.py --group c2 --max-cand 60 > gpurun_out/calib_c2.jsonl 2> gpurun_out/calib_c2.err
