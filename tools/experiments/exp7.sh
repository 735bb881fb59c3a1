#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python tools/sweep.py --case 26214400:0:8 --d2d --reps 10 --hints '{}' --hints '{"threads":512}' --hints '{"in_block":4096}' --hints '{"in_block":16384}'  > gpurun_out/sweep7_copy.jsonl 2>&1
timeout 1500 python tools/calib_sweep.py --group c2 --max-cand 40 --threads 256,512 > gpurun_out/calib7_c2.jsonl 2> gpurun_out/calib7_c2.err
