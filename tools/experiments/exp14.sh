#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 1200 python tools/calib_sweep.py --group c2 --max-cand 160 > gpurun_out/calib14_c2.jsonl 2> gpurun_out/calib14_c2.err
timeout 900 python tools/calib_sweep.py --group c4 --max-cand 100 > gpurun_out/calib14_c4.jsonl 2> gpurun_out/calib14_c4.err
timeout 1200 python tools/calib_sweep.py --recipe 80 --seed 1 --max-cand 80 > gpurun_out/calib14_recipe.jsonl 2> gpurun_out/calib14_recipe.err
timeout 900 python tools/calib_sweep.py --group c3 --max-cand 60 --stride 3 > gpurun_out/calib14_c3.jsonl 2> gpurun_out/calib14_c3.err
