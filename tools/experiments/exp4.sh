#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 1500 python tools/calib_sweep.py --group c2 --max-cand 60 > gpurun_out/calib5_c2.jsonl 2> gpurun_out/calib5_c2.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 -o gpurun_out/p5_od32x128 python tools/sweep.py --case 5120,5120:1,0:8 --reps 1 --hints '{"schema":"OD","in_dim":0,"in_block":32,"out_dim":0,"out_block":128}' > /dev/null 2>&1
