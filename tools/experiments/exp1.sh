#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python tools/sweep.py --group c2 --d2d --reps 10 --hints '{}' --hints '{"variant":1}' --hints '{"variant":2}' --hints '{"variant":3}' > gpurun_out/sweep_c2.jsonl 2> gpurun_out/sweep_c2.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_ -s 3 -c 1 -o gpurun_out/prof_od python tools/sweep.py --case 5120,5120:1,0:8 --reps 2 > gpurun_out/ncu_od.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_ -s 3 -c 1 -o gpurun_out/prof_fml python tools/sweep.py --case 320,320,256:0,2,1:8 --reps 2 > gpurun_out/ncu_fml.log 2>&1
