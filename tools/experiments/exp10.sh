#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 -o gpurun_out/p10_pipe2001 python tools/sweep.py --case 5120,5120:1,0:8 --reps 1 --hints '{"schema":"OD","in_dim":0,"in_block":128,"out_dim":0,"out_block":64,"threads":512,"variant":2}' > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 -o gpurun_out/p10_direct2004 python tools/sweep.py --group c2 --limit 4 --stride 1 --reps 1 > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "execute_host" > gpurun_out/pytest_host.log 2>&1
