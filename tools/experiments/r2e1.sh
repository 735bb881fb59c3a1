#!/bin/bash
# round 2, call 1: full GPU suite incl. whole-tensor full-size parity, smoke
set -x
mkdir -p gpurun_out/r2e1
nproc > gpurun_out/r2e1/nproc.txt; free -g >> gpurun_out/r2e1/nproc.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2e1/smoke.log 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q --durations=40 > gpurun_out/r2e1/gputest.log 2>&1
echo rc=$?
tail -50 gpurun_out/r2e1/gputest.log
