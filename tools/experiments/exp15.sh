#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
g++ -O2 -std=c++17 -I include tools/plantime.cpp -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -Wl,-rpath,'$ORIGIN/../paper_conf_ipps_veduradasskhpkn18_b200' -o tools/plantime
printf "8 6 16 16 16 16 16 16 0 2 5 1 4 3\n8 6 16 16 16 16 16 16 4 1 2 5 3 0\n8 6 24 24 24 24 24 24 4 1 2 5 3 0\n8 2 5120 5120 1 0\n8 6 16 20 16 20 16 16 2 0 4 1 5 3\n4 5 64 64 64 64 128 4 3 2 1 0\n" | ./tools/plantime > gpurun_out/plantime.txt 2>&1
timeout 1500 python tools/suite.py --groups c1,c2,c3,c4,c5,fig13,fig5 --out gpurun_out/suite.jsonl > gpurun_out/suite.err 2>&1
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
