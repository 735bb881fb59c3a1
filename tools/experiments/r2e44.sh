#!/bin/bash
# round 2, call 44: final code -- smoke, the full GPU suite, single use on configs 3 / 4 and the
# 15^6 / 16^6 sweeps (fast-level k_vec pre-ranking), headline bench line
O=gpurun_out/r2e44
mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/singleuse.cpp \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/singleuse
timeout 300 tools/singleuse 50 5 < tools/c4_shapes.txt > $O/singleuse_c4.txt 2>&1
timeout 300 tools/singleuse 50 5 < tools/c3_shapes.txt > $O/singleuse_c3.txt 2>&1
timeout 900 tools/singleuse 20 3 < tools/sweep16_shapes.txt > $O/singleuse_720-16.txt 2>&1
timeout 900 tools/singleuse 20 3 < tools/sweep15_shapes.txt > $O/singleuse_720-15.txt 2>&1
timeout 900 tools/singleuse 20 3 < tools/sweep17_shapes.txt > $O/singleuse_720-17.txt 2>&1
TTLG_BENCH_CASES=1 timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
timeout 2400 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -2 $O/pytest_gpu.log; tail -1 $O/smoke.log
