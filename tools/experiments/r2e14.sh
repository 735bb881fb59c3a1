#!/bin/bash
# round 2, call 14: full check -- GPU suite incl. whole-tensor parity, per-case tables of every
# workload, single-use through the C ABI, Fig. 12, default bench
mkdir -p gpurun_out/r2e14
timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/r2e14/gputest.log 2>&1
echo "gputest rc=$?"; tail -2 gpurun_out/r2e14/gputest.log
build() { g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/$1.cpp \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/$1 2>/dev/null; }
build fig12; build singleuse
timeout 300 tools/singleuse 50 5 < tools/c3_shapes.txt > gpurun_out/r2e14/singleuse_c3.txt 2>&1
for e in 15 16 17; do timeout 900 tools/singleuse 20 3 < tools/sweep${e}_shapes.txt > gpurun_out/r2e14/singleuse_720-$e.txt 2>&1; done
timeout 600 tools/fig12 3 > gpurun_out/r2e14/fig12.jsonl 2>&1
for w in c2 c3 c4 c1 fig13 720-15 720-16 720-17; do
  timeout 600 python tools/cases.py --workload $w --out gpurun_out/r2e14/cases_$w.json > gpurun_out/r2e14/cases_$w.log 2>&1
  tail -1 gpurun_out/r2e14/cases_$w.log | cut -c1-250
done
timeout 900 python bench.py > gpurun_out/r2e14/bench.json 2> gpurun_out/r2e14/bench.err
timeout 900 python bench.py --workload sharded > gpurun_out/r2e14/bench_sharded.json 2> gpurun_out/r2e14/bench_sharded.err
tail -c 600 gpurun_out/r2e14/bench.json; tail -c 1500 gpurun_out/r2e14/bench_sharded.json
