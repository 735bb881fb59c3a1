#!/bin/bash
# round 2, call 2: per-case floor table (graph of R launches per case vs same-size D2D graph)
# for every workload; single-use vs repeated-use through the C ABI (config 3)
mkdir -p gpurun_out/r2e2
g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/singleuse.cpp \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/singleuse 2>/dev/null
tools/singleuse 50 5 < tools/c3_shapes.txt > gpurun_out/r2e2/singleuse_c3.txt 2>&1
for w in c2 c3 c4 720-15 720-16 720-17 fig13 c1; do
  python tools/cases.py --workload $w --out gpurun_out/r2e2/cases_$w.json > gpurun_out/r2e2/cases_$w.log 2>&1
  tail -1 gpurun_out/r2e2/cases_$w.log | cut -c1-600
done
cat gpurun_out/r2e2/singleuse_c3.txt
