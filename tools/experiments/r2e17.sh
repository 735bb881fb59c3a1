#!/bin/bash
# round 2, call 17: k_vec-only challenge; single-use fast effort = refine 12 / rank 8 without the
# padding search; single-use tables, per-case tables, model error on c1 / fig13
mkdir -p gpurun_out/r2e17
build() { g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/$1.cpp \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/$1 2>/dev/null; }
build fig12; build singleuse
timeout 300 tools/singleuse 50 5 < tools/c3_shapes.txt > gpurun_out/r2e17/singleuse_c3.txt 2>&1
for e in 15 16 17; do timeout 900 tools/singleuse 20 3 < tools/sweep${e}_shapes.txt > gpurun_out/r2e17/singleuse_720-$e.txt 2>&1; done
timeout 600 tools/fig12 3 > gpurun_out/r2e17/fig12.jsonl 2>&1
for w in c3 720-16; do
  timeout 600 python tools/cases.py --workload $w --out gpurun_out/r2e17/cases_$w.json > gpurun_out/r2e17/cases_$w.log 2>&1
  tail -1 gpurun_out/r2e17/cases_$w.log | cut -c1-250
done
