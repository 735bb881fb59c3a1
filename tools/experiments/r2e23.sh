#!/bin/bash
# round 2, call 23: single use with the second fast-effort level (passes < 35 us: refine 8,
# rank 6) on the 15^6 sweep (the only one under the threshold) and c3 (unaffected control)
O=gpurun_out/r2e23
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
build() { g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/$1.cpp \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/$1 2>/dev/null; }
build singleuse
timeout 900 tools/singleuse 20 3 < tools/sweep15_shapes.txt > $O/singleuse_720-15.txt 2>&1
timeout 300 tools/singleuse 50 5 < tools/c3_shapes.txt > $O/singleuse_c3.txt 2>&1
tail -3 $O/singleuse_720-15.txt
bash tools/experiments/r2e21.sh
