#!/bin/bash
# round 2, call 40: single use on 16^6 at the fast-2 planning level (refine 8 / rank 6) vs the
# default fast-1 level for passes of 35-150 us -- same box, back to back
O=gpurun_out/r2e40
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/singleuse.cpp \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/singleuse
timeout 900 tools/singleuse 20 3 < tools/sweep16_shapes.txt > $O/singleuse_720-16_f1.txt 2>&1
TTLG_FAST_LEVEL=2 timeout 900 tools/singleuse 20 3 < tools/sweep16_shapes.txt > $O/singleuse_720-16_f2.txt 2>&1
timeout 300 tools/singleuse 50 5 < tools/c3_shapes.txt > $O/singleuse_c3_f1.txt 2>&1
TTLG_FAST_LEVEL=2 timeout 300 tools/singleuse 50 5 < tools/c3_shapes.txt > $O/singleuse_c3_f2.txt 2>&1
