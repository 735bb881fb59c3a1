#!/bin/bash
# round 2, call 41: second fast planning level up to 45-us passes (16^6 fp64, config-4 n0 = 2):
# single use on config 4 (new default vs level 1 forced), 16^6 sweep and config 3 at the new default
O=gpurun_out/r2e41
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/singleuse.cpp \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/singleuse
timeout 300 tools/singleuse 50 5 < tools/c4_shapes.txt > $O/singleuse_c4.txt 2>&1
TTLG_FAST_LEVEL=1 timeout 300 tools/singleuse 50 5 < tools/c4_shapes.txt > $O/singleuse_c4_f1.txt 2>&1
timeout 300 tools/singleuse 50 5 < tools/c3_shapes.txt > $O/singleuse_c3.txt 2>&1
timeout 900 tools/singleuse 20 3 < tools/sweep16_shapes.txt > $O/singleuse_720-16.txt 2>&1
timeout 900 tools/singleuse 20 3 < tools/sweep15_shapes.txt > $O/singleuse_720-15.txt 2>&1
