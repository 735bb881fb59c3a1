#!/bin/bash
# round 2, call 42: rank-dependent second fast level (rank >= 4 below 45 us) and the full k_vec
# list on level 1: single use on configs 3 / 4 and the 720-perm sweeps
O=gpurun_out/r2e42
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/singleuse.cpp \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/singleuse
timeout 300 tools/singleuse 50 5 < tools/c4_shapes.txt > $O/singleuse_c4.txt 2>&1
timeout 300 tools/singleuse 50 5 < tools/c3_shapes.txt > $O/singleuse_c3.txt 2>&1
timeout 900 tools/singleuse 20 3 < tools/sweep16_shapes.txt > $O/singleuse_720-16.txt 2>&1
timeout 900 tools/singleuse 20 3 < tools/sweep15_shapes.txt > $O/singleuse_720-15.txt 2>&1
timeout 900 tools/singleuse 20 3 < tools/sweep17_shapes.txt > $O/singleuse_720-17.txt 2>&1
