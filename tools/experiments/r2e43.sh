#!/bin/bash
# round 2, call 43: single use on configs 3 / 4 at the final planning levels; every candidate
# of the config-4 16-byte-element cases below 0.9 of D2D (4011, 4021)
O=gpurun_out/r2e43
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/singleuse.cpp \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/singleuse
timeout 300 tools/singleuse 50 5 < tools/c4_shapes.txt > $O/singleuse_c4.txt 2>&1
timeout 300 tools/singleuse 50 5 < tools/c3_shapes.txt > $O/singleuse_c3.txt 2>&1
timeout 900 python tools/bulk_sweep.py --workload c4 --variants 0,7 --only 4011,4021,4007 --max-cand 200 --reps 5 > $O/sweep_c4w16.jsonl 2> $O/sweep_c4w16.err
