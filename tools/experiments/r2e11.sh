#!/bin/bash
# round 2, call 11: N3 (Fig. 12 curve, single-use 720-perm sweeps), compute-sanitizer
# over every kernel family, ncu captures of k_vec / k_bulk, smoke
mkdir -p gpurun_out/r2e11
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2e11/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/r2e11/smoke.log
build() { g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/$1.cpp \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/$1 2>/dev/null; }
build fig12; build singleuse
timeout 600 tools/fig12 3 > gpurun_out/r2e11/fig12.jsonl 2>&1; echo "fig12 rc=$?"
for e in 15 16 17; do timeout 900 tools/singleuse 20 3 < tools/sweep${e}_shapes.txt > gpurun_out/r2e11/singleuse_720-$e.txt 2>&1; echo "single $e rc=$?"; done
timeout 300 tools/singleuse 50 5 < tools/c3_shapes.txt > gpurun_out/r2e11/singleuse_c3.txt 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_cases.py > gpurun_out/r2e11/san_$tool.log 2>&1
  echo "sanitizer $tool rc=$?"; tail -2 gpurun_out/r2e11/san_$tool.log
done
prof() {  # tag workload case hints
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 \
    -o /tmp/prof_$1 python tools/one_case.py $2 $3 3 "$4" > gpurun_out/r2e11/prof_$1.log 2>&1
  python tools/ncu_summary.py /tmp/prof_$1.ncu-rep > gpurun_out/r2e11/sum_$1.txt 2>&1
  ncu -i /tmp/prof_$1.ncu-rep --page raw --csv > gpurun_out/r2e11/raw_$1.csv 2>/dev/null
}
prof vec_c4_fms5 c4 4016 '{}'
prof vec_c4_fms3 c4 4006 '{}'
prof bulkq_2k c2 2001 '{"variant": 5, "in_dim": 0, "in_block": 256, "out_dim": 0, "out_block": 32}'
prof quad_c2 c2 2001 '{}'
ls gpurun_out/r2e11 | wc -l
