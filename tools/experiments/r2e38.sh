#!/bin/bash
# round 2, call 38: final-state evidence (1 B200): smoke, headline bench (+ reference arm), ncu launch
# list of one bench step + full captures of the dominant kernel, k_blk and k_tmap, every workload's
# bench line, per-case tables, single use through the C ABI, Fig. 12, the full GPU test suite
O=gpurun_out/${1:-r2e38}
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total,driver_version --format=csv > $O/gpu.txt 2>&1
nproc >> $O/gpu.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
TTLG_BENCH_CASES=1 timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -k regex:k_ -s 171 -c 57 --csv --log-file $O/launches.csv \
  python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-graph --tune 0 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_quad -s 30 -c 1 -o /tmp/prof_quad \
  python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-graph --tune 0 > /dev/null 2>&1
python tools/ncu_summary.py /tmp/prof_quad.ncu-rep > $O/ncu_k_quad_summary.txt 2>&1
prof() {  # tag workload case-id hints
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 \
    -o /tmp/prof_$1 python tools/one_case.py $2 $3 3 "$4" > $O/prof_$1.log 2>&1
  python tools/ncu_summary.py /tmp/prof_$1.ncu-rep > $O/ncu_$1_summary.txt 2>&1
}
prof k_blk_c3_3008 c3 3008 '{}'
prof k_tmap_c2_2001 c2 2001 '{"variant": 10}'
prof k_quad_c2_2001 c2 2001 '{"variant": 3}'
for w in ccsdt smallfvi c1 fig13 720-15 720-16 720-17; do
  TTLG_BENCH_CASES=1 timeout 900 python bench.py --workload $w --steps 10 --warmup 3 --e2e-steps 1 --tune 0 > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 900 python bench.py --workload sharded --steps 10 --warmup 3 > $O/bench_sharded.json 2> $O/bench_sharded.err
for w in c2 c3 c4 c1 fig13 720-15 720-16 720-17; do
  timeout 600 python tools/cases.py --workload $w --out $O/cases_$w.json > /dev/null 2>&1
done
build() { g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/$1.cpp \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/$1 2>/dev/null; }
build fig12; build singleuse
timeout 300 tools/singleuse 50 5 < tools/c3_shapes.txt > $O/singleuse_c3.txt 2>&1
for e in 15 16 17; do timeout 900 tools/singleuse 20 3 < tools/sweep${e}_shapes.txt > $O/singleuse_720-$e.txt 2>&1; done
timeout 600 tools/fig12 3 > $O/fig12.jsonl 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -2 $O/pytest_gpu.log; tail -1 $O/smoke.log; du -sh $O
