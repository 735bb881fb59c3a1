#!/bin/bash
O=gpurun_out/exp32; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
TTLG_BENCH_CASES=1 timeout 900 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench.json 2> $O/bench.err
for w in ccsdt smallfvi; do TTLG_BENCH_CASES=1 timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_$w.json 2> $O/bench_$w.err; done
g++ -O2 -std=c++17 -I include tools/plantime.cpp -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o /tmp/plantime 2>/dev/null
for c in "8 6 16 16 16 16 16 16 4 1 2 5 3 0" "8 6 16 16 16 16 16 16 2 1 0 5 4 3" "8 2 5120 5120 1 0" "8 5 32 32 25 32 32 2 0 4 1 3" "4 3 4 4096 4096 1 2 0"; do
  echo "$c" | /tmp/plantime >> $O/plantime.txt 2>&1
done
timeout 900 python tools/suite.py --groups c3 --out $O/suite.jsonl > $O/suite.log 2>&1
