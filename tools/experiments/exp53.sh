#!/bin/bash
# A/B: deep input-run candidates (one more input dim blocked by tile volume) vs HEAD (libttlg_ab0.so)
O=gpurun_out/exp53
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
L0=$PWD/paper_conf_ipps_veduradasskhpkn18_b200/libttlg_ab0.so
for rep in 1 2; do
  for v in 0 1; do
    for w in ttc57 ccsdt smallfvi; do
      if [ $v = 0 ]; then export TTLG_LIB=$L0; else unset TTLG_LIB; fi
      TTLG_BENCH_CASES=1 timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_${w}_v${v}_r$rep.json 2> $O/bench_${w}_v${v}_r$rep.err
    done
  done
done
unset TTLG_LIB
