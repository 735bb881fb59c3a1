#!/bin/bash
# A/B: warp-staged coalesced loads (k_deint) / stores (k_inter) vs HEAD (libttlg_ab0.so)
O=gpurun_out/exp65; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "deint or inter or smoke or config1" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
L0=$PWD/paper_conf_ipps_veduradasskhpkn18_b200/libttlg_ab0.so
for rep in 1 2; do for v in 0 1; do
  if [ $v = 0 ]; then export TTLG_LIB=$L0; else unset TTLG_LIB; fi
  TTLG_BENCH_CASES=1 timeout 600 python bench.py --workload smallfvi --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_smallfvi_v${v}_r$rep.json 2> $O/e_$v$rep.err
  for n1 in 2 3 5 6; do python tools/sweep.py --case 16777216,$n1:1,0:4 --reps 10 >> $O/inter_v${v}_r$rep.jsonl 2>> $O/sweep.err; done
done; done
unset TTLG_LIB
