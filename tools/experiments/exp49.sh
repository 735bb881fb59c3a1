#!/bin/bash
# k_deint: GPU parity (full suite) + A/B small-FVI vs HEAD without k_deint (libttlg_ab0.so)
O=gpurun_out/exp49
mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
L0=$PWD/paper_conf_ipps_veduradasskhpkn18_b200/libttlg_ab0.so
for rep in 1 2; do
  for v in 0 1; do
    if [ $v = 0 ]; then export TTLG_LIB=$L0; else unset TTLG_LIB; fi
    TTLG_BENCH_CASES=1 timeout 600 python bench.py --workload smallfvi --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_smallfvi_v${v}_r$rep.json 2> $O/bench_smallfvi_v${v}_r$rep.err
  done
done
unset TTLG_LIB
# the deint kernel alone at config-4 sizes, n0 = 2..8, fp32 and fp64 (ncu-free event timing)
timeout 600 python tools/calib_sweep.py --group c4 --ids 4003,4004,4008,4009,4013,4014,4018,4019,4023,4024 --max-cand 400 > $O/c4_deint.jsonl 2> $O/c4_deint.err
