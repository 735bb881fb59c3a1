#!/bin/bash
# A/B e2e (ttlg_execute_host): general split dim vs outermost-dims only (libttlg_ab0.so)
O=gpurun_out/exp61; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
L0=$PWD/paper_conf_ipps_veduradasskhpkn18_b200/libttlg_ab0.so
for rep in 1 2; do
  for v in 0 1; do
    if [ $v = 0 ]; then export TTLG_LIB=$L0; else unset TTLG_LIB; fi
    timeout 900 python bench.py --steps 2 --warmup 3 --e2e-steps 3 --no-cpu-baseline --tune 0 > $O/bench_v${v}_r$rep.json 2> $O/bench_v${v}_r$rep.err
    timeout 300 python tools/e2e_probe.py > $O/e2e_v${v}_r$rep.txt 2>&1
  done
done
