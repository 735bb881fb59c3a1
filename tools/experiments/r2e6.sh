#!/bin/bash
# round 2, call 6: ncu of k_bulk (TMA rows / cp.async rows) on 5120^2 fp64
mkdir -p gpurun_out/r2e6
prof() {  # tag env workload case hints
  env $2 timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 \
    -o /tmp/prof_$1 python tools/one_case.py $3 $4 3 "$5" > gpurun_out/r2e6/prof_$1.log 2>&1
  python tools/ncu_summary.py /tmp/prof_$1.ncu-rep > gpurun_out/r2e6/sum_$1.txt 2>&1
  ncu -i /tmp/prof_$1.ncu-rep --page raw --csv > gpurun_out/r2e6/raw_$1.csv 2>/dev/null
  ncu -i /tmp/prof_$1.ncu-rep --page source --csv > gpurun_out/r2e6/src_$1.csv 2>/dev/null
  gzip -f gpurun_out/r2e6/src_$1.csv
}
prof bq_tma TTLG_BULK_TMA=1 c2 2001 '{"variant": 5}'
prof bq_cpa TTLG_BULK_TMA=0 c2 2001 '{"variant": 5}'
prof bq_big TTLG_BULK_TMA=1 c2 2001 '{"variant": 5, "in_dim": 0, "in_block": 256, "out_dim": 0, "out_block": 32}'
prof quad X=1 c2 2001 '{}'
for h in '{"variant": 5}' '{"variant": 5, "in_dim": 0, "in_block": 256, "out_dim": 0, "out_block": 32}' '{"variant": 5, "in_dim": 0, "in_block": 512, "out_dim": 0, "out_block": 32}' '{"variant": 6, "in_dim": 0, "in_block": 256, "out_dim": 0, "out_block": 32}'; do
  python tools/cases.py --workload c2 --only 2001,2037 --hints "$h" 2>&1 | tail -3 | cut -c1-250
done
