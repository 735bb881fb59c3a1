#!/bin/bash
# round 2, call 24: small-tensor latency floor (tools/latency.cu); Fig. 13 127^4 `0 2 1 3` (the
# FML miss): every candidate timed, ncu of k_direct and k_rows
O=gpurun_out/r2e24
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
nvcc -O2 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I include tools/latency.cu \
  -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -Xlinker -rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 \
  -o tools/latency > $O/latency_build.log 2>&1
timeout 120 tools/latency > $O/latency.txt 2>&1; cat $O/latency.txt | head -60
timeout 900 python tools/bulk_sweep.py --workload fig13 --variants 0 --max-cand 150 --only 7004,7006 > $O/all_fig13.jsonl 2> $O/all_fig13.err
TTLG_ROWS=1 timeout 300 python tools/cases.py --workload fig13 --out $O/cases_fig13_rows.json > /dev/null 2>&1
timeout 300 python tools/cases.py --workload fig13 --out $O/cases_fig13.json > /dev/null 2>&1
prof() {  # tag workload case-id [env]
  env $4 timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 \
    -o /tmp/prof_$1 python tools/one_case.py $2 $3 3 > $O/prof_$1.log 2>&1
  python tools/ncu_summary.py /tmp/prof_$1.ncu-rep > $O/sum_$1.txt 2>&1
  head -1 $O/sum_$1.txt
}
prof f13_127_direct fig13 7006
prof f13_127_rows fig13 7006 TTLG_ROWS=1
prof f13_63_direct fig13 7004
prof c1_1001 c1 1001
prof c1_1016 c1 1016
gzip -f $O/*.jsonl
