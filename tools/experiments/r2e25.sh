#!/bin/bash
# round 2, call 25: FML rows with more bytes in flight -- k_rows with 4 rows per lane group
# (TTLG_ROWS=1) and k_direct with 16 loads per thread (TTLG_DIRECT_U=16): parity, then the
# Fig. 13 sizes and the odd sweeps A/B
O=gpurun_out/r2e25
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "rows" > $O/t_rows.log 2>&1; tail -1 $O/t_rows.log
TTLG_ROWS=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_fullsize.py -x -q -k "fml or direct or sweep or fig13 or variants" > $O/t_rows_env.log 2>&1; tail -1 $O/t_rows_env.log
TTLG_DIRECT_U=16 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_fullsize.py -x -q -k "fml or direct or sweep or fig13 or variants" > $O/t_u16_env.log 2>&1; tail -1 $O/t_u16_env.log
for w in fig13 720-15 720-17; do
  timeout 600 python tools/cases.py --workload $w --out $O/cases_${w}_base.json > /dev/null 2>&1
  TTLG_ROWS=1 timeout 600 python tools/cases.py --workload $w --out $O/cases_${w}_rows.json > /dev/null 2>&1
  TTLG_DIRECT_U=16 timeout 600 python tools/cases.py --workload $w --out $O/cases_${w}_u16.json > /dev/null 2>&1
done
