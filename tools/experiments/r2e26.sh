#!/bin/bash
# round 2, call 26: FML row-length sweep (tools/cases.py --workload fmlrows): k_direct (default),
# k_rows with 4 rows in flight (TTLG_ROWS=1), forced FML schema for both, and the auto pick
O=gpurun_out/r2e26
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
TTLG_ROWS=1 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "rows or fml or direct" > $O/t_rows_env.log 2>&1; tail -1 $O/t_rows_env.log
timeout 600 python tools/cases.py --workload fmlrows --out $O/auto.json > /dev/null 2>&1
timeout 600 python tools/cases.py --workload fmlrows --hints '{"schema": "FML"}' --out $O/fml_direct.json > /dev/null 2>&1
TTLG_ROWS=1 timeout 600 python tools/cases.py --workload fmlrows --hints '{"schema": "FML"}' --out $O/fml_rows.json > /dev/null 2>&1
TTLG_ROWS=1 timeout 600 python tools/cases.py --workload fig13 --out $O/fig13_rows.json > /dev/null 2>&1
