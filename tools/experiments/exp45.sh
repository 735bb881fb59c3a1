#!/bin/bash
# CCSD(T) weak cases: every candidate of 24^6 543210 / 102435 and 48^3x16^3 543210 (best achievable vs model pick)
O=gpurun_out/exp45
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python tools/calib_sweep.py --group c3 --ids 3014,3016,3030 --max-cand 80 --top > $O/c3_top.jsonl 2> $O/c3_top.err
timeout 900 python tools/calib_sweep.py --group c3 --ids 3014,3030 --max-cand 60 > $O/c3_spread.jsonl 2> $O/c3_spread.err
