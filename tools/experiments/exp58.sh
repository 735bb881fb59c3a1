#!/bin/bash
# tiles per CTA for the model's own tiles (k_quad / k_tile)
O=gpurun_out/exp58; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python tools/tpc_sweep.py --workload ttc57 --stride 2 > $O/tpc_ttc57.jsonl 2> $O/tpc.err
timeout 900 python tools/tpc_sweep.py --workload ccsdt --stride 3 > $O/tpc_ccsdt.jsonl 2>> $O/tpc.err
