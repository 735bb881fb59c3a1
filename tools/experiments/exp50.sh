#!/bin/bash
# Fig. 5-style model check + round check with k_deint (s4d)
O=gpurun_out/s4d; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python tools/fig5.py > $O/fig5.jsonl 2> $O/fig5.err
bash tools/round_check.sh s4d
