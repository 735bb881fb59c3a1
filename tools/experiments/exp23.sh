#!/bin/bash
# ncu full captures of the 5120^2 fp64 transpose: best measured tile vs auto plan
O=gpurun_out/exp23; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
H1='{"schema": "OD", "in_dim": 0, "in_block": 32, "out_dim": 0, "out_block": 64, "threads": 256, "variant": 1}'
H2='{"schema": "OD", "in_dim": 0, "in_block": 64, "out_dim": 0, "out_block": 128, "threads": 512, "variant": 1}'
H3='{"schema": "OD", "in_dim": 0, "in_block": 64, "out_dim": 0, "out_block": 128, "threads": 512, "variant": 2}'
i=0
for H in "$H1" "$H2" "$H3"; do
  i=$((i+1))
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_pipe -s 3 -c 1 -o $O/p$i \
    python tools/sweep.py --case 5120,5120:1,0:8 --hints "$H" --reps 2 > $O/p$i.log 2>&1
done
