#!/bin/bash
# k_quad vs k_tile on 5120^2 fp64 and AoS->SoA fp32: ncu full captures + c4 sweep
O=gpurun_out/exp27; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
H1='{"schema": "OD", "in_dim": 0, "in_block": 64, "out_dim": 0, "out_block": 32, "threads": 256, "variant": 1}'
H2='{"schema": "OD", "in_dim": 0, "in_block": 64, "out_dim": 0, "out_block": 32, "threads": 256, "variant": 3}'
i=0
for H in "$H1" "$H2"; do
  i=$((i+1))
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_ -s 3 -c 1 -o $O/p$i \
    python tools/sweep.py --case 5120,5120:1,0:8 --hints "$H" --reps 2 > $O/p$i.log 2>&1
  python tools/sweep.py --case 5120,5120:1,0:8 --hints "$H" --reps 20 > $O/t$i.log 2>&1
done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_ -s 3 -c 1 -o $O/p3 \
    python tools/sweep.py --case 4,4096,4096:1,2,0:4 --hints '{"variant": 3}' --reps 2 > $O/p3.log 2>&1
timeout 900 python tools/calib_sweep.py --group c4 --max-cand 400 --reps 5 > $O/sweep_c4.jsonl 2> $O/sweep_c4.err
