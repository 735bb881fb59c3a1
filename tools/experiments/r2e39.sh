#!/bin/bash
# round 2, call 39: k_tmap with 2 / 3 CTAs per SM (TTLG_TMA_CTAS; smaller rings, more consumer
# warps per SM) -- every tmap candidate vs the auto plan on configs 2 and 3
O=gpurun_out/r2e39
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "tmap_partial" > $O/t_tmap.log 2>&1; tail -1 $O/t_tmap.log
for c in 2 3; do
  TTLG_TMA_CTAS=$c timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "tmap_partial" > $O/t_tmap_$c.log 2>&1; tail -1 $O/t_tmap_$c.log
  for w in c2 c3; do
    TTLG_TMA_CTAS=$c timeout 900 python tools/bulk_sweep.py --workload $w --variants 10 --max-cand 40 --reps 5 > $O/sweep_${w}_cta$c.jsonl 2> $O/sweep_${w}_cta$c.err
  done
done
