#!/bin/bash
# round 2, call 37: k_tmap ring slack fix (1024-byte rounding inside the allocation); tree set 3
# (graph-timed small tensors) ranks / reports < 32 MB, set 2 restored; bench hybrid per-case timing
O=gpurun_out/r2e37
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tmap or config1 or single_use or graph or blk or bulk" > $O/t_sel.log 2>&1; tail -2 $O/t_sel.log
python tools/sanitize_cases.py > $O/sanitize_cases.log 2>&1; tail -2 $O/sanitize_cases.log
for w in c1 fig13 smallfvi ttc57; do
  TTLG_BENCH_CASES=1 timeout 900 python bench.py --workload $w --steps 10 --warmup 3 --e2e-steps 1 --tune 0 --no-cpu-baseline > $O/bench_$w.json 2> $O/bench_$w.err
done
for w in c1 c4 fig13; do
  timeout 600 python tools/cases.py --workload $w --out $O/cases_$w.json > /dev/null 2> $O/cases_$w.err
done
for w in c2 c4 c3; do
  timeout 900 python tools/bulk_sweep.py --workload $w --variants 10 --max-cand 40 --reps 5 > $O/sweep_$w.jsonl 2> $O/sweep_$w.err
done
