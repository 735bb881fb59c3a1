#!/bin/bash
# round 2, call 36: k_tmap with the swizzle span = box row (16/32/64/128 B, input run in dim 0);
# tree set 2 refit with graph-timed small tensors (cal35); bench per-case timing as per-case graphs
O=gpurun_out/r2e36
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "tmap or config1 or smallfvi or single_use or graph" > $O/t_sel.log 2>&1; tail -2 $O/t_sel.log
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
