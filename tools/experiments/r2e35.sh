#!/bin/bash
# round 2, call 35: k_tmap (TMA tensor-map box loads, variant 10) -- parity, sanitizer,
# every k_tmap candidate of the config workloads vs the auto plan (graph timing)
O=gpurun_out/r2e35
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "tmap" > $O/t_tmap.log 2>&1; tail -3 $O/t_tmap.log
timeout 300 compute-sanitizer --tool memcheck python tools/sanitize_cases.py > $O/memcheck.log 2>&1; tail -1 $O/memcheck.log
timeout 300 compute-sanitizer --tool racecheck python tools/sanitize_cases.py > $O/racecheck.log 2>&1; tail -1 $O/racecheck.log
timeout 300 compute-sanitizer --tool synccheck python tools/sanitize_cases.py > $O/synccheck.log 2>&1; tail -1 $O/synccheck.log
for w in c2 c4 c3; do
  timeout 900 python tools/bulk_sweep.py --workload $w --variants 10 --max-cand 40 --reps 5 > $O/sweep_$w.jsonl 2> $O/sweep_$w.err
done
