#!/bin/bash
# round 2, call 29: k_blk (one warp per closed leading block) -- parity, sanitizer, per-case
O=gpurun_out/r2e29
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "blk" > $O/t_blk.log 2>&1; tail -1 $O/t_blk.log
timeout 600 python -m pytest tests/test_strided.py -x -q -m gpu > $O/t_strided.log 2>&1; tail -1 $O/t_strided.log
timeout 300 compute-sanitizer --tool memcheck python tools/sanitize_cases.py > $O/memcheck.log 2>&1; tail -2 $O/memcheck.log
timeout 300 compute-sanitizer --tool racecheck python tools/sanitize_cases.py > $O/racecheck.log 2>&1; tail -2 $O/racecheck.log
for w in 720-16 720-15 720-17 c3 c2 fig13 c1; do
  timeout 600 python tools/cases.py --workload $w --out $O/cases_$w.json > /dev/null 2> $O/cases_$w.err
done
timeout 1500 python -m pytest tests/test_fullsize.py -x -q > $O/t_full.log 2>&1; tail -1 $O/t_full.log
