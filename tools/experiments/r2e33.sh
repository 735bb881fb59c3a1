#!/bin/bash
# round 2, call 33: k_blk (register stages, swizzle for 16-byte chunks, kBlkFactor 1.13) --
# parity, sanitizer, every workload's per-case table
O=gpurun_out/r2e33
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "blk" > $O/t_blk.log 2>&1; tail -1 $O/t_blk.log
timeout 600 python -m pytest tests/test_strided.py -x -q -m gpu > $O/t_strided.log 2>&1; tail -1 $O/t_strided.log
timeout 300 compute-sanitizer --tool memcheck python tools/sanitize_cases.py > $O/memcheck.log 2>&1; tail -1 $O/memcheck.log
timeout 300 compute-sanitizer --tool racecheck python tools/sanitize_cases.py > $O/racecheck.log 2>&1; tail -1 $O/racecheck.log
timeout 300 compute-sanitizer --tool synccheck python tools/sanitize_cases.py > $O/synccheck.log 2>&1; tail -1 $O/synccheck.log
for w in 720-16 720-15 720-17 c2 c3 c4 c1 fig13; do
  timeout 600 python tools/cases.py --workload $w --out $O/cases_$w.json > /dev/null 2> $O/cases_$w.err
done
