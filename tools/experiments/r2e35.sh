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
# cal35: the small-tensor calibration re-timed as CUDA graphs of 20 back-to-back launches
# (cal33 timed one launch between events after a sync: host launch latency included)
export TTLG_VEC=1 TTLG_BULK=1
run() { timeout 1200 python tools/calib_sweep.py "$@" ; }
run --recipe 100 --seed 12 --lo-mb 0.25 --hi-mb 32 --log-size --max-cand 40 --graph 20 > $O/cal35_small.jsonl 2> $O/cal35_small.err
run --group c1 --max-cand 40 --graph 20 > $O/cal35_c1.jsonl 2> $O/cal35_c1.err
run --recipe 20 --seed 11 --max-cand 12 --graph 5 > $O/cal35_recipe_check.jsonl 2> $O/cal35_recipe_check.err
wc -l $O/*.jsonl
gzip -f $O/cal35_*.jsonl
# full ncu captures (reports kept) of two odd-extent weak cases: stall reasons, source hot spots
for t in "720-17 6585 s17_451230" "720-15 6585 s15_451230"; do
  set -- $t
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 \
    -o $O/prof_$3 python tools/one_case.py $1 $2 3 > $O/prof_$3.log 2>&1
  python tools/ncu_summary.py $O/prof_$3.ncu-rep > $O/sum_$3.txt 2>&1
done
