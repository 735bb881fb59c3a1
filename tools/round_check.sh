#!/bin/bash
# One full GPU round on 1 B200 (run under gpurun): build, smoke, bench (+ reference arm),
# ncu launch list of one bench step, one full capture of the dominant kernel, GPU parity tests.
# Usage: bash tools/round_check.sh [TAG]   (outputs under gpurun_out/TAG/)
T=${1:-r}
O=gpurun_out/$T
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total,driver_version --format=csv > $O/gpu.txt 2>&1
nproc >> $O/gpu.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
TTLG_BENCH_CASES=1 timeout 900 python bench.py --steps 10 --warmup 3 > $O/bench.json 2> $O/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err
# launch list: skip the 3 warm-up steps (3 x 57 launches), record one step
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -k regex:k_ -s 171 -c 57 --csv --log-file $O/launches.csv \
  python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
for k in ${NCU_KERNELS:-quad}; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_$k -s 30 -c 1 -o $O/prof_$k \
    python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
done
for w in ccsdt smallfvi; do TTLG_BENCH_CASES=1 timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_$w.json 2> $O/bench_$w.err; done
timeout 1500 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
