#!/bin/bash
# bench + launch list + one full ncu capture per kernel family (1 GPU)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total,driver_version --format=csv > gpurun_out/gpu.txt 2>&1
TTLG_BENCH_CASES=1 timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
# launch list: skip the 3 warm-up steps (3 x 57 launches), record one step
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:k_ -s 171 -c 57 --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
for k in pipe direct; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_$k -s 30 -c 1 -o gpurun_out/prof_$k python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
done
