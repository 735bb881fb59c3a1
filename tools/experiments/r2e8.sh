#!/bin/bash
# round 2, call 8: k_vec parity; every k_vec candidate and every classic candidate of the weak cases
mkdir -p gpurun_out/r2e8
timeout 400 python -m pytest tests/test_gpu_parity.py -x -q -k "bulk or variants_forced" > gpurun_out/r2e8/gputest.log 2>&1 || { tail -30 gpurun_out/r2e8/gputest.log; exit 1; }
tail -2 gpurun_out/r2e8/gputest.log
timeout 900 python tools/bulk_sweep.py --workload c4 --variants 7 --max-cand 80 > gpurun_out/r2e8/vec_c4.jsonl 2> gpurun_out/r2e8/vec_c4.err
timeout 600 python tools/bulk_sweep.py --workload c2 --variants 7 --max-cand 60 --only 2024,2047,2051,2053,2057,2022,2049 > gpurun_out/r2e8/vec_c2.jsonl 2> gpurun_out/r2e8/vec_c2.err
timeout 900 python tools/bulk_sweep.py --workload c3 --variants 7 --max-cand 60 --only 3004,3007,3008,3012,3014,3016,3024,3032,3040 > gpurun_out/r2e8/vec_c3.jsonl 2> gpurun_out/r2e8/vec_c3.err
timeout 900 python tools/bulk_sweep.py --workload c2 --variants 0 --max-cand 150 --only 2024,2047,2053,2051,2057 > gpurun_out/r2e8/all_c2.jsonl 2> gpurun_out/r2e8/all_c2.err
timeout 900 python tools/bulk_sweep.py --workload c4 --variants 0 --max-cand 150 --only 4002,4006,4007,4011,4016,4017 > gpurun_out/r2e8/all_c4.jsonl 2> gpurun_out/r2e8/all_c4.err
timeout 900 python tools/bulk_sweep.py --workload c3 --variants 0 --max-cand 150 --only 3008,3014 > gpurun_out/r2e8/all_c3.jsonl 2> gpurun_out/r2e8/all_c3.err
gzip -f gpurun_out/r2e8/*.jsonl
