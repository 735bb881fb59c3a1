#!/bin/bash
# round 2, call 18: calibration cal34 -- the linear screen's top candidates of configs 2-4 and
# the 720-perm sweeps (every 6th perm), current kernels (k_vec included)
mkdir -p gpurun_out/r2e18
export TTLG_VEC=1
run() { timeout 1500 python tools/calib_sweep.py "$@" ; }
run --group c2 --max-cand 48 --top > gpurun_out/r2e18/cal34_c2top.jsonl 2> gpurun_out/r2e18/c2.err
run --group c3 --max-cand 48 --top > gpurun_out/r2e18/cal34_c3top.jsonl 2> gpurun_out/r2e18/c3.err
run --group c4 --max-cand 48 --top > gpurun_out/r2e18/cal34_c4top.jsonl 2> gpurun_out/r2e18/c4.err
python - <<'PY'
import sys; sys.path.insert(0, '.')
from synth import configs
with open('/tmp/sweep_ids.txt', 'w') as f:
    f.write(",".join(str(c.case_id) for c in configs.sweep720(16)[::6]))
PY
wc -l gpurun_out/r2e18/*.jsonl
gzip -f gpurun_out/r2e18/*.jsonl
