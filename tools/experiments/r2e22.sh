#!/bin/bash
# round 2, call 22: k_phase (16-byte loads at any row alignment) -- parity, A/B on the odd sweeps
mkdir -p gpurun_out/r2e22
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "phase or variants or odd or rank6 or 720 or scaled or misaligned or config1 or execute_batch or graph" > gpurun_out/r2e22/gputest.log 2>&1
rc=$?; echo "gputest rc=$rc"; tail -3 gpurun_out/r2e22/gputest.log; [ $rc -ne 0 ] && exit 1
timeout 600 python -m pytest tests/test_fullsize.py -x -q -k "720_sweep" > gpurun_out/r2e22/fullsize.log 2>&1; echo "fullsize rc=$?"; tail -1 gpurun_out/r2e22/fullsize.log
for w in 720-17 720-15; do
  for m in 0 1; do
    TTLG_PHASE=$m timeout 600 python tools/cases.py --workload $w --out gpurun_out/r2e22/cases_${w}_ph$m.json > /dev/null 2>&1
  done
done
timeout 300 compute-sanitizer --tool memcheck python -c "
import sys; sys.path.insert(0,'.')
import torch, paper_conf_ipps_veduradasskhpkn18_b200 as t
from synth import gen_tensor_torch
for ext,perm in (([17,17,17,17],[3,1,2,0]),([15,15,15],[2,0,1]),([17,6,9,5],[1,3,0,2])):
  n=1
  for e in ext: n*=e
  A=gen_tensor_torch(1,n,8,device='cuda'); B=torch.empty_like(A)
  t.plan('f64',ext,perm,variant=8).execute(A.data_ptr(),B.data_ptr(),0)
torch.cuda.synchronize(); print('ok')
" > gpurun_out/r2e22/memcheck.log 2>&1; tail -2 gpurun_out/r2e22/memcheck.log
