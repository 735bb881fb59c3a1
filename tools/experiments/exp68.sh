#!/bin/bash
# deep k_pipe tiles for closed leading blocks (1 0 2 4 3 5 family): parity + CCSD(T) bench
O=gpurun_out/exp68; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
for r in 1 2; do
TTLG_BENCH_CASES=1 timeout 600 python bench.py --workload ccsdt --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_ccsdt_r$r.json 2> $O/bench_ccsdt.err
done
python - > $O/check.txt 2>&1 <<'PY'
import sys; sys.path.insert(0, '.')
import numpy as np, torch, oracle
import paper_conf_ipps_veduradasskhpkn18_b200 as t
from synth import gen_tensor_torch
for ext in ([24]*6, [32,32,32,16,16,16]):
    perm=[1,0,2,4,3,5]; n=int(np.prod(ext))
    A=gen_tensor_torch(5, n, 8, device='cuda'); B=torch.empty_like(A)
    p=t.plan('f64', ext, perm); p.execute(A.data_ptr(), B.data_ptr(), 0); torch.cuda.synchronize()
    idx=np.random.default_rng(0).integers(0, n, 200000)
    src=oracle.source_index(ext, perm, idx)
    a=A.view(torch.int64).cpu().numpy(); b=B.view(torch.int64).cpu().numpy()
    print(ext, p.describe()['kernel'], p.describe()['tile_extents'], bool((b[idx]==a[src]).all()))
PY
