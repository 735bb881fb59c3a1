#!/bin/bash
# execute_host with a general split dim: parity + e2e probe + bench e2e
O=gpurun_out/exp60; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "execute_host" > $O/pytest_host.log 2>&1; echo "rc=$?" >> $O/pytest_host.log
timeout 300 python tools/e2e_probe.py > $O/e2e.txt 2>&1
timeout 900 python bench.py --steps 3 --warmup 3 --e2e-steps 2 --no-cpu-baseline --tune 0 > $O/bench.json 2> $O/bench.err
