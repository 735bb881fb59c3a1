#!/bin/bash
O=gpurun_out/exp69; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python tools/sweep.py --case 80,16,80,256:1,0,3,2:8 --reps 10 >> $O/sweep.jsonl 2>> $O/err
for k in 2 3 4 6; do for v in 1 2; do
python tools/sweep.py --case 80,16,80,256:1,0,3,2:8 --reps 10 --hints "{\"in_dim\": 2, \"in_block\": $k, \"out_dim\": 0, \"variant\": $v}" >> $O/sweep.jsonl 2>> $O/err
done; done
python -m pytest tests/test_gpu_parity.py -m gpu -q -k "closed_block" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
