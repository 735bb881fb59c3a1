#!/bin/bash
# round 2, call 30: k_blk with NB blocks per warp iteration (>= 8 chunks per lane in flight, registers)
O=gpurun_out/r2e30
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "blk" > $O/t_blk.log 2>&1; tail -1 $O/t_blk.log
ONLY16=$(python -c "
import sys; sys.path.insert(0,'.')
from synth import configs
print(','.join(str(c.case_id) for c in configs.sweep720(16) if c.perm[:2]==(1,0)))")
for w in 720-16 720-17 720-15; do
  timeout 600 python tools/cases.py --workload $w --only $ONLY16 --out $O/cases_$w.json > /dev/null 2> $O/cases_$w.err
done
timeout 300 python tools/cases.py --workload c3 --only 3008,3016,3024,3032,3040 --out $O/cases_c3.json > /dev/null 2>&1
timeout 300 python tools/cases.py --workload c1 --out $O/cases_c1.json > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_blk -s 2 -c 1 \
  -o /tmp/prof_blk python tools/one_case.py 720-16 6122 3 > $O/prof_blk.log 2>&1
python tools/ncu_summary.py /tmp/prof_blk.ncu-rep > $O/sum_blk_6122.txt 2>&1
head -40 $O/sum_blk_6122.txt
