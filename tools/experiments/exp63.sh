#!/bin/bash
# k_inter (SoA -> AoS): GPU parity + speed vs the previous auto plan (libttlg_ab0.so)
O=gpurun_out/exp63; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
L0=$PWD/paper_conf_ipps_veduradasskhpkn18_b200/libttlg_ab0.so
for n1 in 2 3 4 5 6 8; do
  TTLG_LIB=$L0 python tools/sweep.py --case 16777216,$n1:1,0:4 --reps 10 >> $O/old.jsonl 2>> $O/sweep.err
  python tools/sweep.py --case 16777216,$n1:1,0:4 --reps 10 >> $O/new.jsonl 2>> $O/sweep.err
  python tools/sweep.py --case 4096,$n1,4096:1,0,2:4 --reps 10 >> $O/new.jsonl 2>> $O/sweep.err
  TTLG_LIB=$L0 python tools/sweep.py --case 4096,$n1,4096:1,0,2:4 --reps 10 >> $O/old.jsonl 2>> $O/sweep.err
done
