#!/bin/bash
# round 2, call 46: A/B the k_direct cap for odd-length output rows (TTLG_FML_CAP) on the
# workloads whose plans it changes (Fig. 13 sizes, 720 perms of 15^6 / 17^6), per-case graph timing
O=gpurun_out/r2e46
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for w in fig13 720-15 720-17; do
  for c in 0 1; do
    TTLG_FML_CAP=$c timeout 900 python tools/cases.py --workload $w --out $O/cases_${w}_cap$c.json > /dev/null 2> $O/cases_${w}_cap$c.err
  done
done
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "fig13 or odd or rank6 or 720" > $O/t_sel.log 2>&1; tail -1 $O/t_sel.log
