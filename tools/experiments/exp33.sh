#!/bin/bash
# A/B: store cache policy (st.global.cs vs plain) and 16-byte cp.async (.ca vs .cg)
O=gpurun_out/exp33; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()"
python -c "
import importlib.util
spec = importlib.util.spec_from_file_location('b', 'paper_conf_ipps_veduradasskhpkn18_b200/build.py')
b = importlib.util.module_from_spec(spec); spec.loader.exec_module(b)
b.build(out='/tmp/libttlg_wb.so', defines=['TTLG_ST_WB=1'])
b.build(out='/tmp/libttlg_cg.so', defines=['TTLG_CP16_CG=1'])
"
for v in base wb cg base wb cg; do
  L=""; [ $v != base ] && L=/tmp/libttlg_$v.so
  for w in ttc57 smallfvi; do
    TTLG_LIB=$L timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 >> $O/$v.$w.jsonl 2>> $O/err.log
  done
done
