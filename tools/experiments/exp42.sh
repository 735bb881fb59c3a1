#!/bin/bash
# model vs measure-mode picks back to back (ttc57, smallfvi); single- vs repeated-use suite on config 3
O=gpurun_out/exp42
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python tools/regret_b2b.py --workload ttc57 > $O/regret_ttc57.jsonl 2> $O/regret.err
timeout 900 python tools/regret_b2b.py --workload smallfvi > $O/regret_smallfvi.jsonl 2>> $O/regret.err
timeout 900 python tools/suite.py --groups c3 --out $O/suite_c3.jsonl > $O/suite_c3.log 2>&1
