#!/bin/bash
# PCIe limits vs the e2e host path
O=gpurun_out/exp59; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/pcie_probe.py > $O/pcie.txt 2>&1
timeout 300 python tools/e2e_probe.py > $O/e2e.txt 2>&1
