#!/usr/bin/env python
"""Run one workload case a few times with direct launches (for ncu captures):
    python tools/one_case.py <workload> <case_id> [reps] [hints-json]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))


def main():
    import torch
    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from synth import gen_tensor_torch, case_seed
    from cases import workload

    wl, cid = sys.argv[1], int(sys.argv[2])
    reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
    hints = json.loads(sys.argv[4]) if len(sys.argv) > 4 else {}
    c = [x for x in workload(wl) if x.case_id == cid][0]
    A = gen_tensor_torch(case_seed(c.case_id), c.n_elems, c.elem_bytes, device="cuda:0")
    B = torch.empty_like(A)
    p = ttlg.plan("f64" if c.elem_bytes == 8 else "f32", c.extents, c.perm, **hints)
    torch.cuda.synchronize()
    for _ in range(reps):
        p.execute(A.data_ptr(), B.data_ptr(), 0)
    torch.cuda.synchronize()
    print(c.label(), json.dumps(p.describe()))


if __name__ == "__main__":
    main()
