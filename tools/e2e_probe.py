import sys, time, torch
sys.path.insert(0, '.')
import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
from synth import configs, gen_tensor_torch, case_seed
st = torch.cuda.current_stream()
for c in configs.config2()[::8]:
    A = gen_tensor_torch(case_seed(c.case_id), c.n_elems, c.elem_bytes, device='cuda')
    B = torch.empty_like(A)
    hA = torch.empty(A.numel(), dtype=A.dtype, pin_memory=True); hA.copy_(A)
    hB = torch.empty_like(hA).pin_memory()
    p = ttlg.plan('f64', c.extents, c.perm)
    for _ in range(2): p.execute_host(hA.data_ptr(), hB.data_ptr(), A.data_ptr(), B.data_ptr(), st.cuda_stream)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(3): p.execute_host(hA.data_ptr(), hB.data_ptr(), A.data_ptr(), B.data_ptr(), st.cuda_stream)
    torch.cuda.synchronize()
    t = (time.perf_counter() - t0) / 3
    print(c.label(), 'e2e %.1f GB/s' % (c.alg_bytes / t / 1e9), 'ms %.2f' % (t * 1e3), flush=True)
