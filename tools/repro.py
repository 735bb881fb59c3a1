import sys, json, torch, numpy as np
sys.path.insert(0, '.')
import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
from synth import gen_tensor_torch
ext, perm, eb = json.loads(sys.argv[1]), json.loads(sys.argv[2]), int(sys.argv[3])
hints = json.loads(sys.argv[4]) if len(sys.argv) > 4 else {}
n = int(np.prod(ext))
A = gen_tensor_torch(1, n, eb, device='cuda:0'); B = torch.empty_like(A)
p = ttlg.plan('f64' if eb == 8 else 'f32', ext, perm, **hints)
d = p.describe(); print({k: d[k] for k in ['schema','kernel','threads','fused_extents','fused_perm','tile_extents','in_run','out_run','num_tiles','grid','smem_bytes']}, flush=True)
p.execute(A.data_ptr(), B.data_ptr(), torch.cuda.current_stream().cuda_stream)
torch.cuda.synchronize(); print('ok')
