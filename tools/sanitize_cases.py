#!/usr/bin/env python
"""Small launches of every kernel family for compute-sanitizer (memcheck,
racecheck, synccheck): k_direct, k_tile, k_pipe, k_quad, k_deint, k_inter,
k_bulk (TMA rows and cp.async rows, quad and gather consumers), k_blk, k_tmap
(TMA tensor-map boxes), ragged tiles,
strided sub-tensor plans and batched launches.

  compute-sanitizer --tool memcheck python tools/sanitize_cases.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from synth import gen_tensor_torch

    s = torch.cuda.current_stream().cuda_stream
    cases = [  # (extents, perm, elem bytes, hints)
        ([37, 29, 23], [2, 1, 0], 8, {}),                     # OD, ragged
        ([37, 29, 23], [2, 1, 0], 8, {"variant": 1}),         # k_tile
        ([37, 29, 23], [2, 1, 0], 8, {"variant": 2}),         # k_pipe
        ([48, 40, 24], [2, 1, 0], 4, {"variant": 3}),         # k_quad fp32
        ([40, 36, 22], [1, 0, 2], 8, {"variant": 3}),         # k_quad fp64, ragged blocks
        ([12, 14, 16, 10], [1, 0, 3, 2], 4, {}),              # OA
        ([3, 64, 96], [0, 2, 1], 4, {}),                      # FMS 12-byte pencils
        ([40, 30, 20], [0, 2, 1], 4, {}),                     # FML
        ([3, 400, 5], [1, 0, 2], 4, {"variant": 4}),          # k_deint
        ([4096, 3, 8], [1, 0, 2], 4, {"variant": 4}),         # k_inter
        ([64, 96], [1, 0], 8, {"variant": 5}),                # k_bulk quad
        ([3, 256, 96], [2, 1, 0], 4, {"variant": 5}),
        ([40, 36, 22], [2, 0, 1], 4, {"variant": 6}),         # k_bulk gather
        ([8, 30, 50], [0, 2, 1], 4, {"variant": 6}),
        ([256, 24, 6], [1, 0, 2], 8, {"variant": 5, "in_dim": 0, "in_block": 256,
                                      "out_dim": 0, "out_block": 24}),  # TMA rows (2 KB)
        ([24, 24, 12, 4, 3, 2], [1, 0, 2, 4, 3, 5], 8, {"variant": 2}),  # deep k_pipe tiles
        ([16, 16, 5, 7], [1, 0, 3, 2], 8, {"variant": 9}),   # k_blk, 16-byte chunks
        ([15, 15, 6, 5], [1, 0, 3, 2], 8, {"variant": 9}),   # k_blk, 8-byte chunks
        ([8, 8, 8, 9], [2, 1, 0, 3], 4, {"variant": 9}),     # k_blk, 3-D inner perm
        ([24, 24, 12, 4, 3, 2], [1, 0, 2, 4, 3, 5], 8, {}),  # auto (k_blk)
        ([64, 72, 5], [1, 0, 2], 8, {"variant": 10}),        # k_tmap (TMA boxes)
        ([80, 4, 16, 20, 16], [3, 2, 0, 4, 1], 8, {"variant": 10}),  # k_tmap panels
        ([24, 40, 7], [1, 0, 2], 4, {"variant": 10}),        # k_tmap fp32, ragged
    ]
    for ext, perm, eb, hints in cases:
        n = 1
        for e in ext:
            n *= e
        A = gen_tensor_torch(5, n, eb, device="cuda:0")
        B = torch.empty_like(A)
        try:
            p = ttlg.plan("f64" if eb == 8 else "f32", ext, perm, **hints)
        except ttlg.TtlgError as e:
            print("skip", ext, perm, hints, e)
            continue
        p.execute(A.data_ptr(), B.data_ptr(), s)
        p.execute_batch([A.data_ptr()], [B.data_ptr()], s)
        torch.cuda.synchronize()
        print("ok", ext, perm, hints, p.describe()["kernel"])
    # strided sub-tensor plan (the fused exchange's form) and a misaligned view
    base = gen_tensor_torch(7, 64 * 48 * 40, 4, device="cuda:0").view(40, 48, 64)
    x = base[:, 8:40, 4:60]
    y = ttlg.transpose_tensor(x, (2, 0, 1))
    A = gen_tensor_torch(8, 4 * 256 * 96 + 1, 4, device="cuda:0")
    B = torch.empty_like(A)
    ttlg.plan("f32", [4, 256, 96], [0, 2, 1]).execute(A[1:].data_ptr(), B[1:].data_ptr(), s)
    torch.cuda.synchronize()
    print("ok strided / misaligned", tuple(y.shape))


if __name__ == "__main__":
    main()
