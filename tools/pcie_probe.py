"""PCIe probe: H2D / D2H alone and concurrent (pinned), contiguous and 2-D strided."""
import time, torch
n = 1 << 28  # 2 GiB of fp64? no: 256M * 4B = 1 GiB fp32
h = torch.empty(n, dtype=torch.float32, pin_memory=True)
h2 = torch.empty(n, dtype=torch.float32, pin_memory=True)
d = torch.empty(n, dtype=torch.float32, device='cuda')
d2 = torch.empty(n, dtype=torch.float32, device='cuda')
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def t(f, reps=3):
    f(); torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps): f()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps
gb = n * 4 / 1e9
print('H2D %.1f GB/s' % (gb / t(lambda: d.copy_(h, non_blocking=True))))
print('D2H %.1f GB/s' % (gb / t(lambda: h.copy_(d, non_blocking=True))))
def both():
    with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
print('H2D+D2H concurrent: %.1f GB/s each way' % (gb / t(both)))
for w in [4096, 16384, 65536, 262144]:
    rows = n * 4 // (4 * w)  # pitch 4w bytes, copy width w bytes
    def f2():
        torch.cuda.cudart().cudaMemcpy2DAsync(d.data_ptr(), w, h.data_ptr(), 4 * w, w, rows // 1, 1, 0) if False else None
    import ctypes
    cudart = ctypes.CDLL('libcudart.so.12')
    def f3():
        cudart.cudaMemcpy2DAsync(ctypes.c_void_p(d.data_ptr()), ctypes.c_size_t(w), ctypes.c_void_p(h.data_ptr()), ctypes.c_size_t(4 * w), ctypes.c_size_t(w), ctypes.c_size_t(rows), 1, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
    print('H2D 2D width %7d: %.1f GB/s' % (w, rows * w / 1e9 / t(f3)))
