// runbench.cu -- DRAM access-pattern microbenchmark (tools only): a
// "run-granular transpose": A = [R][C] chunks of `run` bytes (chunk-contiguous
// reads), B = [C][R] chunks (every chunk lands `R*run` bytes after the
// previous one).  16-byte vector loads/stores, no shared memory, one CTA per
// tile of 32 x 32 chunks.  Isolates what short output runs cost in DRAM.
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

__global__ void chunk_transpose(const uint4 *__restrict__ a, uint4 *__restrict__ b, int R, int C,
                                int vpr /* uint4 per run */) {
  // tile = 32 rows x 32 cols of chunks; blockIdx.x over col tiles, y over row tiles
  const int r0 = blockIdx.y * 32, c0 = blockIdx.x * 32;
  const int per = 32 * 32 * vpr;
  for (int i = threadIdx.x; i < per; i += blockDim.x) {
    // consecutive threads walk along a row of A (contiguous)
    const int v = i % vpr, c = (i / vpr) % 32, r = i / (vpr * 32);
    const int gr = r0 + r, gc = c0 + c;
    if (gr >= R || gc >= C) continue;
    const uint4 x = __ldcs(a + ((size_t)gr * C + gc) * vpr + v);
    __stcs(b + ((size_t)gc * R + gr) * vpr + v, x);
  }
}

int main() {
  const size_t bytes = 256ull << 20;
  uint4 *a, *b;
  cudaMalloc(&a, bytes);
  cudaMalloc(&b, bytes);
  cudaMemset(a, 1, bytes);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int run : {32, 64, 128, 256, 512, 1024, 2048, 4096}) {
    const int vpr = run / 16;
    const size_t chunks = bytes / run;
    int C = 1;
    while ((size_t)C * C < chunks) C <<= 1;  // ~square
    int R = (int)(chunks / C);
    dim3 grid((C + 31) / 32, (R + 31) / 32);
    for (int t : {256, 512}) {
      for (int i = 0; i < 3; i++) chunk_transpose<<<grid, t>>>(a, b, R, C, vpr);
      cudaEventRecord(e0);
      for (int i = 0; i < 10; i++) chunk_transpose<<<grid, t>>>(a, b, R, C, vpr);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      printf("run %5d B threads %d: %.0f GB/s\n", run, t, 2.0 * R * C * run / (ms / 10 * 1e-3) / 1e9);
    }
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
