// copybench.cu -- micro-benchmark of copy-kernel skeletons on B200 (tools only,
// not part of the library): which grid/unroll/cache-hint structure reaches the
// same-size cudaMemcpy D2D rate.  Informs k_direct / k_pipe design.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o copybench tools/copybench.cu
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

template <int U, bool CS>
__global__ void persist(const uint4 *__restrict__ a, uint4 *__restrict__ b, size_t n) {
  size_t stride = (size_t)gridDim.x * blockDim.x * U;
  for (size_t base = (size_t)blockIdx.x * blockDim.x * U + threadIdx.x; base < n; base += stride) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
      size_t i = base + (size_t)u * blockDim.x;
      if (i < n) v[u] = CS ? __ldcs(a + i) : a[i];
    }
#pragma unroll
    for (int u = 0; u < U; u++) {
      size_t i = base + (size_t)u * blockDim.x;
      if (i < n) {
        if (CS) __stcs(b + i, v[u]); else b[i] = v[u];
      }
    }
  }
}

// one chunk per block (non-persistent), chunk = blockDim * U vectors
template <int U, bool CS>
__global__ void chunked(const uint4 *__restrict__ a, uint4 *__restrict__ b, size_t n) {
  size_t base = (size_t)blockIdx.x * blockDim.x * U + threadIdx.x;
  uint4 v[U];
#pragma unroll
  for (int u = 0; u < U; u++) {
    size_t i = base + (size_t)u * blockDim.x;
    if (i < n) v[u] = CS ? __ldcs(a + i) : a[i];
  }
#pragma unroll
  for (int u = 0; u < U; u++) {
    size_t i = base + (size_t)u * blockDim.x;
    if (i < n) {
      if (CS) __stcs(b + i, v[u]); else b[i] = v[u];
    }
  }
}

// cp.async double-buffered persistent copy through shared memory
__global__ void pipe_copy(const uint4 *__restrict__ a, uint4 *__restrict__ b, size_t n, int tile) {
  extern __shared__ uint4 sm[];
  uint4 *buf[2] = {sm, sm + tile};
  size_t ntiles = (n + tile - 1) / tile;
  size_t t = blockIdx.x;
  auto issue = [&](size_t tt, uint4 *dst) {
    for (int i = threadIdx.x; i < tile; i += blockDim.x) {
      size_t g = tt * tile + i;
      if (g < n) {
        unsigned s = (unsigned)__cvta_generic_to_shared(dst + i);
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(a + g));
      }
    }
  };
  if (t < ntiles) issue(t, buf[0]);
  asm volatile("cp.async.commit_group;\n" ::: "memory");
  for (int k = 0; t < ntiles; k++, t += gridDim.x) {
    size_t nx = t + gridDim.x;
    if (nx < ntiles) issue(nx, buf[(k + 1) & 1]);
    asm volatile("cp.async.commit_group;\n" ::: "memory");
    asm volatile("cp.async.wait_group 1;\n" ::: "memory");
    __syncthreads();
    for (int i = threadIdx.x; i < tile; i += blockDim.x) {
      size_t g = t * tile + i;
      if (g < n) __stcs(b + g, buf[k & 1][i]);
    }
    __syncthreads();
  }
  asm volatile("cp.async.wait_group 0;\n" ::: "memory");
}

// k_tile skeleton for a plain copy: one tile per CTA, LDG -> regs -> STS,
// sync, LDS -> STG (smem round trip), many CTAs (non-persistent)
template <int U>
__global__ void smem_copy(const uint4 *__restrict__ a, uint4 *__restrict__ b, size_t n) {
  extern __shared__ uint4 sm[];
  const int tile = blockDim.x * U;
  size_t base = (size_t)blockIdx.x * tile;
  uint4 v[U];
#pragma unroll
  for (int u = 0; u < U; u++) {
    size_t i = base + u * blockDim.x + threadIdx.x;
    if (i < n) v[u] = __ldcs(a + i);
  }
#pragma unroll
  for (int u = 0; u < U; u++) sm[u * blockDim.x + threadIdx.x] = v[u];
  __syncthreads();
#pragma unroll
  for (int u = 0; u < U; u++) {
    int k = (u * blockDim.x + threadIdx.x + 17 * (threadIdx.x >> 5)) % tile;  // shuffled read
    size_t i = base + k;
    if (i < n) __stcs(b + i, sm[k]);
  }
}

// cp.async single-tile-per-CTA copy (non-persistent)
__global__ void cpasync_copy(const uint4 *__restrict__ a, uint4 *__restrict__ b, size_t n, int tile) {
  extern __shared__ uint4 sm[];
  size_t base = (size_t)blockIdx.x * tile;
  for (int i = threadIdx.x; i < tile; i += blockDim.x) {
    if (base + i < n) {
      unsigned s = (unsigned)__cvta_generic_to_shared(sm + i);
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(a + base + i));
    }
  }
  asm volatile("cp.async.commit_group;\n" ::: "memory");
  asm volatile("cp.async.wait_group 0;\n" ::: "memory");
  __syncthreads();
  for (int i = threadIdx.x; i < tile; i += blockDim.x)
    if (base + i < n) __stcs(b + base + i, sm[i]);
}

template <typename F>
float timeit(F f, int reps) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int i = 0; i < 3; i++) f();
  cudaEventRecord(e0);
  for (int i = 0; i < reps; i++) f();
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  return ms / reps;
}

int main(int argc, char **argv) {
  size_t bytes = (argc > 1 ? atoll(argv[1]) : 200) << 20;
  size_t n = bytes / 16;
  uint4 *a, *b;
  cudaMalloc(&a, bytes);
  cudaMalloc(&b, bytes);
  cudaMemset(a, 1, bytes);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  auto gbs = [&](float ms) { return 2.0 * bytes / (ms * 1e-3) / 1e9; };
  printf("bytes %zu\n", bytes);
  printf("memcpy D2D           %.0f GB/s\n", gbs(timeit([&] { cudaMemcpyAsync(b, a, bytes, cudaMemcpyDeviceToDevice); }, 20)));
  for (int threads : {128, 256, 512}) {
    for (int k : {1, 2, 4, 8, 16, 32}) {
      int grid = sms * k;
      printf("persist U4 cs  t%-4d g%-5d %.0f\n", threads, grid, gbs(timeit([&] { persist<4, true><<<grid, threads>>>(a, b, n); }, 20)));
      printf("persist U4 nc  t%-4d g%-5d %.0f\n", threads, grid, gbs(timeit([&] { persist<4, false><<<grid, threads>>>(a, b, n); }, 20)));
      printf("persist U8 cs  t%-4d g%-5d %.0f\n", threads, grid, gbs(timeit([&] { persist<8, true><<<grid, threads>>>(a, b, n); }, 20)));
      printf("persist U1 nc  t%-4d g%-5d %.0f\n", threads, grid, gbs(timeit([&] { persist<1, false><<<grid, threads>>>(a, b, n); }, 20)));
    }
    for (int U : {1, 2, 4, 8}) {
      size_t chunk = (size_t)threads * U;
      int grid = (int)((n + chunk - 1) / chunk);
      float ms = 0;
      if (U == 1) ms = timeit([&] { chunked<1, false><<<grid, threads>>>(a, b, n); }, 20);
      if (U == 2) ms = timeit([&] { chunked<2, false><<<grid, threads>>>(a, b, n); }, 20);
      if (U == 4) ms = timeit([&] { chunked<4, false><<<grid, threads>>>(a, b, n); }, 20);
      if (U == 8) ms = timeit([&] { chunked<8, false><<<grid, threads>>>(a, b, n); }, 20);
      printf("chunked U%d nc   t%-4d g%-7d %.0f\n", U, threads, grid, gbs(ms));
      if (U == 4) printf("chunked U4 cs   t%-4d g%-7d %.0f\n", threads, grid, gbs(timeit([&] { chunked<4, true><<<grid, threads>>>(a, b, n); }, 20)));
    }
  }
  for (int threads : {256, 512}) {
    for (int U : {4, 8}) {
      size_t tile = (size_t)threads * U;
      int grid = (int)((n + tile - 1) / tile);
      float ms = U == 4 ? timeit([&] { smem_copy<4><<<grid, threads, tile * 16>>>(a, b, n); }, 20)
                        : timeit([&] { smem_copy<8><<<grid, threads, tile * 16>>>(a, b, n); }, 20);
      printf("smem_copy U%d t%-4d tile %zuKB g%-6d %.0f\n", U, threads, tile * 16 / 1024, grid, gbs(ms));
    }
  }
  cudaFuncSetAttribute(cpasync_copy, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  for (int tileKB : {4, 8, 16, 32}) {
    int tile = tileKB * 1024 / 16;
    int grid = (int)((n + tile - 1) / tile);
    for (int threads : {128, 256, 512})
      printf("cpasync_copy tile %2dKB t%-4d g%-6d %.0f\n", tileKB, threads, grid,
             gbs(timeit([&] { cpasync_copy<<<grid, threads, tile * 16>>>(a, b, n, tile); }, 20)));
  }
  cudaFuncSetAttribute(pipe_copy, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  for (int tileKB : {8, 16, 32, 48}) {
    int tile = tileKB * 1024 / 16;
    for (int threads : {256, 512}) {
      int occ = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, pipe_copy, threads, 2 * tile * 16);
      int grid = sms * occ;
      printf("pipe tile %2dKB t%-4d occ %d %.0f\n", tileKB, threads, occ,
             gbs(timeit([&] { pipe_copy<<<grid, threads, 2 * tile * 16>>>(a, b, n, tile); }, 20)));
    }
  }
  cudaError_t e = cudaGetLastError();
  printf("err %s\n", cudaGetErrorString(e));
  return 0;
}
