// Small-tensor latency floor (config 1 / Fig. 13 sizes): where do the ~3.4 us
// per ttlg_execute of a 512 KiB tensor go, against 1.3 us for a same-size D2D
// cudaMemcpyAsync?  Every row is ONE CUDA graph of R back-to-back nodes
// (median of T replays), reported per node:
//   empty kernel, 8-byte / 2.5-KB __grid_constant__ parameter
//   a 16-byte vector copy kernel (grid = SMs), 8-byte / 2.5-KB parameter
//   cudaMemcpyAsync D2D of the same bytes
//   ttlg_execute of 16^4 fp64 for a few permutations (plan: the model's)
//
//   nvcc -O2 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I include tools/latency.cu \
//     -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -Xlinker -rpath,$PWD/paper_... -o tools/latency
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <functional>
#include <vector>

#include "ttlg.h"

#define CK(x)                                                              \
  do {                                                                     \
    cudaError_t e_ = (x);                                                  \
    if (e_ != cudaSuccess) {                                               \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
      exit(1);                                                             \
    }                                                                      \
  } while (0)

struct Big {
  char pad[2560];
  const float4 *a;
  float4 *b;
  long n;
};
struct Small {
  const float4 *a;
  float4 *b;
  long n;
};

__global__ void k_empty_small(Small p) {}
__global__ void k_empty_big(const __grid_constant__ Big p) {}
__global__ void k_copy_small(Small p) {
  for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < p.n; i += (long)gridDim.x * blockDim.x)
    p.b[i] = p.a[i];
}
__global__ void k_copy_big(const __grid_constant__ Big p) {
  for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < p.n; i += (long)gridDim.x * blockDim.x)
    p.b[i] = p.a[i];
}

static double graph_us(cudaStream_t s, int R, int T, const std::function<void()> &body) {
  cudaGraph_t g;
  cudaGraphExec_t ge;
  CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
  for (int r = 0; r < R; r++) body();
  CK(cudaStreamEndCapture(s, &g));
  CK(cudaGraphInstantiate(&ge, g, 0));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(cudaGraphLaunch(ge, s));
  CK(cudaStreamSynchronize(s));
  std::vector<float> v;
  for (int t = 0; t < T; t++) {
    CK(cudaEventRecord(e0, s));
    CK(cudaGraphLaunch(ge, s));
    CK(cudaEventRecord(e1, s));
    CK(cudaEventSynchronize(e1));
    float ms;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    v.push_back(ms);
  }
  std::sort(v.begin(), v.end());
  CK(cudaGraphExecDestroy(ge));
  CK(cudaGraphDestroy(g));
  return 1e3 * v[v.size() / 2] / R;
}

int main(int argc, char **argv) {
  const int R = 20, T = 21;
  int sms;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  const int sizes[] = {16, 15, 32, 31};
  for (int e : sizes) {
    const long n = (long)e * e * e * e;
    const size_t bytes = n * 8;
    void *A, *B;
    CK(cudaMalloc(&A, bytes + 64));
    CK(cudaMalloc(&B, bytes + 64));
    CK(cudaMemset(A, 1, bytes));
    Small sp{(const float4 *)A, (float4 *)B, (long)(bytes / 16)};
    Big bp;
    memset(&bp, 0, sizeof bp);
    bp.a = sp.a;
    bp.b = sp.b;
    bp.n = sp.n;
    printf("## %d^4 fp64 (%zu bytes)\n", e, bytes);
    auto row = [&](const char *name, double us) {
      printf("%-34s %8.3f us  %8.1f GB/s\n", name, us, 2.0 * bytes / (us * 1e3));
    };
    row("empty kernel, 24 B param", graph_us(s, R, T, [&] { k_empty_small<<<1, 32, 0, s>>>(sp); }));
    row("empty kernel, 2.6 KB param", graph_us(s, R, T, [&] { k_empty_big<<<1, 32, 0, s>>>(bp); }));
    row("empty kernel x SMs, 2.6 KB", graph_us(s, R, T, [&] { k_empty_big<<<sms, 512, 0, s>>>(bp); }));
    for (int thr : {256, 512}) {
      char nm[64];
      snprintf(nm, sizeof nm, "copy16 SMs x %d, 24 B", thr);
      row(nm, graph_us(s, R, T, [&] { k_copy_small<<<sms, thr, 0, s>>>(sp); }));
      snprintf(nm, sizeof nm, "copy16 SMs x %d, 2.6 KB", thr);
      row(nm, graph_us(s, R, T, [&] { k_copy_big<<<sms, thr, 0, s>>>(bp); }));
      snprintf(nm, sizeof nm, "copy16 2xSMs x %d, 24 B", thr);
      row(nm, graph_us(s, R, T, [&] { k_copy_small<<<2 * sms, thr, 0, s>>>(sp); }));
    }
    row("cudaMemcpyAsync D2D", graph_us(s, R, T, [&] {
          CK(cudaMemcpyAsync(B, A, bytes, cudaMemcpyDeviceToDevice, s));
        }));
    const char *perms[] = {"0123", "0213", "1023", "3210", "2301", "0321"};
    for (const char *ps : perms) {
      int64_t ext[4] = {e, e, e, e};
      int32_t perm[4];
      for (int k = 0; k < 4; k++) perm[k] = ps[k] - '0';
      ttlg_plan_t p;
      if (ttlg_plan(&p, TTLG_F64, 4, ext, perm) != TTLG_OK) continue;
      ttlg_plan_info info;
      ttlg_plan_describe(p, &info);
      char nm[96];
      static const char *kn[] = {"direct", "tile", "pipe", "quad", "deint", "bulkq", "bulkg", "vec", "phase"};
      snprintf(nm, sizeof nm, "ttlg %s %s g%d t%d p%dB", ps, kn[info.kernel], info.grid, info.threads,
               info.param_bytes);
      row(nm, graph_us(s, R, T, [&] { ttlg_execute(p, A, B, s); }));
      ttlg_plan_destroy(p);
    }
    CK(cudaFree(A));
    CK(cudaFree(B));
  }
  return 0;
}
