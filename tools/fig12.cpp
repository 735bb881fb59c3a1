// fig12.cpp -- PAPER.md Fig. 12 (L1615-1617, L1878-1891) on B200 through the C
// ABI: achieved bandwidth of K repeated transpositions of a 16^6 fp64 tensor,
// plan cost included, as a function of K = 1 ... 4096, for perms
// `0 2 5 1 4 3` (Fig. 12a, matching FVI) and `4 1 2 5 3 0` (Fig. 12b).
// Three curves (the paper compares TTLG with cuTT-measure and cuTT-heuristic):
//   model   : ttlg_plan (model-driven, no execution) + K x ttlg_execute;
//   measure : ttlg_plan + ttlg_plan_tune (executes 8 short-listed candidates
//             and keeps the fastest: the "measure" plan mode) + K x ttlg_execute;
//   single  : K x ttlg_transpose (each call plans, launches and destroys).
// GB/s = K * 2 * N * 8 / (host wall clock from the first API call to
// cudaStreamSynchronize) / 1e9 (L1501-1505); median of `trials`.
//   g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/fig12.cpp \
//       -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
//       -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/fig12
//   tools/fig12 [trials]  -> JSON lines
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "ttlg.h"

static double now_s() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

int main(int argc, char **argv) {
  const int trials = argc > 1 ? atoi(argv[1]) : 3;
  const int64_t ext[6] = {16, 16, 16, 16, 16, 16};
  const int32_t perms[2][6] = {{0, 2, 5, 1, 4, 3}, {4, 1, 2, 5, 3, 0}};
  const int64_t N = 1 << 24;
  const double bytes = 2.0 * N * 8;
  void *A, *B;
  if (cudaMalloc(&A, N * 8) != cudaSuccess || cudaMalloc(&B, N * 8) != cudaSuccess) return 2;
  cudaMemset(A, 0x3c, N * 8);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  // warm-up: module load, function attributes, device profile
  for (int w = 0; w < 3; w++)
    for (auto &pm : perms) ttlg_transpose(TTLG_F64, 6, ext, pm, A, B, s);
  cudaStreamSynchronize(s);
  for (int pi = 0; pi < 2; pi++) {
    const int32_t *pm = perms[pi];
    for (int K = 1; K <= 4096; K *= 2) {
      for (int mode = 0; mode < 3; mode++) {
        std::vector<double> ts;
        for (int t = 0; t < trials; t++) {
          cudaStreamSynchronize(s);
          const double t0 = now_s();
          if (mode == 2) {
            for (int k = 0; k < K; k++) ttlg_transpose(TTLG_F64, 6, ext, pm, A, B, s);
          } else {
            ttlg_plan_t p;
            if (ttlg_plan(&p, TTLG_F64, 6, ext, pm) != TTLG_OK) return 1;
            if (mode == 1 && ttlg_plan_tune(&p, A, B, s, 8, nullptr) != TTLG_OK) return 1;
            for (int k = 0; k < K; k++) ttlg_execute(p, A, B, s);
            cudaStreamSynchronize(s);
            ttlg_plan_destroy(p);
          }
          cudaStreamSynchronize(s);
          ts.push_back(now_s() - t0);
        }
        std::sort(ts.begin(), ts.end());
        const double t = ts[ts.size() / 2];
        printf("{\"perm\": \"%d %d %d %d %d %d\", \"calls\": %d, \"mode\": \"%s\", "
               "\"seconds\": %.6e, \"gbs\": %.2f}\n",
               pm[0], pm[1], pm[2], pm[3], pm[4], pm[5], K,
               mode == 0 ? "model" : (mode == 1 ? "measure" : "single"), t, K * bytes / t / 1e9);
        fflush(stdout);
      }
    }
  }
  cudaFree(A);
  cudaFree(B);
  return 0;
}
