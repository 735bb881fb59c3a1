// singleuse.cpp -- single-use vs repeated-use through the C ABI (SURVEY §8(d),
// PAPER.md L1592-1593 / L1605-1606; VERDICT r1 "Next round" 6): per shape,
//   repeated = one ttlg_plan, then K ttlg_execute calls;
//   single   = K ttlg_transpose calls (each plans, launches, destroys; no cache);
// both host wall clock from the first call to cudaStreamSynchronize, / K; plus
// ttlg_plan + ttlg_plan_destroy over 1000 calls (min / median, full effort).
//   g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/singleuse.cpp \
//       -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -L /usr/local/cuda/lib64 -lcudart \
//       -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/singleuse
//   echo "8 6 16 16 16 16 16 16 4 1 2 5 3 0" | tools/singleuse [K] [trials]
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "ttlg.h"

static double now_us() {
  return std::chrono::duration<double, std::micro>(
             std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

int main(int argc, char **argv) {
  const int K = argc > 1 ? atoi(argv[1]) : 50;
  const int trials = argc > 2 ? atoi(argv[2]) : 5;
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  void *A = nullptr, *B = nullptr;
  size_t cap = 0;
  int es, rank;
  printf("# esize rank extents perm | repeated_us single_us ratio | plan_min_us plan_med_us\n");
  while (scanf("%d %d", &es, &rank) == 2) {
    std::vector<int64_t> ext(rank);
    std::vector<int32_t> perm(rank);
    for (auto &e : ext) scanf("%ld", &e);
    for (auto &p : perm) scanf("%d", &p);
    const ttlg_dtype dt = es == 8 ? TTLG_F64 : TTLG_F32;
    size_t bytes = es;
    for (auto e : ext) bytes *= (size_t)e;
    if (bytes > cap) {
      cudaFree(A);
      cudaFree(B);
      if (cudaMalloc(&A, bytes) != cudaSuccess || cudaMalloc(&B, bytes) != cudaSuccess) return 2;
      cudaMemset(A, 0x3c, bytes);
      cap = bytes;
    }
    ttlg_plan_t p;
    if (ttlg_plan(&p, dt, rank, ext.data(), perm.data()) != TTLG_OK) return 1;
    std::vector<double> rep, sgl;
    for (int t = 0; t < trials; t++) {
      for (int i = 0; i < 3; i++) ttlg_execute(p, A, B, s);
      cudaStreamSynchronize(s);
      double t0 = now_us();
      for (int i = 0; i < K; i++) ttlg_execute(p, A, B, s);
      cudaStreamSynchronize(s);
      rep.push_back((now_us() - t0) / K);
      for (int i = 0; i < 3; i++) ttlg_transpose(dt, rank, ext.data(), perm.data(), A, B, s);
      cudaStreamSynchronize(s);
      t0 = now_us();
      for (int i = 0; i < K; i++) ttlg_transpose(dt, rank, ext.data(), perm.data(), A, B, s);
      cudaStreamSynchronize(s);
      sgl.push_back((now_us() - t0) / K);
    }
    ttlg_plan_destroy(p);
    std::vector<double> pt;
    for (int i = 0; i < 1000; i++) {
      double t0 = now_us();
      ttlg_plan_t q;
      ttlg_plan(&q, dt, rank, ext.data(), perm.data());
      ttlg_plan_destroy(q);
      pt.push_back(now_us() - t0);
    }
    std::sort(rep.begin(), rep.end());
    std::sort(sgl.begin(), sgl.end());
    std::sort(pt.begin(), pt.end());
    const double r = rep[rep.size() / 2], sg = sgl[sgl.size() / 2];
    printf("%d %d", es, rank);
    for (auto e : ext) printf(" %ld", (long)e);
    for (auto q : perm) printf(" %d", q);
    printf(" | %.2f %.2f %.4f | %.2f %.2f\n", r, sg, sg / r, pt[0], pt[pt.size() / 2]);
    fflush(stdout);
  }
  cudaFree(A);
  cudaFree(B);
  return 0;
}
