// plantime_single.cpp -- host-only timing of the single-use planning path
// (ttlg_transpose's plan at the effort level it picks; no GPU needed: with no
// device the call plans, then returns TTLG_ERR_DEVICE at execute).  Prints
// per shape: min / median microseconds over N calls.  HOST-ONLY: on a machine
// with a GPU the fake operand pointers would be launched on -- never run it there.
//   g++ -O2 -std=c++17 -I include tools/plantime_single.cpp -L paper_conf_ipps_veduradasskhpkn18_b200 \
//       -lttlg -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/plantime_single
//   tools/plantime_single [N] < tools/c3_shapes.txt
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "ttlg.h"

int main(int argc, char **argv) {
  const int N = argc > 1 ? atoi(argv[1]) : 200;
  int es, rank;
  while (scanf("%d %d", &es, &rank) == 2) {
    std::vector<int64_t> ext(rank);
    std::vector<int32_t> perm(rank);
    for (auto &e : ext) scanf("%ld", &e);
    for (auto &p : perm) scanf("%d", &p);
    const ttlg_dtype dt = es == 8 ? TTLG_F64 : TTLG_F32;
    std::vector<double> us;
    for (int i = 0; i < N; i++) {
      auto t0 = std::chrono::steady_clock::now();
      ttlg_transpose(dt, rank, ext.data(), perm.data(), (const void *)0x100000,
                     (void *)0x7f0000000000ull, nullptr);
      auto t1 = std::chrono::steady_clock::now();
      us.push_back(std::chrono::duration<double, std::micro>(t1 - t0).count());
    }
    std::sort(us.begin(), us.end());
    printf("%d %d", es, rank);
    for (auto e : ext) printf(" %ld", e);
    for (auto p : perm) printf(" %d", p);
    printf(" | %.2f %.2f\n", us[0], us[us.size() / 2]);
    fflush(stdout);
  }
  return 0;
}
