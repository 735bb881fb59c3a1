// plantime.cpp -- host-side plan-time microbenchmark: time
// ttlg_plan + ttlg_plan_destroy with std::chrono over 1000 calls per shape
// (min and median, microseconds).  The single-use mode pays this per call.
//   g++ -O2 -std=c++17 -I include tools/plantime.cpp -L paper_conf_ipps_veduradasskhpkn18_b200 \
//       -lttlg -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o tools/plantime
//   echo "8 6 16 16 16 16 16 16 4 1 2 5 3 0" | tools/plantime     (esize rank extents... perm...)
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <vector>

#include "ttlg.h"

int main() {
  int es, rank;
  while (scanf("%d %d", &es, &rank) == 2) {
    std::vector<int64_t> ext(rank);
    std::vector<int32_t> perm(rank);
    for (auto &e : ext) scanf("%ld", &e);
    for (auto &p : perm) scanf("%d", &p);
    const ttlg_dtype dt = es == 8 ? TTLG_F64 : TTLG_F32;
    std::vector<double> us;
    for (int i = 0; i < 1000; i++) {
      auto t0 = std::chrono::steady_clock::now();
      ttlg_plan_t p;
      if (ttlg_plan(&p, dt, rank, ext.data(), perm.data()) != TTLG_OK) return 1;
      ttlg_plan_destroy(p);
      auto t1 = std::chrono::steady_clock::now();
      us.push_back(std::chrono::duration<double, std::micro>(t1 - t0).count());
    }
    std::sort(us.begin(), us.end());
    printf("%.2f %.2f\n", us[0], us[us.size() / 2]);
    fflush(stdout);
  }
  return 0;
}
