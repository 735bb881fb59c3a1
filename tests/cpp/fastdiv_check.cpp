// Exhaustive-ish check of the planner's multiply-shift division (ttlg_internal.h)
// against exact integer division, for every divisor used by tile/row decoding
// (2 .. 2^16 and large ones) and dividends up to 2^31 - 1.
#include <cstdio>
#include <cstdint>
#include <random>
#include "../../paper_conf_ipps_veduradasskhpkn18_b200/csrc/ttlg_internal.h"

int main() {
  std::mt19937_64 rng(1);
  long bad = 0, n = 0;
  auto check = [&](uint32_t d) {
    ttlg::FastDiv f = ttlg::make_fastdiv(d);
    uint32_t xs[] = {0u, 1u, d - 1, d, d + 1, 2 * d - 1, 0x7fffffffu, 0x7ffffffeu};
    for (uint32_t x : xs) {
      if (x > 0x7fffffffu) continue;
      n++;
      if (ttlg::fastdiv_host(x, f) != x / d) bad++;
    }
    for (int i = 0; i < 64; i++) {
      uint32_t x = (uint32_t)(rng() & 0x7fffffffu);
      n++;
      if (ttlg::fastdiv_host(x, f) != x / d) bad++;
    }
  };
  for (uint32_t d = 2; d < 70000; d++) check(d);
  for (int i = 0; i < 100000; i++) check(2 + (uint32_t)(rng() % 0x7ffffffdu));
  printf("%ld %ld\n", n, bad);
  return bad != 0;
}
