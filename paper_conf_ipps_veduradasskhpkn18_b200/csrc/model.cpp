// model.cpp -- B200 performance model; see model.h.
#include "model.h"

#include <algorithm>
#include <cmath>

#include "model_coeffs.h"

namespace ttlg {

// DRAM bytes moved for one contiguous run of R bytes: whole 32-byte sectors,
// plus half a sector on average when the run is not sector-aligned, with a
// 64-byte floor (HBM burst) -- the B200 restatement of Table I's transaction
// counts, which count 128-byte K40 transactions.
static double run_cost(double R) {
  double c = 32.0 * std::ceil(R / 32.0);
  if (std::fmod(R, 32.0) != 0.0) c += 16.0;
  return std::max(c, 64.0);
}

ModelFeatures model_features(const ModelInput &mi, const DeviceProfile &dev) {
  ModelFeatures F;
  for (double &x : F.f) x = 0.0;
  const double W = mi.W;
  const double tiles = (double)mi.num_tiles;
  const double fill = mi.fillA;
  double read_bytes, write_bytes, rows, slots;
  auto group = [](double L) { return L >= 32 ? 32.0 : std::pow(2.0, std::ceil(std::log2(L))); };
  if (mi.kind == KK_DIRECT) {
    read_bytes = tiles * fill * run_cost(mi.V * W);
    rows = tiles * fill * mi.RB;
    slots = 0.0;
  } else {
    read_bytes = tiles * fill * mi.RA * run_cost(mi.LA * W);
    rows = tiles * fill * (mi.RA + mi.RB);
    const double gA = group(mi.LA), gB = group(mi.LB);
    // idle lane slots of the warp-row mapping (the paper's "Cycles" feature,
    // L1336-1353, counted per lane group instead of per 32x32 tile)
    slots = tiles * (mi.RA * (std::ceil(mi.LA / gA) * gA - mi.LA) +
                     mi.RB * (std::ceil(mi.LB / gB) * gB - mi.LB));
  }
  write_bytes = tiles * fill * mi.RB * run_cost(mi.LB * W);
  const double bw = dev.hbm_gbs * 1e9;
  // bytes in flight (Little's law with the loaded-DRAM latency): k_direct and
  // k_tile keep up to 8 access elements per thread of loads outstanding, the
  // cp.async pipeline of k_pipe a whole tile per CTA
  const double per_cta = (mi.kind == KK_PIPE) ? (double)mi.V
                                              : std::min<double>(mi.V, kModelUnroll * mi.threads);
  const double inflight = (double)mi.occ * per_cta * W;
  const double bw_lat = dev.sms * inflight / kModelLatency;
  const double bw_eff = std::min(bw, bw_lat);
  // wave quantisation: tiles handed out over the resident CTA slots
  const double slots_chip = (double)dev.sms * std::max(1, mi.occ);
  const double steps = tiles / slots_chip;
  const double wave = std::ceil(steps) / steps;
  const double tiles_per_cta = std::ceil(steps);
  F.f[0] = 1.0;
  F.f[1] = (read_bytes + write_bytes) / bw_eff * wave;
  F.f[2] = tiles_per_cta / std::max(1, mi.occ);
  F.f[3] = slots / dev.sms;
  F.f[4] = rows / dev.sms;
  return F;
}

double predict_seconds(const ModelInput &mi, const DeviceProfile &dev) {
  const ModelFeatures F = model_features(mi, dev);
  const double *c = (mi.kind == KK_DIRECT) ? kCoefDirect
                    : (mi.kind == KK_TILE) ? kCoefTile
                                           : kCoefPipe;
  double t = 0.0;
  for (int i = 0; i < kModelNumFeatures; i++) t += c[i] * F.f[i];
  // the model can never beat one pass of the algorithmic bytes at copy speed
  const double floor_t = 2.0 * (double)mi.N * mi.W / (dev.hbm_gbs * 1e9);
  return std::max(t, floor_t);
}

}  // namespace ttlg
