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
static double run_cost(int64_t R) {
  int64_t c = (R + 31) / 32 * 32;
  if (R & 31) c += 16;
  return (double)(c < 64 ? 64 : c);
}

ModelFeatures model_features(const ModelInput &mi, const DeviceProfile &dev) {
  ModelFeatures F;
  for (double &x : F.f) x = 0.0;
  const double W = mi.W;
  const double tiles = (double)mi.num_tiles;
  const double fill = mi.fillA;
  const double sms = dev.sms;
  auto group = [](double L) {  // lanes per row: next power of two, at most 32
    double g = 1.0;
    while (g < L && g < 32.0) g *= 2.0;
    return g;
  };
  double read_bytes, runsA, opsA;
  if (mi.kind == KK_DIRECT) {
    read_bytes = tiles * fill * run_cost((int64_t)mi.V * mi.W);
    runsA = tiles * fill;
    opsA = tiles * mi.V / 32.0;
  } else {
    read_bytes = tiles * fill * mi.RA * run_cost((int64_t)mi.LA * mi.W);
    runsA = tiles * fill * mi.RA;
    // flat load walk: ceil(V / threads) access elements (k_quad: 16-byte chunks) per thread
    const double vk = mi.qk > 0 ? (double)mi.V / mi.qk : (double)mi.V;  // 16-byte chunks
    opsA = tiles * std::ceil(vk / mi.threads) * (mi.threads / 32.0);
  }
  const double write_bytes = tiles * fill * mi.RB * run_cost((int64_t)mi.LB * mi.W);
  const double runsB = tiles * fill * mi.RB;
  double opsB;
  if (mi.kind == KK_DIRECT) {
    const double gB = group(mi.LB);
    opsB = tiles * mi.RB * std::ceil(mi.LB / gB) / (32.0 / gB);
  } else if (mi.kind == KK_VEC || mi.kind == KK_BULKG) {
    // one 16-byte output chunk per thread, B-rows strided by threads / chunks-per-row
    const double rs = std::floor((double)mi.threads * std::max(1, mi.qk) / mi.LB);
    opsB = tiles * std::ceil(mi.RB / std::max(1.0, rs)) * (mi.threads / 32.0);
  } else if (mi.LB <= mi.threads) {
    // one output position per thread, B-rows (k_quad: groups of K B-rows) strided by threads / LB
    const double rs = std::floor((double)mi.threads / mi.LB);
    const double rows = mi.kind == KK_QUAD ? (double)mi.RB / std::max(1, mi.qk) : (double)mi.RB;
    opsB = tiles * std::ceil(rows / rs) * (mi.threads / 32.0);
  } else if (mi.kind == KK_QUAD) {
    opsB = tiles * ((double)mi.RB / std::max(1, mi.qk)) * std::ceil((double)mi.LB / mi.threads) *
           (mi.threads / 32.0);
  } else {
    opsB = tiles * mi.RB * std::ceil((double)mi.LB / mi.threads) * (mi.threads / 32.0);
  }
  const double sector = read_bytes + write_bytes;
  const double alg = 2.0 * mi.N * W;
  const double bw = dev.hbm_gbs * 1e9;
  // bytes in flight (Little's law with the loaded-DRAM latency): the staged
  // kernels keep a whole tile of cp.async loads in flight per CTA, k_direct up
  // to 8 access elements per thread
  const double per_cta = (mi.kind == KK_DIRECT)
                             ? std::min<double>(mi.V, kModelUnroll * mi.threads)
                             : (double)mi.V;
  const double inflight = (double)mi.occ * per_cta * W;
  const double bw_lat = sms * inflight / kModelLatency;
  // wave quantisation: tiles handed out over the resident CTA slots
  const double slots = sms * std::max(1, mi.occ);
  const double steps = tiles / slots;
  const double wave = std::ceil(steps) / steps;
  // shared-memory wavefronts beyond the conflict-free ideal (the paper's bank
  // conflicts of Orthogonal-Arbitrary, L1016-1020), per SM
  const double conf = (mi.kind == KK_DIRECT)
                          ? 0.0
                          : (mi.N / 32.0) * (mi.conf_load + mi.conf_store - 2.0) / sms;
  F.f[0] = 1.0;                                                // launch + fixed costs
  F.f[1] = alg / bw;                                           // one pass at copy speed
  F.f[2] = (sector - alg) / bw;                                // partial-sector waste
  F.f[3] = (runsA + runsB) / sms;                              // DRAM runs per SM
  F.f[4] = tiles / sms;                                        // tiles per SM
  F.f[5] = std::max(0.0, sector / std::min(bw, bw_lat) - sector / bw);  // too few bytes in flight
  F.f[6] = (wave - 1.0) * sector / bw;                         // tail wave
  F.f[7] = std::ceil(steps);                                   // sequential tiles per CTA slot
  F.f[8] = conf;                                               // extra smem wavefronts per SM
  F.f[9] = (opsA + opsB) / sms;                                // warp-level row work per SM
  return F;
}

double predict_seconds(const ModelInput &mi, const DeviceProfile &dev) {
  const ModelFeatures F = model_features(mi, dev);
  const double *c = (mi.kind == KK_DIRECT)  ? kCoefDirect
                    : (mi.kind == KK_TILE)  ? kCoefTile
                    : (mi.kind == KK_QUAD)  ? kCoefQuad
                    : (mi.kind == KK_BULKQ || mi.kind == KK_TMA) ? kCoefBulkQ
                    : (mi.kind == KK_BULKG) ? kCoefBulkG
                    : (mi.kind == KK_VEC)   ? kCoefVec
                                            : kCoefPipe;
  double t = 0.0;
  for (int i = 0; i < kModelNumFeatures; i++) t += c[i] * F.f[i];
  // the model can never beat one pass of the algorithmic bytes at copy speed
  const double floor_t = 2.0 * (double)mi.N * mi.W / (dev.hbm_gbs * 1e9);
  return std::max(t, floor_t);
}

}  // namespace ttlg

// ---- ranking stage: boosted regression trees (model_gbt.h) --------------------
#include "model_gbt.h"
#include "model_gbt2.h"
#include "model_gbt3.h"

namespace ttlg {

// Plan descriptor fed to the trees; tools/calibrate_gbt.py desc() mirrors it.
void model_descriptor(const ModelInput &mi, const DeviceProfile &dev, double *d) {
  const ModelFeatures F = model_features(mi, dev);
  const double W = mi.W, V = mi.V;
  const double occ = std::max(1, mi.occ), th = mi.threads;
  const double LAb = (mi.kind == KK_DIRECT ? V : (double)mi.LA) * W;
  const double bytes = 2.0 * (double)mi.N * W;
  d[0] = mi.kind;
  d[1] = std::log2(W);
  d[2] = std::log2(LAb);
  d[3] = std::log2((double)mi.LB * W);
  d[4] = std::log2(V * W);
  d[5] = th / 256.0;
  d[6] = occ;
  d[7] = occ * th / 2048.0;
  d[8] = std::log2((double)mi.num_tiles);
  d[9] = F.f[2] / std::max(F.f[1], 1e-12);
  d[10] = F.f[8] / std::max(1.0, bytes / 1e9);
  d[11] = (double)mi.num_tiles / (dev.sms * occ);
  const double RA = V / (mi.kind == KK_DIRECT ? V : (double)mi.LA), RB = V / (double)mi.LB;
  d[12] = std::log2(V / th);                       // elements per thread
  d[13] = (RA + RB + (double)mi.LB) / th;          // per-CTA table entries per thread
  d[14] = mi.fillA;                                // useful fraction of the tile grid
  d[15] = std::ceil((double)mi.num_tiles / std::max(1, mi.grid));  // tiles per CTA
  d[16] = std::log2(bytes);  // total traffic: launch-dominated / L2-resident below ~2x L2
  d[17] = mi.nstage;         // k_bulk ring stages (0: other kernels)
}

double predict_ranked_seconds(const ModelInput &mi, const DeviceProfile &dev) {
  double t;
  predict_ranked_batch(&mi, 1, dev, &t);
  return t;
}

// The candidates' traversals of one tree are independent: interleaving them
// (tree-major, a fixed group of kB candidates so that the node indices stay in
// registers) lets the core overlap their dependent node loads.  Groups are
// padded with copies of their last candidate; every candidate's sum is
// accumulated in tree order, exactly as a one-at-a-time walk would.
template <int NT, int D>
static void gbt_batch(const ModelInput *mis, int n, const DeviceProfile &dev, double *out,
                      double init, const int8_t (&F_)[NT][(1 << D) - 1],
                      const float (&T_)[NT][(1 << D) - 1], const float (&V_)[NT][1 << D]) {
  constexpr int kB = 8;
  constexpr int NI = (1 << D) - 1;
  float d[kB][kGbtDesc];
  double s[kB];
  for (int b0 = 0; b0 < n; b0 += kB) {
    const int m = std::min(kB, n - b0);
    for (int c = 0; c < m; c++) {
      double dd[kGbtDesc];
      model_descriptor(mis[b0 + c], dev, dd);
      for (int k = 0; k < kGbtDesc; k++) d[c][k] = (float)dd[k];  // sklearn splits on float32
    }
    for (int c = m; c < kB; c++)
      for (int k = 0; k < kGbtDesc; k++) d[c][k] = d[m - 1][k];
    for (int c = 0; c < kB; c++) s[c] = init;
    for (int t = 0; t < NT; t++) {
      const int8_t *F = F_[t];
      const float *T = T_[t];
      int idx[kB];
#pragma GCC unroll 8
      for (int c = 0; c < kB; c++) idx[c] = 0;
#pragma GCC unroll 8
      for (int l = 0; l < D; l++) {
#pragma GCC unroll 8
        for (int c = 0; c < kB; c++) {
          const int i = idx[c];
          idx[c] = 2 * i + 1 + (d[c][F[i]] > T[i]);
        }
      }
#pragma GCC unroll 8
      for (int c = 0; c < kB; c++) s[c] += V_[t][idx[c] - NI];
    }
    for (int c = 0; c < m; c++) {
      const ModelInput &mi = mis[b0 + c];
      const double ideal = 2.0 * (double)mi.N * mi.W / (dev.hbm_gbs * 1e9);
      out[b0 + c] = std::exp(std::max(s[c], 0.0)) * ideal;  // never below one pass at copy speed
    }
  }
}

void predict_ranked_batch(const ModelInput *mis, int n, const DeviceProfile &dev, double *out) {
  gbt_batch<kGbtTrees, kGbtDepth>(mis, n, dev, out, kGbtInit, kGbtF, kGbtT, kGbtV);
}

void predict_ranked2_batch(const ModelInput *mis, int n, const DeviceProfile &dev, double *out) {
  gbt_batch<kGbt2Trees, kGbt2Depth>(mis, n, dev, out, kGbt2Init, kGbt2F, kGbt2T, kGbt2V);
}

void predict_ranked3_batch(const ModelInput *mis, int n, const DeviceProfile &dev, double *out) {
  gbt_batch<kGbt3Trees, kGbt3Depth>(mis, n, dev, out, kGbt3Init, kGbt3F, kGbt3T, kGbt3V);
}

}  // namespace ttlg
