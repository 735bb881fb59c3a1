// model.h -- B200 performance model (§V, re-derived).
//
// The paper fits, per kernel, a linear regression of time on features of the
// chosen slices (Volume, NumBlocks, input/output slice, "Cycles" for idle
// lanes on partial tiles; Table II).  On B200 the transposition is
// HBM-bound, so the features are bytes-first: the DRAM sectors the schedule
// touches (run lengths -> 32-byte sectors), the bytes-in-flight limit
// (occupancy x staged elements), tail waves of the persistent grid, per-tile
// synchronisation overhead and idle lanes.  Coefficients are fitted offline
// on B200 measurements (tools/calibrate.py) and shipped in model_coeffs.h.
#pragma once

#include <stdint.h>

#include "ttlg_internal.h"

namespace ttlg {

struct ModelInput {
  int kind, schema, W;
  int64_t N;  // access elements
  int V, LA, LB, RA, RB;
  int64_t num_tiles;
  int threads, smem_bytes, occ, grid;
  double fillA;  // useful fraction of the tile grid (partial tiles)
  double conf_load, conf_store;  // smem wavefronts / ideal for one warp access (>= 1)
  int qk;                        // k_quad chunk elements (0: scalar kernels)
  int nstage;                    // k_bulk: tile buffers in the ring
};

struct ModelFeatures {
  double f[12];  // see model.cpp
};

// Feature vector (units: seconds at the reference bandwidth, or counts).
ModelFeatures model_features(const ModelInput &mi, const DeviceProfile &dev);
double predict_seconds(const ModelInput &mi, const DeviceProfile &dev);
// ranking stage (boosted trees over model_descriptor); seconds
constexpr int kGbtDesc = 18;  // descriptor length (tools/calibrate_gbt.py desc())
void model_descriptor(const ModelInput &mi, const DeviceProfile &dev, double *d);
double predict_ranked_seconds(const ModelInput &mi, const DeviceProfile &dev);
void predict_ranked_batch(const ModelInput *mis, int n, const DeviceProfile &dev, double *out);
// second tree set (model_gbt2.h: refit with k_vec / k_bulk and small tensors in the
// data): decides whether a k_vec candidate beats the first set's winner
void predict_ranked2_batch(const ModelInput *mis, int n, const DeviceProfile &dev, double *out);
// third tree set (model_gbt3.h: the second set's data with the tensors below
// 32 MB re-timed as CUDA graphs of back-to-back launches, cal35 -- an event
// pair around one launch after a sync also times the host's launch latency):
// ranks and reports plans moving less than kSmallTraffic bytes
void predict_ranked3_batch(const ModelInput *mis, int n, const DeviceProfile &dev, double *out);
// k_vec replaces the winner only when predicted this much faster by the second set
constexpr double kVecMargin = 0.95;
// ... and is considered only when the first set predicts its winner below this
// fraction of the copy speed
constexpr double kVecChallenge = 0.8;
// plans moving less than this many bytes (2 N s) are ranked by the second set
constexpr double kSmallTraffic = 32.0 * 1024 * 1024;

// k_deint (one streaming pass, 16-byte accesses both ways): time = this
// factor x the one-pass ideal 2*N*s / HBM bandwidth -- measured on B200 at
// the config-4 sizes, n0 = 2..5: 5.41-5.63 TB/s back to back (exp49)
constexpr double kDeintFactor = 1.18;
// k_blk (one streaming pass, one warp per closed leading block): the same
// form, measured on B200 (r2e30, graph timing): 16^6 / 24^6 fp64 `1 0 ...`
// 5.65-5.7 TB/s, 15^6 / 17^6 5.8-6.0 TB/s -> 1.10-1.16 x the ideal
constexpr double kBlkFactor = 1.13;

}  // namespace ttlg
