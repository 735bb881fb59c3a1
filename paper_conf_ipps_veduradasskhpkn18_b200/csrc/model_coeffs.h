// model_coeffs.h -- coefficients of the B200 performance model (model.cpp).
// Initial physically-motivated values; replaced by tools/calibrate.py with a
// least-squares fit on B200 measurements (§V L1402-1419 method).
#pragma once

namespace ttlg {
constexpr int kModelNumFeatures = 5;
constexpr double kModelLatency = 1.0e-6;     // loaded DRAM latency (s)
constexpr double kModelUnroll = 8.0;         // loads in flight per thread (k_direct, k_tile)
// features: [launch, memory-time, tiles-per-CTA/occ, idle-lane-slots/SM, rows/SM]
constexpr double kCoefDirect[kModelNumFeatures] = {2.5e-6, 1.0, 0.15e-6, 0.0, 0.3e-9};
constexpr double kCoefTile[kModelNumFeatures] = {2.5e-6, 1.0, 0.30e-6, 0.05e-9, 0.3e-9};
constexpr double kCoefPipe[kModelNumFeatures] = {2.5e-6, 1.0, 0.30e-6, 0.05e-9, 0.3e-9};
constexpr const char *kModelSource = "default (uncalibrated)";
}  // namespace ttlg
