// model_coeffs.h -- coefficients of the B200 performance model (model.cpp).
// Initial physically-motivated values; replaced by tools/calibrate.py with a
// least-squares fit on B200 measurements (§V L1402-1419 method).
#pragma once

namespace ttlg {
constexpr int kModelNumFeatures = 10;
constexpr double kModelLatency = 1.0e-6;     // loaded DRAM latency (s)
constexpr double kModelUnroll = 8.0;         // loads in flight per thread (k_direct, k_tile)
// features: see model.cpp model_features()
constexpr double kCoefDirect[kModelNumFeatures] = {5e-6, 1.0, 1.0, 0, 0, 0.1, 1.0, 1e-6, 0, 0};
constexpr double kCoefTile[kModelNumFeatures] = {10e-6, 1.0, 0.3, 1e-9, 0, 0.2, 2.0, 2e-6, 1e-9, 0};
constexpr double kCoefPipe[kModelNumFeatures] = {10e-6, 0.6, 0.3, 0.6e-9, 1e-8, 0, 1.5, 2e-6, 1e-9, 0};
constexpr const char *kModelSource = "default (uncalibrated)";
}  // namespace ttlg
