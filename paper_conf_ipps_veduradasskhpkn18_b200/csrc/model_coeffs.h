// model_coeffs.h -- coefficients of the B200 performance model (model.cpp).
// Initial physically-motivated values; replaced by tools/calibrate.py with a
// least-squares fit on B200 measurements (§V L1402-1419 method).
#pragma once

namespace ttlg {
constexpr int kModelNumFeatures = 10;
constexpr double kModelLatency = 1.0e-6;     // loaded DRAM latency (s)
constexpr double kModelUnroll = 8.0;         // loads in flight per thread (k_direct, k_tile)
// features: see model.cpp model_features()
constexpr double kCoefDirect[kModelNumFeatures] = {5.054199e-06, 8.291805e-01, 8.132743e-01, 5.695055e-10, 0.000000e+00, 3.662638e-01, 5.259155e-01, 7.577827e-07, 0.000000e+00, 9.814919e-10};
constexpr double kCoefTile[kModelNumFeatures] = {1.126557e-05, 4.881508e-01, 1.188975e-01, 2.779425e-10, 0.000000e+00, 0.000000e+00, 0.000000e+00, 1.963278e-06, 0.000000e+00, 2.138978e-09};
constexpr double kCoefPipe[kModelNumFeatures] = {7.285476e-06, 4.141721e-01, 0.000000e+00, 4.030560e-10, 4.019617e-08, 0.000000e+00, 0.000000e+00, 1.612127e-06, 0.000000e+00, 2.398952e-09};
constexpr const char *kModelSource = "B200 fit (176 cases, 18358 points, rel<=3.0): direct: train 5.8% test 12.7% (n=313+55); tile: train 11.5% test 10.5% (n=4499+1101); pipe: train 11.5% test 11.3% (n=4520+1078); regret 12.2%";
}  // namespace ttlg
