// model_coeffs.h -- coefficients of the B200 performance model (model.cpp).
// Initial physically-motivated values; replaced by tools/calibrate.py with a
// least-squares fit on B200 measurements (§V L1402-1419 method).
#pragma once

namespace ttlg {
constexpr int kModelNumFeatures = 10;
constexpr double kModelLatency = 1.0e-6;     // loaded DRAM latency (s)
constexpr double kModelUnroll = 8.0;         // loads in flight per thread (k_direct, k_tile)
// features: see model.cpp model_features()
constexpr double kCoefDirect[kModelNumFeatures] = {6.347335e-06, 8.843837e-01, 0.000000e+00, 1.981821e-10, 0.000000e+00, 7.767651e-01, 2.173065e-01, 2.140969e-07, 0.000000e+00, 1.156034e-09};
constexpr double kCoefTile[kModelNumFeatures] = {9.119138e-06, 8.575126e-01, 0.000000e+00, 4.233825e-11, 0.000000e+00, 3.127599e-01, 0.000000e+00, 3.477675e-07, 4.100381e-10, 1.423466e-09};
constexpr double kCoefPipe[kModelNumFeatures] = {8.107715e-06, 8.890406e-01, 0.000000e+00, 0.000000e+00, 0.000000e+00, 1.413858e-01, 2.939497e-01, 0.000000e+00, 4.139314e-10, 1.699514e-09};
constexpr double kCoefQuad[kModelNumFeatures] = {1.022917e-05, 8.662868e-01, 0.000000e+00, 1.546947e-10, 0.000000e+00, 3.629821e-01, 3.003596e-01, 3.371972e-07, 0.000000e+00, 2.147497e-09};
constexpr const char *kModelSource = "B200 fit (282 cases, 38128 points, rel<=1.5): direct: train 4.3% test 4.2% (n=482+62); tile: train 7.9% test 7.6% (n=5959+1653); pipe: train 7.8% test 7.6% (n=5785+1612); quad: train 7.7% test 6.7% (n=2225+678); regret 14.7%";
}  // namespace ttlg
