// model_coeffs.h -- coefficients of the B200 performance model (model.cpp).
// Initial physically-motivated values; replaced by tools/calibrate.py with a
// least-squares fit on B200 measurements (§V L1402-1419 method).
#pragma once

namespace ttlg {
constexpr int kModelNumFeatures = 10;
constexpr double kModelLatency = 1.0e-6;     // loaded DRAM latency (s)
constexpr double kModelUnroll = 8.0;         // loads in flight per thread (k_direct, k_tile)
// features: see model.cpp model_features()
constexpr double kCoefDirect[kModelNumFeatures] = {4.373133e-06, 8.920645e-01, 1.756448e+00, 4.022023e-10, 0.000000e+00, 4.490829e-01, 4.286812e-01, 6.175414e-07, 0.000000e+00, 7.828605e-10};
constexpr double kCoefTile[kModelNumFeatures] = {8.873988e-06, 7.329123e-01, 4.412852e-01, 3.203440e-10, 0.000000e+00, 8.750968e-02, 2.233884e-01, 1.136793e-06, 2.295258e-10, 1.333646e-09};
constexpr double kCoefPipe[kModelNumFeatures] = {8.021830e-06, 8.330551e-01, 7.908181e-01, 2.106668e-10, 5.316145e-08, 2.988828e-02, 0.000000e+00, 3.750311e-07, 1.897926e-10, 1.544756e-09};
constexpr const char *kModelSource = "B200 fit (176 cases, 17252 points, rel<=1.5): direct: train 4.3% test 10.3% (n=266+59); tile: train 7.7% test 7.3% (n=2358+594); pipe: train 7.4% test 7.1% (n=2365+558); regret 9.8%";
}  // namespace ttlg
