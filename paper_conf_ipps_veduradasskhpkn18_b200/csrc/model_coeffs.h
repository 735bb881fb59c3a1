// model_coeffs.h -- coefficients of the B200 performance model (model.cpp).
// Initial physically-motivated values; replaced by tools/calibrate.py with a
// least-squares fit on B200 measurements (§V L1402-1419 method).
#pragma once

namespace ttlg {
constexpr int kModelNumFeatures = 10;
constexpr double kModelLatency = 1.0e-6;     // loaded DRAM latency (s)
constexpr double kModelUnroll = 8.0;         // loads in flight per thread (k_direct, k_tile)
// features: see model.cpp model_features()
constexpr double kCoefDirect[kModelNumFeatures] = {6.864575e-06, 8.651936e-01, 9.614488e-01, 9.125569e-11, 1.499405e-10, 4.959539e-01, 2.254551e-01, 6.084763e-07, 0.000000e+00, 1.051936e-09};
constexpr double kCoefTile[kModelNumFeatures] = {9.051371e-06, 5.877510e-01, 1.426655e-01, 5.176052e-10, 0.000000e+00, 0.000000e+00, 4.584064e-02, 1.809984e-06, 2.257271e-11, 1.886434e-09};
constexpr double kCoefPipe[kModelNumFeatures] = {6.578404e-06, 5.461088e-01, 0.000000e+00, 4.396413e-10, 2.259999e-08, 0.000000e+00, 0.000000e+00, 1.564538e-06, 0.000000e+00, 2.021733e-09};
constexpr const char *kModelSource = "B200 fit (402 cases, 31238 points, rel<=3.0): direct: train 5.4% test 7.9% (n=1012+117); tile: train 12.0% test 12.0% (n=10498+2869); pipe: train 11.3% test 11.9% (n=7331+2168); regret 12.5%";
}  // namespace ttlg
