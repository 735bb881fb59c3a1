// model_coeffs.h -- coefficients of the B200 performance model (model.cpp).
// Initial physically-motivated values; replaced by tools/calibrate.py with a
// least-squares fit on B200 measurements (§V L1402-1419 method).
#pragma once

namespace ttlg {
constexpr int kModelNumFeatures = 10;
constexpr double kModelLatency = 1.0e-6;     // loaded DRAM latency (s)
constexpr double kModelUnroll = 8.0;         // loads in flight per thread (k_direct, k_tile)
// features: see model.cpp model_features()
constexpr double kCoefDirect[kModelNumFeatures] = {5.965063e-06, 8.795839e-01, 1.626998e+00, 3.761750e-10, 0.000000e+00, 3.970539e-01, 3.584750e-01, 6.288623e-07, 0.000000e+00, 8.114223e-10};
constexpr double kCoefTile[kModelNumFeatures] = {1.012157e-05, 9.854213e-01, 8.898444e-01, 2.130786e-10, 0.000000e+00, 2.457571e-01, 2.408219e-01, 6.020275e-07, 2.316475e-10, 1.457804e-09};
constexpr double kCoefPipe[kModelNumFeatures] = {8.357488e-06, 7.803404e-01, 8.418410e-01, 2.733867e-10, 4.795938e-08, 6.562379e-02, 0.000000e+00, 5.173482e-07, 1.903181e-10, 1.656333e-09};
constexpr const char *kModelSource = "B200 fit (176 cases, 17492 points, rel<=1.5): direct: train 4.2% test 11.0% (n=259+46); tile: train 7.9% test 8.0% (n=1487+384); pipe: train 8.0% test 8.1% (n=2676+668); regret 10.0%";
}  // namespace ttlg
