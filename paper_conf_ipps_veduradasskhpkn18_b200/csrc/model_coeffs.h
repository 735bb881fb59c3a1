// model_coeffs.h -- coefficients of the B200 performance model (model.cpp).
// Initial physically-motivated values; replaced by tools/calibrate.py with a
// least-squares fit on B200 measurements (§V L1402-1419 method).
#pragma once

namespace ttlg {
constexpr int kModelNumFeatures = 10;
constexpr double kModelLatency = 1.0e-6;     // loaded DRAM latency (s)
constexpr double kModelUnroll = 8.0;         // loads in flight per thread (k_direct, k_tile)
// features: see model.cpp model_features()
constexpr double kCoefDirect[kModelNumFeatures] = {3.487685e-06, 8.104583e-01, 7.212736e-01, 6.918417e-10, 0.000000e+00, 2.609106e-01, 6.292655e-01, 8.807121e-07, 0.000000e+00, 1.041337e-09};
constexpr double kCoefTile[kModelNumFeatures] = {1.016694e-05, 5.255828e-01, 1.731233e-01, 4.057429e-10, 0.000000e+00, 0.000000e+00, 2.724066e-01, 1.943307e-06, 5.811676e-11, 1.716047e-09};
constexpr double kCoefPipe[kModelNumFeatures] = {6.559314e-06, 4.518758e-01, 0.000000e+00, 5.001977e-10, 4.830940e-08, 0.000000e+00, 0.000000e+00, 1.442755e-06, 0.000000e+00, 2.204548e-09};
constexpr const char *kModelSource = "B200 fit (176 cases, 18270 points, rel<=3.0): direct: train 6.0% test 13.2% (n=322+58); tile: train 11.6% test 10.8% (n=4549+1089); pipe: train 12.1% test 11.6% (n=4421+1077); regret 11.3%";
}  // namespace ttlg
