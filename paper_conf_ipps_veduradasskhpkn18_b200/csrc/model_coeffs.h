// model_coeffs.h -- coefficients of the B200 performance model (model.cpp).
// Initial physically-motivated values; replaced by tools/calibrate.py with a
// least-squares fit on B200 measurements (§V L1402-1419 method).
#pragma once

namespace ttlg {
constexpr int kModelNumFeatures = 10;
constexpr double kModelLatency = 1.0e-6;     // loaded DRAM latency (s)
constexpr double kModelUnroll = 8.0;         // loads in flight per thread (k_direct, k_tile)
// features: see model.cpp model_features()
constexpr double kCoefDirect[kModelNumFeatures] = {9.164375e-06, 8.819829e-01, 3.164949e-01, 8.371602e-11, 0.000000e+00, 8.554402e-01, 1.056894e-01, 1.642348e-07, 0.000000e+00, 1.013443e-09};
constexpr double kCoefTile[kModelNumFeatures] = {9.982902e-06, 8.427038e-01, 4.334665e-02, 8.618741e-11, 0.000000e+00, 4.841563e-01, 1.016202e-01, 2.755672e-07, 3.866049e-10, 1.430394e-09};
constexpr double kCoefPipe[kModelNumFeatures] = {1.026968e-05, 8.775007e-01, 0.000000e+00, 0.000000e+00, 0.000000e+00, 1.356205e-01, 9.692115e-02, 0.000000e+00, 3.283680e-10, 1.622797e-09};
constexpr double kCoefQuad[kModelNumFeatures] = {9.362660e-06, 8.433642e-01, 0.000000e+00, 2.139055e-10, 0.000000e+00, 4.747816e-01, 3.070801e-01, 2.384217e-07, 0.000000e+00, 2.564201e-09};
constexpr double kCoefBulkQ[kModelNumFeatures] = {1.098686e-05, 9.381789e-01, 0.000000e+00, 3.511322e-10, 0.000000e+00, 0.000000e+00, 8.499278e-01, 1.079595e-07, 0.000000e+00, 6.053561e-10};
constexpr double kCoefBulkG[kModelNumFeatures] = {1.103068e-05, 9.460298e-01, 2.133818e-01, 4.293525e-10, 0.000000e+00, 6.871199e-02, 2.902389e-01, 0.000000e+00, 0.000000e+00, 1.428276e-09};
constexpr double kCoefVec[kModelNumFeatures] = {1.002946e-05, 9.768813e-01, 1.070989e+00, 1.026754e-10, 0.000000e+00, 4.146743e-01, 1.519608e-01, 3.293139e-07, 0.000000e+00, 1.326551e-09};
constexpr const char *kModelSource = "B200 fit (828 cases, 75110 points, rel<=1.5): direct: train 5.6% test 5.4% (n=1610+356); tile: train 8.3% test 8.0% (n=13449+3182); pipe: train 8.1% test 7.7% (n=11526+2739); quad: train 8.2% test 7.7% (n=5340+1293); bulkq: train 7.0% test 6.6% (n=130+32); bulkg: train 6.7% test 7.5% (n=590+124); vec: train 7.5% test 6.8% (n=1338+377); regret 20.6%";
}  // namespace ttlg
