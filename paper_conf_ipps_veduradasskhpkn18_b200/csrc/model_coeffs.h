// model_coeffs.h -- coefficients of the B200 performance model (model.cpp).
// Initial physically-motivated values; replaced by tools/calibrate.py with a
// least-squares fit on B200 measurements (§V L1402-1419 method).
#pragma once

namespace ttlg {
constexpr int kModelNumFeatures = 10;
constexpr double kModelLatency = 1.0e-6;     // loaded DRAM latency (s)
constexpr double kModelUnroll = 8.0;         // loads in flight per thread (k_direct, k_tile)
// features: see model.cpp model_features()
constexpr double kCoefDirect[kModelNumFeatures] = {6.621356e-06, 8.801143e-01, 8.640416e-02, 1.966767e-10, 0.000000e+00, 8.763387e-01, 2.180839e-01, 2.113898e-07, 0.000000e+00, 1.182271e-09};
constexpr double kCoefTile[kModelNumFeatures] = {8.564110e-06, 8.672552e-01, 4.235581e-02, 3.343247e-11, 0.000000e+00, 3.600222e-01, 8.875134e-02, 2.948236e-07, 3.549572e-10, 1.462520e-09};
constexpr double kCoefPipe[kModelNumFeatures] = {7.472125e-06, 9.025470e-01, 0.000000e+00, 0.000000e+00, 0.000000e+00, 1.375855e-01, 4.479036e-01, 0.000000e+00, 3.127622e-10, 1.671868e-09};
constexpr double kCoefQuad[kModelNumFeatures] = {8.068869e-06, 8.957848e-01, 0.000000e+00, 1.501453e-10, 0.000000e+00, 3.723977e-01, 1.773548e-01, 2.590639e-07, 0.000000e+00, 2.316751e-09};
constexpr double kCoefBulkQ[kModelNumFeatures] = {1.098686e-05, 9.381789e-01, 0.000000e+00, 3.511322e-10, 0.000000e+00, 0.000000e+00, 8.499278e-01, 1.079595e-07, 0.000000e+00, 6.053561e-10};
constexpr double kCoefBulkG[kModelNumFeatures] = {1.103068e-05, 9.460298e-01, 2.133818e-01, 4.293525e-10, 0.000000e+00, 6.871199e-02, 2.902389e-01, 0.000000e+00, 0.000000e+00, 1.428276e-09};
constexpr double kCoefVec[kModelNumFeatures] = {1.002946e-05, 9.768813e-01, 1.070989e+00, 1.026754e-10, 0.000000e+00, 4.146743e-01, 1.519608e-01, 3.293139e-07, 0.000000e+00, 1.326551e-09};
constexpr const char *kModelSource = "B200 fit (362 cases, 43650 points, rel<=1.5): direct: train 4.7% test 7.8% (n=854+167); tile: train 7.9% test 8.0% (n=7618+1987); pipe: train 7.7% test 7.8% (n=6688+1699); quad: train 8.0% test 7.2% (n=2853+906); regret 15.9%; k_vec / k_bulk: cal33 fit (828 cases, 75110 points, rel<=1.5): vec test 6.8%, bulkq 6.6%, bulkg 7.5%";
}  // namespace ttlg
