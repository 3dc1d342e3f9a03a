// calibrate.cpp -- offline calibration of the FMPQ channel permutation and precision tags
// (host C++, no device).  P:L138-144 / Fig. 4(d): outlier channels, located on sampled
// calibration activations, are permuted into as few 128-channel blocks as possible; those
// blocks are tagged INT8 and the rest INT4.  Outlier rule (reading R8/R16): amax[k] > ratio *
// median(amax), the paper's "tenfold" being ratio = 10.
#include <algorithm>
#include <cmath>
#include <vector>
#include "internal.h"

using namespace comet;

extern "C" comet_status_t comet_calibrate_perm(const float* amax_host, int64_t K, double ratio,
                                               int32_t* perm_host, uint8_t* tags_host,
                                               int64_t* n_outliers) {
  if (!amax_host || !perm_host || !tags_host) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  if (K < kBlockK || K % kBlockK != 0 || K > (int64_t)kBlockK * kMaxBlocks)
    return fail(COMET_ERR_UNSUPPORTED_SHAPE, "K must be a positive multiple of 128, <= 131072");
  if (!(ratio > 0.0) || !std::isfinite(ratio)) return fail(COMET_ERR_INVALID_ARG, "ratio must be finite and > 0");
  std::vector<double> v((size_t)K);
  for (int64_t k = 0; k < K; ++k) {
    const float a = amax_host[k];
    if (!std::isfinite(a) || a < 0.f) return fail(COMET_ERR_INVALID_ARG, "amax values must be finite and >= 0");
    v[(size_t)k] = (double)a;
  }
  // median: the K/2-th order statistic (and its predecessor for even K)
  std::vector<double> s = v;
  const size_t h = (size_t)K / 2;
  std::nth_element(s.begin(), s.begin() + h, s.end());
  double med = s[h];
  if (K % 2 == 0) {
    const double lo = *std::max_element(s.begin(), s.begin() + h);
    med = (lo + med) / 2.0;
  }
  const double thr = ratio * med;
  int64_t n = 0;
  for (int64_t k = 0; k < K; ++k)
    if (v[(size_t)k] > thr) perm_host[n++] = (int32_t)k;
  int64_t j = n;
  for (int64_t k = 0; k < K; ++k)
    if (!(v[(size_t)k] > thr)) perm_host[j++] = (int32_t)k;
  const int64_t nb = K / kBlockK, n8 = (n + kBlockK - 1) / kBlockK;
  for (int64_t b = 0; b < nb; ++b) tags_host[b] = b < n8 ? 1 : 0;
  if (n_outliers) *n_outliers = n;
  return COMET_OK;
}
