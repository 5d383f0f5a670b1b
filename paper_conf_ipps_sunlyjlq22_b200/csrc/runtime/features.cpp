// features.cpp -- stencil representation (§IV-C):
// the fixed-size binary tensor of Fig. 6 and the Table II feature set, the
// inputs StencilMART's models consume next to the label this library produces.
//
//   "we convert the offset of the accessed neighbor points from the central
//    point into the location of the non-zero elements of a tensor";
//   a 2-D stencil of maximum order 4 becomes a 9 x 9 tensor.
//   Table II: order (maximum extent of non-zeros), nnz, sparsity
//   (density of non-zeros in the tensor), nnz_order-n, nnzRatio_order-n.
// Readings: extent = Chebyshev ring; the tensor is the fixed
// (2*4+1)^d embedding, so sparsity = nnz / 9^d; nnzRatio_order-n =
// nnz_order-n / |ring n| with |ring n| = (2n+1)^d - (2n-1)^d.
#include <cstring>

#include "internal.h"

using namespace smart_rt;

static int check(int ndim, int order, const uint8_t* access) {
  if ((ndim != 2 && ndim != 3) || order < 1 || order > 4 || !access)
    SM_FAIL(STENCIL_E_INVAL, "ndim in {2,3}, order in 1..4, access non-null");
  const int w = 2 * order + 1, n = ndim == 3 ? w * w * w : w * w;
  for (int t = 0; t < n; ++t)
    if (access[t] > 1) SM_FAIL(STENCIL_E_INVAL, "access tensor must be binary");
  return STENCIL_OK;
}

extern "C" int stencil_features(int ndim, int order, const uint8_t* access, stencil_features_t* out) {
  clear_error();
  SM_TRY(check(ndim, order, access));
  if (!out) SM_FAIL(STENCIL_E_INVAL, "null output");
  memset(out, 0, sizeof *out);
  const int w = 2 * order + 1, n = ndim == 3 ? w * w * w : w * w;
  int maxring = 0;
  for (int t = 0; t < n; ++t) {
    if (!access[t]) continue;
    int a = ndim == 3 ? t / (w * w) - order : 0;
    int b = (t / w) % w - order, c = t % w - order;
    if (a < 0) a = -a;
    if (b < 0) b = -b;
    if (c < 0) c = -c;
    int ring = a > b ? a : b;
    ring = ring > c ? ring : c;
    out->nnz += 1;
    if (ring > 0) out->nnz_order[ring - 1] += 1;
    if (ring > maxring) maxring = ring;
  }
  out->order = maxring;
  const double full = ndim == 3 ? 729.0 : 81.0;
  out->sparsity = out->nnz / full;
  for (int k = 1; k <= 4; ++k) {
    const long s1 = 2 * k + 1, s0 = 2 * k - 1;
    const double ring_size = ndim == 3 ? (double)(s1 * s1 * s1 - s0 * s0 * s0) : (double)(s1 * s1 - s0 * s0);
    out->nnz_ratio[k - 1] = out->nnz_order[k - 1] / ring_size;
  }
  return STENCIL_OK;
}

extern "C" int stencil_embed_tensor(int ndim, int order, const uint8_t* access, uint8_t* out9) {
  clear_error();
  SM_TRY(check(ndim, order, access));
  if (!out9) SM_FAIL(STENCIL_E_INVAL, "null output");
  const int w = 2 * order + 1, sh = 4 - order;
  memset(out9, 0, ndim == 3 ? 729 : 81);
  if (ndim == 3) {
    for (int a = 0; a < w; ++a)
      for (int b = 0; b < w; ++b)
        for (int c = 0; c < w; ++c) out9[((a + sh) * 9 + b + sh) * 9 + c + sh] = access[(a * w + b) * w + c];
  } else {
    for (int b = 0; b < w; ++b)
      for (int c = 0; c < w; ++c) out9[(b + sh) * 9 + c + sh] = access[b * w + c];
  }
  return STENCIL_OK;
}
