// attn_exact.cuh -- the exact CUDA-core path of one attention row, shared by
// the two attention kernels (attention.cu, attention_tc.cu): rows whose
// fixed-reference softmax overflowed fp16 (row sum not finite) are
// recomputed here.  Eqn 1 with the reachability mask, reading R1.
#pragma once
#include <cuda_fp16.h>

#include "internal.h"

namespace predtop {
namespace {

// Exact row on the CUDA cores (rare path): fp32 scores from the fp16 q, k
// (log2 units), two passes over the allowed keys (max, then sum and P.V).
template <int DH>
__device__ __noinline__ void exact_row(const __half* __restrict__ qkv, int64_t n0, int N, int row, int h,
                                       int dmodel, const uint64_t* __restrict__ Mrow, __half* __restrict__ outrow) {
  float q[DH];
  const __half* qr = qkv + (n0 + row) * 3 * dmodel + h * DH;
#pragma unroll
  for (int j = 0; j < DH; ++j) q[j] = __half2float(qr[j]);
  auto allowed = [&](int k) { return ((Mrow[k >> 6] >> mask_pos(k & 63)) & 1ull) != 0ull; };
  auto score = [&](int k) {
    const __half* kr = qkv + (n0 + k) * 3 * dmodel + dmodel + h * DH;
    float s = 0.f;
#pragma unroll
    for (int j = 0; j < DH; ++j) s = fmaf(q[j], __half2float(kr[j]), s);
    return s;
  };
  float mx = -INFINITY;
  for (int k = 0; k < N; ++k)
    if (allowed(k)) mx = fmaxf(mx, score(k));
  float l = 0.f, o[DH];
#pragma unroll
  for (int j = 0; j < DH; ++j) o[j] = 0.f;
  for (int k = 0; k < N; ++k) {
    if (!allowed(k)) continue;
    const float p = exp2f(score(k) - mx);
    l += p;
    const __half* vr = qkv + (n0 + k) * 3 * dmodel + 2 * dmodel + h * DH;
#pragma unroll
    for (int j = 0; j < DH; ++j) o[j] = fmaf(p, __half2float(vr[j]), o[j]);
  }
  const float inv = 1.f / l;
#pragma unroll
  for (int j = 0; j < DH; ++j) outrow[j] = __float2half_rn(o[j] * inv);
}

}  // namespace
}  // namespace predtop
