// plan.cu -- K9: white-box pipeline model, Eqn 4 (SV):
//     T_p = sum_{i<=S_p} t_{p,i} + (B_p - 1) * max_i t_{p,i}
// evaluated per plan in fp64 in the canonical order of reading R13 (sort the
// fp32 stage latencies ascending, add them left to right with round-to-
// nearest, then one rounded multiply and one rounded add -- no FMA), so the
// result is a function of the multiset of stage latencies and bit-identical
// to the CPU oracle.  Plus a deterministic argmin by (T, plan id).
#include <climits>

#include "internal.h"

namespace predtop {

__global__ void k_plan(int64_t P, const int64_t* __restrict__ plan_ptr,
                       const int32_t* __restrict__ plan_stage, const int32_t* __restrict__ B,
                       const float* __restrict__ t, int64_t num_stages, double* __restrict__ T,
                       unsigned long long* first_bad) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < P;
       p += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b0 = plan_ptr[p], S = plan_ptr[p + 1] - b0;
    const int32_t mb = B[p];
    bool ok = S >= 1 && S <= PREDTOP_MAX_PLAN_STAGES && mb >= 1;
    float buf[PREDTOP_MAX_PLAN_STAGES];
    int n = 0;
    for (int64_t i = 0; ok && i < S; ++i) {
      const int32_t s = plan_stage[b0 + i];
      if (s < 0 || s >= num_stages) { ok = false; break; }
      // insertion into the sorted prefix (ascending)
      const float v = t[s];
      int j = n - 1;
      while (j >= 0 && buf[j] > v) { buf[j + 1] = buf[j]; --j; }
      buf[j + 1] = v;
      ++n;
    }
    if (!ok) {
      T[p] = __longlong_as_double(0x7ff8000000000000ll);  // NaN
      atomicMin(first_bad, (unsigned long long)p);
      continue;
    }
    double sum = 0.0;
    for (int i = 0; i < n; ++i) sum = __dadd_rn(sum, (double)buf[i]);
    const double m = (double)buf[n - 1];
    T[p] = __dadd_rn(sum, __dmul_rn((double)(mb - 1), m));
  }
}

predtop_status plan_launch(int64_t P, const int64_t* plan_ptr, const int32_t* plan_stage,
                           const int32_t* B, const float* t, int64_t num_stages, double* T,
                           int64_t* first_bad, cudaStream_t st) {
  if (P <= 0) return PREDTOP_OK;
  const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(P, 128), 148 * 8));
{
    ProfScope _p(PK_PLAN, st);
    k_plan<<<blocks, 128, 0, st>>>(P, plan_ptr, plan_stage, B, t, num_stages, T,
                                 reinterpret_cast<unsigned long long*>(first_bad));
    PT_LAUNCH_CHECK();
  }
  return PREDTOP_OK;
}

// argmin by (T, index); NaN never wins; all-NaN -> -1.  Single CTA, fixed
// reduction tree: deterministic.
__device__ __forceinline__ bool better(double a, int64_t ia, double b, int64_t ib) {
  if (ib < 0) return ia >= 0;
  if (ia < 0) return false;
  return a < b || (a == b && ia < ib);
}

__global__ void __launch_bounds__(1024) k_argmin(int64_t n, const double* __restrict__ T,
                                                 int64_t* best) {
  __shared__ double sv[32];
  __shared__ int64_t si[32];
  double bv = 0.0;
  int64_t bi = -1;
  for (int64_t i = threadIdx.x; i < n; i += blockDim.x) {
    const double v = T[i];
    if (v == v && better(v, i, bv, bi)) { bv = v; bi = i; }
  }
  for (int o = 16; o > 0; o >>= 1) {
    const double ov = __shfl_xor_sync(0xffffffffu, bv, o);
    const int64_t oi = __shfl_xor_sync(0xffffffffu, bi, o);
    if (better(ov, oi, bv, bi)) { bv = ov; bi = oi; }
  }
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (lane == 0) { sv[w] = bv; si[w] = bi; }
  __syncthreads();
  if (w == 0) {
    bv = lane < (int)(blockDim.x >> 5) ? sv[lane] : 0.0;
    bi = lane < (int)(blockDim.x >> 5) ? si[lane] : -1;
    for (int o = 16; o > 0; o >>= 1) {
      const double ov = __shfl_xor_sync(0xffffffffu, bv, o);
      const int64_t oi = __shfl_xor_sync(0xffffffffu, bi, o);
      if (better(ov, oi, bv, bi)) { bv = ov; bi = oi; }
    }
    if (lane == 0) *best = bi;
  }
}

predtop_status argmin_launch(int64_t n, const double* T, int64_t* best, cudaStream_t st) {
{
    ProfScope _p(PK_ARGMIN, st);
    k_argmin<<<1, 1024, 0, st>>>(n, T, best);
    PT_LAUNCH_CHECK();
  }
  return PREDTOP_OK;
}

}  // namespace predtop
