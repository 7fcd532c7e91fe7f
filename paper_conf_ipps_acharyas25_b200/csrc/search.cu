// search.cu -- inter-stage plan search over a shared stage table (SURVEY 8(f)
// f1; predtop_plan_search).  P:194: Alpa's inter-operator optimizer chooses the
// pipeline plan under the 1F1B model; it enumerates every stage
// (layer range) on every submesh; PredTOP predicts all of them and
// applies Eqn 4.  A plan slices L layers into contiguous stages, each on a
// choice c (mesh / intra-op configuration, Tables II-III) using dev[c]
// devices with sum dev = D, and costs T = sum t_s + (B-1) max t_s (Eqn 4).
//
// Algorithm (Alpa's): every feasible table entry is a candidate bound t_max;
// for each, a DP over (first layer k, devices left d)
//     F(L, 0) = 0,  F(k, d) = min_{j >= k, c: t[k][j][c] <= t_max, dev[c] <= d}
//                             t[k][j][c] + F(j+1, d - dev[c])
// gives the least stage sum with every stage <= t_max, and
// T* = min_{t_max} F(0, D) + (B-1) t_max.  The minimum over t_max is exact:
// the optimal plan p* is admissible at t_max = max(p*), and every candidate
// value bounds the true Eqn 4 of the plan it stands for from above.
//
// Table layout: [num_tables][K][stride], stage (i, j) of choice c at
// c * stride + tri(i, j), tri(i, j) = i L - i (i-1)/2 + (j - i).
//
//   k_search_cand   one warp per (problem, candidate): the DP in shared memory,
//                   lanes over the (j, c) transitions, warp min-reductions
//   k_search_pick   one CTA per problem: argmin over candidates by
//                   (T, t_max, candidate id), then the winning DP once more
//                   with argmin recording, and the backtrack to the plan
//
// Arithmetic: fp32 latencies added in fp64 (round to nearest) and one
// (B-1) t_max product; R20 states when these sums are exact (then T*
// is bit-identical to exhaustive enumeration, the oracle).
#include <climits>

#include "internal.h"

namespace predtop {

namespace {

constexpr double kInf = __builtin_huge_val();

struct SearchArgs {
  int L, K, D;
  int32_t dev[PREDTOP_SEARCH_MAX_CHOICES];
  const float* t;           // [num_tables][K][stride], stage (i, j) at tri(i, j) of row c
  int64_t stride;           // >= NT
  int64_t num_tables;
  const int32_t* table_of;  // [P] or nullptr (problem p uses table p)
  const int32_t* B;         // [P]
  int64_t P;
  int NT;                   // L(L+1)/2 stages
  int64_t C;                // candidates per problem = K * NT (every table entry)
  double* Tc;               // [P][C]
};

__device__ __forceinline__ bool problem_ok(const SearchArgs& a, int64_t p, const float** tp, int* B) {
  const int64_t tb = a.table_of ? (int64_t)a.table_of[p] : p;
  *B = a.B[p];
  if (tb < 0 || tb >= a.num_tables || *B < 1) return false;
  *tp = a.t + tb * (int64_t)a.K * a.stride;
  return true;
}

// One warp: F(k, d) for k = L..0 (row stride D+1) under the bound tmax;
// arg (nullable) records the winning transition (j - k) * K + c, the first
// in (j, c) order among equal sums.  Returns F(0, D).
__device__ double warp_dp(const SearchArgs& a, const int32_t* dev, const float* __restrict__ tp,
                          float tmax, double* F, int16_t* arg) {
  const int lane = threadIdx.x & 31;
  const int L = a.L, K = a.K, D = a.D, D1 = a.D + 1;
  for (int d = lane; d <= D; d += 32) F[L * D1 + d] = d == 0 ? 0.0 : kInf;
  __syncwarp();
  for (int k = L - 1; k >= 0; --k) {
    const int nitems = (L - k) * K;
    const int tk = k * L - k * (k - 1) / 2;  // tri(k, k): stages (k, j) are tk + (j - k)
    if (lane == 0) {
      F[k * D1] = kInf;
      if (arg) arg[k * D1] = -1;
    }
    for (int d = 1; d <= D; ++d) {
      double best = kInf;
      int bkey = INT_MAX;
      for (int it = lane; it < nitems; it += 32) {
        const int j = k + it / K, c = it - (it / K) * K;
        const int dv = dev[c];
        if (dv > d) continue;
        const float v = __ldg(tp + (size_t)c * a.stride + tk + (j - k));
        if (!(v >= 0.f && v <= tmax)) continue;  // infeasible (NaN, < 0, inf) or above the bound
        const double f = F[(j + 1) * D1 + d - dv];
        if (f == kInf) continue;
        const double s = __dadd_rn((double)v, f);
        if (s < best) { best = s; bkey = it; }  // lanes visit `it` ascending: first minimum kept
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        const double ob = __shfl_xor_sync(0xffffffffu, best, o);
        const int ok = __shfl_xor_sync(0xffffffffu, bkey, o);
        if (ob < best || (ob == best && ok < bkey)) { best = ob; bkey = ok; }
      }
      if (lane == 0) {
        F[k * D1 + d] = best;
        if (arg) arg[k * D1 + d] = (int16_t)(best == kInf ? -1 : bkey);
      }
    }
    __syncwarp();
  }
  return F[D];
}

__global__ void __launch_bounds__(128) k_search_cand(SearchArgs a) {
  extern __shared__ __align__(16) unsigned char sm_search[];
  __shared__ int32_t s_dev[PREDTOP_SEARCH_MAX_CHOICES];
  if (threadIdx.x < PREDTOP_SEARCH_MAX_CHOICES) s_dev[threadIdx.x] = a.dev[threadIdx.x];
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  double* F = reinterpret_cast<double*>(sm_search) + (size_t)warp * (a.L + 1) * (a.D + 1);
  const int64_t total = a.P * a.C;
  for (int64_t w = blockIdx.x * 4ll + warp; w < total; w += gridDim.x * 4ll) {
    const int64_t p = w / a.C, ci = w - p * a.C;
    const float* tp;
    int B;
    double T;
    if (!problem_ok(a, p, &tp, &B)) {
      T = __longlong_as_double(0x7ff8000000000000ll);  // NaN: invalid problem
    } else {
      const int c = (int)(ci / a.NT), s = (int)(ci - (int64_t)c * a.NT);
      const float tmax = tp[(size_t)c * a.stride + s];
      T = kInf;
      if (tmax >= 0.f && tmax < __int_as_float(0x7f800000)) {
        const double f = warp_dp(a, s_dev, tp, tmax, F, nullptr);
        if (f != kInf) T = __dadd_rn(f, __dmul_rn((double)(B - 1), (double)tmax));
      }
    }
    if (lane == 0) a.Tc[w] = T;
    __syncwarp();
  }
}

__device__ __forceinline__ bool cand_better(double T, float tm, int64_t ci, double bT, float btm, int64_t bci) {
  if (bci < 0) return ci >= 0;
  if (ci < 0) return false;
  return T < bT || (T == bT && (tm < btm || (tm == btm && ci < bci)));
}

__global__ void __launch_bounds__(256) k_search_pick(SearchArgs a, double* T_out, int32_t* S_out,
                                                     int32_t* end_out, int32_t* choice_out) {
  extern __shared__ __align__(16) unsigned char sm_search[];
  __shared__ int32_t s_dev[PREDTOP_SEARCH_MAX_CHOICES];
  __shared__ double s_T[8];
  __shared__ float s_tm[8];
  __shared__ long long s_ci[8];
  const int64_t p = blockIdx.x;
  if (threadIdx.x < PREDTOP_SEARCH_MAX_CHOICES) s_dev[threadIdx.x] = a.dev[threadIdx.x];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const float* tp;
  int B;
  const bool ok = problem_ok(a, p, &tp, &B);
  if (!ok) {
    if (threadIdx.x == 0) { T_out[p] = __longlong_as_double(0x7ff8000000000000ll); S_out[p] = 0; }
    return;
  }
  // argmin over candidates by (T, t_max, id); +inf (no admissible plan) never wins
  double bT = kInf;
  float btm = 0.f;
  int64_t bci = -1;
  const double* Tc = a.Tc + p * a.C;
  for (int64_t ci = threadIdx.x; ci < a.C; ci += blockDim.x) {
    const double T = Tc[ci];
    if (!(T < kInf)) continue;
    const int c = (int)(ci / a.NT);
    const float tm = tp[(size_t)c * a.stride + (ci - (int64_t)c * a.NT)];
    if (cand_better(T, tm, ci, bT, btm, bci)) { bT = T; btm = tm; bci = ci; }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const double oT = __shfl_xor_sync(0xffffffffu, bT, o);
    const float otm = __shfl_xor_sync(0xffffffffu, btm, o);
    const long long oci = __shfl_xor_sync(0xffffffffu, (long long)bci, o);
    if (cand_better(oT, otm, oci, bT, btm, bci)) { bT = oT; btm = otm; bci = oci; }
  }
  if (lane == 0) { s_T[warp] = bT; s_tm[warp] = btm; s_ci[warp] = bci; }
  __syncthreads();
  if (warp != 0) return;
  bT = lane < 8 ? s_T[lane] : kInf;
  btm = lane < 8 ? s_tm[lane] : 0.f;
  bci = lane < 8 ? s_ci[lane] : -1;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const double oT = __shfl_xor_sync(0xffffffffu, bT, o);
    const float otm = __shfl_xor_sync(0xffffffffu, btm, o);
    const long long oci = __shfl_xor_sync(0xffffffffu, (long long)bci, o);
    if (cand_better(oT, otm, oci, bT, btm, bci)) { bT = oT; btm = otm; bci = oci; }
  }
  if (bci < 0) {  // no plan uses exactly D devices with feasible stages
    if (lane == 0) { T_out[p] = kInf; S_out[p] = 0; }
    return;
  }
  // the winning DP again, recording transitions, then the backtrack
  const int D1 = a.D + 1;
  double* F = reinterpret_cast<double*>(sm_search);
  int16_t* arg = reinterpret_cast<int16_t*>(F + (size_t)(a.L + 1) * D1);
  warp_dp(a, s_dev, tp, btm, F, arg);
  if (lane == 0) {
    int k = 0, d = a.D, S = 0;
    int32_t* eo = end_out + p * a.L;
    int32_t* co = choice_out + p * a.L;
    while (k < a.L && S < a.L) {
      const int key = arg[k * D1 + d];
      if (key < 0) break;  // unreachable when bci >= 0
      const int j = k + key / a.K, c = key % a.K;
      eo[S] = j;
      co[S] = c;
      ++S;
      d -= s_dev[c];
      k = j + 1;
    }
    T_out[p] = bT;
    S_out[p] = S;
  }
}

}  // namespace

size_t search_workspace_bytes(int64_t P, int L, int K) {
  return align_up((size_t)P * (size_t)K * ((size_t)L * (L + 1) / 2) * sizeof(double), 256);
}

predtop_status search_launch(int64_t P, int L, int K, const int32_t* dev, int D, const float* t,
                             int64_t stride, int64_t num_tables, const int32_t* table_of, const int32_t* B,
                             double* T_out, int32_t* S_out, int32_t* end_out, int32_t* choice_out,
                             void* ws, cudaStream_t st) {
  if (P <= 0) return PREDTOP_OK;
  SearchArgs a{};
  a.L = L; a.K = K; a.D = D;
  for (int c = 0; c < PREDTOP_SEARCH_MAX_CHOICES; ++c) a.dev[c] = c < K ? dev[c] : 1 << 20;
  a.t = t; a.stride = stride; a.num_tables = num_tables;
  a.NT = L * (L + 1) / 2; a.table_of = table_of; a.B = B; a.P = P;
  a.C = (int64_t)K * a.NT;
  a.Tc = reinterpret_cast<double*>(ws);
  const size_t fbytes = (size_t)(L + 1) * (D + 1) * sizeof(double);
  const size_t cand_smem = 4 * fbytes, pick_smem = fbytes + align_up((size_t)(L + 1) * (D + 1) * 2, 16);
  PT_SMEM_ATTR(k_search_cand, cand_smem);
  PT_SMEM_ATTR(k_search_pick, pick_smem);
  const int64_t warps = P * a.C;
  const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(warps, 4), 148 * 16));
  {
    ProfScope _p(PK_SEARCH_CAND, st);
    k_search_cand<<<blocks, 128, cand_smem, st>>>(a);
    PT_LAUNCH_CHECK();
  }
  {
    ProfScope _p(PK_SEARCH_PICK, st);
    k_search_pick<<<(unsigned)P, 256, pick_smem, st>>>(a, T_out, S_out, end_out, choice_out);
    PT_LAUNCH_CHECK();
  }
  return PREDTOP_OK;
}

}  // namespace predtop
