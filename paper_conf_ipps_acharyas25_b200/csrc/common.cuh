// common.cuh -- internal helpers of libpredtop (not part of the ABI).
#pragma once
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <stdint.h>

#include "../../include/predtop.h"

namespace predtop {

// Kernel-launch accounting (predtop_launch_count): every launch site calls
// note_launch() so callers can count the library's kernels in a timed region.
void note_launch(int n = 1);

// Optional per-kernel timing (predtop_profile_enable): a CUDA event pair on
// the launching stream around each launch site, read back by
// predtop_profile_read.  Off by default (no events are recorded).
enum ProfKind {
  PK_DAG_META, PK_DAG_DEPTH, PK_DAG_CLOSURE, PK_DAG_MASK, PK_DAG_CLASSIFY, PK_DAG_WORK,
  PK_PE, PK_EMBED, PK_GEMM_QKV, PK_ATTN, PK_GEMM_O_LN, PK_GEMM_FF1, PK_GEMM_FF2_LN,
  PK_READOUT, PK_PLAN, PK_ARGMIN, PK_COPY, PK_LAYER_TAIL, PK_DAG_SMALL, PK_DAG_FLAGS,
  PK_SEARCH_CAND, PK_SEARCH_PICK, PK_PRUNE, PK_COUNT
};
struct ProfScope {
  int kind;
  cudaStream_t st;
  void* ev0 = nullptr;
  ProfScope(int k, cudaStream_t s);
  ~ProfScope();
};

// Thread-local last-error message.
void set_error(const char* fmt, ...);

// Raise `func`'s dynamic shared-memory limit to at least `bytes` on the
// current device.  The attribute is per device, so the cache is keyed by
// (device, kernel); thread-safe (api.cu).
cudaError_t smem_attr(const void* func, int bytes);
// SM count of the current device (cached per device); 0 on error.
int num_sms();
#define PT_SMEM_ATTR(func, bytes) PT_CUDA_TRY(::predtop::smem_attr((const void*)(func), (int)(bytes)))

#define PT_CUDA_TRY(expr)                                                        \
  do {                                                                           \
    cudaError_t _e = (expr);                                                     \
    if (_e != cudaSuccess) {                                                     \
      ::predtop::set_error("%s failed: %s (%s:%d)", #expr, cudaGetErrorString(_e), \
                           __FILE__, __LINE__);                                  \
      return PREDTOP_ERR_CUDA;                                                   \
    }                                                                            \
  } while (0)

#define PT_LAUNCH_CHECK()                                                        \
  do {                                                                           \
    ::predtop::note_launch();                                                    \
    cudaError_t _e = cudaGetLastError();                                         \
    if (_e != cudaSuccess) {                                                     \
      ::predtop::set_error("kernel launch failed: %s (%s:%d)", cudaGetErrorString(_e), \
                           __FILE__, __LINE__);                                  \
      return PREDTOP_ERR_CUDA;                                                   \
    }                                                                            \
  } while (0)

__host__ __device__ static inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }
__host__ __device__ static inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// A bump allocator over a caller workspace (device pointers are only offsets here).
struct Carver {
  char* base;
  size_t used = 0;
  explicit Carver(void* b) : base((char*)b) {}
  template <class T>
  T* take(size_t count, size_t align = 256) {
    used = align_up(used, align);
    T* p = base ? (T*)(base + used) : nullptr;
    used += sizeof(T) * count;
    return p;
  }
};

}  // namespace predtop
