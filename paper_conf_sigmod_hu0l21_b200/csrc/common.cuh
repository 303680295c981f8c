// common.cuh — shared device/host plumbing for libtc_b200 (sm_100a).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <stdexcept>
#include <string>

namespace tc {

// ---------------------------------------------------------------- errors
struct Error : std::runtime_error {
  int status;
  Error(int s, const std::string &msg) : std::runtime_error(msg), status(s) {}
};

void cuda_fail(cudaError_t e, const char *what, const char *file, int line);

#define TC_CUDA(x)                                                   \
  do {                                                               \
    cudaError_t _e = (x);                                            \
    if (_e != cudaSuccess) ::tc::cuda_fail(_e, #x, __FILE__, __LINE__); \
  } while (0)

extern unsigned long long g_launch_count;  // kernels launched by the library (prof.cu)
#define TC_LAUNCH_CHECK()                   \
  do {                                      \
    ++::tc::g_launch_count;                 \
    TC_CUDA(cudaGetLastError());            \
  } while (0)

#define TC_REQUIRE(cond, status, msg) \
  do {                                \
    if (!(cond)) throw ::tc::Error((status), (msg)); \
  } while (0)

// TC_* status values mirrored from include/tc.h
enum { ST_OK = 0, ST_INVALID = 1, ST_OOM = 2, ST_CUDA = 3, ST_NCCL = 4, ST_STATE = 5 };

// ---------------------------------------------------------------- device buffers
// Device memory cache (alloc.cu): stream-ordered reuse of blocks across graphs and steps.
void *dev_alloc(size_t bytes, cudaStream_t s);
void dev_free(void *p, size_t bytes, cudaStream_t s);
void dev_trim();
size_t dev_cached_bytes();

// Buffer owned by the graph (or a stage), allocated from / returned to the cache on its stream.
template <typename T>
struct DevBuf {
  T *p = nullptr;
  size_t n = 0;
  cudaStream_t s = nullptr;
  DevBuf() = default;
  DevBuf(const DevBuf &) = delete;
  DevBuf &operator=(const DevBuf &) = delete;
  DevBuf(DevBuf &&o) noexcept { swap(o); }
  DevBuf &operator=(DevBuf &&o) noexcept {
    if (this != &o) { release(); swap(o); }
    return *this;
  }
  ~DevBuf() { release(); }
  void swap(DevBuf &o) {
    std::swap(p, o.p); std::swap(n, o.n); std::swap(s, o.s);
  }
  void alloc(size_t count, cudaStream_t stream) {
    release();
    s = stream;
    n = count;
    if (count == 0) return;
    try {
      p = (T *)dev_alloc(count * sizeof(T), stream);
    } catch (...) {
      p = nullptr; n = 0;
      throw;
    }
  }
  void release() {
    if (p) dev_free(p, n * sizeof(T), s);
    p = nullptr; n = 0;
  }
  T *get() const { return p; }
  size_t bytes() const { return n * sizeof(T); }
};

// ---------------------------------------------------------------- profiling (prof.cu)
extern int g_opt_kernel_profile;
// RAII event pair around one or more launches of kernel `name` (no-op unless enabled).
struct ProfScope {
  const char *name_;
  cudaStream_t s_;
  double bytes_;
  void *a_ = nullptr, *b_ = nullptr;
  ProfScope(const char *name, cudaStream_t s, double bytes);
  ~ProfScope();
  ProfScope(const ProfScope &) = delete;
  ProfScope &operator=(const ProfScope &) = delete;
};

// ---------------------------------------------------------------- launch helpers
int num_sms();

inline unsigned grid_for(uint64_t work, unsigned block, unsigned per_sm_blocks = 8) {
  uint64_t want = (work + block - 1) / block;
  uint64_t cap = (uint64_t)num_sms() * per_sm_blocks;
  if (want < 1) want = 1;
  return (unsigned)(want < cap ? want : cap);
}

inline int bits_for(uint64_t maxval) {  // bits needed to represent 0..maxval
  int b = 0;
  while (b < 64 && (maxval >> b)) ++b;
  return b ? b : 1;
}

// ---------------------------------------------------------------- device utils
__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ unsigned warp_id() { return threadIdx.x >> 5; }

__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_u64(uint64_t *p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

__device__ __forceinline__ uint32_t warp_max(uint32_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = max(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

template <typename T>
__device__ __forceinline__ T warp_inclusive_scan(T v) {
  unsigned l = lane_id();
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T t = __shfl_up_sync(0xffffffffu, v, o);
    if (l >= (unsigned)o) v += t;
  }
  return v;
}

// Decoupled look-back status word: [63:62] flag (0 none, 1 aggregate, 2 inclusive), [61:0] value.
constexpr uint64_t LB_AGG = 1ull << 62;
constexpr uint64_t LB_INC = 2ull << 62;
constexpr uint64_t LB_VAL = (1ull << 62) - 1;

// Exclusive prefix of tile `tile` (called by ONE thread) over status[] with
// stride `stride` between consecutive tiles; publishes the inclusive value.
__device__ __forceinline__ uint64_t lookback_exclusive(uint64_t *status, uint64_t tile, size_t stride,
                                                       uint64_t local) {
  if (tile == 0) {
    st_relaxed_u64(status, LB_INC | local);
    return 0;
  }
  st_relaxed_u64(status + tile * stride, LB_AGG | local);
  uint64_t excl = 0;
  int64_t j = (int64_t)tile - 1;
  while (true) {
    uint64_t s = ld_relaxed_u64(status + (uint64_t)j * stride);
    uint64_t f = s & ~LB_VAL;
    if (f == 0) continue;
    excl += s & LB_VAL;
    if (f == LB_INC) break;
    --j;
  }
  st_relaxed_u64(status + tile * stride, LB_INC | (excl + local));
  return excl;
}

}  // namespace tc
