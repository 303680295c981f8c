// alloc.cu — the library's device memory cache.
//
// Every step of the path allocates the same large transient buffers (sort keys, radix
// scratch, CSR, work items) graph after graph.  cudaMallocAsync showed a device-side cost
// of up to tens of ms per step when the stream-ordered pool grew (ncu/CUDA events:
// "alloc_keys" 1-38 ms), so DevBuf draws from this cache instead: blocks are kept per
// (device, rounded size), a freed block records an event on its stream and a later
// allocation on another stream waits on that event (stream-ordered reuse).  cudaMalloc is
// only called when no block of the size is cached; on OOM the cache is emptied and the
// allocation retried.  tc_set_option("trim_memory", 1) releases all cached blocks.
#include <map>
#include <mutex>
#include <vector>

#include "common.cuh"

namespace tc {
namespace {
struct Block {
  void *p;
  cudaStream_t s;
  cudaEvent_t ev;
};
std::mutex g_mu;
std::map<std::pair<int, size_t>, std::vector<Block>> g_free;  // (device, bytes) -> blocks
size_t g_cached = 0;

size_t round_bytes(size_t b) {
  if (b >= (2u << 20)) return (b + (2u << 20) - 1) & ~(size_t)((2u << 20) - 1);
  return (b + 511) & ~(size_t)511;
}

void release_all_locked() {
  for (auto &kv : g_free)
    for (auto &bl : kv.second) {
      cudaEventSynchronize(bl.ev);
      cudaEventDestroy(bl.ev);
      cudaFree(bl.p);
    }
  g_free.clear();
  g_cached = 0;
  cudaGetLastError();
}
}  // namespace

void *dev_alloc(size_t bytes, cudaStream_t s) {
  if (!bytes) return nullptr;
  int dev = 0;
  TC_CUDA(cudaGetDevice(&dev));
  const size_t rb = round_bytes(bytes);
  {
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_free.find({dev, rb});
    if (it != g_free.end() && !it->second.empty()) {
      Block bl = it->second.back();
      it->second.pop_back();
      g_cached -= rb;
      if (bl.s != s) TC_CUDA(cudaStreamWaitEvent(s, bl.ev, 0));
      cudaEventDestroy(bl.ev);
      return bl.p;
    }
  }
  void *p = nullptr;
  cudaError_t e = cudaMalloc(&p, rb);
  if (e == cudaErrorMemoryAllocation) {
    cudaGetLastError();
    {
      std::lock_guard<std::mutex> lk(g_mu);
      release_all_locked();
    }
    e = cudaMalloc(&p, rb);
  }
  if (e == cudaErrorMemoryAllocation) {
    cudaGetLastError();
    throw Error(ST_OOM, "device allocation of " + std::to_string(rb) + " bytes failed");
  }
  TC_CUDA(e);
  return p;
}

void dev_free(void *p, size_t bytes, cudaStream_t s) {
  if (!p) return;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) {
    cudaGetLastError();
    return;
  }
  cudaEvent_t ev;
  if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess || cudaEventRecord(ev, s) != cudaSuccess) {
    cudaGetLastError();
    cudaStreamSynchronize(s);
    cudaFree(p);
    return;
  }
  const size_t rb = round_bytes(bytes);
  std::lock_guard<std::mutex> lk(g_mu);
  g_free[{dev, rb}].push_back(Block{p, s, ev});
  g_cached += rb;
}

void dev_trim() {
  std::lock_guard<std::mutex> lk(g_mu);
  release_all_locked();
}

size_t dev_cached_bytes() {
  std::lock_guard<std::mutex> lk(g_mu);
  return g_cached;
}

}  // namespace tc
