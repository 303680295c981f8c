// build.cu — steps a1-a3: raw samples -> simple undirected graph.
//
//   canonicalize : key = (min(u,v) << b) | max(u,v), b = bits(n-1); a self-loop maps to the
//                  all-ones sentinel (it cannot be an edge key since u < v) so no compaction
//                  pass is needed; ids >= n raise an error flag (TC_ERR_INVALID).  Fused into
//                  the radix sort's histogram and first pass (no key array is materialised).
//   radix sort   : 2b significant bits (prims.cu)
//   unique       : first key of every run (duplicates and both directions merged, Q1),
//                  fused with the degrees d(v) (run-aggregated atomics)
#include "internal.h"
#include "prims.cuh"

namespace tc {
namespace {

// m = runs - (last run is the sentinel)
__global__ void trim_sentinel_kernel(const uint64_t *uniq, uint64_t *d_count, uint64_t sentinel) {
  uint64_t c = *d_count;
  if (c > 0 && uniq[c - 1] == sentinel) *d_count = c - 1;
}

__global__ void max_kernel(const uint32_t *__restrict__ a, uint64_t n, unsigned *out) {
  uint32_t mx = 0;
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) mx = max(mx, a[i]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if (lane_id() == 0 && mx) atomicMax(out, mx);
}

}  // namespace

uint32_t device_max_u32(const uint32_t *a, uint64_t n, cudaStream_t s) {
  DevBuf<unsigned> r;
  r.alloc(1, s);
  TC_CUDA(cudaMemsetAsync(r.get(), 0, sizeof(unsigned), s));
  if (n) {
    max_kernel<<<grid_for(n, 256, 4), 256, 0, s>>>(a, n, r.get());
    TC_LAUNCH_CHECK();
  }
  unsigned h = 0;
  TC_CUDA(cudaMemcpyAsync(&h, r.get(), sizeof(unsigned), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  return h;
}

void build_graph(Graph &g, const uint32_t *d_src, const uint32_t *d_dst, uint64_t M) {
  cudaStream_t s = g.stream;
  const uint32_t n = g.n;
  g.bits = bits_for(n > 0 ? n - 1 : 0);
  g.samples = M;
  const int b = g.bits;
  const uint64_t sentinel = (b * 2 >= 64) ? ~0ull : ((1ull << (2 * b)) - 1);

  DevBuf<uint64_t> keys, tmp;
  {
    ProfScope prof("alloc_keys", s, 0.0);
    keys.alloc(M ? M : 1, s);
    tmp.alloc(M ? M : 1, s);
  }
  DevBuf<unsigned> err;
  err.alloc(1, s);
  DevBuf<uint64_t> d_m;
  d_m.alloc(1, s);
  TC_CUDA(cudaMemsetAsync(err.get(), 0, sizeof(unsigned), s));
  g.deg.alloc(n ? n : 1, s);
  TC_CUDA(cudaMemsetAsync(g.deg.get(), 0, g.deg.bytes(), s));
  // a1+a2: canonicalise inside the radix sort's histogram and first pass
  uint64_t *sorted = radix_sort_edges(d_src, d_dst, M, n, b, sentinel, keys.get(), tmp.get(), err.get(), s);
  uint64_t *uniq = (sorted == keys.get()) ? tmp.get() : keys.get();
  // a2+a3: unique runs and undirected degrees in one pass
  unique_sorted_u64(sorted, uniq, M, d_m.get(), s, g.deg.get(), b, sentinel);
  trim_sentinel_kernel<<<1, 1, 0, s>>>(uniq, d_m.get(), sentinel);
  TC_LAUNCH_CHECK();
  unsigned h_err = 0;
  uint64_t h_m = 0;
  TC_CUDA(cudaMemcpyAsync(&h_err, err.get(), sizeof(unsigned), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaMemcpyAsync(&h_m, d_m.get(), sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  TC_REQUIRE(h_err == 0, ST_INVALID, "tc_graph_from_edges: vertex id >= num_vertices");
  g.m = h_m;
  // keep the unique run as the edge array; release the other buffer
  if (uniq == keys.get()) g.edges = std::move(keys);
  else g.edges = std::move(tmp);
  g.max_degree_ready = false;
  g.state = G_BUILT;
}

void ensure_max_degree(Graph &g) {
  if (g.max_degree_ready) return;
  g.max_degree = device_max_u32(g.deg.get(), g.n, g.stream);
  g.max_degree_ready = true;
}

}  // namespace tc
