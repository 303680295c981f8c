// prims.cuh — device-wide primitives used by the CSR build:
// LSD radix sort (one-sweep, decoupled look-back), exclusive scan, unique-select.
#pragma once
#include "common.cuh"

namespace tc {

// Exclusive scan of n counts into n+1 uint64 offsets (out[n] = total).
void scan_u32_to_u64(const uint32_t *in, uint64_t *out, uint64_t n, cudaStream_t s);
void scan_u64(const uint64_t *in, uint64_t *out, uint64_t n, cudaStream_t s);

// Stable LSD radix sort of N uint64 keys on bits [begin_bit, end_bit).  `tmp` holds N
// keys.  Returns the buffer (keys or tmp) that holds the sorted result.
uint64_t *radix_sort_u64(uint64_t *keys, uint64_t *tmp, uint64_t N, int begin_bit, int end_bit,
                         cudaStream_t s);

// Sort of raw edge samples canonicalised on the fly (a1+a2): key (min << bits) | max,
// self-loops / ids >= nv -> `sentinel` (ids >= nv also set *err).  Result in buf0 or buf1.
uint64_t *radix_sort_edges(const uint32_t *src, const uint32_t *dst, uint64_t M, uint32_t nv, int bits,
                           uint64_t sentinel, uint64_t *buf0, uint64_t *buf1, unsigned *err, cudaStream_t s);

// Unique on a sorted array: out receives the first key of every run; *d_count (device)
// receives the number of runs.  deg != nullptr: also accumulate undirected degrees of the
// kept (u << bits) | v keys other than `sentinel`.
void unique_sorted_u64(const uint64_t *in, uint64_t *out, uint64_t N, uint64_t *d_count, cudaStream_t s,
                       uint32_t *deg = nullptr, int bits = 0, uint64_t sentinel = 0);

// Orientation split of sorted undirected keys (a << bits) | b (a < b): forward edges
// (prim[a] <= prim[b]) keep key and order in F, reversed ones become (b << bits) | a in R in
// input order.  Returns |F| (|R| = m - |F|).  Synchronises the stream.
uint64_t split_oriented(const uint64_t *edges, uint64_t m, int bits, const uint64_t *prim, uint64_t *F, uint64_t *R,
                        cudaStream_t s);

// Block-wide exclusive scan helper (256 threads) used by several kernels.
template <typename T>
__device__ __forceinline__ T block256_exclusive_scan(T v, T *s_warp /*8 entries*/, T *total) {
  T inc = warp_inclusive_scan(v);
  if (lane_id() == 31) s_warp[warp_id()] = inc;
  __syncthreads();
  if (warp_id() == 0) {
    T x = lane_id() < 8 ? s_warp[lane_id()] : T(0);
    T xi = warp_inclusive_scan(x);
    if (lane_id() < 8) s_warp[lane_id()] = xi - x;
    if (lane_id() == 7) *total = xi;
  }
  __syncthreads();
  T r = inc - v + s_warp[warp_id()];
  return r;
}

}  // namespace tc
