// radix_lab.cu — standalone A/B harness for the one-sweep radix pass and for the random
// access patterns a bucketed CSR build would use (NOT part of the product library).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Ipaper_conf_sigmod_hu0l21_b200/csrc \
//        tools/radix_lab.cu -o tools/radix_lab && tools/radix_lab
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "common.cuh"

namespace tc {
void cuda_fail(cudaError_t e, const char *what, const char *file, int line) {
  fprintf(stderr, "%s: %s at %s (%s:%d)\n", cudaGetErrorName(e), cudaGetErrorString(e), what, file, line);
  exit(1);
}
int num_sms() { return 148; }
}  // namespace tc
using namespace tc;

constexpr int T_THREADS = 256;
constexpr int T_WARPS = T_THREADS / 32;

template <typename T>
__device__ __forceinline__ T bscan256(T v, T *s_warp, T *total) {
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
  return inc - v + s_warp[warp_id()];
}

__device__ __forceinline__ uint32_t rank_or(uint32_t d, bool valid, uint32_t *whist, uint32_t *mask, unsigned lane,
                                            unsigned lt_mask) {
  if (valid) atomicOr(&mask[d], 1u << lane);
  __syncwarp();
  const unsigned peers = valid ? mask[d] : 0u;
  __syncwarp();
  uint32_t old = 0;
  const unsigned lead = __ffs(peers) - 1;
  if (valid && lane == lead) {
    old = whist[d];
    whist[d] = old + __popc(peers);
    mask[d] = 0;
  }
  old = __shfl_sync(0xffffffffu, old, valid ? lead : lane);
  return old + __popc(peers & lt_mask);
}

__device__ __forceinline__ uint32_t rank_ballot(uint32_t d, bool valid, uint32_t *whist, unsigned lane,
                                                unsigned lt_mask) {
  unsigned peers = __ballot_sync(0xffffffffu, valid);
  if (!valid) peers = ~peers;
#pragma unroll
  for (int b = 0; b < 8; ++b) {
    unsigned bit = (d >> b) & 1u;
    unsigned bb = __ballot_sync(0xffffffffu, bit);
    peers &= bit ? bb : ~bb;
  }
  const unsigned lead = __ffs(peers) - 1;
  uint32_t old = 0;
  if (lane == lead && valid) {
    old = whist[d];
    whist[d] = old + __popc(peers);
  }
  old = __shfl_sync(0xffffffffu, old, lead);
  return old + __popc(peers & lt_mask);
}

__device__ __forceinline__ uint32_t rank_match(uint32_t d, bool valid, uint32_t *whist, unsigned lane,
                                               unsigned lt_mask) {
  unsigned peers = __match_any_sync(0xffffffffu, valid ? d : 0xffffffffu);
  const unsigned lead = __ffs(peers) - 1;
  uint32_t old = 0;
  if (lane == lead && valid) {
    old = whist[d];
    whist[d] = old + __popc(peers);
  }
  old = __shfl_sync(0xffffffffu, old, lead);
  return old + __popc(peers & lt_mask);
}

// RANK: 0 or-mask, 1 ballot, 2 match.  EARLY: 1 smem-atomic early counts, 0 counts from
// the per-warp histograms after ranking.
template <int RANK, int EARLY, int T_ITEMS, int MINB, int SKIP>
__global__ __launch_bounds__(T_THREADS, MINB) void pass_kernel(const uint64_t *__restrict__ in, uint64_t *__restrict__ out,
                                                            uint64_t n, int shift,
                                                            const unsigned long long *__restrict__ goff,
                                                            uint64_t *status, uint32_t *tile_ctr) {
  constexpr int T_TILE = T_THREADS * T_ITEMS;
  __shared__ uint64_t s_keys[T_TILE < 4096 ? 4096 : T_TILE];
  __shared__ uint32_t s_whist[T_WARPS][256];
  __shared__ uint32_t s_cnt[256];
  __shared__ uint64_t s_gbase[256];
  __shared__ uint32_t s_warp32[8];
  __shared__ uint32_t s_total32;
  __shared__ uint32_t s_tile;
  const unsigned w = warp_id(), l = lane_id(), t = threadIdx.x;
  if (t == 0) s_tile = atomicAdd(tile_ctr, 1u);
  uint32_t *s_mask = reinterpret_cast<uint32_t *>(s_keys);
#pragma unroll
  for (int i = 0; i < T_WARPS; ++i) s_whist[i][t] = 0;
  if (RANK == 0) {
#pragma unroll
    for (int i = 0; i < 2 * T_WARPS; ++i) s_mask[i * 256 + t] = 0;
  }
  if (EARLY) s_cnt[t] = 0;
  __syncthreads();
  const uint64_t tile = s_tile;
  const uint64_t base = tile * T_TILE;
  const bool full = base + T_TILE <= n;
  uint64_t k[T_ITEMS];
  uint32_t r[T_ITEMS];
  const uint64_t wbase = base + w * (32 * T_ITEMS) + l;
  if (full) {
#pragma unroll
    for (int i = 0; i < T_ITEMS; ++i) k[i] = __ldcs(in + wbase + i * 32);
  } else {
#pragma unroll
    for (int i = 0; i < T_ITEMS; ++i) k[i] = (wbase + i * 32 < n) ? __ldcs(in + wbase + i * 32) : ~0ull;
  }
  uint64_t *st = status + t;
  uint32_t tcount = 0, lstart = 0;
  if (EARLY) {
#pragma unroll
    for (int i = 0; i < T_ITEMS; ++i)
      if (full || wbase + i * 32 < n) atomicAdd(&s_cnt[(uint32_t)(k[i] >> shift) & 255u], 1u);
    __syncthreads();
    tcount = s_cnt[t];
    st_relaxed_u64(st + tile * 256, (tile == 0 ? LB_INC : LB_AGG) | tcount);
    lstart = bscan256<uint32_t>(tcount, s_warp32, &s_total32);
  }
  const unsigned lt_mask = (1u << l) - 1u;
  uint32_t *whist = s_whist[w];
  uint32_t *mask0 = s_mask + w * 256, *mask1 = s_mask + (T_WARPS + w) * 256;
  // SKIP==5: first look-back window prefetched before ranking (consumed after it)
  uint64_t pv0 = 0, pv1 = 0, pv2 = 0, pv3 = 0;
  if (SKIP == 5 && EARLY && tile > 0) {
    const uint64_t *p = st + (tile - 1) * 256;
    pv0 = ld_relaxed_u64(p);
    pv1 = tile > 1 ? ld_relaxed_u64(p - 256) : 0ull;
    pv2 = tile > 2 ? ld_relaxed_u64(p - 512) : 0ull;
    pv3 = tile > 3 ? ld_relaxed_u64(p - 768) : 0ull;
  }
  if (RANK == 3 || RANK == 4) {
    // batched: peers of all items first (ALU/vote only), then the leaders' atomics with
    // return (independent, pipelined), then the broadcasts
    unsigned pe[T_ITEMS];
#pragma unroll
    for (int i = 0; i < T_ITEMS; ++i) {
      const uint32_t d = (uint32_t)(k[i] >> shift) & 255u;
      const bool valid = full || wbase + i * 32 < n;
      unsigned peers;
      if (RANK == 3) {
        peers = __ballot_sync(0xffffffffu, valid);
        if (!valid) peers = ~peers;
#pragma unroll
        for (int b = 0; b < 8; ++b) {
          const unsigned bb = __ballot_sync(0xffffffffu, (d >> b) & 1u);
          peers &= ((d >> b) & 1u) ? bb : ~bb;
        }
      } else {
        peers = __match_any_sync(0xffffffffu, valid ? d : 0xffffffffu);
      }
      pe[i] = peers;
    }
#pragma unroll
    for (int i = 0; i < T_ITEMS; ++i) {
      const uint32_t d = (uint32_t)(k[i] >> shift) & 255u;
      const bool valid = full || wbase + i * 32 < n;
      const unsigned lead = __ffs(pe[i]) - 1;
      uint32_t old = 0;
      if (valid && l == lead) old = atomicAdd(&whist[d], (uint32_t)__popc(pe[i]));
      r[i] = old;
    }
#pragma unroll
    for (int i = 0; i < T_ITEMS; ++i) {
      const unsigned lead = __ffs(pe[i]) - 1;
      r[i] = __shfl_sync(0xffffffffu, r[i], lead) + __popc(pe[i] & lt_mask);
    }
  } else
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i) {
    const uint32_t d = (uint32_t)(k[i] >> shift) & 255u;
    const bool valid = full || wbase + i * 32 < n;
    if (SKIP == 2) r[i] = 0;
    else if (RANK == 0) r[i] = rank_or(d, valid, whist, (i & 1) ? mask1 : mask0, l, lt_mask);
    else if (RANK == 1) r[i] = rank_ballot(d, valid, whist, l, lt_mask);
    else r[i] = rank_match(d, valid, whist, l, lt_mask);
  }
  __syncthreads();
  if (!EARLY) {
    uint32_t c = 0;
#pragma unroll
    for (int ww = 0; ww < T_WARPS; ++ww) c += s_whist[ww][t];
    tcount = c;
    st_relaxed_u64(st + tile * 256, (tile == 0 ? LB_INC : LB_AGG) | tcount);
    lstart = bscan256<uint32_t>(tcount, s_warp32, &s_total32);
  }
  uint32_t run = lstart;
#pragma unroll
  for (int ww = 0; ww < T_WARPS; ++ww) {
    uint32_t c = s_whist[ww][t];
    s_whist[ww][t] = run;
    run += c;
  }
  uint64_t e = 0;
  if (SKIP == 1) e = tile * 16;
  else if (tile > 0) {
    const uint64_t *p = st + (tile - 1) * 256;
    uint32_t left = (uint32_t)tile;
    bool pre = SKIP == 5 && EARLY;
    while (true) {
      uint64_t v0, v1, v2, v3;
      if (pre) {
        v0 = pv0; v1 = pv1; v2 = pv2; v3 = pv3;
        pre = false;
      } else {
        v0 = ld_relaxed_u64(p);
        v1 = left > 1 ? ld_relaxed_u64(p - 256) : 0ull;
        v2 = left > 2 ? ld_relaxed_u64(p - 512) : 0ull;
        v3 = left > 3 ? ld_relaxed_u64(p - 768) : 0ull;
      }
      const uint32_t h0 = (uint32_t)(v0 >> 32), h1 = (uint32_t)(v1 >> 32), h2 = (uint32_t)(v2 >> 32),
                     h3 = (uint32_t)(v3 >> 32);
      if (h0 < 0x40000000u) {
        __nanosleep(32);
        continue;
      }
      e += v0 & LB_VAL;
      if (h0 >= 0x80000000u) break;
      if (h1 < 0x40000000u) { p -= 256; left -= 1; continue; }
      e += v1 & LB_VAL;
      if (h1 >= 0x80000000u) break;
      if (h2 < 0x40000000u) { p -= 512; left -= 2; continue; }
      e += v2 & LB_VAL;
      if (h2 >= 0x80000000u) break;
      if (h3 < 0x40000000u) { p -= 768; left -= 3; continue; }
      e += v3 & LB_VAL;
      if (h3 >= 0x80000000u) break;
      p -= 1024;
      left -= 4;
    }
    st_relaxed_u64(st + tile * 256, LB_INC | (e + tcount));
  }
  s_gbase[t] = goff[t] + e - lstart;
  __syncthreads();
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i) {
    uint32_t d = (uint32_t)(k[i] >> shift) & 255u;
    if (full || wbase + i * 32 < n) s_keys[s_whist[w][d] + r[i]] = k[i];
  }
  __syncthreads();
  const uint32_t valid_count = full ? T_TILE : (uint32_t)(n - base);
#pragma unroll 4
  for (uint32_t j = t; j < valid_count; j += T_THREADS) {
    uint64_t key = s_keys[j];
    uint64_t idx = s_gbase[(uint32_t)(key >> shift) & 255u] + j;
    if (SKIP == 1) idx &= (n - 1);
    if (SKIP == 3) idx = base + j;
    if (SKIP == 4) { if (key == 0x1234567ull) out[0] = idx; }
    else out[idx] = key;
  }
}

__global__ void hist_kernel(const uint64_t *__restrict__ k, uint64_t n, int shift, unsigned long long *h) {
  __shared__ uint32_t s[256];
  s[threadIdx.x] = 0;
  __syncthreads();
  for (uint64_t i = blockIdx.x * 256ull + threadIdx.x; i < n; i += gridDim.x * 256ull)
    atomicAdd(&s[(k[i] >> shift) & 255], 1u);
  __syncthreads();
  atomicAdd(&h[threadIdx.x], (unsigned long long)s[threadIdx.x]);
}

__global__ void gen_kernel(uint64_t *k, uint64_t n, uint64_t mask) {
  for (uint64_t i = blockIdx.x * 256ull + threadIdx.x; i < n; i += gridDim.x * 256ull) {
    uint64_t x = i * 0x9E3779B97F4A7C15ull + 12345;
    x ^= x >> 31; x *= 0xBF58476D1CE4E5B9ull; x ^= x >> 29; x *= 0x94D049BB133111EBull; x ^= x >> 32;
    k[i] = x & mask;
  }
}

__device__ __forceinline__ uint64_t mix(uint64_t x) {
  x ^= x >> 31; x *= 0xBF58476D1CE4E5B9ull; x ^= x >> 29; x *= 0x94D049BB133111EBull; x ^= x >> 32;
  return x;
}
__global__ void copy_kernel(const uint64_t *__restrict__ a, uint64_t *__restrict__ b, uint64_t n) {
  for (uint64_t i = blockIdx.x * 256ull + threadIdx.x; i < n; i += gridDim.x * 256ull) b[i] = __ldcs(a + i);
}
__global__ void redg_kernel(uint32_t *cnt, uint64_t n, uint32_t nv) {
  for (uint64_t i = blockIdx.x * 256ull + threadIdx.x; i < n; i += gridDim.x * 256ull)
    atomicAdd(&cnt[mix(i) % nv], 1u);
}
__global__ void atomg_store_kernel(uint32_t *cnt, uint32_t *dst, uint64_t n, uint32_t nv) {
  for (uint64_t i = blockIdx.x * 256ull + threadIdx.x; i < n; i += gridDim.x * 256ull) {
    uint32_t v = (uint32_t)(mix(i) % nv);
    uint32_t p = atomicAdd(&cnt[v], 1u);
    dst[(uint64_t)v * 16 + (p & 15)] = (uint32_t)i;
  }
}
__global__ void rstore_kernel(uint32_t *dst, uint64_t n, uint64_t m) {
  for (uint64_t i = blockIdx.x * 256ull + threadIdx.x; i < n; i += gridDim.x * 256ull) dst[mix(i) % m] = (uint32_t)i;
}
__global__ void rgather_kernel(const uint32_t *src, uint64_t n, uint64_t m, unsigned long long *sink) {
  uint32_t acc = 0;
  for (uint64_t i = blockIdx.x * 256ull + threadIdx.x; i < n; i += gridDim.x * 256ull) acc += src[mix(i) % m];
  if (acc == 0x12345678u) atomicAdd(sink, 1ull);
}
// 64 B random segment gather (a list of 16 u32) by half-warps
__global__ void rgather64_kernel(const uint32_t *src, uint64_t nseg, uint64_t m, unsigned long long *sink) {
  uint32_t acc = 0;
  for (uint64_t i = blockIdx.x * 256ull + threadIdx.x; i < nseg * 16; i += gridDim.x * 256ull) {
    uint64_t seg = mix(i >> 4) % (m / 16);
    acc += src[seg * 16 + (i & 15)];
  }
  if (acc == 0x12345678u) atomicAdd(sink, 1ull);
}

struct Timer {
  cudaEvent_t a, b;
  Timer() { cudaEventCreate(&a); cudaEventCreate(&b); }
  void start() { cudaEventRecord(a); }
  float stop() { cudaEventRecord(b); cudaEventSynchronize(b); float ms; cudaEventElapsedTime(&ms, a, b); return ms; }
};


// ---------------------------------------------------------------- persistent + TMA prefetch
__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
  unsigned a = (unsigned)__cvta_generic_to_shared(bar);
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, unsigned bytes) {
  unsigned a = (unsigned)__cvta_generic_to_shared(bar);
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(a), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_g2s(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
  unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  unsigned b = (unsigned)__cvta_generic_to_shared(bar);
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(d),
               "l"(src), "r"(bytes), "r"(b)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, unsigned phase) {
  unsigned a = (unsigned)__cvta_generic_to_shared(bar);
  asm volatile(
      "{\n.reg .pred p;\nWAIT_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra WAIT_%=;\n}\n" ::"r"(a),
      "r"(phase)
      : "memory");
}

constexpr int P_ITEMS = 16;
constexpr int P_TILE = T_THREADS * P_ITEMS;
// dynamic smem: stage[NST][P_TILE] u64, masks [2][8][256] u32
template <int MINB, int NST, int BAL = 0>
__global__ __launch_bounds__(T_THREADS, MINB) void pass_p(const uint64_t *__restrict__ in, uint64_t *__restrict__ out,
                                                          uint64_t n, int shift,
                                                          const unsigned long long *__restrict__ goff,
                                                          uint64_t *status, uint32_t *tile_ctr, uint32_t ntiles) {
  extern __shared__ __align__(128) uint64_t dsm[];
  uint64_t *stage = dsm;                                              // NST * P_TILE
  uint32_t *s_mask = reinterpret_cast<uint32_t *>(dsm + NST * P_TILE);  // 2*8*256
  __shared__ uint32_t s_whist[T_WARPS][256];
  __shared__ uint32_t s_cnt[256];
  __shared__ uint64_t s_gbase[256];
  __shared__ uint32_t s_warp32[8];
  __shared__ uint32_t s_total32;
  __shared__ uint32_t s_tiles[NST];
  __shared__ __align__(8) uint64_t s_bar[NST];
  const unsigned w = warp_id(), l = lane_id(), t = threadIdx.x;
  if (!BAL) {
#pragma unroll
    for (int i = 0; i < 2 * T_WARPS; ++i) s_mask[i * 256 + t] = 0;
  }
#pragma unroll
  for (int i = 0; i < T_WARPS; ++i) s_whist[i][t] = 0;
  s_cnt[t] = 0;
  if (t == 0) {
    for (int sidx = 0; sidx < NST; ++sidx) mbar_init(&s_bar[sidx], 1);
  }
  __syncthreads();
  // prologue: claim and request NST-1 tiles
  if (t == 0) {
    for (int sidx = 0; sidx < NST - 1; ++sidx) {
      uint32_t tl = atomicAdd(tile_ctr, 1u);
      s_tiles[sidx] = tl;
      if (tl < ntiles) {
        uint64_t b0 = (uint64_t)tl * P_TILE;
        uint32_t cnt = (uint32_t)min((uint64_t)P_TILE, n - b0);
        mbar_expect_tx(&s_bar[sidx], cnt * 8);
        tma_g2s(stage + sidx * P_TILE, in + b0, cnt * 8, &s_bar[sidx]);
      }
    }
  }
  uint32_t phase_bits = 0;
  const unsigned lt_mask = (1u << l) - 1u;
  uint32_t *whist = s_whist[w];
  uint32_t *mask0 = s_mask + w * 256, *mask1 = s_mask + (T_WARPS + w) * 256;
  for (uint32_t it = 0;; ++it) {
    const int cs = it % NST;
    // claim + request the tile NST-1 ahead into the stage freed by the previous iteration
    if (t == 0) {
      const int ns = (it + NST - 1) % NST;
      uint32_t tl = atomicAdd(tile_ctr, 1u);
      s_tiles[ns] = tl;
      if (tl < ntiles) {
        uint64_t b0 = (uint64_t)tl * P_TILE;
        uint32_t cnt = (uint32_t)min((uint64_t)P_TILE, n - b0);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_expect_tx(&s_bar[ns], cnt * 8);
        tma_g2s(stage + ns * P_TILE, in + b0, cnt * 8, &s_bar[ns]);
      }
    }
    __syncthreads();
    const uint32_t tile32 = s_tiles[cs];
    if (tile32 >= ntiles) break;
    const uint64_t tile = tile32;
    const uint64_t base = tile * P_TILE;
    const bool full = base + P_TILE <= n;
    mbar_wait(&s_bar[cs], (phase_bits >> cs) & 1u);
    phase_bits ^= 1u << cs;
    uint64_t *sk = stage + cs * P_TILE;
    uint64_t k[P_ITEMS];
    uint32_t r[P_ITEMS];
    const uint32_t wl = w * (32 * P_ITEMS) + l;
#pragma unroll
    for (int i = 0; i < P_ITEMS; ++i) k[i] = (full || base + wl + i * 32 < n) ? sk[wl + i * 32] : ~0ull;
#pragma unroll
    for (int i = 0; i < P_ITEMS; ++i)
      if (full || base + wl + i * 32 < n) atomicAdd(&s_cnt[(uint32_t)(k[i] >> shift) & 255u], 1u);
    __syncthreads();
    const uint32_t tcount = s_cnt[t];
    uint64_t *st = status + t;
    st_relaxed_u64(st + tile * 256, (tile == 0 ? LB_INC : LB_AGG) | tcount);
    const uint32_t lstart = bscan256<uint32_t>(tcount, s_warp32, &s_total32);
    s_cnt[t] = 0;
#pragma unroll
    for (int i = 0; i < P_ITEMS; ++i)
      r[i] = BAL ? rank_ballot((uint32_t)(k[i] >> shift) & 255u, full || base + wl + i * 32 < n, whist, l, lt_mask)
                 : rank_or((uint32_t)(k[i] >> shift) & 255u, full || base + wl + i * 32 < n, whist, (i & 1) ? mask1 : mask0,
                     l, lt_mask);
    __syncthreads();
    uint32_t run = lstart;
#pragma unroll
    for (int ww = 0; ww < T_WARPS; ++ww) {
      uint32_t c = s_whist[ww][t];
      s_whist[ww][t] = run;
      run += c;
    }
    uint64_t e = 0;
    if (tile > 0) {
      const uint64_t *p = st + (tile - 1) * 256;
      uint32_t left = (uint32_t)tile;
      while (true) {
        const uint64_t v0 = ld_relaxed_u64(p);
        const uint64_t v1 = left > 1 ? ld_relaxed_u64(p - 256) : 0ull;
        const uint64_t v2 = left > 2 ? ld_relaxed_u64(p - 512) : 0ull;
        const uint64_t v3 = left > 3 ? ld_relaxed_u64(p - 768) : 0ull;
        const uint32_t h0 = (uint32_t)(v0 >> 32), h1 = (uint32_t)(v1 >> 32), h2 = (uint32_t)(v2 >> 32),
                       h3 = (uint32_t)(v3 >> 32);
        if (h0 < 0x40000000u) {
          __nanosleep(32);
          continue;
        }
        e += v0 & LB_VAL;
        if (h0 >= 0x80000000u) break;
        if (h1 < 0x40000000u) { p -= 256; left -= 1; continue; }
        e += v1 & LB_VAL;
        if (h1 >= 0x80000000u) break;
        if (h2 < 0x40000000u) { p -= 512; left -= 2; continue; }
        e += v2 & LB_VAL;
        if (h2 >= 0x80000000u) break;
        if (h3 < 0x40000000u) { p -= 768; left -= 3; continue; }
        e += v3 & LB_VAL;
        if (h3 >= 0x80000000u) break;
        p -= 1024;
        left -= 4;
      }
      st_relaxed_u64(st + tile * 256, LB_INC | (e + tcount));
    }
    s_gbase[t] = goff[t] + e - lstart;
    // keys are in registers: the stage buffer becomes the exchange buffer
#pragma unroll
    for (int i = 0; i < P_ITEMS; ++i) {
      uint32_t d = (uint32_t)(k[i] >> shift) & 255u;
      if (full || base + wl + i * 32 < n) sk[s_whist[w][d] + r[i]] = k[i];
    }
    __syncthreads();
    const uint32_t valid_count = full ? P_TILE : (uint32_t)(n - base);
#pragma unroll 4
    for (uint32_t j = t; j < valid_count; j += T_THREADS) {
      uint64_t key = sk[j];
      out[s_gbase[(uint32_t)(key >> shift) & 255u] + j] = key;
    }
#pragma unroll
    for (int i = 0; i < T_WARPS; ++i) s_whist[i][t] = 0;
  }
}

template <int MINB, int NST, int BAL = 0>
float run_pass_p(const uint64_t *in, uint64_t *out, uint64_t n, int shift, unsigned long long *goff,
                 uint64_t *scratch, int reps) {
  uint32_t ntiles = (uint32_t)((n + P_TILE - 1) / P_TILE);
  size_t dsm = (size_t)NST * P_TILE * 8 + (BAL ? 0 : 2 * 8 * 256 * 4);
  TC_CUDA(cudaFuncSetAttribute(pass_p<MINB, NST, BAL>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsm));
  int occ = 0;
  TC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, pass_p<MINB, NST, BAL>, T_THREADS, dsm));
  Timer tm;
  float best = 1e9;
  for (int r = 0; r < reps; ++r) {
    cudaMemsetAsync(scratch, 0, (1 + (uint64_t)ntiles * 256) * 8);
    tm.start();
    pass_p<MINB, NST, BAL><<<148 * occ, T_THREADS, dsm>>>(in, out, n, shift, goff, scratch + 1, (uint32_t *)scratch, ntiles);
    float ms = tm.stop();
    if (ms < best) best = ms;
  }
  TC_CUDA(cudaGetLastError());
  printf("  (persistent occ %d CTAs/SM, smem %zu)\n", occ, dsm);
  return best;
}

template <int RANK, int EARLY, int T_ITEMS = 16, int MINB = 4, int SKIP = 0>
float run_pass(const uint64_t *in, uint64_t *out, uint64_t n, int shift, unsigned long long *goff, uint64_t *scratch,
               int reps) {
  constexpr int T_TILE = T_THREADS * T_ITEMS;
  uint64_t ntiles = (n + T_TILE - 1) / T_TILE;
  Timer tm;
  float best = 1e9;
  for (int r = 0; r < reps; ++r) {
    cudaMemsetAsync(scratch, 0, (1 + ntiles * 256) * 8);
    tm.start();
    pass_kernel<RANK, EARLY, T_ITEMS, MINB, SKIP><<<(unsigned)ntiles, T_THREADS>>>(in, out, n, shift, goff, scratch + 1, (uint32_t *)scratch);
    float ms = tm.stop();
    if (ms < best) best = ms;
  }
  TC_CUDA(cudaGetLastError());
  return best;
}

int main() {
  const uint64_t n = 1ull << 26;
  uint64_t *a, *b, *ref, *scratch;
  unsigned long long *h;
  TC_CUDA(cudaMalloc(&a, n * 8));
  TC_CUDA(cudaMalloc(&b, n * 8));
  TC_CUDA(cudaMalloc(&ref, n * 8));
  uint64_t ntiles = (n + 2047) / 2048;
  TC_CUDA(cudaMalloc(&scratch, (1 + ntiles * 256) * 8));
  TC_CUDA(cudaMalloc(&h, 256 * 8));
  gen_kernel<<<4096, 256>>>(a, n, (1ull << 44) - 1);
  const int shift = 8;
  cudaMemset(h, 0, 256 * 8);
  hist_kernel<<<1184, 256>>>(a, n, shift, h);
  std::vector<unsigned long long> hh(256);
  cudaMemcpy(hh.data(), h, 256 * 8, cudaMemcpyDeviceToHost);
  unsigned long long acc = 0;
  for (int i = 0; i < 256; ++i) { unsigned long long c = hh[i]; hh[i] = acc; acc += c; }
  cudaMemcpy(h, hh.data(), 256 * 8, cudaMemcpyHostToDevice);
  Timer tm;
  {
    float best = 1e9;
    for (int r = 0; r < 5; ++r) { tm.start(); copy_kernel<<<148 * 8, 256>>>(a, b, n); best = std::min(best, tm.stop()); }
    printf("copy 8B keys: %.3f ms  %.0f GB/s\n", best, 16.0 * n / best / 1e6);
  }
  const int reps = 7;
  float t00 = run_pass<0, 1>(a, ref, n, shift, h, scratch, reps);
  printf("pass or-mask early   : %.3f ms  %.0f GB/s\n", t00, 16.0 * n / t00 / 1e6);
  auto check = [&](const char *name, float ms) {
    std::vector<uint64_t> x(n), y(n);
    cudaMemcpy(x.data(), b, n * 8, cudaMemcpyDeviceToHost);
    cudaMemcpy(y.data(), ref, n * 8, cudaMemcpyDeviceToHost);
    bool ok = x == y;
    printf("pass %-16s: %.3f ms  %.0f GB/s  %s\n", name, ms, 16.0 * n / ms / 1e6, ok ? "OK" : "MISMATCH");
  };
  check("or-mask late", run_pass<0, 0>(a, b, n, shift, h, scratch, reps));
  check("ballot early", run_pass<1, 1>(a, b, n, shift, h, scratch, reps));
  check("ballot late", run_pass<1, 0>(a, b, n, shift, h, scratch, reps));
  check("or items12 minb5", run_pass<0, 1, 12, 5>(a, b, n, shift, h, scratch, reps));
  check("or items8 minb6", run_pass<0, 1, 8, 6>(a, b, n, shift, h, scratch, reps));
  check("or items16 minb3", run_pass<0, 1, 16, 3>(a, b, n, shift, h, scratch, reps));
  check("ballot items12 minb5", run_pass<1, 1, 12, 5>(a, b, n, shift, h, scratch, reps));
  check("SKIP lookback", run_pass<0, 1, 16, 4, 1>(a, b, n, shift, h, scratch, reps));
  check("prefetch-lookback", run_pass<0, 1, 16, 4, 5>(a, b, n, shift, h, scratch, reps));
  check("prefetch-lookback bal", run_pass<1, 1, 16, 4, 5>(a, b, n, shift, h, scratch, reps));
  check("persist 2st minb2", run_pass_p<2, 2>(a, b, n, shift, h, scratch, reps));
  check("persist bal 2st minb3", run_pass_p<3, 2, 1>(a, b, n, shift, h, scratch, reps));
  check("persist 2st minb3", run_pass_p<3, 2>(a, b, n, shift, h, scratch, reps));
  check("SEQ write", run_pass<0, 1, 16, 4, 3>(a, b, n, shift, h, scratch, reps));
  check("NO write", run_pass<0, 1, 16, 4, 4>(a, b, n, shift, h, scratch, reps));
  check("SKIP rank", run_pass<0, 1, 16, 4, 2>(a, b, n, shift, h, scratch, reps));

  // random access patterns (n = 2^26 operations)
  uint32_t *cnt, *big;
  const uint32_t nv = 1u << 22;
  const uint64_t bigm = 1ull << 26;  // 256 MiB of u32
  TC_CUDA(cudaMalloc(&cnt, nv * 4));
  TC_CUDA(cudaMalloc(&big, bigm * 4));
  auto timeit = [&](const char *name, auto fn) {
    float best = 1e9;
    for (int r = 0; r < 5; ++r) { cudaMemset(cnt, 0, nv * 4); tm.start(); fn(); best = std::min(best, tm.stop()); }
    TC_CUDA(cudaGetLastError());
    printf("%-40s %.3f ms  %.1f Gop/s\n", name, best, n / best / 1e6);
  };
  timeit("REDG random into 16 MiB", [&] { redg_kernel<<<148 * 8, 256>>>(cnt, n, nv); });
  timeit("ATOMG random + dependent 4B store", [&] { atomg_store_kernel<<<148 * 8, 256>>>(cnt, big, n, nv); });
  timeit("random 4B store into 256 MiB", [&] { rstore_kernel<<<148 * 8, 256>>>(big, n, bigm); });
  timeit("random 4B gather from 256 MiB", [&] { rgather_kernel<<<148 * 8, 256>>>(big, n, bigm, h); });
  timeit("random 64B-segment gather (ops=u32)", [&] { rgather64_kernel<<<148 * 8, 256>>>(big, n / 16, bigm, h); });
  return 0;
}
