// prims.cu — one-sweep LSD radix sort, look-back scan and unique-select for sm_100a.
//
// All three are single-pass over their input per digit/scan using decoupled look-back
// (tiles obtain their index from an atomic counter, publish an aggregate, then the
// inclusive prefix), so each radix pass reads and writes the keys exactly once
// (16 B per key per pass of HBM traffic), plus one up-front read for all digit
// histograms.  Digits are 8 bits; only the significant bits are sorted (the CSR
// build packs (u, v) into 2*ceil(log2 n) bits).
#include "prims.cuh"

namespace tc {

namespace {

constexpr int T_THREADS = 256;
constexpr int T_ITEMS = 16;
constexpr int T_TILE = T_THREADS * T_ITEMS;  // 4096
constexpr int T_WARPS = T_THREADS / 32;
constexpr int MAX_PASSES = 8;

// ------------------------------------------------------------------ key sources
// Radix-sort input loaders: plain keys, or raw edge samples canonicalised on the fly
// (step a1 fused into the histogram and the first pass: (min << b) | max, self-loop or
// out-of-range id -> all-ones sentinel; out-of-range ids also raise *err).
struct KeySrc {
  const uint64_t *__restrict__ k;
  __device__ __forceinline__ uint64_t load(uint64_t i) const { return __ldcs(k + i); }
};
struct EdgeSrc {
  const uint32_t *__restrict__ src;
  const uint32_t *__restrict__ dst;
  uint32_t n;
  int bits;
  uint64_t sentinel;
  unsigned *err;  // set only by the histogram kernel
  __device__ __forceinline__ uint64_t load(uint64_t i) const {
    uint32_t u = __ldcs(src + i), v = __ldcs(dst + i);
    if (u >= n || v >= n) {
      if (err) atomicOr(err, 1u);
      return sentinel;
    }
    if (u == v) return sentinel;
    return ((uint64_t)min(u, v) << bits) | max(u, v);
  }
};

// ------------------------------------------------------------------ scan
template <typename TI>
__global__ __launch_bounds__(T_THREADS) void scan_kernel(const TI *__restrict__ in,
                                                             uint64_t *__restrict__ out, uint64_t n,
                                                             uint64_t *status, uint32_t *tile_ctr) {
  __shared__ uint64_t s_warp[8];
  __shared__ uint64_t s_total;
  __shared__ uint32_t s_tile;
  __shared__ uint64_t s_excl;
  if (threadIdx.x == 0) s_tile = atomicAdd(tile_ctr, 1u);
  __syncthreads();
  uint64_t tile = s_tile;
  uint64_t base = tile * T_TILE + (uint64_t)threadIdx.x * T_ITEMS;
  uint64_t v[T_ITEMS];
  uint64_t sum = 0;
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i) {
    uint64_t idx = base + i;
    v[i] = idx < n ? (uint64_t)in[idx] : 0ull;
    sum += v[i];
  }
  uint64_t excl_t = block256_exclusive_scan<uint64_t>(sum, s_warp, &s_total);
  if (threadIdx.x == 0) s_excl = lookback_exclusive(status, tile, 1, s_total);
  __syncthreads();
  uint64_t run = s_excl + excl_t;
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i) {
    uint64_t idx = base + i;
    if (idx <= n) out[idx] = run;  // out[n] = total
    run += v[i];
  }
}

// ------------------------------------------------------------------ unique
// Warp-wide decoupled look-back over one status word per tile (flag | value): lane i
// examines predecessor tile - 1 - i, so one round trip covers 32 tiles.  Called by one
// whole warp; returns the exclusive prefix of `tile` (all lanes) and publishes its
// inclusive value.
__device__ __forceinline__ uint64_t warp_lookback(uint64_t *status, uint64_t tile, uint64_t local) {
  const unsigned l = lane_id();
  if (tile == 0) {
    if (l == 0) st_relaxed_u64(status, LB_INC | local);
    return 0;
  }
  if (l == 0) st_relaxed_u64(status + tile, LB_AGG | local);
  uint64_t excl = 0;
  int64_t j = (int64_t)tile - 1;
  while (true) {
    const uint64_t v = (j - (int64_t)l >= 0) ? ld_relaxed_u64(status + (j - l)) : LB_INC;
    const uint32_t h = (uint32_t)(v >> 32);
    const unsigned notready = __ballot_sync(0xffffffffu, h < 0x40000000u);
    const unsigned incm = __ballot_sync(0xffffffffu, h >= 0x80000000u);
    const int lim = incm ? __ffs(incm) - 1 : 32;  // nearest inclusive value
    const unsigned below = lim == 32 ? 0xffffffffu : ((1u << lim) - 1u);
    if (notready & (below | (incm ? (1u << lim) : 0u))) {
      __nanosleep(32);
      continue;
    }
    excl += warp_sum((int)l <= lim ? (v & LB_VAL) : 0ull);
    if (incm) break;
    j -= 32;
  }
  if (l == 0) st_relaxed_u64(status + tile, LB_INC | (excl + local));
  return excl;
}

// Unique-select; optionally (deg != nullptr) the undirected degrees of the kept edges
// (step a3 fused): keys are (u << bits) | v, u < v; the sentinel key is dropped from deg.
// Warp w of a tile owns 512 consecutive keys, lane l item i = key w*512 + 32*i + l
// (coalesced loads and stores); the predecessor of a key comes from the neighbouring lane.
// deg[v] takes one atomic per kept key; deg[u] one per run of equal u within a 32-key row.
__global__ __launch_bounds__(T_THREADS) void unique_kernel(const uint64_t *__restrict__ in,
                                                           uint64_t *__restrict__ out, uint64_t n,
                                                           uint64_t *status, uint32_t *tile_ctr,
                                                           uint64_t ntiles, uint64_t *d_count, uint32_t *deg,
                                                           int bits, uint64_t sentinel) {
  __shared__ uint32_t s_wcnt[T_WARPS];
  __shared__ uint64_t s_base;
  __shared__ uint32_t s_tile;
  if (threadIdx.x == 0) s_tile = atomicAdd(tile_ctr, 1u);
  __syncthreads();
  const uint64_t tile = s_tile;
  const unsigned w = warp_id(), l = lane_id();
  const uint64_t wb = tile * T_TILE + (uint64_t)w * (32 * T_ITEMS);
  uint64_t k[T_ITEMS];
  unsigned hm[T_ITEMS];
  uint64_t before = 0;
  if (l == 0 && wb > 0 && wb <= n) before = in[wb - 1];
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i) {
    const uint64_t idx = wb + 32 * i + l;
    k[i] = idx < n ? __ldcs(in + idx) : 0ull;
  }
  uint32_t wcnt = 0;
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i) {
    const uint64_t idx = wb + 32 * i + l;
    uint64_t prev = __shfl_up_sync(0xffffffffu, k[i], 1);
    const uint64_t last_prev_row = __shfl_sync(0xffffffffu, i ? k[i - 1] : before, 31);
    if (l == 0) prev = i ? last_prev_row : before;
    const bool head = idx < n && (idx == 0 || k[i] != prev);
    hm[i] = __ballot_sync(0xffffffffu, head);
    wcnt += __popc(hm[i]);
  }
  if (l == 0) s_wcnt[w] = wcnt;
  __syncthreads();
  if (w == 0) {
    const uint32_t c = l < T_WARPS ? s_wcnt[l] : 0u;
    const uint32_t inc = warp_inclusive_scan(c);
    const uint32_t total = __shfl_sync(0xffffffffu, inc, 31);
    const uint64_t excl = warp_lookback(status, tile, total);
    if (l < T_WARPS) s_wcnt[l] = inc - c;
    if (l == 0) {
      s_base = excl;
      if (tile == ntiles - 1) *d_count = excl + total;
    }
  }
  __syncthreads();
  uint64_t pos = s_base + s_wcnt[w];
  const unsigned lt = (1u << l) - 1u;
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i) {
    if (hm[i] >> l & 1u) out[pos + __popc(hm[i] & lt)] = k[i];
    pos += __popc(hm[i]);
  }
  if (deg) {
    const uint64_t mask = (1ull << bits) - 1;
#pragma unroll
    for (int i = 0; i < T_ITEMS; ++i) {
      const bool keep = (hm[i] >> l & 1u) && k[i] != sentinel;
      const uint32_t u = (uint32_t)(k[i] >> bits), v = (uint32_t)(k[i] & mask);
      if (keep) atomicAdd(&deg[v], 1u);
      // runs of equal u along the row (keys ascending): the run's last lane adds its kept count
      const unsigned km = __ballot_sync(0xffffffffu, keep);
      if (!km) continue;
      const uint32_t un = __shfl_down_sync(0xffffffffu, u, 1);
      const uint32_t up = __shfl_up_sync(0xffffffffu, u, 1);
      const unsigned starts = __ballot_sync(0xffffffffu, l == 0 || up != u);
      const bool last = l == 31 || un != u;
      if (last) {
        const unsigned upto = l == 31 ? 0xffffffffu : ((2u << l) - 1u);
        const int rs = 31 - __clz(starts & upto);
        const unsigned c = __popc(km & upto & ~((1u << rs) - 1u));
        if (c) atomicAdd(&deg[u], c);
      }
    }
  }
}

// ------------------------------------------------------------------ orientation split
// Sorted undirected keys (a << bits) | b, a < b, are split by the orientation rule
// u -> v iff (prim[u], u) < (prim[v], v): forward edges (a -> b) keep their key and their
// order in F; reversed edges (b -> a) become (b << bits) | a in R, in input order (so each
// source's group is ascending in a after a stable sort of R on the source bits).  One
// look-back on the forward count per tile; the reversed position is (index - forward).
__global__ __launch_bounds__(T_THREADS) void split_kernel(const uint64_t *__restrict__ in, uint64_t n, int bits,
                                                          const uint64_t *__restrict__ prim, uint64_t *__restrict__ F,
                                                          uint64_t *__restrict__ R, uint64_t *status,
                                                          uint32_t *tile_ctr, uint64_t ntiles, uint64_t *d_nf) {
  __shared__ uint32_t s_wcnt[T_WARPS];
  __shared__ uint64_t s_base;
  __shared__ uint32_t s_tile;
  if (threadIdx.x == 0) s_tile = atomicAdd(tile_ctr, 1u);
  __syncthreads();
  const uint64_t tile = s_tile;
  const unsigned w = warp_id(), l = lane_id();
  const uint64_t wb = tile * T_TILE + (uint64_t)w * (32 * T_ITEMS);
  const uint64_t mask = (1ull << bits) - 1;
  uint64_t k[T_ITEMS];
  unsigned fm[T_ITEMS];
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i) {
    const uint64_t idx = wb + 32 * i + l;
    k[i] = idx < n ? __ldcs(in + idx) : 0ull;
  }
  uint32_t wcnt = 0;
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i) {
    const uint64_t idx = wb + 32 * i + l;
    bool fwd = false;
    if (idx < n) {
      const uint32_t a = (uint32_t)(k[i] >> bits), b = (uint32_t)(k[i] & mask);
      fwd = prim[a] <= prim[b];
      if (!fwd) k[i] = ((uint64_t)b << bits) | a;
    }
    fm[i] = __ballot_sync(0xffffffffu, fwd);
    wcnt += __popc(fm[i]);
  }
  if (l == 0) s_wcnt[w] = wcnt;
  __syncthreads();
  if (w == 0) {
    const uint32_t c = l < T_WARPS ? s_wcnt[l] : 0u;
    const uint32_t inc = warp_inclusive_scan(c);
    const uint32_t total = __shfl_sync(0xffffffffu, inc, 31);
    const uint64_t excl = warp_lookback(status, tile, total);
    if (l < T_WARPS) s_wcnt[l] = inc - c;
    if (l == 0) {
      s_base = excl;
      if (tile == ntiles - 1) *d_nf = excl + total;
    }
  }
  __syncthreads();
  uint64_t fpos = s_base + s_wcnt[w];  // forward edges before this warp's first key
  const unsigned lt = (1u << l) - 1u;
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i) {
    const uint64_t row = wb + 32 * i;  // keys before this row: row; forward among them: fpos
    const uint64_t idx = row + l;
    if (idx < n) {
      const uint32_t fb = __popc(fm[i] & lt);
      if (fm[i] >> l & 1u) F[fpos + fb] = k[i];
      else R[(row - fpos) + (l - fb)] = k[i];
    }
    fpos += __popc(fm[i]);
  }
}

// ------------------------------------------------------------------ radix sort
// Up-front digit histograms for every pass; per-warp private smem counters.
template <class Src>
__global__ __launch_bounds__(T_THREADS) void rs_hist_kernel(Src keys, uint64_t n, int begin_bit, int passes,
                                                            unsigned long long *ghist) {
  extern __shared__ uint32_t s_h[];  // [T_WARPS/2][passes][256]
  const int groups = T_WARPS / 2;
  for (int i = threadIdx.x; i < groups * passes * 256; i += T_THREADS) s_h[i] = 0;
  __syncthreads();
  uint32_t *mine = s_h + (warp_id() / 2) * passes * 256;
  // 8 independent loads in flight per thread before the shared-memory counting
  constexpr int U = 8;
  const uint64_t stride = (uint64_t)gridDim.x * T_THREADS;
  uint64_t i = (uint64_t)blockIdx.x * T_THREADS + threadIdx.x;
  for (; i + (U - 1) * stride < n; i += U * stride) {
    uint64_t k[U];
#pragma unroll
    for (int u = 0; u < U; ++u) k[u] = keys.load(i + u * stride);
#pragma unroll
    for (int u = 0; u < U; ++u)
      for (int p = 0; p < passes; ++p) atomicAdd(&mine[p * 256 + ((k[u] >> (begin_bit + 8 * p)) & 255u)], 1u);
  }
  for (; i < n; i += stride) {
    uint64_t k = keys.load(i);
    for (int p = 0; p < passes; ++p) atomicAdd(&mine[p * 256 + ((k >> (begin_bit + 8 * p)) & 255u)], 1u);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < passes * 256; i += T_THREADS) {
    uint32_t c = 0;
    for (int g = 0; g < groups; ++g) c += s_h[g * passes * 256 + i];
    if (c) atomicAdd(&ghist[i], (unsigned long long)c);
  }
}

__global__ void rs_hist_scan_kernel(unsigned long long *ghist, int passes) {
  // one block of 256 threads: exclusive scan of each pass' 256 bins, in place
  __shared__ uint64_t s_warp[8];
  __shared__ uint64_t s_total;
  for (int p = 0; p < passes; ++p) {
    uint64_t v = ghist[p * 256 + threadIdx.x];
    uint64_t e = block256_exclusive_scan<uint64_t>(v, s_warp, &s_total);
    __syncthreads();
    ghist[p * 256 + threadIdx.x] = e;
    __syncthreads();
  }
}

// Stable rank of one warp-striped item across the warp: lanes with equal digit found with
// 8 ballots (cheaper than match.any on sm_100a's MIO pipe), the group leader bumps the
// warp's smem counter once, the old value is broadcast back.  Items are processed in
// order by the same warp, so equal digits keep input order (LSD stability).
template <bool FULL>
__device__ __forceinline__ uint32_t rank_item(uint32_t d, bool valid, uint32_t *whist, unsigned lt_mask) {
  unsigned peers = FULL ? 0xffffffffu : __ballot_sync(0xffffffffu, valid);
  if (!FULL && !valid) peers = ~peers;
#pragma unroll
  for (int b = 0; b < 8; ++b) {
    unsigned bit = (d >> b) & 1u;
    unsigned bb = __ballot_sync(0xffffffffu, bit);
    peers &= bit ? bb : ~bb;
  }
  unsigned lead = __ffs(peers) - 1;
  uint32_t old = 0;
  if (lane_id() == lead && (FULL || valid)) old = atomicAdd(&whist[d], (uint32_t)__popc(peers));
  old = __shfl_sync(0xffffffffu, old, lead);
  return old + __popc(peers & lt_mask);
}

// Same rank with a shared-memory peer mask instead of 8 ballots: every lane ORs its bit
// into mask[d]; after a warp barrier the mask IS the peer set.  The leader advances the
// warp's counter and clears the mask (masks double-buffered across consecutive items so
// the clear never races the next item's ORs).  ~12 instructions per key instead of ~30.
__device__ __forceinline__ uint32_t rank_item_or(uint32_t d, bool valid, uint32_t *whist, uint32_t *mask,
                                                 unsigned lane, unsigned lt_mask) {
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

template <class Src>
__global__ __launch_bounds__(T_THREADS, 4) void rs_pass_kernel(Src in, uint64_t *__restrict__ out, uint64_t n,
                                                               int shift,
                                                               const unsigned long long *__restrict__ goff,
                                                               uint64_t *status, uint32_t *tile_ctr) {
  __shared__ uint64_t s_keys[T_TILE];
  __shared__ uint32_t s_whist[T_WARPS][256];
  __shared__ uint32_t s_cnt[256];
  __shared__ uint64_t s_gbase[256];
  __shared__ uint32_t s_warp32[8];
  __shared__ uint32_t s_total32;
  __shared__ uint32_t s_tile;
  const unsigned w = warp_id(), l = lane_id(), t = threadIdx.x;
  if (t == 0) s_tile = atomicAdd(tile_ctr, 1u);
  // ranking peer masks [2 buffers][warp][digit] alias the key staging area, which is only
  // written after ranking completes
  uint32_t *s_mask = reinterpret_cast<uint32_t *>(s_keys);
#pragma unroll
  for (int i = 0; i < T_WARPS; ++i) s_whist[i][t] = 0;
#pragma unroll
  for (int i = 0; i < 2 * T_WARPS; ++i) s_mask[i * 256 + t] = 0;
  s_cnt[t] = 0;
  __syncthreads();
  const uint64_t tile = s_tile;
  const uint64_t base = tile * T_TILE;
  const bool full = base + T_TILE <= n;

  uint64_t k[T_ITEMS];
  uint32_t r[T_ITEMS];
  const uint64_t wbase = base + w * (32 * T_ITEMS) + l;  // warp-striped: stable order
  if (full) {
#pragma unroll
    for (int i = 0; i < T_ITEMS; ++i) k[i] = in.load(wbase + i * 32);
  } else {
#pragma unroll
    for (int i = 0; i < T_ITEMS; ++i) k[i] = (wbase + i * 32 < n) ? in.load(wbase + i * 32) : ~0ull;
  }
  // early tile histogram -> publish the aggregate before the (long) ranking so that
  // successors' look-back rarely waits (one-sweep "early counts")
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i)
    if (full || wbase + i * 32 < n) atomicAdd(&s_cnt[(uint32_t)(k[i] >> shift) & 255u], 1u);
  __syncthreads();
  const uint32_t tcount = s_cnt[t];
  uint64_t *st = status + t;  // status laid out [tile][256]
  st_relaxed_u64(st + tile * 256, (tile == 0 ? LB_INC : LB_AGG) | tcount);
  // tile-local start of digit t (known before ranking thanks to the early counts)
  const uint32_t lstart = block256_exclusive_scan<uint32_t>(tcount, s_warp32, &s_total32);

  const unsigned lt_mask = (1u << l) - 1u;
  uint32_t *whist = s_whist[w];
  uint32_t *mask0 = s_mask + w * 256, *mask1 = s_mask + (T_WARPS + w) * 256;
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i)
    r[i] = rank_item_or((uint32_t)(k[i] >> shift) & 255u, full || wbase + i * 32 < n, whist, (i & 1) ? mask1 : mask0,
                        l, lt_mask);
  __syncthreads();
  // digit t: tile-local start + exclusive prefix over warps -> per-warp scatter base
  uint32_t run = lstart;
#pragma unroll
  for (int ww = 0; ww < T_WARPS; ++ww) {
    uint32_t c = s_whist[ww][t];
    s_whist[ww][t] = run;
    run += c;
  }
  // look-back for digit t, four predecessors per round trip; flags tested on the high
  // word, 32-bit bookkeeping (the walk is executed by every thread, so its instruction
  // count matters as much as its round trips)
  uint64_t e = 0;
  if (tile > 0) {
    const uint64_t *p = st + (tile - 1) * 256;  // this digit's word of the newest predecessor
    uint32_t left = (uint32_t)tile;             // predecessors not yet examined (p is valid)
    while (true) {
      const uint64_t v0 = ld_relaxed_u64(p);
      const uint64_t v1 = left > 1 ? ld_relaxed_u64(p - 256) : 0ull;
      const uint64_t v2 = left > 2 ? ld_relaxed_u64(p - 512) : 0ull;
      const uint64_t v3 = left > 3 ? ld_relaxed_u64(p - 768) : 0ull;
      const uint32_t h0 = (uint32_t)(v0 >> 32), h1 = (uint32_t)(v1 >> 32), h2 = (uint32_t)(v2 >> 32),
                     h3 = (uint32_t)(v3 >> 32);
      // flag (top two bits): 0 not out, 1 aggregate, 2 inclusive
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
  s_gbase[t] = goff[t] + e - lstart;  // global position of tile slot j of digit t = s_gbase[t] + j
  __syncthreads();
#pragma unroll
  for (int i = 0; i < T_ITEMS; ++i) {
    uint32_t d = (uint32_t)(k[i] >> shift) & 255u;
    if (full || wbase + i * 32 < n) s_keys[s_whist[w][d] + r[i]] = k[i];
  }
  __syncthreads();
  if (full) {
#pragma unroll 4
    for (uint32_t j = t; j < T_TILE; j += T_THREADS) {
      uint64_t key = s_keys[j];
      out[s_gbase[(uint32_t)(key >> shift) & 255u] + j] = key;
    }
  } else {
    const uint32_t valid_count = (uint32_t)(n - base);
    for (uint32_t j = t; j < valid_count; j += T_THREADS) {
      uint64_t key = s_keys[j];
      out[s_gbase[(uint32_t)(key >> shift) & 255u] + j] = key;
    }
  }
}

}  // namespace

template <typename TI>
static void scan_impl(const TI *in, uint64_t *out, uint64_t n, cudaStream_t s) {
  uint64_t ntiles = (n + 1 + T_TILE - 1) / T_TILE;  // +1: the total at out[n]
  DevBuf<uint64_t> scratch;
  scratch.alloc(ntiles + 1, s);
  TC_CUDA(cudaMemsetAsync(scratch.get(), 0, scratch.bytes(), s));
  ProfScope prof("scan", s, (double)n * sizeof(TI) + 8.0 * (n + 1));
  scan_kernel<TI><<<(unsigned)ntiles, T_THREADS, 0, s>>>(in, out, n, scratch.get() + 1,
                                                         (uint32_t *)scratch.get());
  TC_LAUNCH_CHECK();
}

void scan_u32_to_u64(const uint32_t *in, uint64_t *out, uint64_t n, cudaStream_t s) {
  scan_impl<uint32_t>(in, out, n, s);
}
void scan_u64(const uint64_t *in, uint64_t *out, uint64_t n, cudaStream_t s) {
  scan_impl<uint64_t>(in, out, n, s);
}

void unique_sorted_u64(const uint64_t *in, uint64_t *out, uint64_t n, uint64_t *d_count, cudaStream_t s,
                       uint32_t *deg, int bits, uint64_t sentinel) {
  if (n == 0) {
    TC_CUDA(cudaMemsetAsync(d_count, 0, sizeof(uint64_t), s));
    return;
  }
  uint64_t ntiles = (n + T_TILE - 1) / T_TILE;
  DevBuf<uint64_t> scratch;
  scratch.alloc(ntiles + 1, s);
  TC_CUDA(cudaMemsetAsync(scratch.get(), 0, scratch.bytes(), s));
  ProfScope prof("unique", s, 8.0 * n);
  unique_kernel<<<(unsigned)ntiles, T_THREADS, 0, s>>>(in, out, n, scratch.get() + 1, (uint32_t *)scratch.get(),
                                                       ntiles, d_count, deg, bits, sentinel);
  TC_LAUNCH_CHECK();
}

uint64_t split_oriented(const uint64_t *edges, uint64_t m, int bits, const uint64_t *prim, uint64_t *F, uint64_t *R,
                        cudaStream_t s) {
  if (m == 0) return 0;
  uint64_t ntiles = (m + T_TILE - 1) / T_TILE;
  DevBuf<uint64_t> scratch;  // [tile counter | forward count][status ntiles]
  scratch.alloc(ntiles + 2, s);
  TC_CUDA(cudaMemsetAsync(scratch.get(), 0, scratch.bytes(), s));
  {
    ProfScope prof("split", s, 16.0 * m);
    split_kernel<<<(unsigned)ntiles, T_THREADS, 0, s>>>(edges, m, bits, prim, F, R, scratch.get() + 2,
                                                        (uint32_t *)scratch.get(), ntiles, scratch.get() + 1);
    TC_LAUNCH_CHECK();
  }
  uint64_t nf = 0;
  TC_CUDA(cudaMemcpyAsync(&nf, scratch.get() + 1, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  return nf;
}

template <class Src>
static uint64_t *radix_sort_impl(Src first, uint64_t *out0, uint64_t *out1, uint64_t n, int begin_bit, int end_bit,
                                 cudaStream_t s) {
  int passes = (end_bit - begin_bit + 7) / 8;
  TC_REQUIRE(passes >= 1 && passes <= MAX_PASSES, ST_INVALID, "radix sort: bad bit range");
  uint64_t ntiles = (n + T_TILE - 1) / T_TILE;
  DevBuf<unsigned long long> hist;
  hist.alloc((size_t)passes * 256, s);
  TC_CUDA(cudaMemsetAsync(hist.get(), 0, hist.bytes(), s));
  size_t hsm = (size_t)(T_WARPS / 2) * passes * 256 * sizeof(uint32_t);
  static bool attr_set = false;
  if (!attr_set) {
    int mx = (int)((T_WARPS / 2) * MAX_PASSES * 256 * sizeof(uint32_t));
    TC_CUDA(cudaFuncSetAttribute(rs_hist_kernel<KeySrc>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx));
    TC_CUDA(cudaFuncSetAttribute(rs_hist_kernel<EdgeSrc>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx));
    attr_set = true;
  }
  {
    ProfScope prof("radix_hist", s, 8.0 * n);
    rs_hist_kernel<Src><<<grid_for(n, T_THREADS, 4), T_THREADS, hsm, s>>>(first, n, begin_bit, passes, hist.get());
    TC_LAUNCH_CHECK();
  }
  rs_hist_scan_kernel<<<1, 256, 0, s>>>(hist.get(), passes);
  TC_LAUNCH_CHECK();
  DevBuf<uint64_t> scratch;  // [tile counter][status ntiles*256]
  {
    ProfScope prof("radix_scratch", s, 0.0);
    scratch.alloc(1 + ntiles * 256, s);
  }
  uint64_t *prev = nullptr;
  for (int p = 0; p < passes; ++p) {
    uint64_t *dst = (p % 2 == 0) ? out0 : out1;
    {
      ProfScope prof("radix_memset", s, 8.0 * scratch.n);
      TC_CUDA(cudaMemsetAsync(scratch.get(), 0, scratch.bytes(), s));
    }
    ProfScope prof("radix_pass", s, 16.0 * n);
    if (p == 0) {
      rs_pass_kernel<Src><<<(unsigned)ntiles, T_THREADS, 0, s>>>(first, dst, n, begin_bit, hist.get(),
                                                                 scratch.get() + 1, (uint32_t *)scratch.get());
    } else {
      rs_pass_kernel<KeySrc><<<(unsigned)ntiles, T_THREADS, 0, s>>>(KeySrc{prev}, dst, n, begin_bit + 8 * p,
                                                                    hist.get() + p * 256, scratch.get() + 1,
                                                                    (uint32_t *)scratch.get());
    }
    TC_LAUNCH_CHECK();
    prev = dst;
  }
  return prev;
}

uint64_t *radix_sort_u64(uint64_t *keys, uint64_t *tmp, uint64_t n, int begin_bit, int end_bit, cudaStream_t s) {
  if (n <= 1 || end_bit <= begin_bit) return keys;
  return radix_sort_impl(KeySrc{keys}, tmp, keys, n, begin_bit, end_bit, s);
}

uint64_t *radix_sort_edges(const uint32_t *src, const uint32_t *dst, uint64_t M, uint32_t nv, int bits,
                           uint64_t sentinel, uint64_t *buf0, uint64_t *buf1, unsigned *err, cudaStream_t s) {
  if (M == 0) return buf0;
  return radix_sort_impl(EdgeSrc{src, dst, nv, bits, sentinel, err}, buf0, buf1, M, 0, 2 * bits, s);
}

}  // namespace tc
