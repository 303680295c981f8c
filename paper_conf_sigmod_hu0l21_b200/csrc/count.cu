// count.cu — steps a8-a10: schedule and binary-search intersection count (the hot loop).
//
// T = Σ_u Σ_{v ∈ N+(u)} |N+(u) ∩ N+(v)| on the oriented CSR (every triangle once, at its
// source).  The computing pattern is the paper's "copy-synchronize-search"
// (Hu's fine-grained method): N+(u) is staged in shared memory, then every wedge
// u->v->w (w ∈ N+(v)) is checked by a binary search for w in the staged N+(u)
// (binary-search list intersection).  B200 mapping:
//
//  * warp per source vertex u (d~(u) < SMALL_CAP): N+(u) in a per-warp shared-memory slice;
//    the wedges of 32 consecutive v's are flattened (warp inclusive scan of d~(v)) so each
//    lane takes one wedge per step: coalesced reads of N+(v), a 5-step owner search and a
//    ceil(log2 d~(u))-step binary search in shared memory.  Work is fetched in chunks from
//    a degree-binned worklist (heaviest log2-bin first, cf. logarithmic radix binning P:63).
//  * CTA per source vertex u (d~(u) >= SMALL_CAP): N+(u) staged in pieces of PIECE elements
//    by a TMA bulk copy (cp.async.bulk + mbarrier), all warps stream the N+(v) lists against
//    the piece (the piece of Hu's method).
//  * RANGE schedule: CTA i takes the k consecutive labels of bucket i (the block model of
//    P:182-186 that A-order optimises); each warp takes vertices of its bucket round-robin;
//    lists too long for a warp slice are searched in global memory.
//  * counts: u32 per lane per task, u64 per warp, block reduction, ONE 64-bit atomic per CTA.
//  * per-vertex t(v): +1 at w and v per match (global atomics), warp total at u.
#include <algorithm>
#include <vector>

#include "internal.h"
#include "prims.cuh"

namespace tc {

int g_opt_small_cap = 1024;  // power of two

namespace {

constexpr int CT_THREADS = 256;       // small / range kernels: 8 warps
constexpr int CT_WARPS = CT_THREADS / 32;
constexpr int LG_THREADS = 512;       // large kernel: 16 warps
constexpr int LG_WARPS = LG_THREADS / 32;
constexpr uint32_t PIECE = 16384;     // large kernel: N+(u) piece in shared memory (64 KB)
constexpr uint32_t CHUNK = 8;         // worklist entries per atomic fetch

struct WarpScratch {  // per-warp owner-search tables for one 32-v chunk
  uint64_t vb[32];
  uint32_t pre[32];
  uint32_t v[32];
};

__device__ __forceinline__ uint32_t ldg_u32(const uint32_t *p) { return __ldg(p); }

// Branchless search: does `w` occur in the ascending list s[0..L), L >= 1?
__device__ __forceinline__ bool bsearch_list(const uint32_t *s, uint32_t L, uint32_t w) {
  const uint32_t *p = s;
  uint32_t len = L;
  while (len > 1) {
    uint32_t h = len >> 1;
    p = (p[h] <= w) ? p + h : p;
    len -= h;
  }
  return *p == w;
}

// Count the wedges u->v->w of one chunk of up to 32 v's (lane-held `v`, `valid`) whose
// w lies in list[0..L) (w restricted to [lo, hi]).  Returns this lane's matches.
template <bool PV>
__device__ __forceinline__ uint32_t warp_chunk(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col,
                                               uint32_t v, bool valid, const uint32_t *list, uint32_t L, uint32_t lo,
                                               uint32_t hi, WarpScratch &ws, unsigned long long *tv) {
  const unsigned lane = lane_id();
  uint64_t vb = 0;
  uint32_t dv = 0;
  if (valid) {
    vb = offs[v];
    dv = (uint32_t)(offs[v + 1] - vb);
  }
  uint32_t inc = warp_inclusive_scan(dv);
  uint32_t total = __shfl_sync(0xffffffffu, inc, 31);
  ws.vb[lane] = vb;
  ws.pre[lane] = inc;
  if (PV) ws.v[lane] = v;
  __syncwarp();
  uint32_t cnt = 0;
  for (uint32_t j = lane; j < total; j += 32) {
    uint32_t o = 0;
#pragma unroll
    for (uint32_t step = 16; step; step >>= 1) o = (ws.pre[o + step - 1] <= j) ? o + step : o;
    uint32_t excl = o ? ws.pre[o - 1] : 0u;
    uint32_t w = ldg_u32(col + ws.vb[o] + (j - excl));
    if (w >= lo && w <= hi && bsearch_list(list, L, w)) {
      ++cnt;
      if (PV) {
        atomicAdd(&tv[w], 1ull);
        atomicAdd(&tv[ws.v[o]], 1ull);
      }
    }
  }
  __syncwarp();
  return cnt;
}

// Process source vertex u with one warp; list = shared slice (SMEM) or global N+(u).
template <bool PV>
__device__ __forceinline__ uint64_t warp_vertex(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col,
                                                uint32_t u, uint32_t *slice, uint32_t cap, WarpScratch &ws,
                                                unsigned long long *tv) {
  const unsigned lane = lane_id();
  const uint64_t a = offs[u];
  const uint32_t L = (uint32_t)(offs[u + 1] - a);
  if (L < 2) return 0;
  const uint32_t *list;
  if (L <= cap) {
    for (uint32_t j = lane; j < L; j += 32) slice[j] = ldg_u32(col + a + j);
    __syncwarp();
    list = slice;
  } else {
    list = col + a;
  }
  const uint32_t lo = list[0], hi = list[L - 1];
  uint32_t cnt = 0;
  for (uint32_t c0 = 0; c0 < L; c0 += 32) {
    bool valid = c0 + lane < L;
    uint32_t v = valid ? list[c0 + lane] : 0u;
    cnt += warp_chunk<PV>(offs, col, v, valid, list, L, lo, hi, ws, tv);
  }
  __syncwarp();
  uint64_t c = cnt;
  if (PV) {
    uint64_t tot = warp_sum(c);
    if (lane == 0 && tot) atomicAdd(&tv[u], (unsigned long long)tot);
  }
  return c;
}

__device__ __forceinline__ void block_add_u64(uint64_t v, unsigned long long *T) {
  __shared__ unsigned long long s_part[32];
  v = warp_sum(v);
  if (lane_id() == 0) s_part[warp_id()] = v;
  __syncthreads();
  if (warp_id() == 0) {
    unsigned nw = blockDim.x / 32;
    uint64_t x = lane_id() < nw ? s_part[lane_id()] : 0;
    x = warp_sum(x);
    if (lane_id() == 0 && x) atomicAdd(T, (unsigned long long)x);
  }
}

// --------------------------------------------------------------- schedule (a8)
__device__ __forceinline__ int deg_bin(uint32_t d) { return 31 - __clz(d); }  // floor(log2 d), d >= 1

__global__ void bin_hist_kernel(const uint64_t *__restrict__ offs, uint32_t ub, uint32_t ue, unsigned *hist) {
  __shared__ unsigned s_h[32];
  if (threadIdx.x < 32) s_h[threadIdx.x] = 0;
  __syncthreads();
  for (uint64_t u = (uint64_t)ub + blockIdx.x * blockDim.x + threadIdx.x; u < ue; u += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t d = (uint32_t)(offs[u + 1] - offs[u]);
    if (d >= 2) atomicAdd(&s_h[deg_bin(d)], 1u);
  }
  __syncthreads();
  if (threadIdx.x < 32 && s_h[threadIdx.x]) atomicAdd(&hist[threadIdx.x], s_h[threadIdx.x]);
}

// cursor[bin] = start of bin in the worklist, bins in DESCENDING order (heaviest first)
__global__ void bin_scan_kernel(const unsigned *hist, unsigned *cursor) {
  unsigned lane = threadIdx.x;  // 32 threads; lane = 31 - bin
  unsigned c = hist[31 - lane];
  unsigned inc = warp_inclusive_scan(c);
  cursor[31 - lane] = inc - c;
}

__global__ void bin_scatter_kernel(const uint64_t *__restrict__ offs, uint32_t ub, uint32_t ue, unsigned *cursor,
                                   uint32_t *__restrict__ work) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t base = (uint64_t)ub + blockIdx.x * blockDim.x + (threadIdx.x & ~31u); base < ue; base += stride) {
    uint64_t u = base + lane_id();
    uint32_t d = u < ue ? (uint32_t)(offs[u + 1] - offs[u]) : 0u;
    int bin = d >= 2 ? deg_bin(d) : -1;
    unsigned peers = __match_any_sync(0xffffffffu, bin);
    unsigned leader = __ffs(peers) - 1;
    unsigned pos = 0;
    if (bin >= 0 && lane_id() == leader) pos = atomicAdd(&cursor[bin], (unsigned)__popc(peers));
    pos = __shfl_sync(0xffffffffu, pos, leader);
    if (bin >= 0) work[pos + __popc(peers & ((1u << lane_id()) - 1u))] = (uint32_t)u;
  }
}

// --------------------------------------------------------------- count kernels (a9)
template <bool PV>
__global__ __launch_bounds__(CT_THREADS) void count_small_kernel(const uint64_t *__restrict__ offs,
                                                                 const uint32_t *__restrict__ col,
                                                                 const uint32_t *__restrict__ work, uint32_t nwork,
                                                                 unsigned *work_ctr, uint32_t cap,
                                                                 unsigned long long *T, unsigned long long *tv) {
  extern __shared__ uint32_t s_dyn[];
  __shared__ WarpScratch s_ws[CT_WARPS];
  uint32_t *slice = s_dyn + warp_id() * cap;
  WarpScratch &ws = s_ws[warp_id()];
  uint64_t acc = 0;
  while (true) {
    unsigned base = 0;
    if (lane_id() == 0) base = atomicAdd(work_ctr, CHUNK);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (base >= nwork) break;
    unsigned end = min(base + CHUNK, nwork);
    for (unsigned i = base; i < end; ++i) acc += warp_vertex<PV>(offs, col, work[i], slice, cap, ws, tv);
  }
  block_add_u64(acc, T);
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
  unsigned a = (unsigned)__cvta_generic_to_shared(bar);
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, unsigned bytes) {
  unsigned a = (unsigned)__cvta_generic_to_shared(bar);
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(a), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_bulk_g2s(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
  unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  unsigned b = (unsigned)__cvta_generic_to_shared(bar);
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(d),
               "l"(src), "r"(bytes), "r"(b)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, unsigned phase) {
  unsigned a = (unsigned)__cvta_generic_to_shared(bar);
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(a),
      "r"(phase)
      : "memory");
}

// CTA per heavy source vertex; N+(u) staged piece by piece with a TMA bulk copy.
template <bool PV>
__global__ __launch_bounds__(LG_THREADS) void count_large_kernel(const uint64_t *__restrict__ offs,
                                                                 const uint32_t *__restrict__ col,
                                                                 const uint32_t *__restrict__ work, uint32_t nwork,
                                                                 unsigned *work_ctr, unsigned long long *T,
                                                                 unsigned long long *tv) {
  extern __shared__ __align__(128) uint32_t s_piece[];  // PIECE + 8 words (alignment slack)
  __shared__ WarpScratch s_ws[LG_WARPS];
  __shared__ __align__(8) uint64_t s_bar;
  __shared__ unsigned s_item;
  WarpScratch &ws = s_ws[warp_id()];
  if (threadIdx.x == 0) mbar_init(&s_bar, 1);
  __syncthreads();
  unsigned phase = 0;
  uint64_t acc = 0;
  while (true) {
    if (threadIdx.x == 0) s_item = atomicAdd(work_ctr, 1u);
    __syncthreads();
    unsigned item = s_item;
    __syncthreads();
    if (item >= nwork) break;
    const uint32_t u = work[item];
    const uint64_t a = offs[u];
    const uint32_t L = (uint32_t)(offs[u + 1] - a);
    uint64_t ucnt = 0;
    for (uint32_t p0 = 0; p0 < L; p0 += PIECE) {
      const uint32_t plen = min(PIECE, L - p0);
      // 16-byte aligned bulk copy covering col[a+p0, a+p0+plen)
      const uint64_t first = a + p0;
      const uint64_t abeg = first & ~3ull;             // element index, 16 B aligned
      const uint64_t aend = (first + plen + 3) & ~3ull;
      const uint32_t shift = (uint32_t)(first - abeg);
      if (threadIdx.x == 0) {
        unsigned bytes = (unsigned)((aend - abeg) * 4);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // prior generic reads of the piece
        mbar_expect_tx(&s_bar, bytes);
        tma_bulk_g2s(s_piece, col + abeg, bytes, &s_bar);
      }
      mbar_wait(&s_bar, phase);
      phase ^= 1u;
      const uint32_t *list = s_piece + shift;
      const uint32_t lo = list[0], hi = list[plen - 1];
      uint32_t cnt = 0;
      for (uint32_t c0 = warp_id() * 32; c0 < L; c0 += LG_THREADS) {
        bool valid = c0 + lane_id() < L;
        uint32_t v = valid ? ldg_u32(col + a + c0 + lane_id()) : 0u;
        cnt += warp_chunk<PV>(offs, col, v, valid, list, plen, lo, hi, ws, tv);
      }
      ucnt += cnt;
      __syncthreads();  // piece fully consumed before the next bulk copy overwrites it
    }
    acc += ucnt;
    if (PV) {
      uint64_t tot = warp_sum(ucnt);
      if (lane_id() == 0 && tot) atomicAdd(&tv[u], (unsigned long long)tot);
    }
  }
  block_add_u64(acc, T);
}

// RANGE schedule: CTA per bucket of consecutive labels [boff[i], boff[i+1]) ∩ [ub, ue).
template <bool PV>
__global__ __launch_bounds__(CT_THREADS) void count_range_kernel(const uint64_t *__restrict__ offs,
                                                                 const uint32_t *__restrict__ col,
                                                                 const uint32_t *__restrict__ boff, uint32_t kfixed,
                                                                 uint32_t b0, uint32_t nb, uint32_t ub, uint32_t ue,
                                                                 uint32_t cap, unsigned long long *T,
                                                                 unsigned long long *tv) {
  extern __shared__ uint32_t s_dyn[];
  __shared__ WarpScratch s_ws[CT_WARPS];
  uint32_t *slice = s_dyn + warp_id() * cap;
  WarpScratch &ws = s_ws[warp_id()];
  uint64_t acc = 0;
  for (uint32_t bi = b0 + blockIdx.x; bi < b0 + nb; bi += gridDim.x) {
    uint64_t s0 = boff ? boff[bi] : (uint64_t)bi * kfixed;
    uint64_t s1 = boff ? boff[bi + 1] : (uint64_t)(bi + 1) * kfixed;
    if (s0 < ub) s0 = ub;
    if (s1 > ue) s1 = ue;
    for (uint64_t u = s0 + warp_id(); u < s1; u += CT_WARPS)
      acc += warp_vertex<PV>(offs, col, (uint32_t)u, slice, cap, ws, tv);
  }
  block_add_u64(acc, T);
}

__global__ void gather_tv_kernel(const unsigned long long *__restrict__ tnew, const uint32_t *__restrict__ perm,
                                 uint32_t n, uint64_t *__restrict__ out) {
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
    out[v] = tnew[perm ? perm[v] : v];
}

// --------------------------------------------------------------- work model / analysis
// w(u) = d~(u) + Σ_{v ∈ N+(u)} d~(v); sectors: 32-B sectors the Hu pattern touches with no reuse.
__global__ void work_kernel(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col, uint32_t n,
                            uint64_t *__restrict__ w, unsigned long long *sectors) {
  uint64_t sec = 0;
  unsigned warps = gridDim.x * (blockDim.x / 32);
  for (uint64_t u = (uint64_t)blockIdx.x * (blockDim.x / 32) + warp_id(); u < n; u += warps) {
    uint64_t a = offs[u], e = offs[u + 1];
    uint64_t s = 0, sc = 0;
    for (uint64_t p = a + lane_id(); p < e; p += 32) {
      uint32_t v = col[p];
      uint64_t vb = offs[v], ve = offs[v + 1];
      s += ve - vb;
      // N+(v) list span + the offs pair
      if (ve > vb) sc += ((ve * 4 - 1) >> 5) - ((vb * 4) >> 5) + 1;
      sc += (((uint64_t)v * 8 + 15) >> 5) - (((uint64_t)v * 8) >> 5) + 1;
    }
    s = warp_sum(s);
    sc = warp_sum(sc);
    if (lane_id() == 0) {
      w[u] = s + (e - a);
      if (e - a >= 2) sec += sc + (((e * 4 - 1) >> 5) - ((a * 4) >> 5) + 1) + 1;
    }
  }
  if (lane_id() == 0 && sec && sectors) atomicAdd(sectors, (unsigned long long)sec);
}

__global__ void bounds_kernel(const uint64_t *__restrict__ pre, uint32_t n, uint32_t world, uint32_t *bounds) {
  // bounds[g] = first u with pre[u] >= g * total / world (pre = exclusive prefix, pre[n] = total)
  uint32_t g = blockIdx.x * blockDim.x + threadIdx.x;
  if (g > world) return;
  if (g == 0) { bounds[0] = 0; return; }
  if (g == world) { bounds[world] = n; return; }
  unsigned __int128 target128 = (unsigned __int128)pre[n] * g / world;
  uint64_t target = (uint64_t)target128;
  uint32_t lo = 0, hi = n;
  while (lo < hi) {
    uint32_t mid = lo + (hi - lo) / 2;
    if (pre[mid] < target) lo = mid + 1;
    else hi = mid;
  }
  bounds[g] = lo;
}

}  // namespace

static void configure_kernels() {
  static bool done = false;
  if (done) return;
  size_t large_smem = (PIECE + 8) * sizeof(uint32_t);
  TC_CUDA(cudaFuncSetAttribute(count_large_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)large_smem));
  TC_CUDA(cudaFuncSetAttribute(count_large_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)large_smem));
  int small_max = 200 * 1024;
  TC_CUDA(cudaFuncSetAttribute(count_small_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, small_max));
  TC_CUDA(cudaFuncSetAttribute(count_small_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, small_max));
  TC_CUDA(cudaFuncSetAttribute(count_range_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, small_max));
  TC_CUDA(cudaFuncSetAttribute(count_range_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, small_max));
  done = true;
}

static int occupancy(const void *fn, int threads, size_t smem) {
  int blocks = 0;
  TC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks, fn, threads, smem));
  return blocks > 0 ? blocks : 1;
}

uint64_t count_graph(Graph &g, uint32_t ub, uint32_t ue, uint64_t *d_tv, float *kernel_ms, uint64_t *launches) {
  cudaStream_t s = g.stream;
  configure_kernels();
  if (ue > g.n) ue = g.n;
  uint64_t nlaunch = 0;
  DevBuf<unsigned long long> dT;
  dT.alloc(1, s);
  TC_CUDA(cudaMemsetAsync(dT.get(), 0, sizeof(unsigned long long), s));
  unsigned long long *tv = reinterpret_cast<unsigned long long *>(d_tv);
  const uint32_t cap = (uint32_t)g_opt_small_cap;
  int sched = g.schedule;
  if (sched == TC_SCHED_AUTO) sched = (g.reorder_rule == TC_REORDER_PAPER) ? TC_SCHED_RANGE : TC_SCHED_BUCKETED;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  if (kernel_ms) {
    TC_CUDA(cudaEventCreate(&e0));
    TC_CUDA(cudaEventCreate(&e1));
  }
  if (ub < ue && g.m) {
    if (sched == TC_SCHED_RANGE) {
      const uint32_t *boff = nullptr;
      uint32_t k = 32, b0 = 0, nb = 0;
      if (!g.h_bucket_off.empty()) {
        boff = g.bucket_off.get();
        const auto &hb = g.h_bucket_off;
        uint32_t nbk = (uint32_t)hb.size() - 1;
        // buckets intersecting [ub, ue)
        b0 = (uint32_t)(std::upper_bound(hb.begin(), hb.end(), ub) - hb.begin());
        b0 = b0 ? b0 - 1 : 0;
        uint32_t b1 = (uint32_t)(std::lower_bound(hb.begin(), hb.end(), ue) - hb.begin());
        if (b1 > nbk) b1 = nbk;
        nb = b1 > b0 ? b1 - b0 : 0;
      } else {
        b0 = ub / k;
        nb = (ue + k - 1) / k - b0;
      }
      if (nb) {
        size_t smem = (size_t)CT_WARPS * cap * sizeof(uint32_t);
        int occ = occupancy(tv ? (const void *)count_range_kernel<true> : (const void *)count_range_kernel<false>,
                            CT_THREADS, smem);
        unsigned grid = (unsigned)std::min<uint64_t>(nb, (uint64_t)num_sms() * occ);
        if (kernel_ms) TC_CUDA(cudaEventRecord(e0, s));
        ProfScope prof("count_range", s, 0.0);
        if (tv)
          count_range_kernel<true><<<grid, CT_THREADS, smem, s>>>(g.offs.get(), g.col.get(), boff, k, b0, nb, ub, ue,
                                                                   cap, dT.get(), tv);
        else
          count_range_kernel<false><<<grid, CT_THREADS, smem, s>>>(g.offs.get(), g.col.get(), boff, k, b0, nb, ub, ue,
                                                                    cap, dT.get(), nullptr);
        TC_LAUNCH_CHECK();
        if (kernel_ms) TC_CUDA(cudaEventRecord(e1, s));
        ++nlaunch;
      }
    } else {
      // degree-binned worklist (heaviest bin first)
      DevBuf<unsigned> hist;  // [0..31] hist, [32..63] cursor, [64] small ctr, [65] large ctr
      hist.alloc(66, s);
      TC_CUDA(cudaMemsetAsync(hist.get(), 0, hist.bytes(), s));
      bin_hist_kernel<<<grid_for(ue - ub, 256, 4), 256, 0, s>>>(g.offs.get(), ub, ue, hist.get());
      TC_LAUNCH_CHECK();
      bin_scan_kernel<<<1, 32, 0, s>>>(hist.get(), hist.get() + 32);
      TC_LAUNCH_CHECK();
      std::vector<unsigned> hh(32);
      TC_CUDA(cudaMemcpyAsync(hh.data(), hist.get(), 32 * sizeof(unsigned), cudaMemcpyDeviceToHost, s));
      TC_CUDA(cudaStreamSynchronize(s));
      uint64_t nwork = 0, nlarge = 0;
      int capbin = 31 - __builtin_clz(cap);  // d < cap  <=>  bin < capbin
      for (int b = 0; b < 32; ++b) {
        nwork += hh[b];
        if (b >= capbin) nlarge += hh[b];
      }
      nlaunch += 3;
      if (nwork) {
        DevBuf<uint32_t> work;
        work.alloc(nwork, s);
        bin_scatter_kernel<<<grid_for(ue - ub, 256), 256, 0, s>>>(g.offs.get(), ub, ue, hist.get() + 32, work.get());
        TC_LAUNCH_CHECK();
        ++nlaunch;
        if (kernel_ms) TC_CUDA(cudaEventRecord(e0, s));
        if (nlarge) {
          size_t smem = (PIECE + 8) * sizeof(uint32_t);
          int occ = occupancy(tv ? (const void *)count_large_kernel<true> : (const void *)count_large_kernel<false>,
                              LG_THREADS, smem);
          unsigned grid = (unsigned)std::min<uint64_t>(nlarge, (uint64_t)num_sms() * occ);
          ProfScope prof("count_large", s, 0.0);
          if (tv)
            count_large_kernel<true><<<grid, LG_THREADS, smem, s>>>(g.offs.get(), g.col.get(), work.get(),
                                                                     (uint32_t)nlarge, hist.get() + 65, dT.get(), tv);
          else
            count_large_kernel<false><<<grid, LG_THREADS, smem, s>>>(g.offs.get(), g.col.get(), work.get(),
                                                                      (uint32_t)nlarge, hist.get() + 65, dT.get(),
                                                                      nullptr);
          TC_LAUNCH_CHECK();
          ++nlaunch;
        }
        uint64_t nsmall = nwork - nlarge;
        if (nsmall) {
          size_t smem = (size_t)CT_WARPS * cap * sizeof(uint32_t);
          int occ = occupancy(tv ? (const void *)count_small_kernel<true> : (const void *)count_small_kernel<false>,
                              CT_THREADS, smem);
          uint64_t want = (nsmall + CT_WARPS * CHUNK - 1) / (CT_WARPS * CHUNK);
          unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(want, (uint64_t)num_sms() * occ));
          ProfScope prof("count_small", s, 0.0);
          if (tv)
            count_small_kernel<true><<<grid, CT_THREADS, smem, s>>>(g.offs.get(), g.col.get(), work.get() + nlarge,
                                                                     (uint32_t)nsmall, hist.get() + 64, cap, dT.get(), tv);
          else
            count_small_kernel<false><<<grid, CT_THREADS, smem, s>>>(g.offs.get(), g.col.get(), work.get() + nlarge,
                                                                      (uint32_t)nsmall, hist.get() + 64, cap, dT.get(),
                                                                      nullptr);
          TC_LAUNCH_CHECK();
          ++nlaunch;
        }
        if (kernel_ms) TC_CUDA(cudaEventRecord(e1, s));
      }
    }
  }
  uint64_t hT = 0;
  TC_CUDA(cudaMemcpyAsync(&hT, dT.get(), sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  if (kernel_ms) {
    float ms = 0;
    if (cudaEventQuery(e1) == cudaSuccess && cudaEventElapsedTime(&ms, e0, e1) == cudaSuccess) *kernel_ms = ms;
    else { cudaGetLastError(); *kernel_ms = 0; }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
  }
  if (launches) *launches = nlaunch;
  return hT;
}

void gather_per_vertex(Graph &g, const uint64_t *d_tnew, uint64_t *d_out) {
  if (!g.n) return;
  gather_tv_kernel<<<grid_for(g.n, 256), 256, 0, g.stream>>>(reinterpret_cast<const unsigned long long *>(d_tnew),
                                                             g.identity_perm ? nullptr : g.perm.get(), g.n, d_out);
  TC_LAUNCH_CHECK();
}

void partition_graph(Graph &g, uint32_t world, uint32_t *bounds) {
  cudaStream_t s = g.stream;
  const uint32_t n = g.n;
  DevBuf<uint64_t> w, pre;
  DevBuf<uint32_t> db;
  w.alloc(n ? n : 1, s);
  pre.alloc((uint64_t)n + 1, s);
  db.alloc(world + 1, s);
  if (n) {
    work_kernel<<<grid_for((uint64_t)n * 32, 256), 256, 0, s>>>(g.offs.get(), g.col.get(), n, w.get(), nullptr);
    TC_LAUNCH_CHECK();
  }
  scan_u64(w.get(), pre.get(), n, s);
  bounds_kernel<<<1, 1024, 0, s>>>(pre.get(), n, world, db.get());
  TC_LAUNCH_CHECK();
  TC_CUDA(cudaMemcpyAsync(bounds, db.get(), sizeof(uint32_t) * (world + 1), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
}

void analyze_graph(Graph &g) {
  cudaStream_t s = g.stream;
  const uint32_t n = g.n;
  DevBuf<uint64_t> w, pre;
  DevBuf<unsigned long long> sec;
  w.alloc(n ? n : 1, s);
  pre.alloc((uint64_t)n + 1, s);
  sec.alloc(1, s);
  TC_CUDA(cudaMemsetAsync(sec.get(), 0, 8, s));
  if (n) {
    work_kernel<<<grid_for((uint64_t)n * 32, 256), 256, 0, s>>>(g.offs.get(), g.col.get(), n, w.get(), sec.get());
    TC_LAUNCH_CHECK();
  }
  scan_u64(w.get(), pre.get(), n, s);
  uint64_t tot = 0, hs = 0;
  TC_CUDA(cudaMemcpyAsync(&tot, pre.get() + n, 8, cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaMemcpyAsync(&hs, sec.get(), 8, cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  g.wedges = tot - g.m;
  g.alg_bytes = hs * 32;
}

}  // namespace tc
