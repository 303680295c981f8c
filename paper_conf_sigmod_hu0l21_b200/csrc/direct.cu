// direct.cu — steps a4-a5: edge directing (Algorithm 1).
//
// Every rule is expressed as a total order on vertices: u->v iff (prim[u], u) < (prim[v], v),
// so the directed graph has no 3-cycle by construction.
//   ID      prim = 0                         (id order)
//   DEGREE  prim = d(v)                      (degree order, ties by id, P:19 / Q11)
//   PAPER   prim = (subround << 32) | dsnap  (A-direction)
//
// A-direction, bulk-synchronous form of Algorithm 1.  Each frontier F (line 4-6, line 17)
// is exactly {unpeeled v : res(v) <= threshold}; all of F is peeled in one subround:
//   mark   : sub(v) = subround, dsnap(v) = res(v)   (snapshot at formation, Q7)
//   expand : for v in F, nbr unpeeled and not in F: res(nbr)-- (line 12-14); the decrement
//            that takes res(nbr) from threshold+1 to threshold appends nbr to the next
//            frontier exactly once (line 15-16, Q9)
//   edges inside F are ordered by (dsnap, id) (line 9-11, Q7), edges F->unpeeled go out of F
//   (line 12-13): both are the key order (sub, dsnap, id).
// The threshold is |E| 2^level / |V| compared exactly in integers (Q3/Q4); an empty frontier
// doubles it (line 19).  The sequential oracle (oracle/tc_oracle.c) and this BSP form yield
// the same orientation because decrements commute and dsnap is taken after the previous
// subround completes.
#include "internal.h"
#include "prims.cuh"

namespace tc {


namespace {

enum : uint8_t { V_UNPEELED = 0, V_FRONTIER = 1, V_PEELED = 2 };

__global__ void copy_deg_kernel(const uint32_t *__restrict__ deg, uint64_t *__restrict__ prim, uint32_t n) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    prim[i] = deg[i];
}

__global__ void sym_fill_kernel(const uint64_t *__restrict__ edges, uint64_t m, int bits,
                                unsigned long long *__restrict__ cursor, uint32_t *__restrict__ adj) {
  const uint64_t mask = (1ull << bits) - 1;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  // edges are sorted by u: lanes sharing u reserve their slots with ONE atomic per run
  for (uint64_t base = (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u); base < m; base += stride) {
    const uint64_t i = base + lane_id();
    const bool valid = i < m;
    const uint64_t k = valid ? edges[i] : 0;
    const uint32_t u = valid ? (uint32_t)(k >> bits) : 0xffffffffu, v = (uint32_t)(k & mask);
    const unsigned peers = __match_any_sync(0xffffffffu, u);
    const unsigned lead = __ffs(peers) - 1;
    unsigned long long pu = 0;
    if (valid && lane_id() == lead) pu = atomicAdd(&cursor[u], (unsigned long long)__popc(peers));
    pu = __shfl_sync(0xffffffffu, pu, lead) + __popc(peers & ((1u << lane_id()) - 1u));
    if (valid) {
      adj[pu] = v;
      adj[atomicAdd(&cursor[v], 1ull)] = u;
    }
  }
}

// Warp-aggregated append of `v` when `want` (warp-uniform control flow required).
__device__ __forceinline__ void warp_append(bool want, uint32_t v, uint32_t *list, unsigned *count) {
  unsigned mask = __ballot_sync(0xffffffffu, want);
  if (!mask) return;
  unsigned leader = __ffs(mask) - 1;
  unsigned base = 0;
  if (lane_id() == leader) base = atomicAdd(count, (unsigned)__popc(mask));
  base = __shfl_sync(0xffffffffu, base, leader);
  if (want) list[base + __popc(mask & ((1u << lane_id()) - 1u))] = v;
}

__global__ void frontier_init_kernel(const uint8_t *__restrict__ state, const uint32_t *__restrict__ res,
                                     uint32_t n, uint64_t thr, uint32_t *F, unsigned *nf) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t base = (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u); base < n; base += stride) {
    uint64_t v = base + lane_id();
    bool want = v < n && state[v] == V_UNPEELED && (uint64_t)res[v] <= thr;
    warp_append(want, (uint32_t)v, F, nf);
  }
}

// Marks the frontier (snapshot at formation) and splits it by degree for the three expand
// kernels: d(v) <= 32 -> Fs (flattened, 32 vertices per warp), 32 < d(v) <= HUGE_DEG -> Fb
// (warp per vertex), d(v) > HUGE_DEG -> Fh (the whole grid per vertex: a hub never
// serialises on one warp).  Vertices with d(v) = 0 have nothing to expand.
constexpr uint32_t HUGE_DEG = 4096;
__global__ void mark_kernel(const uint32_t *__restrict__ F, unsigned nf, uint8_t *state,
                            const uint32_t *__restrict__ res, const uint32_t *__restrict__ deg, uint32_t *sub,
                            uint32_t *dsnap, uint32_t r, uint32_t *Fs, uint32_t *Fb, uint32_t *Fh,
                            unsigned *cnt_sb) {
  for (unsigned base = blockIdx.x * blockDim.x + (threadIdx.x & ~31u); base < nf; base += gridDim.x * blockDim.x) {
    const unsigned i = base + lane_id();
    uint32_t v = 0, d = 0;
    if (i < nf) {
      v = F[i];
      state[v] = V_FRONTIER;
      sub[v] = r;
      dsnap[v] = res[v];
      d = deg[v];
    }
    warp_append(i < nf && d != 0 && d <= 32, v, Fs, cnt_sb);
    warp_append(i < nf && d > 32 && d <= HUGE_DEG, v, Fb, cnt_sb + 1);
    warp_append(i < nf && d > HUGE_DEG, v, Fh, cnt_sb + 2);
  }
}

// Decrement of one incident edge (v, nbr) of a frontier vertex (Algorithm 1 line 12-16).
__device__ __forceinline__ bool expand_one(uint32_t nbr, const uint8_t *__restrict__ state, uint32_t *res,
                                           uint64_t thr) {
  if (state[nbr] != V_UNPEELED) return false;
  const uint32_t old = atomicSub(&res[nbr], 1u);
  return (uint64_t)old == thr + 1;
}

// Frontier vertices with d(v) <= 32, 32 per warp: their adjacency lists are flattened
// (warp inclusive scan of the degrees) so every lane handles one incident edge per step;
// the owner of flattened element j is found by a 5-step search over the scan in registers.
__global__ void expand_flat_kernel(const uint32_t *__restrict__ F, const unsigned *__restrict__ nfp,
                                   const uint64_t *__restrict__ soffs, const uint32_t *__restrict__ sadj,
                                   const uint8_t *__restrict__ state, uint32_t *res, uint64_t thr, uint32_t *next,
                                   unsigned *nnext) {
  const unsigned nf = *nfp;
  const unsigned warps = gridDim.x * (blockDim.x / 32);
  const unsigned lane = lane_id();
  for (unsigned g0 = (blockIdx.x * (blockDim.x / 32) + warp_id()) * 32; g0 < nf; g0 += warps * 32) {
    uint64_t a = 0;
    uint32_t d = 0;
    if (g0 + lane < nf) {
      const uint32_t v = F[g0 + lane];
      a = soffs[v];
      d = (uint32_t)(soffs[v + 1] - a);
    }
    const uint32_t inc = warp_inclusive_scan(d);
    const uint32_t total = __shfl_sync(0xffffffffu, inc, 31);
    for (uint32_t j0 = 0; j0 < total; j0 += 32) {
      const uint32_t j = j0 + lane;
      // owner o = number of lanes whose inclusive prefix is <= j (binary search over lanes)
      uint32_t o = 0;
#pragma unroll
      for (int k = 4; k >= 0; --k) {
        const uint32_t q = o + (1u << k);
        const uint32_t pq = __shfl_sync(0xffffffffu, inc, (q - 1) & 31);
        if (q <= 32 && pq <= j) o = q;
      }
      const uint32_t oo = o & 31;
      const uint64_t ao = __shfl_sync(0xffffffffu, a, oo);
      const uint32_t eo = __shfl_sync(0xffffffffu, inc, oo) - __shfl_sync(0xffffffffu, d, oo);
      bool cross = false;
      uint32_t nbr = 0;
      if (j < total) {
        nbr = sadj[ao + (j - eo)];
        cross = expand_one(nbr, state, res, thr);
      }
      warp_append(cross, nbr, next, nnext);
    }
  }
}

// Frontier vertices with d(v) > 32: one warp per vertex; lanes stride over N(v).
__global__ void expand_kernel(const uint32_t *__restrict__ F, const unsigned *__restrict__ nfp,
                              const uint64_t *__restrict__ soffs,
                              const uint32_t *__restrict__ sadj, const uint8_t *__restrict__ state,
                              uint32_t *res, uint64_t thr, uint32_t *next, unsigned *nnext) {
  const unsigned nf = *nfp;
  unsigned warps = gridDim.x * (blockDim.x / 32);
  for (unsigned i = blockIdx.x * (blockDim.x / 32) + warp_id(); i < nf; i += warps) {
    uint32_t v = F[i];
    uint64_t a = soffs[v], e = soffs[v + 1];
    for (uint64_t p0 = a; p0 < e; p0 += 32) {
      uint64_t p = p0 + lane_id();
      bool cross = false;
      uint32_t nbr = 0;
      if (p < e) {
        nbr = sadj[p];
        cross = expand_one(nbr, state, res, thr);
      }
      warp_append(cross, nbr, next, nnext);
    }
  }
}

// Frontier hubs (d(v) > HUGE_DEG), one after another, each spread over every thread of
// the grid; the appends stay warp-aggregated.
__global__ void expand_huge_kernel(const uint32_t *__restrict__ F, const unsigned *__restrict__ nfp,
                                   const uint64_t *__restrict__ soffs, const uint32_t *__restrict__ sadj,
                                   const uint8_t *__restrict__ state, uint32_t *res, uint64_t thr, uint32_t *next,
                                   unsigned *nnext) {
  const unsigned nf = *nfp;
  const uint64_t nthreads = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t tid0 = (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u);
  for (unsigned i = 0; i < nf; ++i) {
    const uint32_t v = F[i];
    const uint64_t a = soffs[v], e = soffs[v + 1];
    for (uint64_t p0 = a + tid0; p0 < e; p0 += nthreads) {
      const uint64_t p = p0 + lane_id();
      bool cross = false;
      uint32_t nbr = 0;
      if (p < e) {
        nbr = sadj[p];
        cross = expand_one(nbr, state, res, thr);
      }
      warp_append(cross, nbr, next, nnext);
    }
  }
}

__global__ void peel_kernel(const uint32_t *__restrict__ F, unsigned nf, uint8_t *state) {
  for (unsigned i = blockIdx.x * blockDim.x + threadIdx.x; i < nf; i += gridDim.x * blockDim.x)
    state[F[i]] = V_PEELED;
}

__global__ void prim_paper_kernel(const uint32_t *__restrict__ sub, const uint32_t *__restrict__ dsnap,
                                  uint64_t *__restrict__ prim, uint32_t n) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    prim[i] = ((uint64_t)sub[i] << 32) | dsnap[i];
}

// d~(src)++ for every edge, src = the endpoint earlier in the (prim, id) order.
__global__ void outdeg_kernel(const uint64_t *__restrict__ edges, uint64_t m, int bits,
                              const uint64_t *__restrict__ prim, uint32_t *__restrict__ od) {
  uint64_t mask = (1ull << bits) - 1;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t k = edges[i];
    uint32_t u = (uint32_t)(k >> bits), v = (uint32_t)(k & mask);  // u < v
    uint32_t s = prim[u] <= prim[v] ? u : v;
    atomicAdd(&od[s], 1u);
  }
}

__global__ void od_from_offs_kernel(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ perm, uint32_t n,
                                    uint32_t *__restrict__ od) {
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t p = perm ? perm[v] : (uint32_t)v;
    od[v] = (uint32_t)(offs[p + 1] - offs[p]);
  }
}

// Eq.1 numerator Σ_u |n d~(u) - m| in 128-bit, one partial per block.
__global__ void eq1_kernel(const uint32_t *__restrict__ od, uint32_t n, uint64_t m, unsigned long long *partials) {
  unsigned __int128 acc = 0;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    unsigned __int128 a = (unsigned __int128)n * od[i];
    acc += a >= m ? a - m : (unsigned __int128)m - a;
  }
  __shared__ unsigned long long s_lo[256], s_hi[256];
  s_lo[threadIdx.x] = (unsigned long long)acc;
  s_hi[threadIdx.x] = (unsigned long long)(acc >> 64);
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned __int128 t = 0;
    for (int i = 0; i < (int)blockDim.x; ++i) t += ((unsigned __int128)s_hi[i] << 64) | s_lo[i];
    partials[2 * blockIdx.x] = (unsigned long long)t;
    partials[2 * blockIdx.x + 1] = (unsigned long long)(t >> 64);
  }
}

void peel_paper(Graph &g) {
  cudaStream_t s = g.stream;
  const uint32_t n = g.n;
  const uint64_t m = g.m;
  // symmetric adjacency N(v) (unsorted lists suffice for peeling)
  DevBuf<uint64_t> soffs;
  soffs.alloc((uint64_t)n + 1, s);
  scan_u32_to_u64(g.deg.get(), soffs.get(), n, s);
  DevBuf<uint32_t> sadj;
  sadj.alloc(2 * m + 1, s);
  {
    DevBuf<unsigned long long> cursor;
    cursor.alloc(n ? n : 1, s);
    TC_CUDA(cudaMemcpyAsync(cursor.get(), soffs.get(), sizeof(uint64_t) * n, cudaMemcpyDeviceToDevice, s));
    if (m) {
      ProfScope prof("sym_fill", s, 8.0 * m + 24.0 * m);
      sym_fill_kernel<<<grid_for(m, 256), 256, 0, s>>>(g.edges.get(), m, g.bits, cursor.get(), sadj.get());
      TC_LAUNCH_CHECK();
    }
  }
  DevBuf<uint32_t> res, F, next, Fs, Fb, Fh;
  DevBuf<uint8_t> state;
  DevBuf<unsigned> counters;  // [0] |F| being built, [1] |next|, [2] |Fs|, [3] |Fb|, [4] |Fh|
  res.alloc(n ? n : 1, s);
  F.alloc(n ? n : 1, s);
  next.alloc(n ? n : 1, s);
  Fs.alloc(n ? n : 1, s);
  Fb.alloc(n ? n : 1, s);
  Fh.alloc(n ? n : 1, s);
  state.alloc(n ? n : 1, s);
  counters.alloc(5, s);
  g.sub.alloc(n ? n : 1, s);
  g.dsnap.alloc(n ? n : 1, s);
  TC_CUDA(cudaMemcpyAsync(res.get(), g.deg.get(), sizeof(uint32_t) * n, cudaMemcpyDeviceToDevice, s));
  TC_CUDA(cudaMemsetAsync(state.get(), 0, n, s));
  // pinned frontier counters, allocated once per host thread (cudaMallocHost is slow)
  static thread_local unsigned *h_cnt = nullptr;
  if (!h_cnt) TC_CUDA(cudaMallocHost(&h_cnt, 2 * sizeof(unsigned)));
  uint64_t peeled = 0;
  uint32_t level = 0, r = 0;
  ProfScope prof("peel", s, 0.0);
  try {
    while (peeled < n) {
      unsigned __int128 num = (unsigned __int128)m << level;
      unsigned __int128 t128 = num / n;
      uint64_t thr = t128 > 0xFFFFFFFFull ? 0xFFFFFFFFull : (uint64_t)t128;
      TC_CUDA(cudaMemsetAsync(counters.get(), 0, 2 * sizeof(unsigned), s));
      frontier_init_kernel<<<grid_for(n, 256), 256, 0, s>>>(state.get(), res.get(), n, thr, F.get(), counters.get());
      TC_LAUNCH_CHECK();
      TC_CUDA(cudaMemcpyAsync(h_cnt, counters.get(), sizeof(unsigned), cudaMemcpyDeviceToHost, s));
      TC_CUDA(cudaStreamSynchronize(s));
      unsigned nf = h_cnt[0];
      while (nf > 0) {
        TC_CUDA(cudaMemsetAsync(counters.get() + 1, 0, 4 * sizeof(unsigned), s));
        mark_kernel<<<grid_for(nf, 256), 256, 0, s>>>(F.get(), nf, state.get(), res.get(), g.deg.get(), g.sub.get(),
                                                      g.dsnap.get(), r, Fs.get(), Fb.get(), Fh.get(),
                                                      counters.get() + 2);
        TC_LAUNCH_CHECK();
        // |Fs| and |Fb| stay on the device: both expands size their grids from nf
        expand_flat_kernel<<<grid_for(((uint64_t)nf + 31) / 32 * 32, 256), 256, 0, s>>>(
            Fs.get(), counters.get() + 2, soffs.get(), sadj.get(), state.get(), res.get(), thr, next.get(),
            counters.get() + 1);
        TC_LAUNCH_CHECK();
        expand_kernel<<<grid_for((uint64_t)nf * 32, 256), 256, 0, s>>>(Fb.get(), counters.get() + 3, soffs.get(),
                                                                       sadj.get(), state.get(), res.get(), thr,
                                                                       next.get(), counters.get() + 1);
        TC_LAUNCH_CHECK();
        expand_huge_kernel<<<num_sms() * 4, 256, 0, s>>>(Fh.get(), counters.get() + 4, soffs.get(), sadj.get(),
                                                         state.get(), res.get(), thr, next.get(), counters.get() + 1);
        TC_LAUNCH_CHECK();
        peel_kernel<<<grid_for(nf, 256), 256, 0, s>>>(F.get(), nf, state.get());
        TC_LAUNCH_CHECK();
        TC_CUDA(cudaMemcpyAsync(h_cnt + 1, counters.get() + 1, sizeof(unsigned), cudaMemcpyDeviceToHost, s));
        TC_CUDA(cudaStreamSynchronize(s));
        peeled += nf;
        ++r;
        F.swap(next);
        nf = h_cnt[1];
      }
      ++level;
      TC_REQUIRE(level < 200, ST_CUDA, "A-direction did not terminate");
    }
  } catch (...) {
    throw;
  }
  g.levels = level;
  g.subrounds = r;
  prim_paper_kernel<<<grid_for(n, 256), 256, 0, s>>>(g.sub.get(), g.dsnap.get(), g.prim.get(), n);
  TC_LAUNCH_CHECK();
}

}  // namespace

void direct_graph(Graph &g, int rule) {
  cudaStream_t s = g.stream;
  const uint32_t n = g.n;
  g.prim.alloc(n ? n : 1, s);
  g.sub.release();
  g.dsnap.release();
  g.levels = g.subrounds = 0;
  if (rule == TC_DIRECT_ID) {
    TC_CUDA(cudaMemsetAsync(g.prim.get(), 0, g.prim.bytes(), s));
  } else if (rule == TC_DIRECT_DEGREE) {
    if (n) copy_deg_kernel<<<grid_for(n, 256), 256, 0, s>>>(g.deg.get(), g.prim.get(), n);
    TC_LAUNCH_CHECK();
  } else {
    peel_paper(g);
  }
  g.od.release();
  g.od_ready = false;  // computed on demand (ensure_od): not needed by NONE ordering
  g.direct_rule = rule;
  g.reorder_rule = -1;
  g.identity_perm = true;
  g.perm.release();
  g.bucket_off.release();
  g.h_bucket_off.clear();
  g.eq3 = -1;
  g.offs.release();
  g.col.release();
  g.csr_mem.release();
  g.csr_ready = false;
  g.state = G_DIRECTED;
}

void ensure_od(Graph &g) {
  if (g.od_ready) return;
  cudaStream_t s = g.stream;
  const uint32_t n = g.n;
  g.od.alloc(n ? n : 1, s);
  if (g.csr_ready) {  // d~ = list lengths of the oriented CSR
    if (n) {
      od_from_offs_kernel<<<grid_for(n, 256), 256, 0, s>>>(g.offs.get(), g.identity_perm ? nullptr : g.perm.get(), n,
                                                           g.od.get());
      TC_LAUNCH_CHECK();
    }
  } else {
    TC_CUDA(cudaMemsetAsync(g.od.get(), 0, g.od.bytes(), s));
    if (g.m) {
      ProfScope prof("outdeg", s, 8.0 * g.m + 16.0 * g.m);
      outdeg_kernel<<<grid_for(g.m, 256), 256, 0, s>>>(g.edges.get(), g.m, g.bits, g.prim.get(), g.od.get());
      TC_LAUNCH_CHECK();
    }
  }
  g.max_outdeg = device_max_u32(g.od.get(), n, s);
  // Eq.1 statistic
  unsigned blocks = grid_for(n, 256, 2);
  DevBuf<unsigned long long> part;
  part.alloc(2 * blocks, s);
  eq1_kernel<<<blocks, 256, 0, s>>>(g.od.get(), n, g.m, part.get());
  TC_LAUNCH_CHECK();
  std::vector<unsigned long long> h(2 * blocks);
  TC_CUDA(cudaMemcpyAsync(h.data(), part.get(), part.bytes(), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  unsigned __int128 t = 0;
  for (unsigned i = 0; i < blocks; ++i) t += ((unsigned __int128)h[2 * i + 1] << 64) | h[2 * i];
  g.eq1_lo = (uint64_t)t;
  g.eq1_hi = (uint64_t)(t >> 64);
  g.od_ready = true;
}

}  // namespace tc
