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
#include <cooperative_groups.h>

#include "internal.h"
#include "prims.cuh"

namespace tc {

int g_opt_peel_coop = 1;  // whole A-direction peel in one cooperative launch
int g_opt_peel_red = -1;  // coop peel: decrements as RED + frontier scan (1), returning atomics (0), auto (-1)

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
// serialises on one warp; hubs are cut into chunks of HUB_CHUNK edges spread over all warps).
// Vertices with d(v) = 0 have nothing to expand.
constexpr uint32_t HUGE_DEG = 1024;
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
// RED = true (the cooperative peel): a fire-and-forget reduction (the warp does not wait
// for the returned value); the vertices that crossed the threshold are found afterwards by
// a scan of the unpeeled vertices (res <= thr), the same set as the crossing test below
template <bool RED = false>
__device__ __forceinline__ bool expand_one(uint32_t nbr, const uint8_t *__restrict__ state, uint32_t *res,
                                           uint64_t thr) {
  if (state[nbr] != V_UNPEELED) return false;
  if (RED) {
    atomicSub(&res[nbr], 1u);  // result unused: compiled to RED
    return false;
  }
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

// Frontier hubs (d(v) > HUGE_DEG): cut into chunks of HUB_CHUNK edges, one warp per chunk
// over the whole grid.  Every CTA builds the chunk prefix of the (few) hubs in shared
// memory and binary-searches it per chunk; with more than HUB_MAX hubs the hubs are taken
// one after another, each spread over every thread of the grid.  Called by whole CTAs.
constexpr uint32_t HUB_CHUNK = 1024, HUB_MAX = 8192;
template <bool RED = false>
__device__ __forceinline__ void expand_hubs(const uint32_t *__restrict__ F, unsigned nh,
                                            const uint64_t *__restrict__ soffs, const uint32_t *__restrict__ sadj,
                                            const uint8_t *__restrict__ state, uint32_t *res, uint64_t thr,
                                            uint32_t *next, unsigned *nnext, uint32_t *s_pre) {
  const unsigned lane = lane_id();
  const uint64_t gthreads = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t gtid0 = (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u);
  if (nh == 0) return;
  if (nh > HUB_MAX) {
    for (unsigned i = 0; i < nh; ++i) {
      const uint32_t v = F[i];
      const uint64_t a = soffs[v], e = soffs[v + 1];
      for (uint64_t p0 = a + gtid0; p0 < e; p0 += gthreads) {
        const uint64_t p = p0 + lane;
        bool cross = false;
        uint32_t nbr = 0;
        if (p < e) {
          nbr = sadj[p];
          cross = expand_one<RED>(nbr, state, res, thr);
        }
        warp_append(cross, nbr, next, nnext);
      }
    }
    return;
  }
  // inclusive prefix of chunk counts: thread t sums a contiguous run, block scan, write back
  __shared__ uint32_t s_tot[32];
  const unsigned per = (nh + blockDim.x - 1) / blockDim.x;
  const unsigned b0 = threadIdx.x * per, b1 = min(nh, b0 + per);
  uint32_t run = 0;
  for (unsigned i = b0; i < b1; ++i) {
    const uint32_t v = F[i];
    run += (uint32_t)((soffs[v + 1] - soffs[v] + HUB_CHUNK - 1) / HUB_CHUNK);
    s_pre[i] = run;
  }
  const uint32_t inc = warp_inclusive_scan(run);
  if (lane == 31) s_tot[warp_id()] = inc;
  __syncthreads();
  if (warp_id() == 0) {
    const unsigned nw = blockDim.x / 32;
    const uint32_t x = lane < nw ? s_tot[lane] : 0u;
    const uint32_t xi = warp_inclusive_scan(x);
    if (lane < nw) s_tot[lane] = xi - x;
  }
  __syncthreads();
  const uint32_t add = inc - run + s_tot[warp_id()];
  for (unsigned i = b0; i < b1; ++i) s_pre[i] += add;
  __syncthreads();
  const uint32_t total = s_pre[nh - 1];
  const unsigned nwarps = (unsigned)(gthreads >> 5);
  for (uint32_t c = (uint32_t)(gtid0 >> 5); c < total; c += nwarps) {
    unsigned lo = 0, hi = nh - 1;  // first i with s_pre[i] > c
    while (lo < hi) {
      const unsigned mid = (lo + hi) >> 1;
      if (s_pre[mid] > c) hi = mid;
      else lo = mid + 1;
    }
    const uint32_t ci = c - (lo ? s_pre[lo - 1] : 0u);
    const uint32_t v = F[lo];
    const uint64_t e = soffs[v + 1];
    const uint64_t a = soffs[v] + (uint64_t)ci * HUB_CHUNK;
    const uint64_t ce = min(e, a + HUB_CHUNK);
    for (uint64_t p0 = a; p0 < ce; p0 += 32) {
      const uint64_t p = p0 + lane;
      bool cross = false;
      uint32_t nbr = 0;
      if (p < ce) {
        nbr = sadj[p];
        cross = expand_one<RED>(nbr, state, res, thr);
      }
      warp_append(cross, nbr, next, nnext);
    }
  }
  __syncthreads();  // s_pre reusable
}

__global__ __launch_bounds__(256) void expand_huge_kernel(const uint32_t *__restrict__ F,
                                                          const unsigned *__restrict__ nfp,
                                                          const uint64_t *__restrict__ soffs,
                                                          const uint32_t *__restrict__ sadj,
                                                          const uint8_t *__restrict__ state, uint32_t *res,
                                                          uint64_t thr, uint32_t *next, unsigned *nnext) {
  __shared__ uint32_t s_pre[HUB_MAX];
  expand_hubs(F, *nfp, soffs, sadj, state, res, thr, next, nnext, s_pre);
}

// ---------------------------------------------------------------- whole peel, one launch
// The same BSP subrounds as the kernels above, run by ONE cooperative grid (every CTA
// resident) with grid-wide barriers between the phases: no host round trip per subround
// (the multi-launch loop paid a launch + a D2H copy + a stream sync per subround, ~30 per
// R-MAT s22 run).  Frontier counters are read by every thread after a barrier and reset by
// thread 0 one phase before their next use (double-buffered where a read and the next
// reset would otherwise race).
struct PeelArgs {
  const uint64_t *soffs;
  const uint32_t *sadj;
  const uint32_t *deg;
  uint32_t *res, *sub, *dsnap;
  uint8_t *state;
  uint32_t *F, *next, *Fs, *Fb, *Fh;
  unsigned *ctr;      // [0,1] init-frontier counts (per level parity), [2,3] next counts, [4..6] split counts
  uint32_t *out;      // [0] levels, [1] subrounds, [2] error
  uint32_t n;
  uint64_t m;
  int red;            // residual-degree decrements as RED + a scan for the next frontier
};

__global__ __launch_bounds__(256) void peel_coop_kernel(PeelArgs A) {
  namespace cg = cooperative_groups;
  __shared__ uint32_t s_pre[HUB_MAX];
  cg::grid_group grid = cg::this_grid();
  const uint64_t gtid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const uint64_t gthreads = (uint64_t)gridDim.x * blockDim.x;
  const unsigned gwarp = (unsigned)(gtid >> 5), nwarps = (unsigned)(gthreads >> 5);
  const unsigned lane = lane_id();
  const uint32_t n = A.n;
  uint64_t peeled = 0;
  uint32_t level = 0, r = 0;
  uint32_t *F = A.F, *next = A.next;
  while (peeled < n) {
    if (level >= 200) {  // cannot happen (thr reaches max degree after <= 64 levels)
      if (gtid == 0) A.out[2] = 1;
      break;
    }
    const unsigned __int128 t128 = ((unsigned __int128)A.m << level) / n;
    const uint64_t thr = t128 > 0xFFFFFFFFull ? 0xFFFFFFFFull : (uint64_t)t128;
    unsigned *cinit = A.ctr + (level & 1);
    // next level's init counter: idle now (last read as this level's predecessor's nf,
    // which every thread did before a grid.sync, or which was 0), and first appended to
    // after the grid.sync below, so the barrier orders this reset before its next use
    if (gtid == 0) A.ctr[(level + 1) & 1] = 0;
    // frontier formation (Algorithm 1 line 4-6)
    for (uint64_t base = gtid & ~31ull; base < n; base += gthreads) {
      const uint64_t v = base + lane;
      const bool want = v < n && A.state[v] == V_UNPEELED && (uint64_t)A.res[v] <= thr;
      warp_append(want, (uint32_t)v, F, cinit);
    }
    grid.sync();
    unsigned nf = *cinit;
    while (nf > 0) {
      unsigned *cnext = A.ctr + 2 + (r & 1);
      // mark + split by degree
      for (uint64_t base = gtid & ~31ull; base < nf; base += gthreads) {
        const uint64_t i = base + lane;
        uint32_t v = 0, d = 0;
        if (i < nf) {
          v = F[i];
          A.state[v] = V_FRONTIER;
          A.sub[v] = r;
          A.dsnap[v] = A.res[v];
          d = A.deg[v];
        }
        warp_append(i < nf && d != 0 && d <= 32, v, A.Fs, A.ctr + 4);
        warp_append(i < nf && d > 32 && d <= HUGE_DEG, v, A.Fb, A.ctr + 5);
        warp_append(i < nf && d > HUGE_DEG, v, A.Fh, A.ctr + 6);
      }
      grid.sync();
      const unsigned ns = A.ctr[4], nb = A.ctr[5], nh = A.ctr[6];
      // expand: d <= 32 flattened, 32 vertices per warp
      for (unsigned g0 = gwarp * 32; g0 < ns; g0 += nwarps * 32) {
        uint64_t a = 0;
        uint32_t d = 0;
        if (g0 + lane < ns) {
          const uint32_t v = A.Fs[g0 + lane];
          a = A.soffs[v];
          d = (uint32_t)(A.soffs[v + 1] - a);
        }
        const uint32_t inc = warp_inclusive_scan(d);
        const uint32_t total = __shfl_sync(0xffffffffu, inc, 31);
        for (uint32_t j0 = 0; j0 < total; j0 += 32) {
          const uint32_t j = j0 + lane;
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
            nbr = A.sadj[ao + (j - eo)];
            cross = A.red ? expand_one<true>(nbr, A.state, A.res, thr) : expand_one<false>(nbr, A.state, A.res, thr);
          }
          warp_append(cross, nbr, next, cnext);
        }
      }
      // 32 < d <= HUGE_DEG: warp per vertex
      for (unsigned i = gwarp; i < nb; i += nwarps) {
        const uint32_t v = A.Fb[i];
        const uint64_t a = A.soffs[v], e = A.soffs[v + 1];
        for (uint64_t p0 = a; p0 < e; p0 += 32) {
          const uint64_t p = p0 + lane;
          bool cross = false;
          uint32_t nbr = 0;
          if (p < e) {
            nbr = A.sadj[p];
            cross = A.red ? expand_one<true>(nbr, A.state, A.res, thr) : expand_one<false>(nbr, A.state, A.res, thr);
          }
          warp_append(cross, nbr, next, cnext);
        }
      }
      // hubs: chunks of HUB_CHUNK edges over every warp of the grid
      if (A.red) expand_hubs<true>(A.Fh, nh, A.soffs, A.sadj, A.state, A.res, thr, next, cnext, s_pre);
      else expand_hubs<false>(A.Fh, nh, A.soffs, A.sadj, A.state, A.res, thr, next, cnext, s_pre);
      grid.sync();
      // peel the frontier (Algorithm 1 line 17-18); reset the split counters and the
      // next-frontier counter of the following subround
      for (uint64_t i = gtid; i < nf; i += gthreads) A.state[F[i]] = V_PEELED;
      if (A.red) {  // next frontier: the unpeeled vertices whose residual degree reached thr
        for (uint64_t base = gtid & ~31ull; base < n; base += gthreads) {
          const uint64_t v = base + lane;
          const bool want = v < n && A.state[v] == V_UNPEELED && (uint64_t)A.res[v] <= thr;
          warp_append(want, (uint32_t)v, next, cnext);
        }
      }
      if (gtid == 0) {
        A.ctr[4] = A.ctr[5] = A.ctr[6] = 0;
        A.ctr[2 + ((r + 1) & 1)] = 0;
      }
      grid.sync();
      peeled += nf;
      nf = *cnext;
      ++r;
      uint32_t *t = F;
      F = next;
      next = t;
    }
    ++level;
  }
  if (gtid == 0) {
    A.out[0] = level;
    A.out[1] = r;
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
  counters.alloc(8, s);
  g.sub.alloc(n ? n : 1, s);
  g.dsnap.alloc(n ? n : 1, s);
  TC_CUDA(cudaMemcpyAsync(res.get(), g.deg.get(), sizeof(uint32_t) * n, cudaMemcpyDeviceToDevice, s));
  TC_CUDA(cudaMemsetAsync(state.get(), 0, n, s));
  if (g_opt_peel_coop) {
    int dev = 0, coop = 0, occ = 0;
    TC_CUDA(cudaGetDevice(&dev));
    TC_CUDA(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, dev));
    TC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, peel_coop_kernel, 256, 0));
    if (coop && occ > 0) {
      DevBuf<uint32_t> out;
      out.alloc(3, s);
      TC_CUDA(cudaMemsetAsync(out.get(), 0, 3 * sizeof(uint32_t), s));
      TC_CUDA(cudaMemsetAsync(counters.get(), 0, counters.bytes(), s));
      PeelArgs A{soffs.get(), sadj.get(), g.deg.get(), res.get(), g.sub.get(), g.dsnap.get(), state.get(),
                 F.get(), next.get(), Fs.get(), Fb.get(), Fh.get(), counters.get(), out.get(), n, m,
                 // auto: RED from 2^25 vertices (the frontier scan costs n per subround; the
                 // waits on returning atomics to hubs dominate only on large graphs)
                 g_opt_peel_red >= 0 ? g_opt_peel_red : (n >= (1u << 25) ? 1 : 0)};
      void *args[] = {&A};
      {
        ProfScope prof("peel", s, 0.0);
        TC_CUDA(cudaLaunchCooperativeKernel((const void *)peel_coop_kernel, dim3(num_sms() * occ), dim3(256), args, 0,
                                            s));
        TC_LAUNCH_CHECK();
      }
      uint32_t h_out[3] = {0, 0, 0};
      TC_CUDA(cudaMemcpyAsync(h_out, out.get(), sizeof(h_out), cudaMemcpyDeviceToHost, s));
      TC_CUDA(cudaStreamSynchronize(s));
      TC_REQUIRE(h_out[2] == 0, ST_CUDA, "A-direction did not terminate");
      g.levels = h_out[0];
      g.subrounds = h_out[1];
      prim_paper_kernel<<<grid_for(n, 256), 256, 0, s>>>(g.sub.get(), g.dsnap.get(), g.prim.get(), n);
      TC_LAUNCH_CHECK();
      return;
    }
  }
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
