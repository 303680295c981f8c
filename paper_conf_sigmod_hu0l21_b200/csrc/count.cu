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
#include <map>
#include <mutex>
#include <tuple>
#include <type_traits>
#include <vector>

#include "count_dev.cuh"
#include "internal.h"
#include "prims.cuh"

namespace tc {

int g_opt_small_cap = 256;   // power of two: d~ below it -> warp items, else CTA items
int g_opt_bracket = 1;       // bracketed binary search for long staged lists
int g_opt_intersect = 0;     // 0 = binary search (the paper's kernel), 1 = sort-merge (P:548-550 comparison)
int g_opt_lean = 1;          // register-lean short-list count_small instantiation (MODE 4)
int g_opt_extra = -1;        // §5.3 balance-point experiment: extra searches per wedge (-1 off)
int g_opt_l2_persist = 0;    // L2 access-policy window over [offs | col] during counts (off: measured slower overall)
int g_opt_shorter = 1;       // count modes: per edge the shorter list is streamed (owner lists)
int g_opt_owner_span = 128;  // owners per warp item (shorter-list schedule)
int g_opt_owner_lspan = 2048;  // owners per CTA item
int g_opt_vtiles = 1;        // classic count: streamed lists in this many L2 label tiles (1 = off)
int g_opt_cuckoo = 64;       // count-only CTA items: cuckoo set of the staged piece, max evictions (0 = off)
int g_opt_e2sort = -1;       // E2 owners grouped by a sort (no returning cursor atomics); -1 auto
int g_opt_otiles = 1;        // shorter-list CTA items: owner-label L2 tiles (0 = auto, 1 = off; default off: measured no faster)
int g_opt_otile_mb = 48;     // auto: MB of col per owner-label tile
int g_opt_otile_min = 4;     // a large x is tiled when it has >= otile_min * tiles owners

using namespace cnt;
namespace {

__global__ void items_hist_kernel(const uint64_t *__restrict__ offs, uint32_t ub, uint32_t ue, uint32_t cap,
                                  unsigned long long *hist, Owners ow) {
  __shared__ unsigned long long s_h[32];
  if (threadIdx.x < 32) s_h[threadIdx.x] = 0;
  __syncthreads();
  for (uint64_t u = (uint64_t)ub + blockIdx.x * blockDim.x + threadIdx.x; u < ue; u += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t d = (uint32_t)(offs[u + 1] - offs[u]);
    uint32_t it = items_of(d, owner_count(ow, (uint32_t)u, d), cap, ow);
    if (ow.nt && d >= cap && ow.lg[u] != 0xffffffffu) it = 0;  // tiled x: its own item list
    if (it) atomicAdd(&s_h[deg_bin(d)], (unsigned long long)it);
  }
  __syncthreads();
  if (threadIdx.x < 32 && s_h[threadIdx.x]) atomicAdd(&hist[threadIdx.x], s_h[threadIdx.x]);
}

// cursor[bin] = start of bin in the item list, bins in DESCENDING order (heaviest first)
__global__ void bin_scan_kernel(const unsigned long long *hist, unsigned long long *cursor) {
  unsigned lane = threadIdx.x;  // 32 threads; lane = 31 - bin
  unsigned long long c = hist[31 - lane];
  unsigned long long inc = warp_inclusive_scan(c);
  cursor[31 - lane] = inc - c;
}

constexpr int SC_PER_THREAD = 8;
__global__ __launch_bounds__(256) void items_scatter_kernel(const uint64_t *__restrict__ offs, uint32_t ub,
                                                            uint32_t ue, uint32_t cap, unsigned long long *cursor,
                                                            uint64_t *__restrict__ items, Owners ow) {
  __shared__ unsigned s_cnt[32];
  __shared__ unsigned long long s_base[32];
  const uint64_t span = 256ull * SC_PER_THREAD;
  for (uint64_t c0 = (uint64_t)ub + blockIdx.x * span; c0 < ue; c0 += (uint64_t)gridDim.x * span) {
    if (threadIdx.x < 32) s_cnt[threadIdx.x] = 0;
    __syncthreads();
    uint32_t off[SC_PER_THREAD], d[SC_PER_THREAD], it[SC_PER_THREAD];
#pragma unroll
    for (int i = 0; i < SC_PER_THREAD; ++i) {
      uint64_t u = c0 + (uint64_t)i * 256 + threadIdx.x;
      d[i] = u < ue ? (uint32_t)(offs[u + 1] - offs[u]) : 0u;
      it[i] = u < ue ? items_of(d[i], owner_count(ow, (uint32_t)u, d[i]), cap, ow) : 0u;
      if (it[i] && ow.nt && d[i] >= cap && ow.lg[u] != 0xffffffffu) it[i] = 0;  // tiled x
      off[i] = it[i] ? atomicAdd(&s_cnt[deg_bin(d[i])], it[i]) : 0u;
    }
    __syncthreads();
    if (threadIdx.x < 32) s_base[threadIdx.x] = s_cnt[threadIdx.x] ? atomicAdd(&cursor[threadIdx.x], (unsigned long long)s_cnt[threadIdx.x]) : 0ull;
    __syncthreads();
#pragma unroll
    for (int i = 0; i < SC_PER_THREAD; ++i) {
      if (!it[i]) continue;
      uint64_t u = c0 + (uint64_t)i * 256 + threadIdx.x;
      uint64_t p = s_base[deg_bin(d[i])] + off[i];
      const uint32_t step = d[i] < cap ? (ow.own ? ow.span : SV) : (ow.own ? ow.lspan : LV);
      for (uint32_t c = 0; c < it[i]; ++c) items[p + c] = (u << 32) | (uint64_t)(c * step);
    }
    __syncthreads();
  }
}

// ---- shorter-list owners (count modes): classification + scatter, warp per source u
__global__ void od_from_offs_kernel(const uint64_t *__restrict__ offs, uint32_t n, uint32_t *__restrict__ od) {
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < n; x += (uint64_t)gridDim.x * blockDim.x)
    od[x] = (uint32_t)(offs[x + 1] - offs[x]);
}
// e1c[u] = #{v in N+(u): 1 <= d~(v) <= d~(u)} (u streams nothing, v's lists are searched in
// N+(u)); e2c[v] += 1 for every u->v with d~(u) < d~(v) (u's list searched in N+(v)).
// Sources with d~(u) < 2 close no triangle.
// Owner-label tiles (option "otiles"): tile t = labels [bnd[t], bnd[t+1]), equal shares of
// col; tile_of = the largest t with bnd[t] <= o (bnd staged in shared memory).
constexpr uint32_t MAX_OTILES = 255;
__device__ __forceinline__ uint32_t tile_of(const uint32_t *sb, uint32_t nt, uint32_t o) {
  uint32_t lo = 0, len = nt;
  while (len > 1) {
    const uint32_t h = len >> 1;
    lo = sb[lo + h] <= o ? lo + h : lo;
    len -= h;
  }
  return lo;
}
__device__ __forceinline__ void stage_bounds(uint32_t *sb, const uint32_t *bnd, uint32_t nt) {
  for (uint32_t t = threadIdx.x; t <= nt; t += blockDim.x) sb[t] = bnd ? bnd[t] : 0u;
  __syncthreads();
}
// per lane: add 1 at row[key] for every lane with the same key (one atomic per distinct key)
__device__ __forceinline__ uint32_t warp_agg_add(bool on, uint32_t key, uint32_t *row) {
  const unsigned peers = __match_any_sync(0xffffffffu, on ? key : 0xffffffffu);
  uint32_t base = 0;
  const int leader = __ffs(peers) - 1;
  if (on && (int)lane_id() == leader) base = atomicAdd(&row[key], (uint32_t)__popc(peers));
  base = __shfl_sync(0xffffffffu, base, leader);
  return base + __popc(peers & ((1u << lane_id()) - 1u));
}
__global__ void tile_bounds_kernel(const uint64_t *__restrict__ offs, uint32_t n, uint64_t m, uint32_t nt,
                                   uint32_t *__restrict__ bnd) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t > nt) return;
  if (t == 0 || t == nt) {
    bnd[t] = t ? n : 0u;
    return;
  }
  const uint64_t target = m * t / nt;
  uint32_t lo = 0, hi = n;  // first label o with offs[o] >= target
  while (lo < hi) {
    const uint32_t mid = lo + (hi - lo) / 2;
    if (offs[mid] < target) lo = mid + 1;
    else hi = mid;
  }
  bnd[t] = lo;
}
// lg[x] = index of x among the sources with d~(x) >= cap (large), else ~0
__global__ void large_flag_kernel(const uint32_t *__restrict__ od, uint32_t n, uint32_t cap, uint32_t *__restrict__ f) {
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < n; x += (uint64_t)gridDim.x * blockDim.x)
    f[x] = od[x] >= cap ? 1u : 0u;
}
__global__ void large_index_kernel(const uint32_t *__restrict__ od, const uint64_t *__restrict__ pre, uint32_t n,
                                   uint32_t cap, uint32_t *__restrict__ lg) {
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < n; x += (uint64_t)gridDim.x * blockDim.x)
    lg[x] = od[x] >= cap ? (uint32_t)pre[x] : 0xffffffffu;
}

// e1c[u] = #{v in N+(u): 1 <= d~(v) <= d~(u)} (u streams nothing, v's lists are searched in
// N+(u)); e2c[v] += 1 for every u->v with d~(u) < d~(v) (u's list searched in N+(v)).
// Sources with d~(u) < 2 close no triangle.  Owner tiles (tcnt != nullptr): also
// tcnt[lg[x]*nt + tile(o)] += 1 for every owner o of a large x.
__global__ void owners_count_kernel(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col,
                                    const uint32_t *__restrict__ od, uint32_t ub, uint32_t ue,
                                    uint32_t *__restrict__ e1c, uint32_t *__restrict__ e2c,
                                    const uint32_t *__restrict__ lg, const uint32_t *__restrict__ bnd, uint32_t nt,
                                    uint32_t *__restrict__ tcnt, uint32_t *__restrict__ e2s) {
  __shared__ uint32_t s_bnd[MAX_OTILES + 1];
  if (tcnt) stage_bounds(s_bnd, bnd, nt);
  const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
  for (uint64_t u = ub + (uint64_t)blockIdx.x * (blockDim.x / 32) + warp_id(); u < ue; u += nw) {
    const uint64_t a = offs[u];
    const uint32_t du = (uint32_t)(offs[u + 1] - a);
    if (du < 2) continue;
    const uint32_t lu = tcnt ? lg[u] : 0xffffffffu;  // warp-uniform
    uint32_t c1 = 0, c2 = 0;
    for (uint32_t j0 = 0; j0 < du; j0 += 32) {
      const uint32_t j = j0 + lane_id();
      uint32_t v = 0, dv = 0;
      if (j < du) {
        v = col[a + j];
        dv = od[v];
      }
      const bool e1 = j < du && dv >= 1 && dv <= du;
      c1 += __popc(__ballot_sync(0xffffffffu, e1));
      c2 += __popc(__ballot_sync(0xffffffffu, j < du && dv > du));
      if (lu != 0xffffffffu) warp_agg_add(e1, e1 ? tile_of(s_bnd, nt, v) : 0u, tcnt + (uint64_t)lu * nt);
      if (j < du && dv > du) {
        atomicAdd(&e2c[v], 1u);
        if (tcnt) {
          const uint32_t lv = lg[v];
          if (lv != 0xffffffffu) atomicAdd(&tcnt[(uint64_t)lv * nt + tile_of(s_bnd, nt, (uint32_t)u)], 1u);
        }
      }
    }
    if (lane_id() == 0) {
      e1c[u] = c1;
      if (e2s) e2s[u] = c2;
    }
  }
}
// per large x: tiled iff it has >= tmin owners (else lg[x] = ~0: untiled); tiled rows get
// toff (exclusive prefix of the tile counts, then the total) and tcnt becomes the row's
// write cursor
__global__ void tile_offsets_kernel(uint32_t n, uint32_t *__restrict__ lg, const uint64_t *__restrict__ ooff,
                                    uint32_t nt, uint32_t tmin, uint32_t *__restrict__ tcnt,
                                    uint32_t *__restrict__ toff) {
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < n; x += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t l = lg[x];
    if (l == 0xffffffffu) continue;
    if (ooff[x + 1] - ooff[x] < tmin) {
      lg[x] = 0xffffffffu;
      continue;
    }
    uint32_t *c = tcnt + (uint64_t)l * nt, *o = toff + (uint64_t)l * (nt + 1);
    uint32_t acc = 0;
    for (uint32_t t = 0; t < nt; ++t) {
      const uint32_t k = c[t];
      o[t] = acc;
      c[t] = acc;
      acc += k;
    }
    o[nt] = acc;
  }
}
// CTA items of the tiled x, tile by tile: per tile the item count, then cursors, then the
// items (x << 32) | (t << 24) | chunk (ceil(owners in tile / lspan) chunks)
__global__ void tile_items_count_kernel(uint32_t n, const uint32_t *__restrict__ lg, const uint32_t *__restrict__ toff,
                                        uint32_t nt, uint32_t lspan, unsigned long long *__restrict__ tile_items) {
  __shared__ unsigned long long s_c[MAX_OTILES];
  for (uint32_t t = threadIdx.x; t < nt; t += blockDim.x) s_c[t] = 0;
  __syncthreads();
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < n; x += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t l = lg[x];
    if (l == 0xffffffffu) continue;
    const uint32_t *o = toff + (uint64_t)l * (nt + 1);
    for (uint32_t t = 0; t < nt; ++t) {
      const uint32_t k = o[t + 1] - o[t];
      if (k) atomicAdd(&s_c[t], (unsigned long long)((k + lspan - 1) / lspan));
    }
  }
  __syncthreads();
  for (uint32_t t = threadIdx.x; t < nt; t += blockDim.x)
    if (s_c[t]) atomicAdd(&tile_items[t], s_c[t]);
}
__global__ void tile_items_scan_kernel(unsigned long long *tile_items, uint32_t nt) {
  // tile_items[0..nt) counts -> [nt .. 2nt) cursors, [2nt] total (one thread: nt <= 255)
  unsigned long long acc = 0;
  for (uint32_t t = 0; t < nt; ++t) {
    tile_items[nt + t] = acc;
    acc += tile_items[t];
  }
  tile_items[2 * nt] = acc;
}
__global__ void tile_items_scatter_kernel(uint32_t n, const uint32_t *__restrict__ lg,
                                          const uint32_t *__restrict__ toff, uint32_t nt, uint32_t lspan,
                                          unsigned long long *__restrict__ cursor, uint64_t *__restrict__ items) {
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < n; x += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t l = lg[x];
    if (l == 0xffffffffu) continue;
    const uint32_t *o = toff + (uint64_t)l * (nt + 1);
    for (uint32_t t = 0; t < nt; ++t) {
      const uint32_t k = o[t + 1] - o[t];
      if (!k) continue;
      const uint32_t ni = (k + lspan - 1) / lspan;
      const unsigned long long p = atomicAdd(&cursor[t], (unsigned long long)ni);
      for (uint32_t c = 0; c < ni; ++c) items[p + c] = (x << 32) | ((uint64_t)t << 24) | c;
    }
  }
}
__global__ void owners_total_kernel(const uint32_t *__restrict__ e1c, uint32_t n, uint32_t *__restrict__ c) {
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < n; x += (uint64_t)gridDim.x * blockDim.x)
    c[x] += e1c[x];
}
// E2 write cursor of x: its owner-list start plus its E1 owners
__global__ void owners_cursor_kernel(const uint64_t *__restrict__ ooff, const uint32_t *__restrict__ e1c,
                                     uint32_t n, unsigned long long *__restrict__ cur) {
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < n; x += (uint64_t)gridDim.x * blockDim.x)
    cur[x] = ooff[x] + e1c[x];
}
// owners of x: its E1 out-neighbours (N+(x) order) then its E2 in-neighbours (any order);
// a tiled x (lg[x] != ~0, owner tiles on): grouped by owner tile through the row cursors
__global__ void owners_scatter_kernel(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col,
                                      const uint32_t *__restrict__ od, uint32_t ub, uint32_t ue,
                                      const uint64_t *__restrict__ ooff, unsigned long long *__restrict__ e2cur,
                                      uint32_t *__restrict__ own, const uint32_t *__restrict__ lg,
                                      const uint32_t *__restrict__ bnd, uint32_t nt, uint32_t *__restrict__ tcur) {
  __shared__ uint32_t s_bnd[MAX_OTILES + 1];
  if (tcur) stage_bounds(s_bnd, bnd, nt);
  const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
  for (uint64_t u = ub + (uint64_t)blockIdx.x * (blockDim.x / 32) + warp_id(); u < ue; u += nw) {
    const uint64_t a = offs[u];
    const uint32_t du = (uint32_t)(offs[u + 1] - a);
    if (du < 2) continue;
    uint64_t p1 = ooff[u];
    const uint32_t lu = tcur ? lg[u] : 0xffffffffu;  // warp-uniform
    for (uint32_t j0 = 0; j0 < du; j0 += 32) {
      const uint32_t j = j0 + lane_id();
      uint32_t v = 0, dv = 0;
      if (j < du) {
        v = col[a + j];
        dv = od[v];
      }
      const bool e1 = j < du && dv >= 1 && dv <= du;
      if (lu != 0xffffffffu) {
        const uint32_t r = warp_agg_add(e1, e1 ? tile_of(s_bnd, nt, v) : 0u, tcur + (uint64_t)lu * nt);
        if (e1) own[p1 + r] = v;
      } else {
        const unsigned m1 = __ballot_sync(0xffffffffu, e1);
        if (e1) own[p1 + __popc(m1 & ((1u << lane_id()) - 1u))] = v;
        p1 += __popc(m1);
      }
      if (j < du && dv > du) {
        const uint32_t lv = tcur ? lg[v] : 0xffffffffu;
        if (lv != 0xffffffffu)
          own[ooff[v] + atomicAdd(&tcur[(uint64_t)lv * nt + tile_of(s_bnd, nt, (uint32_t)u)], 1u)] = (uint32_t)u;
        else
          own[atomicAdd(&e2cur[v], 1ull)] = (uint32_t)u;
      }
    }
  }
}

// E2 owners grouped by a sort instead of returning cursor atomics (option "e2sort"): the
// cursor of a hub x takes every E2 owner of x, and the returned positions serialise there.
// e2s[u] = #E2 edges of source u (owners_count); the E1 scatter also writes the E2 pairs
// (x << vbits) | u compactly at e2pos[u]; an LSD sort on the x bits groups them (stable);
// the placement puts the j-th pair of x at own[ooff[x] + e1c[x] + j].
__global__ void owners_scatter_e2keys_kernel(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col,
                                             const uint32_t *__restrict__ od, uint32_t ub, uint32_t ue,
                                             const uint64_t *__restrict__ ooff, const uint64_t *__restrict__ e2pos,
                                             uint32_t vbits, uint32_t *__restrict__ own, uint64_t *__restrict__ keys) {
  const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
  for (uint64_t u = ub + (uint64_t)blockIdx.x * (blockDim.x / 32) + warp_id(); u < ue; u += nw) {
    const uint64_t a = offs[u];
    const uint32_t du = (uint32_t)(offs[u + 1] - a);
    if (du < 2) continue;
    uint64_t p1 = ooff[u], p2 = e2pos[u];
    for (uint32_t j0 = 0; j0 < du; j0 += 32) {
      const uint32_t j = j0 + lane_id();
      uint32_t v = 0, dv = 0;
      if (j < du) {
        v = col[a + j];
        dv = od[v];
      }
      const bool e1 = j < du && dv >= 1 && dv <= du;
      const bool e2 = j < du && dv > du;
      const unsigned lt = (1u << lane_id()) - 1u;
      const unsigned m1 = __ballot_sync(0xffffffffu, e1), m2 = __ballot_sync(0xffffffffu, e2);
      if (e1) own[p1 + __popc(m1 & lt)] = v;
      if (e2) keys[p2 + __popc(m2 & lt)] = ((uint64_t)v << vbits) | u;
      p1 += __popc(m1);
      p2 += __popc(m2);
    }
  }
}
__global__ void owners_place_e2_kernel(const uint64_t *__restrict__ sorted, uint64_t total, uint32_t vbits,
                                       const uint64_t *__restrict__ ooff, const uint32_t *__restrict__ e1c,
                                       const uint64_t *__restrict__ e2start, uint32_t *__restrict__ own) {
  const uint64_t mask = (1ull << vbits) - 1;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t key = sorted[i];
    const uint64_t x = key >> vbits;
    own[ooff[x] + e1c[x] + (i - e2start[x])] = (uint32_t)(key & mask);
  }
}

// Bitmap intersection (option "intersect" = 2): Bisson's block-per-vertex pattern as the
// paper describes it (Fig.1) and evaluates A-direction on (Fig.13):
// the CTA marks N+(u) in a bitmap of |V| bits, synchronises, then in supersteps of
// BM_THREADS neighbours each thread takes one v in N+(u) and tests every w in N+(v)
// against the bitmap; a barrier closes every superstep, so a superstep lasts as long as
// its longest N+(v) — the intra-block BSP imbalance Eq.1 models.  The bits of
// N+(u) are cleared again before the next u.  Bitmap in shared memory when |V| <= 2^20
// (128 KB), else one |V|-bit slice of global memory per CTA (L2-resident for |V| = 2^22).
constexpr int BM_THREADS = 256;
constexpr uint32_t BM_CHUNK = 16;  // sources per counter fetch
constexpr uint32_t BM_SMEM_MAX_N = 1u << 20;
template <bool SMEM>
__global__ __launch_bounds__(BM_THREADS) void count_bitmap_kernel(const uint64_t *__restrict__ offs,
                                                                  const uint32_t *__restrict__ col, uint32_t ub,
                                                                  uint32_t ue, uint32_t *gbits, uint32_t words,
                                                                  unsigned *ctr, unsigned long long *T) {
  uint32_t *bits = SMEM ? tc_smem : gbits + (uint64_t)blockIdx.x * words;
  __shared__ uint32_t s_c;
  if (SMEM)
    for (uint32_t i = threadIdx.x; i < words; i += BM_THREADS) bits[i] = 0u;
  uint64_t acc = 0;
  const uint32_t nu = ue - ub;
  while (true) {
    __syncthreads();
    if (threadIdx.x == 0) s_c = atomicAdd(ctr, BM_CHUNK);
    __syncthreads();
    const uint32_t c0 = s_c;
    if (c0 >= nu) break;
    const uint32_t c1 = min(nu, c0 + BM_CHUNK);
    for (uint32_t c = c0; c < c1; ++c) {
      const uint32_t u = ub + c;
      const uint64_t a = offs[u];
      const uint32_t L = (uint32_t)(offs[u + 1] - a);
      if (L < 2) continue;  // block-uniform
      for (uint32_t i = threadIdx.x; i < L; i += BM_THREADS) {
        const uint32_t w = __ldg(col + a + i);
        atomicOr(&bits[w >> 5], 1u << (w & 31));
      }
      __syncthreads();
      uint32_t cnt = 0;
      for (uint32_t g0 = 0; g0 < L; g0 += BM_THREADS) {  // one superstep per group of neighbours
        const uint32_t i = g0 + threadIdx.x;
        if (i < L) {
          const uint32_t v = __ldg(col + a + i);
          const uint64_t vb = offs[v];
          const uint32_t dv = (uint32_t)(offs[v + 1] - vb);
          for (uint32_t j = 0; j < dv; ++j) {
            const uint32_t w = __ldg(col + vb + j);
            cnt += (bits[w >> 5] >> (w & 31)) & 1u;
          }
        }
        __syncthreads();
      }
      acc += cnt;
      for (uint32_t i = threadIdx.x; i < L; i += BM_THREADS) bits[__ldg(col + a + i) >> 5] = 0u;
      __syncthreads();
    }
  }
  block_add_u64(acc, T);
}

// ---- edge-unit A-order (TC_SCHED_EDGE_AORDER, Q26)
// A unit is ONE directed edge u -> v (CSR position p, index j = p - offs[u]); its task
// streams N+(v) and binary-searches every w in N+(u).  Superiority S(d~(v)) (the streamed
// list); d~(v) = 0 -> no work, inactive.  Warp per source: lanes over its out-edges.
__global__ void unit_sup_kernel(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col, uint32_t n,
                                const int64_t *__restrict__ stab, uint64_t *__restrict__ items,
                                int64_t *__restrict__ isup, uint8_t *__restrict__ iact) {
  const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x / 32);
  for (uint64_t u = (uint64_t)blockIdx.x * (blockDim.x / 32) + warp_id(); u < n; u += nw) {
    const uint64_t a = offs[u];
    const uint32_t d = (uint32_t)(offs[u + 1] - a);
    for (uint32_t j = lane_id(); j < d; j += 32) {
      const uint32_t v = col[a + j];
      const uint32_t dv = (uint32_t)(offs[v + 1] - offs[v]);
      items[a + j] = (u << 32) | (uint64_t)j;
      isup[a + j] = dv ? stab[dv] : 0;
      iact[a + j] = dv ? 1 : 0;
    }
  }
}
// CTA per bucket of edge units (fetched dynamically); warp per unit: the lanes stream
// N+(v) and binary-search each w in N+(u) in global memory (Fox's edge-centric pattern,
// no staging: a bucket's edges have unrelated sources).  MODE 1: +1 at u, v, w per
// triangle; MODE 2: +1 at the CSR positions of (u,v), (u,w), (v,w).
template <int MODE>
__global__ __launch_bounds__(CT_THREADS) void count_units_kernel(const uint64_t *__restrict__ offs,
                                                                 const uint32_t *__restrict__ col,
                                                                 const uint64_t *__restrict__ units,
                                                                 const uint32_t *__restrict__ uoff, uint32_t nb,
                                                                 uint32_t ub, uint32_t ue, unsigned *bucket_ctr,
                                                                 unsigned long long *T, unsigned long long *tv) {
  __shared__ uint32_t s_bucket;
  uint64_t acc = 0;
  while (true) {
    __syncthreads();
    if (threadIdx.x == 0) s_bucket = atomicAdd(bucket_ctr, 1u);
    __syncthreads();
    const uint32_t bi = s_bucket;
    if (bi >= nb) break;
    for (uint32_t i = uoff[bi] + warp_id(); i < uoff[bi + 1]; i += CT_WARPS) {
      const uint64_t it = units[i];
      const uint32_t u = (uint32_t)(it >> 32), j = (uint32_t)it;
      if (u < ub || u >= ue) continue;  // tc_count_range / tc_count_dist slices
      const uint64_t a = offs[u];
      const uint32_t L = (uint32_t)(offs[u + 1] - a);
      if (L < 2) continue;
      const uint32_t v = col[a + j];
      const uint64_t vb = offs[v];
      const uint32_t dv = (uint32_t)(offs[v + 1] - vb);
      const GlobalSearch search{col + a, L, 0};
      uint32_t cnt = 0;
      for (uint32_t t = lane_id(); t < dv; t += 32) {
        const uint32_t w = col[vb + t];
        uint32_t pos;
        const bool hit = search(w, pos);
        cnt += hit ? 1u : 0u;
        if (MODE == 1 && hit) {
          atomicAdd(&tv[v], 1ull);
          atomicAdd(&tv[w], 1ull);
        }
        if (MODE == 2 && hit) {
          atomicAdd(&tv[a + j], 1ull);
          atomicAdd(&tv[a + pos], 1ull);
          atomicAdd(&tv[vb + t], 1ull);
        }
      }
      if (MODE == 1) {
        const uint32_t tot = warp_sum((uint64_t)cnt);
        if (lane_id() == 0 && tot) atomicAdd(&tv[u], (unsigned long long)tot);
      }
      acc += cnt;
    }
  }
  block_add_u64(acc, T);
}

__global__ void gather_tv_kernel(const unsigned long long *__restrict__ tnew, const uint32_t *__restrict__ perm,
                                 uint32_t n, uint64_t *__restrict__ out) {
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
    out[v] = tnew[perm ? perm[v] : v];
}

// --------------------------------------------------------------- per-edge output order
__global__ void inverse_perm_kernel(const uint32_t *__restrict__ perm, uint32_t n, uint32_t *__restrict__ iperm) {
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
    iperm[perm[v]] = (uint32_t)v;
}

// Per-edge support from CSR positions (final labels) to the canonical order of the simple
// graph's edge list (keys (min << bits) | max over ORIGINAL ids, ascending): one warp per
// source label, every CSR edge located by a binary search of its canonical key.
__global__ void edge_map_kernel(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col, uint32_t n,
                                const uint32_t *__restrict__ iperm, const uint64_t *__restrict__ edges, uint64_t m,
                                int bits, const unsigned long long *__restrict__ te, uint64_t *__restrict__ out) {
  const unsigned warps = gridDim.x * (blockDim.x / 32);
  for (uint64_t x = (uint64_t)blockIdx.x * (blockDim.x / 32) + warp_id(); x < n; x += warps) {
    const uint64_t a = offs[x], e = offs[x + 1];
    const uint32_t ox = iperm ? iperm[x] : (uint32_t)x;
    for (uint64_t p = a + lane_id(); p < e; p += 32) {
      const uint32_t y = col[p];
      const uint32_t oy = iperm ? iperm[y] : y;
      const uint64_t key = ((uint64_t)min(ox, oy) << bits) | max(ox, oy);
      uint64_t lo = 0, hi = m;
      while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (edges[mid] < key) lo = mid + 1;
        else hi = mid;
      }
      out[lo] = te[p];
    }
  }
}

// --------------------------------------------------------------- work model / analysis
// w(u) = d~(u) + Σ_{v ∈ N+(u)} d~(v); sectors: 32-B sectors the Hu pattern touches with no reuse.
// w[u] = d~(u) + Σ_{v ∈ N+(u)} d~(v), with `shorter` Σ min(d~(u), d~(v)) (the partition
// work model of the schedule that runs: the elements streamed per edge); sectors: the count's
// algorithmic DRAM sectors with no reuse: per source with d~ >= 2 its
// staged list + 1, per edge the streamed list + its offs pair — N+(v) (Hu's pattern), or
// with `shorter` the shorter of N+(u), N+(v) (the shorter-list schedule of count_graph).
__global__ void work_kernel(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col, uint32_t n,
                            uint64_t *__restrict__ w, unsigned long long *sectors, int shorter) {
  uint64_t sec = 0;
  unsigned warps = gridDim.x * (blockDim.x / 32);
  for (uint64_t u = (uint64_t)blockIdx.x * (blockDim.x / 32) + warp_id(); u < n; u += warps) {
    uint64_t a = offs[u], e = offs[u + 1];
    uint64_t s = 0, sc = 0;
    for (uint64_t p = a + lane_id(); p < e; p += 32) {
      uint32_t v = col[p];
      uint64_t vb = offs[v], ve = offs[v + 1];
      const bool own_u = shorter && ve - vb > e - a;  // E2: N+(u) is the streamed list
      s += own_u ? e - a : ve - vb;                   // elements streamed for this edge
      const uint64_t sb = own_u ? a : vb, se = own_u ? e : ve, sx = own_u ? u : v;
      // streamed list span + its offs pair
      if (se > sb) sc += ((se * 4 - 1) >> 5) - ((sb * 4) >> 5) + 1;
      sc += ((sx * 8 + 15) >> 5) - ((sx * 8) >> 5) + 1;
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

// Per-device setup: the >48 KB dynamic shared-memory opt-in (cudaFuncSetAttribute) and the
// __constant__ options are per device, so both are tracked per device under a mutex.
static std::mutex g_cfg_mu;
struct DeviceCfg {
  bool configured = false;
  int bracket = 1, intersect = 0, extra = -1, cuckoo = 64;
};
static DeviceCfg g_cfg[64];

static DeviceCfg &device_cfg() {
  int dev = 0;
  TC_CUDA(cudaGetDevice(&dev));
  TC_REQUIRE(dev >= 0 && dev < 64, ST_CUDA, "device ordinal >= 64");
  return g_cfg[dev];
}

static void configure_kernels_locked(DeviceCfg &c) {
  if (c.configured) return;
  const int large_smem = (int)(LG_SMEM_WORDS * sizeof(uint32_t));
  for (int m = 0; m <= 2; ++m)
    TC_CUDA(cudaFuncSetAttribute(large_kernel(m, false), cudaFuncAttributeMaxDynamicSharedMemorySize, large_smem));
  TC_CUDA(cudaFuncSetAttribute(large_kernel(0, true), cudaFuncAttributeMaxDynamicSharedMemorySize, large_smem));
  const int small_max = 200 * 1024;
  for (int m = 0; m <= 4; ++m)
    TC_CUDA(cudaFuncSetAttribute(small_kernel(m, false), cudaFuncAttributeMaxDynamicSharedMemorySize, small_max));
  for (int m : {0, 4})
    TC_CUDA(cudaFuncSetAttribute(small_kernel(m, true), cudaFuncAttributeMaxDynamicSharedMemorySize, small_max));
  for (int m = 0; m <= 2; ++m)
    TC_CUDA(cudaFuncSetAttribute(range_kernel(m), cudaFuncAttributeMaxDynamicSharedMemorySize, small_max));
  TC_CUDA(cudaFuncSetAttribute(count_bitmap_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               (int)(BM_SMEM_MAX_N / 8)));
  c.configured = true;
}

// kernel attributes + the option constants of the current device, once per change (every
// kernel translation unit holds its own copy of the __constant__ options)
static void configure_kernels() {
  std::lock_guard<std::mutex> lk(g_cfg_mu);
  DeviceCfg &c = device_cfg();
  configure_kernels_locked(c);
  const int extra = g_opt_extra >= 0 ? g_opt_extra : c.extra;
  if (g_opt_bracket != c.bracket || g_opt_intersect != c.intersect || extra != c.extra || g_opt_cuckoo != c.cuckoo) {
    small_set_constants(g_opt_bracket, g_opt_intersect, extra < 0 ? 0 : extra, g_opt_cuckoo);
    large_set_constants(g_opt_bracket, g_opt_intersect, extra < 0 ? 0 : extra, g_opt_cuckoo);
    c.cuckoo = g_opt_cuckoo;
    c.bracket = g_opt_bracket;
    c.intersect = g_opt_intersect;
    c.extra = extra;
  }
}

// type-erased launch of a kernel of the kernel translation units (arguments passed with the
// kernel's exact parameter types)
template <class... A>
static void launch(const void *fn, unsigned grid, unsigned block, size_t smem, cudaStream_t s, A... a) {
  void *args[] = {(void *)&a...};
  TC_CUDA(cudaLaunchKernel(fn, dim3(grid), dim3(block), args, smem, s));
}

// L2 access-policy window over the head of the CSR allocation [offs | col...] for the
// duration of the count: the offsets (8 B read per visited list, random) and as much of
// the column array as the persisting carve-out allows stay in the 126 MB L2.  Best effort:
// any failure just leaves the default policy.  Restored (and persisting lines released)
// afterwards so later work on the stream is unaffected.
struct L2Window {
  cudaStream_t s;
  bool on = false;
  L2Window(cudaStream_t st, void *base, size_t bytes) : s(st) {
    if (!g_opt_l2_persist || !bytes || !base) return;
    int dev = 0, maxp = 0, maxw = 0;
    if (cudaGetDevice(&dev) != cudaSuccess ||
        cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev) != cudaSuccess ||
        cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, dev) != cudaSuccess || maxp <= 0 ||
        maxw <= 0) {
      cudaGetLastError();
      return;
    }
    size_t cur = 0;
    if (cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize) == cudaSuccess && cur < (size_t)maxp)
      cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)maxp);
    cudaStreamAttrValue v = {};
    v.accessPolicyWindow.base_ptr = base;
    v.accessPolicyWindow.num_bytes = std::min(bytes, std::min((size_t)maxp, (size_t)maxw));
    v.accessPolicyWindow.hitRatio = 1.0f;
    v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    on = cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v) == cudaSuccess;
    cudaGetLastError();
  }
  ~L2Window() {
    if (!on) return;
    cudaStreamAttrValue v = {};
    v.accessPolicyWindow.num_bytes = 0;
    cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v);
    cudaCtxResetPersistingL2Cache();
    cudaGetLastError();
  }
};

// Largest warp-slice capacity <= cap whose per-CTA shared memory (slices, bracket tables,
// per-vertex/per-edge counters) fits the 200 KB the warp kernels are configured for; lists
// longer than the slice are searched in global memory (the kernels' L > cap path).
static uint32_t fit_cap(uint32_t cap, bool pv) {
  while (cap > 32 && (size_t)CT_WARPS * warp_stride(cap, pv) * sizeof(uint32_t) > 200u * 1024u) cap >>= 1;
  return cap;
}

// Resident CTAs per SM, cached per (kernel, block, smem): queried on every count otherwise.
static int occupancy(const void *fn, int threads, size_t smem) {
  static std::mutex mu;
  static std::map<std::tuple<const void *, int, size_t, int>, int> cache;
  int dev = 0;
  TC_CUDA(cudaGetDevice(&dev));
  const auto key = std::make_tuple(fn, threads, smem, dev);
  {
    std::lock_guard<std::mutex> lk(mu);
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
  }
  int blocks = 0;
  TC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks, fn, threads, smem));
  blocks = blocks > 0 ? blocks : 1;
  std::lock_guard<std::mutex> lk(mu);
  cache[key] = blocks;
  return blocks;
}

uint64_t count_graph(Graph &g, uint32_t ub, uint32_t ue, uint64_t *d_tv, float *kernel_ms, uint64_t *launches,
                     int mode, unsigned long long *d_T) {
  // 0 count, 1 per-vertex (t[n], new labels), 2 per-edge (CSR positions), 3 count with
  // g_opt_extra extra searches per wedge in the warp-item kernel (§5.3 experiment)
  if (mode < 0) mode = d_tv ? 1 : (g_opt_extra >= 0 ? 3 : 0);
  const bool pv = mode == 1 || mode == 2;
  cudaStream_t s = g.stream;
  configure_kernels();
  if (ue > g.n) ue = g.n;
  uint64_t nlaunch = 0;
  DevBuf<unsigned long long> dT_own;
  if (!d_T) {
    dT_own.alloc(1, s);
    TC_CUDA(cudaMemsetAsync(dT_own.get(), 0, sizeof(unsigned long long), s));
  }
  struct {
    unsigned long long *p;
    unsigned long long *get() const { return p; }
  } dT{d_T ? d_T : dT_own.get()};
  unsigned long long *tv = reinterpret_cast<unsigned long long *>(d_tv);
  const uint32_t cap = (uint32_t)g_opt_small_cap;
  // bits of the largest label: absolute bracket tables cover [0, 2^vbits)
  const uint32_t vbits = g.n > 1 ? 32u - (uint32_t)__builtin_clz(g.n - 1) : 1u;
  int sched = g.schedule;
  // AUTO = BUCKETED for every ordering: measured on B200 (R-MAT s22, profiles/), the
  // dynamic heavy-first item schedule beats the static block-per-bucket model A-order
  // targets (RANGE) by 1.3-1.5x, and makes the count time order-independent.
  if (sched == TC_SCHED_AUTO) sched = TC_SCHED_BUCKETED;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  if (kernel_ms) {
    TC_CUDA(cudaEventCreate(&e0));
    TC_CUDA(cudaEventCreate(&e1));
  }
  L2Window l2win(s, g.csr_mem.get(), g.csr_mem.bytes());
  if (ub < ue && g.m && (mode == 0 || mode == 3) && g_opt_intersect == 2) {
    // bitmap intersection (Bisson's block-per-vertex pattern): its own schedule
    const bool in_smem = g.n <= BM_SMEM_MAX_N;
    const uint32_t words = (g.n + 31) / 32;
    const size_t smem = in_smem ? (size_t)words * sizeof(uint32_t) : 0;
    auto fn = in_smem ? count_bitmap_kernel<true> : count_bitmap_kernel<false>;
    int occ = occupancy((const void *)fn, BM_THREADS, smem);
    uint64_t want = ((uint64_t)(ue - ub) + BM_CHUNK - 1) / BM_CHUNK;
    uint64_t grid = std::max<uint64_t>(1, std::min<uint64_t>(want, (uint64_t)num_sms() * occ));
    DevBuf<uint32_t> gbits;
    if (!in_smem) {  // one zeroed |V|-bit slice per CTA, at most 1 GiB in total
      grid = std::max<uint64_t>(1, std::min<uint64_t>(grid, (1ull << 28) / words));
      gbits.alloc(grid * words, s);
      TC_CUDA(cudaMemsetAsync(gbits.get(), 0, gbits.bytes(), s));
    }
    DevBuf<unsigned> ctr;
    ctr.alloc(1, s);
    TC_CUDA(cudaMemsetAsync(ctr.get(), 0, sizeof(unsigned), s));
    if (kernel_ms) TC_CUDA(cudaEventRecord(e0, s));
    ProfScope prof("count_bitmap", s, 0.0);
    fn<<<(unsigned)grid, BM_THREADS, smem, s>>>(g.offs.get(), g.col.get(), ub, ue, gbits.get(), words, ctr.get(),
                                                 dT.get());
    TC_LAUNCH_CHECK();
    if (kernel_ms) TC_CUDA(cudaEventRecord(e1, s));
    ++nlaunch;
  } else if (ub < ue && g.m && sched == TC_SCHED_EDGE_AORDER) {
    build_units(g);
    const uint32_t nb = (uint32_t)g.h_unit_off.size() - 1;
    if (nb) {
      const size_t smem = 0;
      auto fn = mode == 2 ? count_units_kernel<2> : mode == 1 ? count_units_kernel<1> : count_units_kernel<0>;
      int occ = occupancy((const void *)fn, CT_THREADS, smem);
      unsigned grid = (unsigned)std::min<uint64_t>(nb, (uint64_t)num_sms() * occ);
      DevBuf<unsigned> bctr;
      bctr.alloc(1, s);
      TC_CUDA(cudaMemsetAsync(bctr.get(), 0, sizeof(unsigned), s));
      if (kernel_ms) TC_CUDA(cudaEventRecord(e0, s));
      ProfScope prof("count_units", s, 0.0);
      fn<<<grid, CT_THREADS, smem, s>>>(g.offs.get(), g.col.get(), g.units.get(), g.unit_off.get(), nb, ub, ue,
                                        bctr.get(), dT.get(), tv);
      TC_LAUNCH_CHECK();
      if (kernel_ms) TC_CUDA(cudaEventRecord(e1, s));
      ++nlaunch;
    }
  } else if (ub < ue && g.m) {
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
        const uint32_t rcap = fit_cap(cap, pv);
        size_t smem = (size_t)CT_WARPS * warp_stride(rcap, pv) * sizeof(uint32_t);
        const void *range_fn = range_kernel(mode == 2 ? 2 : mode == 1 ? 1 : 0);
        int occ = occupancy(range_fn, CT_THREADS, smem);
        unsigned grid = (unsigned)std::min<uint64_t>(nb, (uint64_t)num_sms() * occ);
        DevBuf<unsigned> bctr;
        bctr.alloc(1, s);
        TC_CUDA(cudaMemsetAsync(bctr.get(), 0, sizeof(unsigned), s));
        if (kernel_ms) TC_CUDA(cudaEventRecord(e0, s));
        ProfScope prof("count_range", s, 0.0);
        launch(range_fn, grid, CT_THREADS, smem, s, (const uint64_t *)g.offs.get(), (const uint32_t *)g.col.get(), boff,
               (uint32_t)k, b0, nb, ub, ue, rcap, bctr.get(), (unsigned long long *)dT.get(), tv, vbits);
        if (kernel_ms) TC_CUDA(cudaEventRecord(e1, s));
        ++nlaunch;
      }
    } else {
      // shorter-list owners (count modes, option "shorter"): per edge the shorter list is
      // streamed and searched in the longer one, which is staged once for all its owners
      Owners ow{nullptr, nullptr, 0, 0, 0, 0xffffffffu};
      DevBuf<uint32_t> od_new, e1c, e2c, own;
      DevBuf<uint32_t> lg, bnd, tcnt, toff;  // owner tiles
      uint32_t nt = 0;
      uint64_t nlarge_x = 0;
      DevBuf<uint64_t> ooff;
      DevBuf<unsigned long long> e2cur;
      uint32_t iub = ub, iue = ue;  // sources of the item list
      // max d~ (label-free; from ensure_od when it ran, else from the CSR): with every list
      // short (max d~ < 64, e.g. ER) the two lists of an edge are alike and the owner pass
      // does not pay back (ER configs[1]: 3.2 -> 4.8 ms), so the classic schedule runs
      uint32_t maxd = g.od_ready ? g.max_outdeg : 0;
      if (g_opt_shorter && mode == 0 && g_opt_intersect == 0 && !g.od_ready && g.n) {
        od_new.alloc(g.n, s);
        od_from_offs_kernel<<<grid_for(g.n, 256), 256, 0, s>>>(g.offs.get(), g.n, od_new.get());
        TC_LAUNCH_CHECK();
        maxd = device_max_u32(od_new.get(), g.n, s);
      }
      if (g_opt_shorter && mode == 0 && g_opt_intersect == 0 && maxd >= 64) {
        const uint32_t n = g.n;
        if (!od_new.get()) {
          od_new.alloc(n, s);
          od_from_offs_kernel<<<grid_for(n, 256), 256, 0, s>>>(g.offs.get(), n, od_new.get());
          TC_LAUNCH_CHECK();
        }
        e1c.alloc(n, s);
        e2c.alloc(n, s);
        e2cur.alloc(n, s);
        ooff.alloc((uint64_t)n + 1, s);
        own.alloc(g.m ? g.m : 1, s);
        ProfScope prof_owners("owners", s, 0.0);
        TC_CUDA(cudaMemsetAsync(e1c.get(), 0, e1c.bytes(), s));
        TC_CUDA(cudaMemsetAsync(e2c.get(), 0, e2c.bytes(), s));
        // owner-label L2 tiles of the CTA items (option "otiles"): col cut into nt equal
        // label tiles; the large x with enough owners get their owners grouped by tile
        nt = g_opt_otiles == 1 ? 0u
             : g_opt_otiles > 1 ? (uint32_t)g_opt_otiles
                                : (uint32_t)((g.m * 4 + ((uint64_t)g_opt_otile_mb << 20) - 1) / ((uint64_t)g_opt_otile_mb << 20));
        if (nt > MAX_OTILES) nt = MAX_OTILES;
        if ((uint64_t)n / (uint64_t)g_opt_owner_lspan >= (1ull << 24)) nt = 0;  // chunk index in 24 bits
        if (nt < 2) nt = 0;
        if (nt) {
          bnd.alloc(nt + 1, s);
          tile_bounds_kernel<<<grid_for(nt + 1, 256), 256, 0, s>>>(g.offs.get(), n, g.m, nt, bnd.get());
          TC_LAUNCH_CHECK();
          lg.alloc(n, s);
          DevBuf<uint64_t> lpre;
          lpre.alloc((uint64_t)n + 1, s);
          large_flag_kernel<<<grid_for(n, 256), 256, 0, s>>>(od_new.get(), n, cap, lg.get());
          TC_LAUNCH_CHECK();
          scan_u32_to_u64(lg.get(), lpre.get(), n, s);
          large_index_kernel<<<grid_for(n, 256), 256, 0, s>>>(od_new.get(), lpre.get(), n, cap, lg.get());
          TC_LAUNCH_CHECK();
          uint64_t nL = 0;
          TC_CUDA(cudaMemcpyAsync(&nL, lpre.get() + n, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
          TC_CUDA(cudaStreamSynchronize(s));
          nlarge_x = nL;
          tcnt.alloc(nL * nt + 1, s);
          toff.alloc(nL * (nt + 1) + 1, s);
          TC_CUDA(cudaMemsetAsync(tcnt.get(), 0, tcnt.bytes(), s));
          nlaunch += 4;
        }
        const unsigned wgrid = grid_for((uint64_t)(ue - ub) * 32, 256, 8);
        // auto: from 2^28 edges (configs[3] count -3.4 ms, configs[4] -33 ms; R-MAT s22 +0.5 ms)
        const bool e2sort = (g_opt_e2sort < 0 ? g.m >= (1ull << 28) : g_opt_e2sort != 0) && !nt && 2 * vbits <= 64;
        DevBuf<uint32_t> e2s;  // E2 edges per source (e2sort)
        if (e2sort) {
          e2s.alloc(n, s);
          TC_CUDA(cudaMemsetAsync(e2s.get(), 0, e2s.bytes(), s));
        }
        owners_count_kernel<<<wgrid, 256, 0, s>>>(g.offs.get(), g.col.get(), od_new.get(), ub, ue, e1c.get(),
                                                  e2c.get(), lg.get(), bnd.get(), nt, nt ? tcnt.get() : nullptr,
                                                  e2sort ? e2s.get() : nullptr);
        TC_LAUNCH_CHECK();
        DevBuf<uint64_t> e2start;
        if (e2sort) {  // group starts of the E2 owners, before e2c becomes the total count
          e2start.alloc((uint64_t)n + 1, s);
          scan_u32_to_u64(e2c.get(), e2start.get(), n, s);
        }
        owners_total_kernel<<<grid_for(n, 256), 256, 0, s>>>(e1c.get(), n, e2c.get());
        TC_LAUNCH_CHECK();
        scan_u32_to_u64(e2c.get(), ooff.get(), n, s);
        owners_cursor_kernel<<<grid_for(n, 256), 256, 0, s>>>(ooff.get(), e1c.get(), n, e2cur.get());
        TC_LAUNCH_CHECK();
        if (nt) {
          const uint64_t tmin = (uint64_t)g_opt_otile_min * nt;
          tile_offsets_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, lg.get(), ooff.get(), nt,
                                                               (uint32_t)std::min<uint64_t>(tmin, 0xffffffffu),
                                                               tcnt.get(), toff.get());
          TC_LAUNCH_CHECK();
          ++nlaunch;
        }
        if (e2sort) {
          DevBuf<uint64_t> e2pos;
          e2pos.alloc((uint64_t)n + 1, s);
          scan_u32_to_u64(e2s.get(), e2pos.get(), n, s);
          uint64_t total = 0;
          TC_CUDA(cudaMemcpyAsync(&total, e2pos.get() + n, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
          TC_CUDA(cudaStreamSynchronize(s));
          DevBuf<uint64_t> k2, t2;
          k2.alloc(total ? total : 1, s);
          t2.alloc(total ? total : 1, s);
          owners_scatter_e2keys_kernel<<<wgrid, 256, 0, s>>>(g.offs.get(), g.col.get(), od_new.get(), ub, ue,
                                                             ooff.get(), e2pos.get(), vbits, own.get(), k2.get());
          TC_LAUNCH_CHECK();
          if (total) {
            const uint64_t *sorted = radix_sort_u64(k2.get(), t2.get(), total, (int)vbits, (int)(2 * vbits), s);
            owners_place_e2_kernel<<<grid_for(total, 256), 256, 0, s>>>(sorted, total, vbits, ooff.get(), e1c.get(),
                                                                       e2start.get(), own.get());
            TC_LAUNCH_CHECK();
          }
          nlaunch += 5;
        } else {
          owners_scatter_kernel<<<wgrid, 256, 0, s>>>(g.offs.get(), g.col.get(), od_new.get(), ub, ue, ooff.get(),
                                                      e2cur.get(), own.get(), lg.get(), bnd.get(), nt,
                                                      nt ? tcnt.get() : nullptr);
          TC_LAUNCH_CHECK();
        }
        nlaunch += 6;
        ow = Owners{ooff.get(), own.get(), (uint32_t)g_opt_owner_span, (uint32_t)g_opt_owner_lspan, 0, 0xffffffffu};
        if (nt) {
          ow.lg = lg.get();
          ow.toff = toff.get();
          ow.nt = nt;
        }
        iub = 0;  // an E2 edge u -> v is counted at v, any label
        iue = n;
      }
      // degree-binned item list (heaviest bin first)
      DevBuf<unsigned long long> hist;  // [0..31] items/bin, [32..63] cursor, [64..66] fetch counters
      hist.alloc(67, s);
      TC_CUDA(cudaMemsetAsync(hist.get(), 0, hist.bytes(), s));
      items_hist_kernel<<<grid_for(iue - iub, 256, 4), 256, 0, s>>>(g.offs.get(), iub, iue, cap, hist.get(), ow);
      TC_LAUNCH_CHECK();
      bin_scan_kernel<<<1, 32, 0, s>>>(hist.get(), hist.get() + 32);
      TC_LAUNCH_CHECK();
      // the item list is scattered before the host reads the bin sizes back (the scatter
      // needs only the device-side cursors), into a buffer sized by the bound
      // sum_u ceil(d~(u)/32) <= m/32 + #{sources with d~ >= 2} <= m/32 + min(#sources, m/2)
      DevBuf<uint64_t> items;
      items.alloc(g.m / SV + std::min<uint64_t>((uint64_t)(iue - iub), g.m / 2) + 1, s);
      {
        uint64_t span = 256ull * SC_PER_THREAD;
        unsigned grid = (unsigned)std::min<uint64_t>((iue - iub + span - 1) / span, (uint64_t)num_sms() * 8);
        items_scatter_kernel<<<grid, 256, 0, s>>>(g.offs.get(), iub, iue, cap, hist.get() + 32, items.get(), ow);
        TC_LAUNCH_CHECK();
        ++nlaunch;
      }
      // CTA items of the tiled x, listed tile by tile ([2nt] total, [2nt+1] fetch counter)
      DevBuf<unsigned long long> titems;
      DevBuf<uint64_t> items_t;
      uint64_t ntiled = 0;
      if (nt) {
        titems.alloc(2 * (uint64_t)nt + 2, s);
        TC_CUDA(cudaMemsetAsync(titems.get(), 0, titems.bytes(), s));
        tile_items_count_kernel<<<grid_for(g.n, 256, 4), 256, 0, s>>>(g.n, lg.get(), toff.get(), nt, ow.lspan,
                                                                         titems.get());
        TC_LAUNCH_CHECK();
        tile_items_scan_kernel<<<1, 1, 0, s>>>(titems.get(), nt);
        TC_LAUNCH_CHECK();
        items_t.alloc(g.m / ow.lspan + nlarge_x * nt + 1, s);
        tile_items_scatter_kernel<<<grid_for(g.n, 256, 4), 256, 0, s>>>(g.n, lg.get(), toff.get(), nt, ow.lspan,
                                                                           titems.get() + nt, items_t.get());
        TC_LAUNCH_CHECK();
        TC_CUDA(cudaMemcpyAsync(&ntiled, titems.get() + 2 * nt, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
        nlaunch += 3;
      }
      std::vector<unsigned long long> hh(32);
      TC_CUDA(cudaMemcpyAsync(hh.data(), hist.get(), 32 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
      TC_CUDA(cudaStreamSynchronize(s));
      uint64_t nitems = 0, nlarge = 0, nheavy = 0;
      const int capbin = 31 - __builtin_clz(cap);  // d < cap  <=>  bin < capbin
      for (int b = 0; b < 32; ++b) {
        nitems += hh[b];
        if (b >= capbin) nlarge += hh[b];
        else if (b >= 5) nheavy += hh[b];  // d~ >= 32: fetched one item at a time
      }
      // warp slices only as large as the longest warp-item list needs (occupancy: an ER
      // graph with d~ < 32 gets 64-word slices, not 1024)
      uint32_t cap_small = 32;
      for (int b = capbin - 1; b >= 0; --b)
        if (hh[b]) {
          cap_small = std::max<uint32_t>(32, std::min<uint32_t>(cap, 1u << (b + 1)));
          break;
        }
      cap_small = fit_cap(cap_small, pv);
      nlaunch += 2;
      if (nitems || ntiled) {
        if (kernel_ms) TC_CUDA(cudaEventRecord(e0, s));
        if (ntiled) {
          size_t smem = LG_SMEM_WORDS * sizeof(uint32_t);
          const void *large_fn = large_kernel(0, true);
          int occ = occupancy(large_fn, LG_THREADS, smem);
          unsigned grid = (unsigned)std::min<uint64_t>(ntiled, (uint64_t)num_sms() * occ);
          ProfScope prof("count_large", s, 0.0);
          launch(large_fn, grid, LG_THREADS, smem, s, (const uint64_t *)g.offs.get(), (const uint32_t *)g.col.get(),
                 (const uint64_t *)items_t.get(), ntiled, titems.get() + 2 * nt + 1, (unsigned long long *)dT.get(), tv,
                 vbits, ow);
          ++nlaunch;
        }
        if (nlarge) {
          size_t smem = LG_SMEM_WORDS * sizeof(uint32_t);
          const void *large_fn = large_kernel(ow.own ? 0 : mode, ow.own != nullptr);
          int occ = occupancy(large_fn, LG_THREADS, smem);
          unsigned grid = (unsigned)std::min<uint64_t>(nlarge, (uint64_t)num_sms() * occ);
          ProfScope prof("count_large", s, 0.0);
          launch(large_fn, grid, LG_THREADS, smem, s, (const uint64_t *)g.offs.get(), (const uint32_t *)g.col.get(),
                 (const uint64_t *)items.get(), nlarge, hist.get() + 64, (unsigned long long *)dT.get(), tv, vbits, ow);
          ++nlaunch;
        }
        uint64_t nsmall = nitems - nlarge;
        if (nsmall) {
          size_t smem = (size_t)CT_WARPS * warp_stride(cap_small, pv) * sizeof(uint32_t);
          // MODE 4: count with every warp-item list <= 32 entries (an ER graph): the
          // short-list-only search dispatch needs 32 registers -> 8 CTAs (64 warps) per SM
          // (a 32-register instantiation for lists <= 256 without the global path was
          // measured 10% slower on R-MAT: issue-bound there, and it spills)
          const bool short_only = g_opt_lean && mode == 0 && cap_small == 32 && g_opt_intersect == 0;
          const int smode = short_only ? 4 : mode;
          const void *small_fn = small_kernel(smode, ow.own != nullptr);
          int occ = occupancy(small_fn, CT_THREADS, smem);
          uint64_t want = (nsmall + CT_WARPS - 1) / CT_WARPS;
          unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(want, (uint64_t)num_sms() * occ));
          ProfScope prof("count_small", s, 0.0);
          // option "vtiles" (classic schedule, count modes, no CTA items): the streamed lists
          // N+(v) in label tiles counted one pass each, so a tile's lists stay in L2
          const uint32_t tiles = (!ow.own && (mode == 0) && !nlarge && g_opt_vtiles > 1) ? (uint32_t)g_opt_vtiles : 1u;
          for (uint32_t t = 0; t < tiles; ++t) {
            Owners owt = ow;
            if (tiles > 1) {
              owt.vlo = (uint32_t)((uint64_t)g.n * t / tiles);
              owt.vhi = (uint32_t)((uint64_t)g.n * (t + 1) / tiles);
              if (t) TC_CUDA(cudaMemsetAsync(hist.get() + 65, 0, 2 * sizeof(unsigned long long), s));
            }
            launch(small_fn, grid, CT_THREADS, smem, s, (const uint64_t *)g.offs.get(), (const uint32_t *)g.col.get(),
                   (const uint64_t *)(items.get() + nlarge), nsmall, nheavy, hist.get() + 65, cap_small,
                   (unsigned long long *)dT.get(), tv, vbits, owt);
          }
          ++nlaunch;
        }
        if (kernel_ms) TC_CUDA(cudaEventRecord(e1, s));
      }
    }
  }
  uint64_t hT = 0;
  if (!d_T) TC_CUDA(cudaMemcpyAsync(&hT, dT.get(), sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
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

// Edge-unit A-order: one unit per directed edge, superiority on the GPU, Algorithm 2 over the
// units on the host (aorder_units, the same greedy as the vertex A-order), active units
// uploaded in bucket order.  Inactive units (d~(v) = 0) are dropped: they add nothing to T.
void build_units(Graph &g) {
  if (g.units_ready) return;
  cudaStream_t s = g.stream;
  const uint32_t n = g.n;
  tc_aorder_params prm = g.aparams;
  if (!g.aparams_set) {
    prm.lambda = 9.682;
    prm.alpha = prm.beta = 0.5;
    prm.bw = nullptr;
    prm.bw_len = 0;
    prm.k = 32;
    prm.order = 0;
  }
  const uint64_t nitems = g.m;
  // superiority per out-degree value (fixed point, λ folded in); max d~ is label-free
  ensure_od(g);
  const uint32_t maxd = g.max_outdeg;
  std::vector<int64_t> htab = superiority_table(maxd, prm);
  DevBuf<int64_t> stab;
  stab.alloc(htab.size(), s);
  TC_CUDA(cudaMemcpyAsync(stab.get(), htab.data(), 8 * htab.size(), cudaMemcpyHostToDevice, s));
  DevBuf<uint64_t> items;
  DevBuf<int64_t> isup;
  DevBuf<uint8_t> iact;
  items.alloc(nitems ? nitems : 1, s);
  isup.alloc(nitems ? nitems : 1, s);
  iact.alloc(nitems ? nitems : 1, s);
  if (nitems) {
    unit_sup_kernel<<<grid_for((uint64_t)n * 32, 256), 256, 0, s>>>(g.offs.get(), g.col.get(), n, stab.get(),
                                                                    items.get(), isup.get(), iact.get());
    TC_LAUNCH_CHECK();
  }
  std::vector<uint64_t> h_items(nitems);
  std::vector<int64_t> h_sup(nitems);
  std::vector<uint8_t> h_act(nitems);
  if (nitems) {
    TC_CUDA(cudaMemcpyAsync(h_items.data(), items.get(), 8 * nitems, cudaMemcpyDeviceToHost, s));
    TC_CUDA(cudaMemcpyAsync(h_sup.data(), isup.get(), 8 * nitems, cudaMemcpyDeviceToHost, s));
    TC_CUDA(cudaMemcpyAsync(h_act.data(), iact.get(), nitems, cudaMemcpyDeviceToHost, s));
  }
  TC_CUDA(cudaStreamSynchronize(s));
  std::vector<uint32_t> pos;
  aorder_units(h_sup, h_act, prm.k, prm.order, pos, g.h_unit_off, g.eq3_units);
  const uint64_t nact = g.h_unit_off.back();
  std::vector<uint64_t> ordered(nact ? nact : 1);
  for (uint64_t i = 0; i < nitems; ++i)
    if (h_act[i]) ordered[pos[i]] = h_items[i];
  g.units.alloc(nact ? nact : 1, s);
  g.unit_off.alloc(g.h_unit_off.size(), s);
  if (nact) TC_CUDA(cudaMemcpyAsync(g.units.get(), ordered.data(), 8 * nact, cudaMemcpyHostToDevice, s));
  TC_CUDA(cudaMemcpyAsync(g.unit_off.get(), g.h_unit_off.data(), 4 * g.h_unit_off.size(), cudaMemcpyHostToDevice, s));
  TC_CUDA(cudaStreamSynchronize(s));  // host vectors must outlive the copies
  g.units_ready = true;
}

void map_edges_canonical(Graph &g, const uint64_t *d_te, uint64_t *d_out) {
  cudaStream_t s = g.stream;
  if (!g.m) return;
  DevBuf<uint32_t> iperm;
  if (!g.identity_perm) {
    iperm.alloc(g.n, s);
    inverse_perm_kernel<<<grid_for(g.n, 256), 256, 0, s>>>(g.perm.get(), g.n, iperm.get());
    TC_LAUNCH_CHECK();
  }
  edge_map_kernel<<<grid_for((uint64_t)g.n * 32, 256), 256, 0, s>>>(
      g.offs.get(), g.col.get(), g.n, g.identity_perm ? nullptr : iperm.get(), g.edges.get(), g.m, g.bits,
      reinterpret_cast<const unsigned long long *>(d_te), d_out);
  TC_LAUNCH_CHECK();
}

void gather_per_vertex(Graph &g, const uint64_t *d_tnew, uint64_t *d_out) {
  if (!g.n) return;
  gather_tv_kernel<<<grid_for(g.n, 256), 256, 0, g.stream>>>(reinterpret_cast<const unsigned long long *>(d_tnew),
                                                             g.identity_perm ? nullptr : g.perm.get(), g.n, d_out);
  TC_LAUNCH_CHECK();
}

// Does a plain count (count-only, bucketed) run the shorter-list schedule?  Option on, binary
// search, and max d~ >= 64 (label-free: from ensure_od when it ran, else from the CSR).
int shorter_schedule(Graph &g) {
  if (!g_opt_shorter || g_opt_intersect != 0 || g.schedule == TC_SCHED_RANGE || g.schedule == TC_SCHED_EDGE_AORDER)
    return 0;
  uint32_t maxd = g.od_ready ? g.max_outdeg : 0;
  if (!g.od_ready && g.n) {
    DevBuf<uint32_t> od_new;
    od_new.alloc(g.n, g.stream);
    od_from_offs_kernel<<<grid_for(g.n, 256), 256, 0, g.stream>>>(g.offs.get(), g.n, od_new.get());
    TC_LAUNCH_CHECK();
    maxd = device_max_u32(od_new.get(), g.n, g.stream);
  }
  return maxd >= 64;
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
    work_kernel<<<grid_for((uint64_t)n * 32, 256), 256, 0, s>>>(g.offs.get(), g.col.get(), n, w.get(), nullptr,
                                                                shorter_schedule(g));
    TC_LAUNCH_CHECK();
  }
  scan_u64(w.get(), pre.get(), n, s);
  bounds_kernel<<<grid_for((uint64_t)world + 1, 256), 256, 0, s>>>(pre.get(), n, world, db.get());
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
    const int shorter = shorter_schedule(g);  // the schedule a plain count runs
    g.alg_model_shorter = shorter;
    work_kernel<<<grid_for((uint64_t)n * 32, 256), 256, 0, s>>>(g.offs.get(), g.col.get(), n, w.get(), sec.get(),
                                                                shorter);
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
