// count_dev.cuh — device side of the count (a8-a10): search functors, the wedge loop,
// warp / CTA work items and the count kernel templates.  Included by count.cu (schedule,
// host driver) and by the kernel translation units count_small.cu / count_large.cu, which
// instantiate the kernels (split for parallel compilation).  See count.cu for the design.
#pragma once
#include <stdint.h>

#include <type_traits>

#include "common.cuh"

namespace tc {
namespace cnt {


constexpr int CT_THREADS = 256;       // small / range kernels: 8 warps
constexpr int CT_WARPS = CT_THREADS / 32;
constexpr int LG_THREADS = 256;       // large kernel: 8 warps
constexpr int LG_WARPS = LG_THREADS / 32;
constexpr uint32_t PIECE = 4096;      // large kernel: N+(u) piece in shared memory (16 KB)
constexpr uint32_t LG_SUB = 8;        // large kernel: v's per dynamically fetched sub-chunk
#ifndef TC_LG_NB
#define TC_LG_NB 8                    // large kernel, count: 32-wedge steps per gather block
#endif
#ifndef TC_LG_SUB_OWN
#define TC_LG_SUB_OWN 16
#endif
constexpr uint32_t LG_SUB_OWN = TC_LG_SUB_OWN;  // ... of the shorter-list schedule (owners)
#ifndef TC_LG_MINB_OWN
#define TC_LG_MINB_OWN 5
#endif
// bracket tables get 2^TS_* buckets per list element (finer buckets: fewer search steps)
constexpr int TS_W = 2;               // warp items
#ifndef TC_TS_L
#define TC_TS_L 1
#endif
constexpr int TS_L = TC_TS_L;         // CTA items (pieces): the table's size in smem
// CTA items: the piece's table takes all the room left after the padded piece (a shorter
// piece leaves more), up to 2^TS_LMAX buckets per element
#ifndef TC_TS_LMAX
#define TC_TS_LMAX 4
#endif
constexpr int TS_LMAX = TC_TS_LMAX;
#ifndef TC_LG_SMEM_WORDS
#define TC_LG_SMEM_WORDS ((PIECE + 72) + ((PIECE << TS_L) + 64) / 2)
#endif
constexpr uint32_t LG_SMEM_WORDS = TC_LG_SMEM_WORDS;  // piece (+pad) + u16 table / the cuckoo tables
constexpr uint32_t CHUNK = 8;         // worklist entries per atomic fetch
constexpr uint32_t CK_MAXL = (PIECE * 9) / 10;  // cuckoo sets: pieces up to 0.9 x 4096 (2 x 4096 slots)

struct WarpScratch {  // per-warp owner-search tables for one 32-v chunk
  uint64_t vb[32];
  uint32_t pre[32];
  uint32_t v[32];
  uint32_t vcnt[32];  // per-vertex mode: matches per owner v (flushed once per chunk)
};

// Owner lists of the shorter-list schedule (count modes): for every staged list N+(x) the
// lists N+(o) whose elements are binary-searched in it.  Per directed edge u->v the SHORTER
// of N+(u), N+(v) is the streamed one ("the shorter of the two lists
// per edge ... probed into the longer list"): d~(v) <= d~(u): owner v of x = u (E1, the
// paper's Hu pattern); d~(u) < d~(v): owner u of x = v (E2).  own == nullptr: the classic
// schedule, owners of u = N+(u) itself.  span / lspan: owners per warp / CTA item.
struct Owners {
  const uint64_t *off;  // off[x] .. off[x+1]: owners of x in own[]
  const uint32_t *own;
  uint32_t span, lspan;
  // classic schedule, count modes: only v in [vlo, vhi) this pass (L2 tiles of the
  // streamed lists, option "vtiles"); [0, 2^32) = every v
  uint32_t vlo = 0, vhi = 0xffffffffu;
  // CTA items in owner-label L2 tiles (option "otiles"; nt = 0: off).  The owners of a tiled
  // x (lg[x] != ~0) are grouped by the label tile of the owner: tile t of x is
  // own[off[x] + toff[lg[x]*(nt+1) + t] .. + toff[.. + t + 1]); its CTA items are
  // (x << 32) | (t << 24) | chunk, listed tile by tile, so the lists streamed at any moment
  // lie in one label tile (<= a few tens of MB of col) and are re-read from L2, not HBM
  const uint32_t *lg = nullptr;
  const uint32_t *toff = nullptr;
  uint32_t nt = 0;
};

__device__ __forceinline__ uint32_t ldg_u32(const uint32_t *p) { return __ldg(p); }

// Dynamic shared memory of every count kernel.  Searches index it directly so the
// compiler emits 32-bit LDS (not generic loads) for the binary-search steps.
extern __shared__ __align__(128) uint32_t tc_smem[];

// Branchless search: does `w` occur in the ascending list s[0..L), L >= 1? (any memory)
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

__device__ __forceinline__ int ceil_log2(uint32_t L) { return L <= 1 ? 0 : 32 - __clz(L - 1); }

// words of dynamic shared memory per warp in the warp-item kernels
// (slice cap+64 words, u16 bracket table cap+64 entries, PV counters cap words)
__host__ __device__ constexpr uint32_t tab_words(uint32_t cap) { return ((cap << TS_W) + 64) / 2; }
__host__ __device__ constexpr uint32_t warp_stride(uint32_t cap, bool pv) {
  return (cap + 64) + tab_words(cap) + (pv ? cap : 0);
}

static __constant__ int g_bracket = 1;  // bracketed binary search on (option "bracket")
static __constant__ int g_merge = 0;    // sort-merge intersection instead of binary search (option "intersect")
static __constant__ int g_extra = 0;    // MODE 3: extra searches per 8 wedges (option "extra_compute", §5.3 p_c)
static __constant__ uint32_t g_sink_mask = 0;
static __constant__ int g_cuckoo = 64;  // count-only CTA items: cuckoo set of the piece, max evictions per insert (0 = off)

// Cuckoo hash set of a staged piece (count-only CTA items, option "cuckoo"): two tables of
// M = 2^b slots in shared memory, w at T1[h1(w)] or T2[h2(w)] (multiplicative hashes), built
// by the CTA with atomicExch evictions (Alcantara et al.'s GPU cuckoo insertion).  A probe is
// two independent 32-bit shared loads, where the bracketed binary search needs one table
// load and S2 + 1 dependent ones: the count kernel is bound by shared-memory wavefronts.
// Load <= 0.45 of the 2M slots (pieces up to 0.9 M elements); a failed insertion falls back
// to the staged sorted piece.
constexpr uint32_t CK_K1 = 0x9E3779B1u, CK_K2 = 0x85EBCA77u;
constexpr uint32_t CK_EMPTY = 0xffffffffu;  // never a vertex id

// Sort-merge intersection (the strategy the paper compares binary search against, §6.2,
// P:548-550, Fig.10): lane l intersects N+(u) (`list`, ascending, shared or global) with
// its own N+(v) (col[vb .. vb+dv), ascending) by a two-pointer merge.  Every lane walks
// its own pair of lists, so a warp runs as long as its longest merge (the divergence the
// paper's argument for binary search rests on).  Count only.
__device__ __forceinline__ uint32_t merge_lane(const uint32_t *list, uint32_t L, const uint32_t *__restrict__ B,
                                               uint32_t dv) {
  uint32_t cnt = 0;
  if (dv == 0 || L == 0) return 0;
  uint32_t i = 0, j = 0, a = list[0], b = __ldg(B);
  while (true) {
    if (a < b) {
      if (++i == L) break;
      a = list[i];
    } else if (a > b) {
      if (++j == dv) break;
      b = __ldg(B + j);
    } else {
      ++cnt;
      if (++i == L || ++j == dv) break;
      a = list[i];
      b = __ldg(B + j);
    }
  }
  return cnt;
}

// Searchers: does w occur in N+(u)?  `pos` = its shared-memory index (PV counters).
struct GlobalSearch {  // N+(u) in global memory (lists longer than a warp slice)
  const uint32_t *list;
  uint32_t L;
  uint32_t sbase;  // pos = sbase + index of the last element <= w (per-edge positions)
  __device__ __forceinline__ bool operator()(uint32_t w, uint32_t &pos) const {
    const uint32_t *p = list;
    uint32_t len = L;
    while (len > 1) {
      const uint32_t h = len >> 1;
      p = (p[h] <= w) ? p + h : p;
      len -= h;
    }
    pos = sbase + (uint32_t)(p - list);
    return *p == w;
  }
};
// Shared-memory loads through 32-bit shared-window byte addresses computed once per
// item (the generic tc_smem[] form made the compiler rebuild the window base from
// SR_CgaCtaId on every probe: 4 uniform instructions per wedge).
__device__ __forceinline__ uint32_t smem_addr(uint32_t word) {
  return (uint32_t)__cvta_generic_to_shared(tc_smem) + 4u * word;
}
__device__ __forceinline__ uint32_t lds32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t lds16(uint32_t a) {
  unsigned short v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a) : "memory");
  return v;
}

// All searches are branch-free and valid for ANY vertex id w (no [lo, hi] pre-filter is
// needed): a w outside the list's range ends on an element != w (ids are < 2^32 - 1, so
// never equal to the +inf padding).
template <int S>
struct Pow2Search {  // full fixed-depth binary search over the +inf-padded slice
  uint32_t sa;       // byte address of slice[0]
  uint32_t sbase;    // word index of slice[0] (PV positions)
  __device__ __forceinline__ bool operator()(uint32_t w, uint32_t &pos) const {
    uint32_t p = sa;
#pragma unroll
    for (int k = S - 1; k >= 0; --k) {
      const uint32_t q = p + (4u << k);
      p = (lds32(q) <= w) ? q : p;
    }
    pos = sbase + ((p - sa) >> 2);
    return lds32(p) == w;
  }
};
// Bracketed binary search: a per-item table maps the value bucket of w to the first list
// position of that bucket (as a byte offset from slice[0]); the binary search then only
// spans the bucket (S2 = ceil(log2 max bucket occupancy) steps instead of
// ceil(log2 d~(u))).  Elements past the bucket are larger than w (buckets are monotone),
// and the slice carries +inf padding past its end, so no bounds checks are needed.
// Relative table (ABS = false): bucket (w - lo) >> sh over the list's own range [lo, hi]; a
// w outside it maps to bucket B (clamped), whose entry is L: the probes then read the +inf
// padding (2^S2 - 1 < 64 entries past L) and end on an element != w.  Absolute table
// (ABS = true, chosen when the list spans the whole label range at the same bucket width):
// bucket w >> sh over [0, 2^vbits), every label has an entry, no subtraction or clamp.
template <int S2, bool ABS>
struct TabSearch {
  uint32_t sa, ta, lo, sh, B, sbase;  // slice / table byte addresses, table size, PV base
  __device__ __forceinline__ bool operator()(uint32_t w, uint32_t &pos) const {
    const uint32_t b = ABS ? (w >> sh) : min((w - lo) >> sh, B);
    uint32_t p = sa + lds16(ta + 2u * b);
#pragma unroll
    for (int k = S2 - 1; k >= 0; --k) {
      const uint32_t q = p + (4u << k);
      p = (lds32(q) <= w) ? q : p;
    }
    pos = sbase + ((p - sa) >> 2);
    return lds32(p) == w;
  }
};

struct CuckooSearch {
  uint32_t t1, t2;  // byte addresses of the two tables
  uint32_t sh;      // 32 - b
  __device__ __forceinline__ bool operator()(uint32_t w, uint32_t &pos) const {
    pos = 0;  // membership only
    const uint32_t a1 = t1 + (((w * CK_K1) >> sh) << 2);
    const uint32_t a2 = t2 + (((w * CK_K2) >> sh) << 2);
    return (lds32(a1) == w) | (lds32(a2) == w);
  }
};

// Wedge loop of one chunk.  Owner tables hold only the non-empty N+(v) of the chunk
// (K entries: start offset, inclusive wedge prefix); each lane walks its owner forward
// incrementally (its wedge index grows by 32 per step), so locating w's list costs ~1
// shared load per wedge instead of a 5-step search.
// MODE 0: count only.  MODE 1, per-vertex (PV) and MODE 2, per-edge (PE): matches are
// first aggregated in shared memory — per owner v in ws.vcnt, per position of w in N+(u)
// at tc_smem[cbase + pos] — and flushed with one global atomic per distinct vertex (PV) or
// edge (PE) per item (hub vertices would otherwise serialise on atomics).  A triangle
// u -> v -> w (w in N+(u)) adds one to each of its edges (u,v), (u,w), (v,w) in PE mode:
// (u,v) through the owner counter, (u,w) through the position counter (or directly at
// CSR position ebase + index when N+(u) is searched in global memory / a CTA piece), and
// (v,w) directly at the wedge's own CSR position (unique per wedge).  `tv` is the output:
// t[n] (PV) or the support of every CSR position (PE).
// N consecutive 32-wedge steps of one lane (j0, j0 + 32, ...): the N loads are issued back
// to back before any search (memory-level parallelism for the gather; the owner walk stays
// incremental).  The tail is branch-free: indices past `last` are clamped to the last wedge
// (a valid address) and their hits masked (a clamped w must not count twice; +inf would
// match the padding).
template <int N, int MODE, class Search>
__device__ __forceinline__ void wedge_block(uint32_t j0, uint32_t last, const uint32_t *__restrict__ col,
                                            const Search &search, WarpScratch &ws, uint32_t &o, uint32_t &o_end,
                                            const uint32_t *&ob, uint32_t &cnt, uint32_t sbase, uint32_t cbase,
                                            unsigned long long *tv, uint64_t ebase) {
  constexpr bool PV = MODE == 1, PE = MODE == 2;
  uint32_t w[N], ow[N];
  uint64_t ep[PE ? N : 1];  // PE: CSR position of the wedge's (v, w) edge
#pragma unroll
  for (int k = 0; k < N; ++k) {
    const uint32_t j = min(j0 + 32 * k, last);
    while (o_end <= j) {
      const uint32_t o_beg = o_end;
      ++o;
      o_end = ws.pre[o];
      ob = col + ws.vb[o] - o_beg;
    }
    ow[k] = o;
    w[k] = ldg_u32(ob + j);
    if (PE) ep[PE ? k : 0] = (uint64_t)(ob - col) + j;
  }
#pragma unroll
  for (int k = 0; k < N; ++k) {
    uint32_t pos;
    const bool hit = search(w[k], pos) && j0 + 32 * k <= last;
    cnt += hit ? 1u : 0u;
    if (MODE == 3) {  // the paper's balance-point experiment (§5.3): p_c extra
      uint32_t acc = 0;  // searches of the staged list per wedge (g_extra in 1/8 units), results kept alive
      const uint32_t wi = (j0 >> 5) + k;  // 32-wedge step index: warp-uniform extra work
      const int ne = (int)((((uint64_t)wi + 1) * (uint32_t)g_extra) >> 3) - (int)(((uint64_t)wi * (uint32_t)g_extra) >> 3);
      for (int e = 0; e < ne; ++e) {
        uint32_t p2;
        acc += search(w[k] ^ (uint32_t)(e + 1), p2) ? 1u : 0u;
      }
      cnt += acc & g_sink_mask;  // 0 at run time, unknown to the compiler: keeps the searches
    }
    if ((PV || PE) && hit) {
      atomicAdd(&ws.vcnt[ow[k]], 1u);
      if (cbase != 0xffffffffu) atomicAdd(&tc_smem[cbase + (pos - sbase)], 1u);
      else if (PV) atomicAdd(&tv[w[k]], 1ull);
      else atomicAdd(&tv[ebase + (pos - sbase)], 1ull);
      if (PE) atomicAdd(&tv[ep[PE ? k : 0]], 1ull);
    }
  }
}

// N consecutive 32-wedge steps that all lie in ONE owner list (warp-uniform): lane l takes
// wedges base + l + 32k, all valid, read from one pointer with immediate offsets; no owner
// walk, no tail masking (count modes only).
template <int N, int MODE, class Search>
__device__ __forceinline__ void fast_block(const uint32_t *__restrict__ p, const Search &search, uint32_t j0,
                                           uint32_t &cnt) {
  uint32_t w[N];
#pragma unroll
  for (int k = 0; k < N; ++k) {
#ifdef TC_EXP_NOLOAD  // decomposition experiment: searches without the gather (T is wrong)
    w[k] = (uint32_t)(((uintptr_t)(p + 32 * k) >> 2) * 2654435761u) >> 8;
#else
    w[k] = ldg_u32(p + 32 * k);
#endif
  }
#pragma unroll
  for (int k = 0; k < N; ++k) {
    uint32_t pos;
#ifdef TC_EXP_NOSEARCH  // decomposition experiment: gathers without the search (T is wrong)
    const bool hit = w[k] == 0x7fffffffu;
    pos = 0;
    (void)search;
#else
    const bool hit = search(w[k], pos);
#endif
    cnt += hit ? 1u : 0u;
    if (MODE == 3) {  // §5.3 balance-point experiment, as in wedge_block
      uint32_t acc = 0;
      const uint32_t wi = (j0 >> 5) + k;
      const int ne = (int)((((uint64_t)wi + 1) * (uint32_t)g_extra) >> 3) - (int)(((uint64_t)wi * (uint32_t)g_extra) >> 3);
      for (int e = 0; e < ne; ++e) {
        uint32_t p2;
        acc += search(w[k] ^ (uint32_t)(e + 1), p2) ? 1u : 0u;
      }
      cnt += acc & g_sink_mask;
    }
  }
}

// All wedges of one chunk in blocks of NB (8 for CTA items), 4, 2 and 1 steps of 32.  The
// owner of each block's first wedge is tracked warp-uniformly; a block that lies entirely
// in that owner's list (long N+(v): most wedges of a skewed graph) takes fast_block, the
// others walk per lane from there (wedge_block).
// L2 prefetch (PF > 0, CTA items): the lists PF owners ahead of the one being gathered are
// requested into L2 (one 128-B line per lane).  Measured slower on B200 (configs[3] count
// 283 / 298 / 301 / 310 ms at PF = 0 / 1 / 2 / 4): off (TC_PF = 0, compiled out).
#ifndef TC_PF
#define TC_PF 0
#endif
template <int MODE, class Search, int NB = 4, int PF = 0>
__device__ __forceinline__ uint32_t wedge_loop(const uint32_t *__restrict__ col, const Search &search, uint32_t sbase,
                                               uint32_t cbase, uint32_t st_lane, uint32_t total,
                                               WarpScratch &ws, unsigned long long *tv, uint64_t ebase,
                                               uint32_t nown = 0) {
  constexpr bool FAST = MODE == 0 || MODE == 3 || MODE == 4;
  uint32_t cnt = 0;
  uint32_t uo = 0, uo_end = ws.pre[0];
  const uint32_t *uob = col + ws.vb[0];  // element j of the uniform owner's list is uob[j]
  const uint32_t last = total - 1, steps = (total + 31) >> 5, lane = lane_id();
  (void)st_lane;  // (a warp-reduction owner lookup for short lists was measured slower)
  auto pf_list = [&](uint32_t o) {  // warp-uniform o
    if (o >= nown) return;
    const uint32_t b0 = o ? ws.pre[o - 1] : 0u;
    const uintptr_t p0 = (uintptr_t)(col + ws.vb[o]);
    const uintptr_t p1 = p0 + 4ull * (ws.pre[o] - b0);
    for (uintptr_t q = (p0 & ~(uintptr_t)127) + 128ull * lane; q < p1; q += 4096)
      asm volatile("prefetch.global.L2 [%0];" ::"l"(q));
  };
  if (PF)
    for (uint32_t d = 1; d <= (uint32_t)PF; ++d) pf_list(d);
  auto block = [&](auto nconst, uint32_t st) {
    constexpr int N = decltype(nconst)::value;
    const uint32_t base = 32 * st;
    while (uo_end <= base) {  // warp-uniform
      const uint32_t b0 = uo_end;
      ++uo;
      uo_end = ws.pre[uo];
      uob = col + ws.vb[uo] - b0;
      if (PF) pf_list(uo + PF);
    }
    if (FAST && uo_end >= base + 32 * N) {
      fast_block<N, MODE>(uob + base + lane, search, base + lane, cnt);
    } else {
      uint32_t o = uo, o_end = uo_end;
      const uint32_t *ob = uob;
      wedge_block<N, MODE>(base + lane, last, col, search, ws, o, o_end, ob, cnt, sbase, cbase, tv, ebase);
    }
  };
  uint32_t st = 0;
  if (NB == 16)  // (variant: 16 gathers in flight per lane)
    for (; st + 16 <= steps; st += 16) block(std::integral_constant<int, 16>(), st);
  if (NB >= 8)  // CTA items (register budget 48): 8 gathers in flight per lane
    for (; st + 8 <= steps; st += 8) block(std::integral_constant<int, 8>(), st);
  for (; st + 4 <= steps; st += 4) block(std::integral_constant<int, 4>(), st);
  if (st + 2 <= steps) {
    block(std::integral_constant<int, 2>(), st);
    st += 2;
  }
  if (st < steps) block(std::integral_constant<int, 1>(), st);
  return cnt;
}

// Builds the bracket table of the staged list s = tc_smem[sbase .. sbase+L) (warp-wide):
// tab[b] = 4 * (first index whose bucket (s - lo) >> sh is >= b), b in [0, B] with
// B = ((hi - lo) >> sh) + 1 (hi >= the list's last element: the absolute table passes
// lo = 0, hi = 2^vbits - 1); returns ceil(log2(max bucket occupancy)).
__device__ __forceinline__ int build_bracket(uint32_t sbase, uint32_t tbase, uint32_t L, uint32_t lo, uint32_t hi,
                                             uint32_t sh) {
  const uint32_t B = ((hi - lo) >> sh) + 1;
  uint16_t *tab = reinterpret_cast<uint16_t *>(tc_smem + tbase);
  for (uint32_t j = lane_id(); j < L; j += 32) {
    const uint32_t bj = (tc_smem[sbase + j] - lo) >> sh;
    const int bp = j ? (int)((tc_smem[sbase + j - 1] - lo) >> sh) : -1;
    for (int b = bp + 1; b <= (int)bj; ++b) tab[b] = (uint16_t)(4 * j);
  }
  // buckets past the last element's (absolute tables) and the sentinel B: 4L
  for (uint32_t b = ((tc_smem[sbase + L - 1] - lo) >> sh) + 1 + lane_id(); b <= B; b += 32) tab[b] = (uint16_t)(4 * L);
  __syncwarp();
  uint32_t mx = 0;
  for (uint32_t b = lane_id(); b < B; b += 32) mx = max(mx, ((uint32_t)tab[b + 1] - tab[b]) >> 2);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  return ceil_log2(mx);
}

// Warp-built bracket table of the staged slice (S = ceil(log2 L) >= 6): absolute when the
// list spans the whole label range (same bucket width), else relative to [lo, hi]; returns
// S2 and sets sh / abs_t.
__device__ __forceinline__ int warp_table(uint32_t sbase, uint32_t tbase, uint32_t L, uint32_t lo, uint32_t hi,
                                          uint32_t vbits, int S, uint32_t &sh, bool &abs_t) {
  const int span_bits = 32 - __clz(hi - lo);  // bits of (hi - lo)
  abs_t = span_bits >= (int)vbits;
  const int tb = abs_t ? (int)vbits : span_bits;
  const uint32_t tlo = abs_t ? 0u : lo;
  const uint32_t thi = abs_t ? (vbits >= 32 ? 0xffffffffu : (1u << vbits) - 1u) : hi;
  sh = tb > S + TS_W ? (uint32_t)(tb - S - TS_W) : 0u;
  const int S2 = build_bracket(sbase, tbase, L, tlo, thi, sh);
  __syncwarp();
  return S2;
}

// Count the wedges u->v->w of one chunk of up to 32 v's (lane-held `v`, `valid`) whose w
// lies in list[0..L) (w restricted to [lo, hi]).  `padded`: list is the shared-memory copy
// tc_smem[sbase ..] padded with +inf to 2^ceil(log2 L) (+64) entries; tbase != ~0: room
// for a bracket table.  Returns this lane's matches.
template <int MODE, int NB = 4, bool CK = false>
__device__ __forceinline__ uint32_t warp_chunk(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col,
                                               uint32_t v, bool valid, const uint32_t *list, uint32_t sbase,
                                               uint32_t tbase, uint32_t cbase, uint32_t L, bool padded, uint32_t lo,
                                               uint32_t hi, WarpScratch &ws, unsigned long long *tv, uint32_t vidx,
                                               uint64_t ua, uint64_t ebase, uint32_t vbits, int S2pre = -1,
                                               uint32_t shpre = 0, int abspre = 0, uint32_t ck_sh = 0) {
  constexpr bool PV = MODE == 1, PE = MODE == 2;
  const unsigned lane = lane_id();
  uint64_t vb = 0;
  uint32_t dv = 0;
  if (valid) {
    vb = offs[v];
    dv = (uint32_t)(offs[v + 1] - vb);
  }
  const uint32_t inc = warp_inclusive_scan(dv);
  const uint32_t total = __shfl_sync(0xffffffffu, inc, 31);
  const unsigned nz = __ballot_sync(0xffffffffu, dv != 0);
  const uint32_t st_lane = dv ? inc - dv : 0xffffffffu;  // wedge index where this lane's list starts
  if (dv) {
    const unsigned pos = __popc(nz & ((1u << lane) - 1u));
    ws.vb[pos] = vb;
    ws.pre[pos] = inc;
    if (PV) ws.v[pos] = v;
    if (PE) ws.v[pos] = vidx;  // index of v in N+(u): the (u,v) edge is CSR position ua + vidx
  }
  if (PV || PE) ws.vcnt[lane] = 0;
  __syncwarp();
  uint32_t cnt = 0;
  if (MODE == 0 && g_merge) return merge_lane(list, L, col + vb, dv);
  if (CK && MODE == 0 && ck_sh && total) {  // cuckoo hash set at tc_smem[sbase ..] (2 x 2^(32-ck_sh) slots)
    const uint32_t t1 = smem_addr(sbase);
    cnt = wedge_loop<MODE, CuckooSearch, NB, TC_PF>(col, CuckooSearch{t1, t1 + (4u << (32 - ck_sh)), ck_sh}, sbase,
                                                    cbase, st_lane, total, ws, tv, ebase, (uint32_t)__popc(nz));
  } else if (total) {
    const int S = padded ? ceil_log2(L) : 0;
    int S2 = S2pre >= 0 ? S2pre : 99;  // S2pre: table prebuilt by the CTA (large kernel)
    uint32_t sh = shpre;
    bool abs_t = abspre != 0;
    uint32_t tlo = lo, thi = hi;
    if (MODE != 4 && S2pre < 0 && S >= 6 && tbase != 0xffffffffu && g_bracket && total >= 2 * L) {
      S2 = warp_table(sbase, tbase, L, lo, hi, vbits, S, sh, abs_t);
      if (abs_t) tlo = 0;
    }
    if (MODE == 4) {  // every staged list has <= 32 entries (host-checked): 1..5 steps only
      switch (S) {
#define TC_SHORT(k) \
  case k: cnt = wedge_loop<MODE, Pow2Search<k>, NB>(col, Pow2Search<k>{smem_addr(sbase), sbase}, sbase, cbase, st_lane, total, ws, tv, ebase); break;
        TC_SHORT(1) TC_SHORT(2) TC_SHORT(3) TC_SHORT(4) TC_SHORT(5)
#undef TC_SHORT
      }
    } else if (S2 <= 6) {
      switch (S2) {
#define TC_TAB(k)                                                                                            \
  case k:                                                                                                    \
    if (abs_t)                                                                                               \
      cnt = wedge_loop<MODE, TabSearch<k, true>, NB>(                                                        \
          col, TabSearch<k, true>{smem_addr(sbase), smem_addr(tbase), 0u, sh, 0u, sbase}, sbase, cbase, st_lane, \
          total, ws, tv, ebase);                                                                             \
    else                                                                                                     \
      cnt = wedge_loop<MODE, TabSearch<k, false>, NB>(                                                       \
          col, TabSearch<k, false>{smem_addr(sbase), smem_addr(tbase), tlo, sh, ((thi - tlo) >> sh) + 1, sbase}, \
          sbase, cbase, st_lane, total, ws, tv, ebase);                                                       \
    break;
        TC_TAB(0) TC_TAB(1) TC_TAB(2) TC_TAB(3) TC_TAB(4) TC_TAB(5) TC_TAB(6)
#undef TC_TAB
      }
    } else {
      switch (S) {
#define TC_CASE(k) \
  case k: cnt = wedge_loop<MODE, Pow2Search<k>, NB>(col, Pow2Search<k>{smem_addr(sbase), sbase}, sbase, cbase, st_lane, total, ws, tv, ebase); break;
        TC_CASE(1) TC_CASE(2) TC_CASE(3) TC_CASE(4) TC_CASE(5) TC_CASE(6) TC_CASE(7)
        TC_CASE(8) TC_CASE(9) TC_CASE(10) TC_CASE(11) TC_CASE(12) TC_CASE(13) TC_CASE(14)
#undef TC_CASE
        default:
          cnt = wedge_loop<MODE, GlobalSearch, NB>(col, GlobalSearch{list, L, sbase}, sbase, 0xffffffffu, st_lane, total, ws, tv, ebase);
      }
    }
  }
  __syncwarp();
  if (PV && lane < (unsigned)__popc(nz) && ws.vcnt[lane]) atomicAdd(&tv[ws.v[lane]], (unsigned long long)ws.vcnt[lane]);
  if (PE && lane < (unsigned)__popc(nz) && ws.vcnt[lane])
    atomicAdd(&tv[ua + ws.v[lane]], (unsigned long long)ws.vcnt[lane]);
  // the flush reads ws.v / ws.vcnt of other owners: order it before the next chunk's writes
  // (compute-sanitizer racecheck WAR hazard across consecutive chunks of a CTA item)
  if (PV || PE) __syncwarp();
  return cnt;
}

// Shorter-list schedule, warp item: N+(x) staged once in the warp's slice (+inf padded, one
// bracket table for the whole item), then the item's owners own[off[x] + c0 ..] in chunks
// of 32: each owner's list is streamed and every element binary-searched in N+(x).
// Count modes only.
template <int MODE>
__device__ __forceinline__ uint64_t warp_item_owners(const uint64_t *__restrict__ offs,
                                                     const uint32_t *__restrict__ col, uint32_t x, uint32_t c0,
                                                     uint32_t sbase, uint32_t cap, WarpScratch &ws, uint32_t vbits,
                                                     const Owners &ow, uint64_t a, uint32_t L) {
  const unsigned lane = lane_id();
  const uint64_t o0 = ow.off[x];
  const uint32_t C = (uint32_t)(ow.off[x + 1] - o0);
  if (c0 >= C) return 0;
  const uint32_t cend = min(C, c0 + ow.span);
  const uint32_t *list;
  bool padded = false;
  int S2 = -1;
  uint32_t sh = 0;
  bool abs_t = false;
  if (L <= cap) {
    const int SL = ceil_log2(L);
    const uint32_t P = (1u << SL) + (SL >= 6 ? 64u : 0u);  // +64: bracket-search slack
    for (uint32_t j = lane; j < P; j += 32) tc_smem[sbase + j] = j < L ? ldg_u32(col + a + j) : 0xffffffffu;
    __syncwarp();
    list = tc_smem + sbase;
    padded = true;
    if (MODE != 4 && SL >= 6 && g_bracket) {
      S2 = warp_table(sbase, sbase + cap + 64, L, list[0], list[L - 1], vbits, SL, sh, abs_t);
      if (S2 > 6) S2 = -1;
    }
  } else {
    list = col + a;
  }
  const uint32_t lo = list[0], hi = list[L - 1];
  uint32_t cnt = 0;
  for (uint32_t cc = c0; cc < cend; cc += 32) {
    const bool valid = cc + lane < cend;
    const uint32_t v = valid ? ldg_u32(ow.own + o0 + cc + lane) : 0u;
    cnt += warp_chunk<MODE>(offs, col, v, valid, list, sbase, padded && S2 >= 0 ? sbase + cap + 64 : 0xffffffffu,
                            0xffffffffu, L, padded, lo, hi, ws, nullptr, 0, a, a, vbits, S2 >= 0 ? S2 : -2, sh,
                            abs_t ? 1 : 0);
    __syncwarp();  // owner tables reused by the next chunk
  }
  return cnt;
}

// One work item: source u, v's N+(u)[c0 .. c0+32) on one warp; N+(u) is searched in the
// warp's shared slice (staged here, padded with +inf to a power of two) when it fits,
// else in global memory.  Per-warp layout (warp_stride words): slice [cap + 64, +inf
// padded], bracket table [cap + 64], PV only: match counters [cap].
template <int MODE, bool OWN = false>
__device__ __forceinline__ uint64_t warp_item(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col,
                                              uint32_t u, uint32_t c0, uint32_t sbase, uint32_t cap,
                                              WarpScratch &ws, unsigned long long *tv, uint32_t vbits,
                                              const Owners &ow) {
  constexpr bool PV = MODE == 1, PE = MODE == 2;
  const unsigned lane = lane_id();
  const uint64_t a = offs[u];
  const uint32_t L = (uint32_t)(offs[u + 1] - a);
  if (L < 2) return 0;
  if constexpr (OWN) return warp_item_owners<MODE>(offs, col, u, c0, sbase, cap, ws, vbits, ow, a, L);
  if (c0 >= L) return 0;
  const uint32_t *list;
  bool padded = false;
  const uint32_t cbase = ((PV || PE) && L <= cap) ? sbase + (cap + 64) + tab_words(cap) : 0xffffffffu;
  if (L <= cap) {
    const int SL = ceil_log2(L);
    const uint32_t P = (1u << SL) + (SL >= 6 ? 64u : 0u);  // +64: bracket-search slack
    for (uint32_t j = lane; j < P; j += 32) {
      tc_smem[sbase + j] = j < L ? ldg_u32(col + a + j) : 0xffffffffu;
      if ((PV || PE) && j < L) tc_smem[cbase + j] = 0;
    }
    __syncwarp();
    list = tc_smem + sbase;
    padded = true;
  } else {
    list = col + a;
  }
  const uint32_t lo = list[0], hi = list[L - 1];
  bool valid = c0 + lane < L;
  const uint32_t v = valid ? list[c0 + lane] : 0u;
  if (MODE == 0 || MODE == 4) valid = valid && v - ow.vlo < ow.vhi - ow.vlo;  // v-tile pass
  uint32_t cnt = warp_chunk<MODE>(offs, col, v, valid, list, sbase, padded ? sbase + cap + 64 : 0xffffffffu, cbase, L,
                                  padded, lo, hi, ws, tv, c0 + lane, a, a, vbits);
  __syncwarp();  // slice reads done before the next item restages it
  if (PV) {
    uint64_t tot = warp_sum((uint64_t)cnt);
    if (lane == 0 && tot) atomicAdd(&tv[u], (unsigned long long)tot);
    if (cbase != 0xffffffffu) {
      for (uint32_t j = lane; j < L; j += 32) {
        uint32_t c = tc_smem[cbase + j];
        if (c) atomicAdd(&tv[tc_smem[sbase + j]], (unsigned long long)c);
      }
      __syncwarp();
    }
  }
  if (PE && cbase != 0xffffffffu) {  // (u,w) edges: CSR position a + index of w in N+(u)
    for (uint32_t j = lane; j < L; j += 32) {
      const uint32_t c = tc_smem[cbase + j];
      if (c) atomicAdd(&tv[a + j], (unsigned long long)c);
    }
    __syncwarp();
  }
  return cnt;
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
// Work items (u, c0): N+(u) is cut into chunks of SV = 32 v's (warp items, d~(u) < cap) or
// LV = 1024 v's (CTA items, d~(u) >= cap), so one heavy source never serialises on one
// warp.  Items are grouped in floor(log2 d~(u)) bins, heaviest bin first (cf. the
// logarithmic radix binning of P:63); within a bin the order is arbitrary (counts are
// order-independent integers).
constexpr uint32_t SV = 32;
constexpr uint32_t LV = 1024;  // v's per CTA item (4 sub-chunk rounds per warp: fewer re-stagings of N+(u))

__device__ __forceinline__ int deg_bin(uint32_t d) { return 31 - __clz(d); }  // floor(log2 d), d >= 1

// owners of x (count) and the item span, given the staged list length d = d~(x)
__device__ __forceinline__ uint32_t owner_count(const Owners &ow, uint32_t x, uint32_t d) {
  return ow.own ? (uint32_t)(ow.off[x + 1] - ow.off[x]) : d;
}
__device__ __forceinline__ uint32_t items_of(uint32_t d, uint32_t c, uint32_t cap, const Owners &ow) {
  if (d < 2 || c == 0) return 0;
  const uint32_t step = d < cap ? (ow.own ? ow.span : SV) : (ow.own ? ow.lspan : LV);
  return (c + step - 1) / step;
}

// --------------------------------------------------------------- count kernels (a9)
// Warp items; items [0, nheavy) are fetched one at a time, the rest CHUNK at a time.
template <int MODE, bool OWN = false>
__global__ __launch_bounds__(CT_THREADS, MODE == 4 ? 8 : (MODE == 0 || MODE == 3) ? 6 : 4) void count_small_kernel(const uint64_t *__restrict__ offs,
                                                                 const uint32_t *__restrict__ col,
                                                                 const uint64_t *__restrict__ items, uint64_t nitems,
                                                                 uint64_t nheavy, unsigned long long *ctr, uint32_t cap,
                                                                 unsigned long long *T, unsigned long long *tv,
                                                                 uint32_t vbits, Owners ow) {
  __shared__ WarpScratch s_ws[CT_WARPS];
  const uint32_t slice = warp_id() * warp_stride(cap, MODE == 1 || MODE == 2);
  WarpScratch &ws = s_ws[warp_id()];
  uint64_t acc = 0;
  while (true) {  // heavy items, one per fetch
    unsigned long long i = 0;
    if (lane_id() == 0) i = atomicAdd(&ctr[0], 1ull);
    i = __shfl_sync(0xffffffffu, i, 0);
    if (i >= nheavy) break;
    uint64_t it = items[i];
    acc += warp_item<MODE, OWN>(offs, col, (uint32_t)(it >> 32), (uint32_t)it, slice, cap, ws, tv, vbits, ow);
  }
  while (true) {  // light items, CHUNK per fetch
    unsigned long long b = 0;
    if (lane_id() == 0) b = nheavy + atomicAdd(&ctr[1], (unsigned long long)CHUNK);
    b = __shfl_sync(0xffffffffu, b, 0);
    if (b >= nitems) break;
    uint64_t e = min((uint64_t)b + CHUNK, nitems);
    for (uint64_t i = b; i < e; ++i) {
      uint64_t it = items[i];
      acc += warp_item<MODE, OWN>(offs, col, (uint32_t)(it >> 32), (uint32_t)it, slice, cap, ws, tv, vbits, ow);
    }
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

// CTA items (u, c0) of heavy sources: v's N+(u)[c0 .. c0+LV) over 16 warps; N+(u) staged
// piece by piece with a TMA bulk copy (cp.async.bulk + mbarrier complete_tx).
template <int MODE, bool OWN = false>
__global__ __launch_bounds__(LG_THREADS, OWN ? TC_LG_MINB_OWN : 5) void count_large_kernel(const uint64_t *__restrict__ offs,
                                                                 const uint32_t *__restrict__ col,
                                                                 const uint64_t *__restrict__ items, uint64_t nitems,
                                                                 unsigned long long *ctr, unsigned long long *T,
                                                                 unsigned long long *tv, uint32_t vbits, Owners ow) {
  uint32_t *s_piece = tc_smem;  // the piece (alignment slack + padding), then the table
  __shared__ WarpScratch s_ws[LG_WARPS];
  __shared__ uint32_t s_red[LG_WARPS];
  __shared__ __align__(8) uint64_t s_bar;
  __shared__ unsigned long long s_item;
  __shared__ uint32_t s_next;  // next sub-chunk of the current piece
  __shared__ uint32_t s_ckfail;  // cuckoo insertion failed (fall back to the sorted piece)
  WarpScratch &ws = s_ws[warp_id()];
  if (threadIdx.x == 0) mbar_init(&s_bar, 1);
  __syncthreads();
  unsigned phase = 0;
  uint64_t acc = 0;
  while (true) {
    if (threadIdx.x == 0) s_item = atomicAdd(ctr, 1ull);
    __syncthreads();
    unsigned long long item = s_item;
    __syncthreads();
    if (item >= nitems) break;
    const uint64_t it = items[item];
    const uint32_t u = (uint32_t)(it >> 32);
    uint32_t cbeg = (uint32_t)it;
    const uint64_t a = offs[u];
    const uint32_t L = (uint32_t)(offs[u + 1] - a);
    // owners: N+(u) itself (classic) or the shorter-list owners of u (count modes), or
    // one label tile of them (tiled x)
    const uint32_t *olist = OWN ? ow.own + ow.off[u] : col + a;
    uint32_t C = OWN ? (uint32_t)(ow.off[u + 1] - ow.off[u]) : L;
    if (OWN && ow.nt) {
      const uint32_t l = ow.lg[u];
      if (l != 0xffffffffu) {
        const uint32_t *tt = ow.toff + (uint64_t)l * (ow.nt + 1) + ((uint32_t)(it >> 24) & 0xffu);
        const uint32_t t0 = tt[0];
        olist += t0;
        C = tt[1] - t0;
        cbeg = ((uint32_t)it & 0xffffffu) * ow.lspan;
      }
    }
    const uint32_t cend = min(C, cbeg + (OWN ? ow.lspan : LV));
    uint64_t ucnt = 0;
    for (uint32_t p0 = 0; p0 < L; p0 += PIECE) {
      const uint32_t plen = min(PIECE, L - p0);
      uint32_t ck_sh = 0;  // cuckoo set of the piece (count only), 0 = sorted piece
      if (MODE == 0 && g_cuckoo && !g_merge && plen <= CK_MAXL && cbeg < cend) {
        const int b = max(6, ceil_log2((plen * 10 + 8) / 9));  // 2^b >= plen / 0.9
        const uint32_t M = 1u << b;
        for (uint32_t j = threadIdx.x; j < 2 * M; j += LG_THREADS) tc_smem[j] = CK_EMPTY;
        if (threadIdx.x == 0) {
          s_ckfail = 0;
          s_next = 0;
        }
        __syncthreads();
        for (uint32_t j = threadIdx.x; j < plen; j += LG_THREADS) {
          uint32_t x = ldg_u32(col + a + p0 + j);
          uint32_t tb = 0;
          for (int it = 0; it < g_cuckoo && x != CK_EMPTY; ++it) {  // the evicted element moves to its other table
            const uint32_t idx = tb ? M + ((x * CK_K2) >> (32 - b)) : ((x * CK_K1) >> (32 - b));
            x = atomicExch(&tc_smem[idx], x);
            tb ^= 1u;
          }
          if (x != CK_EMPTY) s_ckfail = 1;
        }
        __syncthreads();
        if (!s_ckfail) ck_sh = 32 - b;
        __syncthreads();  // s_ckfail read by every thread before any reset
      }
      uint32_t shift = 0;
      const uint32_t *list = s_piece;
      uint32_t lo = 0, hi = 0;
      int S2 = -1;
      uint32_t sh = 0;
      bool abs_t = false;
      uint32_t tbase = 0;
      if (!ck_sh) {
      // 16-byte aligned bulk copy covering col[a+p0, a+p0+plen)
      const uint64_t first = a + p0;
      const uint64_t abeg = first & ~3ull;             // element index, 16 B aligned
      const uint64_t aend = (first + plen + 3) & ~3ull;
      shift = (uint32_t)(first - abeg);
      if (threadIdx.x == 0) {
        unsigned bytes = (unsigned)((aend - abeg) * 4);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // prior generic reads of the piece
        mbar_expect_tx(&s_bar, bytes);
        tma_bulk_g2s(s_piece, col + abeg, bytes, &s_bar);
      }
      mbar_wait(&s_bar, phase);
      if (threadIdx.x == 0) s_next = 0;  // published by the barrier below
      phase ^= 1u;
      list = s_piece + shift;
      // pad the piece with +inf up to a power of two (+64) for the fixed-depth search; the
      // bracket table starts right after it (u16 entries, 4-byte aligned)
      const uint32_t P = (1u << ceil_log2(plen)) + 64;
      for (uint32_t j = plen + threadIdx.x; j < P; j += LG_THREADS) s_piece[shift + j] = 0xffffffffu;
      __syncthreads();
      tbase = shift + P;
      const uint32_t tcap = (LG_SMEM_WORDS - tbase) * 2u;  // table entries that fit
      lo = list[0];
      hi = list[plen - 1];
      // CTA-wide bracket table of the piece (shared by all warps of the item); absolute
      // (bucket w >> sh over [0, 2^vbits)) when the piece spans the whole label range
      const int S = ceil_log2(plen);
      if (g_bracket && S >= 6) {
        const int span_bits = 32 - __clz(hi - lo);
        abs_t = span_bits >= (int)vbits;
        const uint32_t tlo = abs_t ? 0u : lo;
        const uint32_t thi = abs_t ? (vbits >= 32 ? 0xffffffffu : (1u << vbits) - 1u) : hi;
        // finest bucket width 2^sh whose table (entries 0 .. B, B = (span >> sh) + 1) fits in
        // the room left, at most 2^TS_LMAX buckets per element (fewer search steps S2)
        const uint32_t lim = min(tcap - 2u, 1u << (S + TS_LMAX));
        while (((thi - tlo) >> sh) > lim) ++sh;
        const uint32_t B = ((thi - tlo) >> sh) + 1;
        uint16_t *tab = reinterpret_cast<uint16_t *>(tc_smem + tbase);
        for (uint32_t j = threadIdx.x; j < plen; j += LG_THREADS) {
          const uint32_t bj = (list[j] - tlo) >> sh;
          const int bp = j ? (int)((list[j - 1] - tlo) >> sh) : -1;
          for (int b = bp + 1; b <= (int)bj; ++b) tab[b] = (uint16_t)(4 * j);
        }
        for (uint32_t b = ((hi - tlo) >> sh) + 1 + threadIdx.x; b <= B; b += LG_THREADS) tab[b] = (uint16_t)(4 * plen);
        __syncthreads();
        uint32_t mx = 0;
        for (uint32_t b = threadIdx.x; b < B; b += LG_THREADS) mx = max(mx, ((uint32_t)tab[b + 1] - tab[b]) >> 2);
        mx = warp_max(mx);
        if (lane_id() == 0) s_red[warp_id()] = mx;
        __syncthreads();
        mx = 0;
        for (int w = 0; w < LG_WARPS; ++w) mx = max(mx, s_red[w]);
        S2 = ceil_log2(mx);
        if (S2 > 6) S2 = -1;  // pathological skew: plain fixed-depth search
        __syncthreads();
      }
      }  // sorted piece
      uint32_t cnt = 0;
      // the item's v's in sub-chunks of LG_SUB fetched dynamically by the warps: the
      // wedges behind each v vary widely, and a static 32-v share per warp left warps
      // waiting at the end-of-piece barrier
      while (true) {
        uint32_t sc = 0;
        if (lane_id() == 0) sc = atomicAdd(&s_next, 1u);
        constexpr uint32_t SUB = OWN ? LG_SUB_OWN : LG_SUB;
        const uint32_t c0 = cbeg + __shfl_sync(0xffffffffu, sc, 0) * SUB;
        if (c0 >= cend) break;
        const bool valid = lane_id() < SUB && c0 + lane_id() < cend;
        const uint32_t v = valid ? ldg_u32(olist + c0 + lane_id()) : 0u;
        cnt += warp_chunk<MODE, MODE == 0 ? TC_LG_NB : 4, true>(offs, col, v, valid, list, shift, S2 >= 0 ? tbase : 0xffffffffu, 0xffffffffu, plen,
                                true, lo, hi, ws, tv, c0 + lane_id(), a, a + p0, vbits, S2 >= 0 ? S2 : -2, sh,
                                abs_t ? 1 : 0, ck_sh);
      }
      ucnt += cnt;
      __syncthreads();  // piece fully consumed before the next bulk copy overwrites it
    }
    acc += ucnt;
    if (MODE == 1) {
      uint64_t tot = warp_sum(ucnt);
      if (lane_id() == 0 && tot) atomicAdd(&tv[u], (unsigned long long)tot);
    }
  }
  block_add_u64(acc, T);
}

// RANGE schedule: CTA per bucket of consecutive labels [boff[i], boff[i+1]) ∩ [ub, ue).
template <int MODE>
__global__ __launch_bounds__(CT_THREADS) void count_range_kernel(const uint64_t *__restrict__ offs,
                                                                 const uint32_t *__restrict__ col,
                                                                 const uint32_t *__restrict__ boff, uint32_t kfixed,
                                                                 uint32_t b0, uint32_t nb, uint32_t ub, uint32_t ue,
                                                                 uint32_t cap, unsigned *bucket_ctr,
                                                                 unsigned long long *T, unsigned long long *tv,
                                                                 uint32_t vbits) {
  __shared__ WarpScratch s_ws[CT_WARPS];
  __shared__ uint32_t s_bucket;
  const uint32_t slice = warp_id() * warp_stride(cap, MODE == 1 || MODE == 2);
  WarpScratch &ws = s_ws[warp_id()];
  uint64_t acc = 0;
  while (true) {  // buckets fetched dynamically: a CTA takes the next bucket when done
    __syncthreads();
    if (threadIdx.x == 0) s_bucket = b0 + atomicAdd(bucket_ctr, 1u);
    __syncthreads();
    const uint32_t bi = s_bucket;
    if (bi >= b0 + nb) break;
    uint64_t s0 = boff ? boff[bi] : (uint64_t)bi * kfixed;
    uint64_t s1 = boff ? boff[bi + 1] : (uint64_t)(bi + 1) * kfixed;
    if (s0 < ub) s0 = ub;
    if (s1 > ue) s1 = ue;
    // the bucket's (u, 32-v chunk) items, dealt round-robin to the CTA's warps
    uint32_t t = 0;
    for (uint64_t u = s0; u < s1; ++u) {
      uint32_t L = (uint32_t)(offs[u + 1] - offs[u]);
      if (L < 2) continue;
      uint32_t nit = (L + SV - 1) / SV;
      uint32_t first = (warp_id() + CT_WARPS - (t % CT_WARPS)) % CT_WARPS;
      for (uint32_t c = first; c < nit; c += CT_WARPS)
        acc += warp_item<MODE>(offs, col, (uint32_t)u, c * SV, slice, cap, ws, tv, vbits, Owners{nullptr, nullptr, 0, 0});
      t += nit;
    }
  }
  block_add_u64(acc, T);
}


// per-translation-unit kernel tables (count_small.cu, count_large.cu)
const void *small_kernel(int mode, bool own);
const void *range_kernel(int mode);
const void *large_kernel(int mode, bool own);
// the __constant__ options of each kernel translation unit (current device)
void small_set_constants(int bracket, int merge, int extra, int cuckoo);
void large_set_constants(int bracket, int merge, int extra, int cuckoo);

}  // namespace cnt
}  // namespace tc
