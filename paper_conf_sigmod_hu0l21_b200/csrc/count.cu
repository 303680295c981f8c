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

#include "internal.h"
#include "prims.cuh"

namespace tc {

int g_opt_small_cap = 256;   // power of two: d~ below it -> warp items, else CTA items
int g_opt_bracket = 1;       // bracketed binary search for long staged lists
int g_opt_intersect = 0;     // 0 = binary search (the paper's kernel), 1 = sort-merge (P:548-550 comparison)
int g_opt_lean = 1;          // register-lean short-list count_small instantiation (MODE 4)
int g_opt_extra = -1;        // §5.3 balance-point experiment: extra searches per wedge (-1 off)
int g_opt_l2_persist = 0;    // L2 access-policy window over [offs | col] during counts (off: measured slower overall)

namespace {

constexpr int CT_THREADS = 256;       // small / range kernels: 8 warps
constexpr int CT_WARPS = CT_THREADS / 32;
constexpr int LG_THREADS = 256;       // large kernel: 8 warps
constexpr int LG_WARPS = LG_THREADS / 32;
constexpr uint32_t PIECE = 4096;      // large kernel: N+(u) piece in shared memory (16 KB)
constexpr uint32_t LG_SUB = 8;        // large kernel: v's per dynamically fetched sub-chunk
// bracket tables get 2^TS_* buckets per list element (finer buckets: fewer search steps)
constexpr int TS_W = 2;               // warp items
constexpr int TS_L = 1;               // CTA items (pieces)
constexpr uint32_t LG_SMEM_WORDS = (PIECE + 72) + ((PIECE << TS_L) + 64) / 2;  // piece (+pad) + u16 table
constexpr uint32_t CHUNK = 8;         // worklist entries per atomic fetch

struct WarpScratch {  // per-warp owner-search tables for one 32-v chunk
  uint64_t vb[32];
  uint32_t pre[32];
  uint32_t v[32];
  uint32_t vcnt[32];  // per-vertex mode: matches per owner v (flushed once per chunk)
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

__constant__ int g_bracket = 1;  // bracketed binary search on (option "bracket")
__constant__ int g_merge = 0;    // sort-merge intersection instead of binary search (option "intersect")
__constant__ int g_extra = 0;    // MODE 3: extra searches per 8 wedges (option "extra_compute", §5.3 p_c)
__constant__ uint32_t g_sink_mask = 0;

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
  for (int k = 0; k < N; ++k) w[k] = ldg_u32(p + 32 * k);
#pragma unroll
  for (int k = 0; k < N; ++k) {
    uint32_t pos;
    const bool hit = search(w[k], pos);
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
template <int MODE, class Search, int NB = 4>
__device__ __forceinline__ uint32_t wedge_loop(const uint32_t *__restrict__ col, const Search &search, uint32_t sbase,
                                               uint32_t cbase, uint32_t lo, uint32_t hi, uint32_t total,
                                               WarpScratch &ws, unsigned long long *tv, uint64_t ebase) {
  constexpr bool FAST = MODE == 0 || MODE == 3 || MODE == 4;
  uint32_t cnt = 0;
  uint32_t uo = 0, uo_end = ws.pre[0];
  const uint32_t *uob = col + ws.vb[0];  // element j of the uniform owner's list is uob[j]
  const uint32_t last = total - 1, steps = (total + 31) >> 5, lane = lane_id();
  auto block = [&](auto nconst, uint32_t st) {
    constexpr int N = decltype(nconst)::value;
    const uint32_t base = 32 * st;
    while (uo_end <= base) {  // warp-uniform
      const uint32_t b0 = uo_end;
      ++uo;
      uo_end = ws.pre[uo];
      uob = col + ws.vb[uo] - b0;
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
  if (NB == 8)  // CTA items (register budget 48): 8 gathers in flight per lane
    for (; st + 8 <= steps; st += 8) block(std::integral_constant<int, 8>(), st);
  for (; st + 4 <= steps; st += 4) block(std::integral_constant<int, 4>(), st);
  if (st + 2 <= steps) {
    block(std::integral_constant<int, 2>(), st);
    st += 2;
  }
  if (st < steps) block(std::integral_constant<int, 1>(), st);
  (void)lo;
  (void)hi;
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

// Count the wedges u->v->w of one chunk of up to 32 v's (lane-held `v`, `valid`) whose w
// lies in list[0..L) (w restricted to [lo, hi]).  `padded`: list is the shared-memory copy
// tc_smem[sbase ..] padded with +inf to 2^ceil(log2 L) (+64) entries; tbase != ~0: room
// for a bracket table.  Returns this lane's matches.
template <int MODE, int NB = 4>
__device__ __forceinline__ uint32_t warp_chunk(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col,
                                               uint32_t v, bool valid, const uint32_t *list, uint32_t sbase,
                                               uint32_t tbase, uint32_t cbase, uint32_t L, bool padded, uint32_t lo,
                                               uint32_t hi, WarpScratch &ws, unsigned long long *tv, uint32_t vidx,
                                               uint64_t ua, uint64_t ebase, uint32_t vbits, int S2pre = -1,
                                               uint32_t shpre = 0, int abspre = 0) {
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
  if (total) {
    const int S = padded ? ceil_log2(L) : 0;
    int S2 = S2pre >= 0 ? S2pre : 99;  // S2pre: table prebuilt by the CTA (large kernel)
    uint32_t sh = shpre;
    bool abs_t = abspre != 0;
    uint32_t tlo = lo, thi = hi;
    if (MODE != 4 && S2pre < 0 && S >= 6 && tbase != 0xffffffffu && g_bracket && total >= 2 * L) {
      const int span_bits = 32 - __clz(hi - lo);  // bits of (hi - lo)
      // a list spanning the whole label range gets the absolute table (same bucket width)
      abs_t = span_bits >= (int)vbits;
      const int tb = abs_t ? (int)vbits : span_bits;
      if (abs_t) {
        tlo = 0;
        thi = vbits >= 32 ? 0xffffffffu : (1u << vbits) - 1u;
      }
      sh = tb > S + TS_W ? (uint32_t)(tb - S - TS_W) : 0u;
      S2 = build_bracket(sbase, tbase, L, tlo, thi, sh);
      __syncwarp();
    }
    if (MODE == 4) {  // every staged list has <= 32 entries (host-checked): 1..5 steps only
      switch (S) {
#define TC_SHORT(k) \
  case k: cnt = wedge_loop<MODE, Pow2Search<k>, NB>(col, Pow2Search<k>{smem_addr(sbase), sbase}, sbase, cbase, lo, hi, total, ws, tv, ebase); break;
        TC_SHORT(1) TC_SHORT(2) TC_SHORT(3) TC_SHORT(4) TC_SHORT(5)
#undef TC_SHORT
      }
    } else if (S2 <= 6) {
      switch (S2) {
#define TC_TAB(k)                                                                                            \
  case k:                                                                                                    \
    if (abs_t)                                                                                               \
      cnt = wedge_loop<MODE, TabSearch<k, true>, NB>(                                                        \
          col, TabSearch<k, true>{smem_addr(sbase), smem_addr(tbase), 0u, sh, 0u, sbase}, sbase, cbase, lo, hi, \
          total, ws, tv, ebase);                                                                             \
    else                                                                                                     \
      cnt = wedge_loop<MODE, TabSearch<k, false>, NB>(                                                       \
          col, TabSearch<k, false>{smem_addr(sbase), smem_addr(tbase), tlo, sh, ((thi - tlo) >> sh) + 1, sbase}, \
          sbase, cbase, lo, hi, total, ws, tv, ebase);                                                       \
    break;
        TC_TAB(0) TC_TAB(1) TC_TAB(2) TC_TAB(3) TC_TAB(4) TC_TAB(5) TC_TAB(6)
#undef TC_TAB
      }
    } else {
      switch (S) {
#define TC_CASE(k) \
  case k: cnt = wedge_loop<MODE, Pow2Search<k>, NB>(col, Pow2Search<k>{smem_addr(sbase), sbase}, sbase, cbase, lo, hi, total, ws, tv, ebase); break;
        TC_CASE(1) TC_CASE(2) TC_CASE(3) TC_CASE(4) TC_CASE(5) TC_CASE(6) TC_CASE(7)
        TC_CASE(8) TC_CASE(9) TC_CASE(10) TC_CASE(11) TC_CASE(12) TC_CASE(13) TC_CASE(14)
#undef TC_CASE
        default:
          cnt = wedge_loop<MODE, GlobalSearch, NB>(col, GlobalSearch{list, L, sbase}, sbase, 0xffffffffu, lo, hi, total, ws, tv, ebase);
      }
    }
  }
  __syncwarp();
  if (PV && lane < (unsigned)__popc(nz) && ws.vcnt[lane]) atomicAdd(&tv[ws.v[lane]], (unsigned long long)ws.vcnt[lane]);
  if (PE && lane < (unsigned)__popc(nz) && ws.vcnt[lane])
    atomicAdd(&tv[ua + ws.v[lane]], (unsigned long long)ws.vcnt[lane]);
  return cnt;
}

// One work item: source u, v's N+(u)[c0 .. c0+32) on one warp; N+(u) is searched in the
// warp's shared slice (staged here, padded with +inf to a power of two) when it fits,
// else in global memory.  Per-warp layout (warp_stride words): slice [cap + 64, +inf
// padded], bracket table [cap + 64], PV only: match counters [cap].
template <int MODE>
__device__ __forceinline__ uint64_t warp_item(const uint64_t *__restrict__ offs, const uint32_t *__restrict__ col,
                                              uint32_t u, uint32_t c0, uint32_t sbase, uint32_t cap,
                                              WarpScratch &ws, unsigned long long *tv, uint32_t vbits) {
  constexpr bool PV = MODE == 1, PE = MODE == 2;
  const unsigned lane = lane_id();
  const uint64_t a = offs[u];
  const uint32_t L = (uint32_t)(offs[u + 1] - a);
  if (L < 2 || c0 >= L) return 0;
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
  const bool valid = c0 + lane < L;
  const uint32_t v = valid ? list[c0 + lane] : 0u;
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

__device__ __forceinline__ uint32_t items_of(uint32_t d, uint32_t cap) {
  if (d < 2) return 0;
  return d < cap ? (d + SV - 1) / SV : (d + LV - 1) / LV;
}

__global__ void items_hist_kernel(const uint64_t *__restrict__ offs, uint32_t ub, uint32_t ue, uint32_t cap,
                                  unsigned long long *hist) {
  __shared__ unsigned long long s_h[32];
  if (threadIdx.x < 32) s_h[threadIdx.x] = 0;
  __syncthreads();
  for (uint64_t u = (uint64_t)ub + blockIdx.x * blockDim.x + threadIdx.x; u < ue; u += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t d = (uint32_t)(offs[u + 1] - offs[u]);
    uint32_t it = items_of(d, cap);
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
                                                            uint64_t *__restrict__ items) {
  __shared__ unsigned s_cnt[32];
  __shared__ unsigned long long s_base[32];
  const uint64_t span = 256ull * SC_PER_THREAD;
  for (uint64_t c0 = (uint64_t)ub + blockIdx.x * span; c0 < ue; c0 += (uint64_t)gridDim.x * span) {
    if (threadIdx.x < 32) s_cnt[threadIdx.x] = 0;
    __syncthreads();
    uint32_t off[SC_PER_THREAD], d[SC_PER_THREAD];
#pragma unroll
    for (int i = 0; i < SC_PER_THREAD; ++i) {
      uint64_t u = c0 + (uint64_t)i * 256 + threadIdx.x;
      d[i] = u < ue ? (uint32_t)(offs[u + 1] - offs[u]) : 0u;
      uint32_t it = items_of(d[i], cap);
      off[i] = it ? atomicAdd(&s_cnt[deg_bin(d[i])], it) : 0u;
    }
    __syncthreads();
    if (threadIdx.x < 32) s_base[threadIdx.x] = s_cnt[threadIdx.x] ? atomicAdd(&cursor[threadIdx.x], (unsigned long long)s_cnt[threadIdx.x]) : 0ull;
    __syncthreads();
#pragma unroll
    for (int i = 0; i < SC_PER_THREAD; ++i) {
      uint32_t it = items_of(d[i], cap);
      if (!it) continue;
      uint64_t u = c0 + (uint64_t)i * 256 + threadIdx.x;
      uint64_t p = s_base[deg_bin(d[i])] + off[i];
      uint32_t step = d[i] < cap ? SV : LV;
      for (uint32_t c = 0; c < it; ++c) items[p + c] = (u << 32) | (uint64_t)(c * step);
    }
    __syncthreads();
  }
}

// --------------------------------------------------------------- count kernels (a9)
// Warp items; items [0, nheavy) are fetched one at a time, the rest CHUNK at a time.
template <int MODE>
__global__ __launch_bounds__(CT_THREADS, MODE == 4 ? 8 : (MODE == 0 || MODE == 3) ? 6 : 4) void count_small_kernel(const uint64_t *__restrict__ offs,
                                                                 const uint32_t *__restrict__ col,
                                                                 const uint64_t *__restrict__ items, uint64_t nitems,
                                                                 uint64_t nheavy, unsigned long long *ctr, uint32_t cap,
                                                                 unsigned long long *T, unsigned long long *tv,
                                                                 uint32_t vbits) {
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
    acc += warp_item<MODE>(offs, col, (uint32_t)(it >> 32), (uint32_t)it, slice, cap, ws, tv, vbits);
  }
  while (true) {  // light items, CHUNK per fetch
    unsigned long long b = 0;
    if (lane_id() == 0) b = nheavy + atomicAdd(&ctr[1], (unsigned long long)CHUNK);
    b = __shfl_sync(0xffffffffu, b, 0);
    if (b >= nitems) break;
    uint64_t e = min((uint64_t)b + CHUNK, nitems);
    for (uint64_t i = b; i < e; ++i) {
      uint64_t it = items[i];
      acc += warp_item<MODE>(offs, col, (uint32_t)(it >> 32), (uint32_t)it, slice, cap, ws, tv, vbits);
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
template <int MODE>
__global__ __launch_bounds__(LG_THREADS, 5) void count_large_kernel(const uint64_t *__restrict__ offs,
                                                                 const uint32_t *__restrict__ col,
                                                                 const uint64_t *__restrict__ items, uint64_t nitems,
                                                                 unsigned long long *ctr, unsigned long long *T,
                                                                 unsigned long long *tv, uint32_t vbits) {
  uint32_t *s_piece = tc_smem;  // PIECE + 72 words (alignment slack + padding), then the table
  constexpr uint32_t tbase_lg = PIECE + 72;
  __shared__ WarpScratch s_ws[LG_WARPS];
  __shared__ uint32_t s_red[LG_WARPS];
  __shared__ __align__(8) uint64_t s_bar;
  __shared__ unsigned long long s_item;
  __shared__ uint32_t s_next;  // next sub-chunk of the current piece
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
    const uint32_t u = (uint32_t)(it >> 32), cbeg = (uint32_t)it;
    const uint64_t a = offs[u];
    const uint32_t L = (uint32_t)(offs[u + 1] - a);
    const uint32_t cend = min(L, cbeg + LV);
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
      if (threadIdx.x == 0) s_next = 0;  // published by the barrier below
      phase ^= 1u;
      const uint32_t *list = s_piece + shift;
      {  // pad the piece with +inf up to a power of two (+64) for the fixed-depth search
        const uint32_t P = (1u << ceil_log2(plen)) + 64;
        for (uint32_t j = plen + threadIdx.x; j < P; j += LG_THREADS) s_piece[shift + j] = 0xffffffffu;
        __syncthreads();
      }
      const uint32_t lo = list[0], hi = list[plen - 1];
      // CTA-wide bracket table of the piece (shared by all warps of the item); absolute
      // (bucket w >> sh over [0, 2^vbits)) when the piece spans the whole label range
      int S2 = -1;
      uint32_t sh = 0;
      bool abs_t = false;
      const int S = ceil_log2(plen);
      if (g_bracket && S >= 6) {
        const int span_bits = 32 - __clz(hi - lo);
        abs_t = span_bits >= (int)vbits;
        const uint32_t tlo = abs_t ? 0u : lo;
        const uint32_t thi = abs_t ? (vbits >= 32 ? 0xffffffffu : (1u << vbits) - 1u) : hi;
        const int tb = abs_t ? (int)vbits : span_bits;
        sh = tb > S + TS_L ? (uint32_t)(tb - S - TS_L) : 0u;
        const uint32_t B = ((thi - tlo) >> sh) + 1;
        uint16_t *tab = reinterpret_cast<uint16_t *>(tc_smem + tbase_lg);
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
      uint32_t cnt = 0;
      // the item's v's in sub-chunks of LG_SUB fetched dynamically by the warps: the
      // wedges behind each v vary widely, and a static 32-v share per warp left warps
      // waiting at the end-of-piece barrier
      while (true) {
        uint32_t sc = 0;
        if (lane_id() == 0) sc = atomicAdd(&s_next, 1u);
        const uint32_t c0 = cbeg + __shfl_sync(0xffffffffu, sc, 0) * LG_SUB;
        if (c0 >= cend) break;
        const bool valid = lane_id() < LG_SUB && c0 + lane_id() < cend;
        const uint32_t v = valid ? ldg_u32(col + a + c0 + lane_id()) : 0u;
        cnt += warp_chunk<MODE, MODE == 0 ? 8 : 4>(offs, col, v, valid, list, shift, S2 >= 0 ? tbase_lg : 0xffffffffu, 0xffffffffu, plen,
                                true, lo, hi, ws, tv, c0 + lane_id(), a, a + p0, vbits, S2 >= 0 ? S2 : -2, sh,
                                abs_t ? 1 : 0);
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
        acc += warp_item<MODE>(offs, col, (uint32_t)u, c * SV, slice, cap, ws, tv, vbits);
      t += nit;
    }
  }
  block_add_u64(acc, T);
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

// Per-device setup: the >48 KB dynamic shared-memory opt-in (cudaFuncSetAttribute) and the
// __constant__ options are per device, so both are tracked per device under a mutex.
static std::mutex g_cfg_mu;
struct DeviceCfg {
  bool configured = false;
  int bracket = 1, intersect = 0, extra = -1;
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
  size_t large_smem = LG_SMEM_WORDS * sizeof(uint32_t);
  for (auto fn : {count_large_kernel<0>, count_large_kernel<1>, count_large_kernel<2>})
    TC_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)large_smem));
  int small_max = 200 * 1024;
  for (auto fn : {count_small_kernel<0>, count_small_kernel<1>, count_small_kernel<2>, count_small_kernel<3>,
                  count_small_kernel<4>})
    TC_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, small_max));
  for (auto fn : {count_range_kernel<0>, count_range_kernel<1>, count_range_kernel<2>})
    TC_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, small_max));
  TC_CUDA(cudaFuncSetAttribute(count_bitmap_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               (int)(BM_SMEM_MAX_N / 8)));
  c.configured = true;
}

// kernel attributes + the option constants of the current device, once per change
static void configure_kernels() {
  std::lock_guard<std::mutex> lk(g_cfg_mu);
  DeviceCfg &c = device_cfg();
  configure_kernels_locked(c);
  if (g_opt_extra != c.extra && g_opt_extra >= 0) {
    TC_CUDA(cudaMemcpyToSymbol(g_extra, &g_opt_extra, sizeof(int)));
    c.extra = g_opt_extra;
  }
  if (g_opt_bracket != c.bracket) {
    TC_CUDA(cudaMemcpyToSymbol(g_bracket, &g_opt_bracket, sizeof(int)));
    c.bracket = g_opt_bracket;
  }
  if (g_opt_intersect != c.intersect) {
    TC_CUDA(cudaMemcpyToSymbol(g_merge, &g_opt_intersect, sizeof(int)));
    c.intersect = g_opt_intersect;
  }
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
        auto range_fn = mode == 2 ? count_range_kernel<2> : mode == 1 ? count_range_kernel<1> : count_range_kernel<0>;
        int occ = occupancy((const void *)range_fn, CT_THREADS, smem);
        unsigned grid = (unsigned)std::min<uint64_t>(nb, (uint64_t)num_sms() * occ);
        DevBuf<unsigned> bctr;
        bctr.alloc(1, s);
        TC_CUDA(cudaMemsetAsync(bctr.get(), 0, sizeof(unsigned), s));
        if (kernel_ms) TC_CUDA(cudaEventRecord(e0, s));
        ProfScope prof("count_range", s, 0.0);
        range_fn<<<grid, CT_THREADS, smem, s>>>(g.offs.get(), g.col.get(), boff, k, b0, nb, ub, ue, rcap, bctr.get(),
                                                dT.get(), tv, vbits);
        TC_LAUNCH_CHECK();
        if (kernel_ms) TC_CUDA(cudaEventRecord(e1, s));
        ++nlaunch;
      }
    } else {
      // degree-binned item list (heaviest bin first)
      DevBuf<unsigned long long> hist;  // [0..31] items/bin, [32..63] cursor, [64..66] fetch counters
      hist.alloc(67, s);
      TC_CUDA(cudaMemsetAsync(hist.get(), 0, hist.bytes(), s));
      items_hist_kernel<<<grid_for(ue - ub, 256, 4), 256, 0, s>>>(g.offs.get(), ub, ue, cap, hist.get());
      TC_LAUNCH_CHECK();
      bin_scan_kernel<<<1, 32, 0, s>>>(hist.get(), hist.get() + 32);
      TC_LAUNCH_CHECK();
      // the item list is scattered before the host reads the bin sizes back (the scatter
      // needs only the device-side cursors), into a buffer sized by the bound
      // sum_u ceil(d~(u)/32) <= m/32 + #{sources with d~ >= 2} <= m/32 + min(#sources, m/2)
      DevBuf<uint64_t> items;
      items.alloc(g.m / SV + std::min<uint64_t>((uint64_t)(ue - ub), g.m / 2) + 1, s);
      {
        uint64_t span = 256ull * SC_PER_THREAD;
        unsigned grid = (unsigned)std::min<uint64_t>((ue - ub + span - 1) / span, (uint64_t)num_sms() * 8);
        items_scatter_kernel<<<grid, 256, 0, s>>>(g.offs.get(), ub, ue, cap, hist.get() + 32, items.get());
        TC_LAUNCH_CHECK();
        ++nlaunch;
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
      if (nitems) {
        if (kernel_ms) TC_CUDA(cudaEventRecord(e0, s));
        if (nlarge) {
          size_t smem = LG_SMEM_WORDS * sizeof(uint32_t);
          auto large_fn =
              mode == 2 ? count_large_kernel<2> : mode == 1 ? count_large_kernel<1> : count_large_kernel<0>;
          int occ = occupancy((const void *)large_fn, LG_THREADS, smem);
          unsigned grid = (unsigned)std::min<uint64_t>(nlarge, (uint64_t)num_sms() * occ);
          ProfScope prof("count_large", s, 0.0);
          large_fn<<<grid, LG_THREADS, smem, s>>>(g.offs.get(), g.col.get(), items.get(), nlarge, hist.get() + 64,
                                                   dT.get(), tv, vbits);
          TC_LAUNCH_CHECK();
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
          auto small_fn = short_only  ? count_small_kernel<4>
                          : mode == 3 ? count_small_kernel<3>
                          : mode == 2 ? count_small_kernel<2>
                          : mode == 1 ? count_small_kernel<1>
                                      : count_small_kernel<0>;
          int occ = occupancy((const void *)small_fn, CT_THREADS, smem);
          uint64_t want = (nsmall + CT_WARPS - 1) / CT_WARPS;
          unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(want, (uint64_t)num_sms() * occ));
          ProfScope prof("count_small", s, 0.0);
          small_fn<<<grid, CT_THREADS, smem, s>>>(g.offs.get(), g.col.get(), items.get() + nlarge, nsmall, nheavy,
                                                   hist.get() + 65, cap_small, dT.get(), tv, vbits);
          TC_LAUNCH_CHECK();
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
