// internal.h — the tc_graph object and the host-side stage functions of libtc_b200.
#pragma once
#include <stdint.h>

#include <mutex>
#include <vector>

#include "../../include/tc.h"
#include "common.cuh"

namespace tc {

enum GraphState { G_BUILT = 0, G_DIRECTED = 1, G_ORDERED = 2 };

struct StageTimer;  // CUDA-event stage timing (api.cu)

template <typename T>
struct View {  // non-owning slice of a DevBuf
  T *p = nullptr;
  size_t n = 0;
  T *get() const { return p; }
  size_t bytes() const { return n * sizeof(T); }
  void release() { p = nullptr; n = 0; }
};

struct Graph {
  int device = 0;
  cudaStream_t stream = nullptr;
  uint32_t n = 0;
  uint64_t m = 0, samples = 0;
  int bits = 1;  // bits(n-1): packed key (hi << bits) | lo
  GraphState state = G_BUILT;

  // a1-a3: simple undirected graph
  DevBuf<uint64_t> edges;  // m packed keys (u << bits) | v, u < v, ascending
  DevBuf<uint32_t> deg;    // d(v)
  uint32_t max_degree = 0;
  bool max_degree_ready = false;
  bool od_ready = false;  // od / max_outdeg / eq1 are computed lazily (ensure_od)

  // a4-a5: directing
  int direct_rule = -1;
  DevBuf<uint64_t> prim;   // orientation key: u->v iff (prim[u], u) < (prim[v], v)
  DevBuf<uint32_t> od;     // out-degree d~ (original ids)
  DevBuf<uint32_t> sub, dsnap;  // A-direction internals (PAPER only)
  uint32_t levels = 0, subrounds = 0, max_outdeg = 0;
  uint64_t eq1_lo = 0, eq1_hi = 0;

  // a6-a7: ordering + oriented CSR (final labels)
  int reorder_rule = -1;
  bool identity_perm = true;
  DevBuf<uint32_t> perm;          // perm[old] = new (empty if identity)
  std::vector<uint32_t> h_bucket_off;  // A-order buckets (host)
  DevBuf<uint32_t> bucket_off;    // A-order buckets (device)
  int64_t eq3 = -1;
  // oriented CSR in ONE allocation [offs (n+1) u64 | col (m+32) u32] so that one L2
  // access-policy window can keep the offsets (random, 8 B per list) resident
  DevBuf<uint64_t> csr_mem;
  View<uint64_t> offs;            // n+1
  View<uint32_t> col;             // m (+ 32 padding words)
  bool csr_ready = false;

  // a8 schedule
  int schedule = TC_SCHED_AUTO;
  // A-order parameters of the last tc_reorder (bw copied), used by the edge-unit schedule
  tc_aorder_params aparams{};
  std::vector<double> abw;
  bool aparams_set = false;
  // edge-unit A-order (TC_SCHED_EDGE_AORDER): active items in bucket order + offsets
  bool units_ready = false;
  DevBuf<uint64_t> units;
  DevBuf<uint32_t> unit_off;
  std::vector<uint32_t> h_unit_off;
  int64_t eq3_units = -1;

  // results / stats
  uint64_t triangles = 0, wedges = 0, alg_bytes = 0;
  int alg_model_shorter = 0;  // alg_bytes modelled the shorter-list schedule (tc_analyze)
  double ms_build = 0, ms_direct = 0, ms_reorder = 0, ms_count = 0, ms_count_kernel = 0;
  uint64_t count_launches = 0;
};

// build.cu
void build_graph(Graph &g, const uint32_t *d_src, const uint32_t *d_dst, uint64_t M);
void ensure_max_degree(Graph &g);
uint32_t device_max_u32(const uint32_t *a, uint64_t n, cudaStream_t s);
// direct.cu
void direct_graph(Graph &g, int rule);
void ensure_od(Graph &g);  // out-degrees d~ (original ids), max d~, Eq.1 numerator
// reorder.cu
// A-order permutation source: by default the host greedy runs here; tc_reorder_dist runs it
// on rank 0 only and broadcasts pi / bucket_off (AOrderSource filled by api.cu)
struct AOrderSource {
  // produce g.perm (device, n), g.bucket_off (device), g.h_bucket_off, g.eq3 from the
  // host out-degrees; returns false to fall back to the local host greedy
  // h_od[n]: host out-degrees; h_perm[n]: host scratch for pi (both pinned)
  virtual bool produce(Graph &g, const uint32_t *h_od, uint32_t *h_perm, const tc_aorder_params &p) = 0;
  virtual ~AOrderSource() {}
};
void reorder_graph(Graph &g, int rule, const tc_aorder_params &p, AOrderSource *src = nullptr);
void build_oriented_csr(Graph &g);
// aorder.cpp (host, Algorithm 2)
// od[n] -> perm[n] (caller memory, e.g. pinned), bucket_off, Eq.3 objective
void aorder_host(const uint32_t *od, size_t n, const tc_aorder_params &p, uint32_t *perm,
                 std::vector<uint32_t> &bucket_off, int64_t &eq3);
// pinned host staging buffers (grow-only; slot 0 / 1), used under g_pinned_mu (reorder.cu)
uint32_t *pinned_u32(size_t n, int slot);
extern std::mutex g_pinned_mu;
void aorder_units(const std::vector<int64_t> &S, const std::vector<uint8_t> &active, uint32_t k, int order,
                  std::vector<uint32_t> &pos, std::vector<uint32_t> &bucket_off, int64_t &eq3);
std::vector<int64_t> superiority_table(uint32_t maxd, const tc_aorder_params &p);
void aorder_classified(const uint32_t *odm, size_t nmem, const uint32_t *odc, size_t ncomp,
                       const std::vector<int64_t> &table, int64_t smax, int64_t smin1, int64_t smin2, uint32_t k,
                       uint32_t *bmem, uint32_t *rmem, uint32_t *bcomp, uint32_t *rcomp,
                       std::vector<uint32_t> &bucket_off, int64_t &eq3);
// A-order with the classification (lines 3-4) and the relabel (lines 16-20) on the device and
// the sequential greedy on the host: sets g.perm, g.bucket_off, g.h_bucket_off, g.eq3.
// Returns false when not applicable (LPT order: host path).
bool aorder_device(Graph &g, const tc_aorder_params &p);
// count.cu
// d_T: optional device accumulator (zeroed by the caller): the count is added there and not
// read back (returns 0), so a collective can consume it on the stream (tc_count_dist)
uint64_t count_graph(Graph &g, uint32_t u_begin, uint32_t u_end, uint64_t *d_tv /*new labels or null*/,
                     float *kernel_ms, uint64_t *launches, int mode = -1 /*-1: 1 if d_tv else 0; 2 = per-edge*/,
                     unsigned long long *d_T = nullptr);
// per-edge support in CSR positions (final labels) -> canonical order of g.edges (original ids)
void map_edges_canonical(Graph &g, const uint64_t *d_te, uint64_t *d_out);
void gather_per_vertex(Graph &g, const uint64_t *d_tnew, uint64_t *d_out);
void partition_graph(Graph &g, uint32_t world, uint32_t *bounds);
int shorter_schedule(Graph &g);  // a plain count runs the shorter-list schedule
void analyze_graph(Graph &g);
void build_units(Graph &g);  // edge-unit A-order buckets (count.cu)

// options (api.cu)
extern int g_opt_profile;
extern int g_opt_aorder_device;  // A-order classification / relabel on the device (1) or host (0)
extern int g_opt_small_cap;
extern int g_opt_l2_persist;
extern int g_opt_bracket;
extern int g_opt_lean;  // register-lean count_small instantiations
extern int g_opt_extra;  // §5.3 experiment: extra searches per wedge (-1 = production kernel)
extern int g_opt_intersect;  // 0 binary search, 1 sort-merge (count only)
extern int g_opt_peel_red;   // coop peel: RED decrements + frontier scan (1/0, -1 auto)
extern int g_opt_peel_coop;  // A-direction peel as one cooperative launch
extern int g_opt_split;  // orientation split CSR build (original labels)
extern int g_opt_shorter;      // shorter-list owner schedule for count modes
extern int g_opt_owner_span;   // owners per warp item
extern int g_opt_owner_lspan;  // owners per CTA item
extern int g_opt_vtiles;       // classic count: label tiles of the streamed lists (1 = off)
extern int g_opt_cuckoo;       // count-only CTA items: cuckoo hash set of the staged piece
extern int g_opt_e2sort;       // E2 owners grouped by a sort instead of cursor atomics
extern int g_opt_otiles;       // shorter-list CTA items: owner-label L2 tiles (0 = auto, 1 = off)
extern int g_opt_otile_mb;     // auto: MB of col per owner tile
extern int g_opt_otile_min;    // tiled x: >= otile_min * tiles owners

}  // namespace tc
