// aorder.cpp — step a6, A-order (Algorithm 2), host C++.
//
// Algorithm 2 is an inherently sequential greedy: each placement depends on every
// previous one through the bucket priorities ("the priority of the bucket is then
// updated accordingly").  It costs O(|V| log|B|) and the paper counts it as
// preprocessing (Table 5 "total"), so it runs here on the host inside the library,
// fed by the out-degrees the directing kernels produced; the relabel and CSR rebuild that
// follow run on the GPU (reorder.cu).
//
// Priority queues (Alg.2 lines 2 and 10) are realised as a tournament (segment) tree over
// the bucket indices; a bucket that reaches its capacity k is retired from the tree (Q17).
//   phase 1 (line 5-9):   memory-dominated v -> bucket with min (mem_sup, index)
//   phase 2 (line 11-15): computing-dominated v -> bucket with max mem_sup, ties min index
//   relabel (line 16-20): buckets in index order, members in insertion order (Q21);
//                          vertices with d~ = 0 last by id (Q16).
// Memory superiority F_m(d) - λ F_c(d) in 2^-20 fixed point (Q20):
//   F_m = BW(d)^α (Eq.19), F_c = 1/d^β (Eq.20); α = β = 1/2 evaluated literally as
//   sqrt(BW(d)) and sqrt(1/d) (Eq.22); BW(d) = d unless a table is given (Q15).
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <stdexcept>
#include <vector>

#include "../../include/tc.h"

namespace tc {

static int64_t memory_superiority(uint32_t d, const tc_aorder_params &p) {
  double bwv = p.bw ? p.bw[d < p.bw_len ? d : p.bw_len - 1] : (double)d;
  double fm = (p.alpha == 0.5) ? std::sqrt(bwv) : std::pow(bwv, p.alpha);
  double fc = (p.beta == 0.5) ? std::sqrt(1.0 / (double)d) : 1.0 / std::pow((double)d, p.beta);
  return std::llround(std::ldexp(fm - p.lambda * fc, 20));
}

namespace {
// Tournament (segment) tree over the buckets.  Each node stores its winner's key inline,
// so an update touches only the leaf-to-root path (no indirection into mem_sup):
// key = (+mem_sup, index) for the min queue, (-mem_sup, index) for the max queue, the
// lexicographic minimum wins; a full bucket holds the +inf key.
struct Tournament {
  struct Node {
    int64_t key;
    uint32_t idx;
  };
  std::vector<Node> node;
  size_t P = 1;
  bool want_max = false;
  static bool less(const Node &a, const Node &b) { return a.key != b.key ? a.key < b.key : a.idx < b.idx; }
  Node leaf(size_t i, int64_t sup, bool alive) const {
    if (!alive) return Node{INT64_MAX, UINT32_MAX};
    return Node{want_max ? -sup : sup, (uint32_t)i};
  }
  void build(size_t b, const std::vector<int64_t> &sup, const std::vector<uint8_t> &alive) {
    P = 1;
    while (P < b) P <<= 1;
    node.assign(2 * P, Node{INT64_MAX, UINT32_MAX});
    for (size_t i = 0; i < b; ++i) node[P + i] = leaf(i, sup[i], alive[i]);
    for (size_t i = P - 1; i >= 1; --i) node[i] = less(node[2 * i + 1], node[2 * i]) ? node[2 * i + 1] : node[2 * i];
  }
  void update(size_t i, int64_t sup, bool alive) {
    size_t x = P + i;
    node[x] = leaf(i, sup, alive);
    for (x >>= 1; x >= 1; x >>= 1) node[x] = less(node[2 * x + 1], node[2 * x]) ? node[2 * x + 1] : node[2 * x];
  }
  int64_t top() const { return node[1].idx == UINT32_MAX ? -1 : (int64_t)node[1].idx; }
};

// Faster variant when (value, index) packs into 63 bits: one u64 per node (branchless min),
// 4-ary heap layout (half the levels, children in one 32-B run).
struct PackedTournament4 {
  std::vector<uint64_t> node;  // internal nodes [0, nint), leaves [nint, nint + P)
  size_t nint = 0, P = 1;
  int ib = 1;          // index bits
  int64_t off = 0;     // value offset making keys non-negative
  bool want_max = false;
  uint64_t pack(size_t i, int64_t sup, bool alive) const {
    if (!alive) return UINT64_MAX;
    int64_t v = want_max ? -sup : sup;
    return ((uint64_t)(v + off) << ib) | (uint64_t)i;
  }
  void build(size_t b, const std::vector<int64_t> &sup, const std::vector<uint8_t> &alive) {
    P = 1;
    nint = 0;
    while (P < b) {
      nint += P;
      P <<= 2;
    }
    node.assign(nint + P, UINT64_MAX);
    for (size_t i = 0; i < b; ++i) node[nint + i] = pack(i, sup[i], alive[i]);
    for (size_t x = nint; x-- > 0;) node[x] = min4(x);
  }
  uint64_t min4(size_t x) const {
    const uint64_t *c = &node[4 * x + 1];
    uint64_t a = c[0] < c[1] ? c[0] : c[1];
    uint64_t b = c[2] < c[3] ? c[2] : c[3];
    return a < b ? a : b;
  }
  void update(size_t i, int64_t sup, bool alive) {
    size_t x = nint + i;
    node[x] = pack(i, sup, alive);
    while (x > 0) {
      x = (x - 1) >> 2;
      node[x] = min4(x);
    }
  }
  int64_t top() const {
    uint64_t t = node[0];
    return t == UINT64_MAX ? -1 : (int64_t)(t & ((1ull << ib) - 1));
  }
};
}  // namespace

void aorder_host(const std::vector<uint32_t> &od, const tc_aorder_params &p, std::vector<uint32_t> &perm,
                 std::vector<uint32_t> &bucket_off, int64_t &eq3) {
  const size_t n = od.size();
  const uint32_t k = p.k;
  uint32_t maxd = 0;
  for (uint32_t d : od) maxd = std::max(maxd, d);
  // superiority per degree value (table when the degree range is modest)
  std::vector<int64_t> table;
  const bool use_table = maxd <= (1u << 24);
  if (use_table) {
    table.assign((size_t)maxd + 1, 0);
    std::vector<uint8_t> seen((size_t)maxd + 1, 0);
    for (uint32_t d : od) seen[d] = 1;
    for (uint32_t d = 1; d <= maxd; ++d)
      if (seen[d]) table[d] = memory_superiority(d, p);
  }
  auto S = [&](uint32_t d) -> int64_t { return use_table ? table[d] : memory_superiority(d, p); };

  std::vector<uint32_t> vmem, vcomp;  // line 3-4, ascending id
  for (size_t v = 0; v < n; ++v) {
    if (od[v] == 0) continue;
    if (S(od[v]) > 0) vmem.push_back((uint32_t)v);
    else vcomp.push_back((uint32_t)v);
  }
  if (p.order == 1) {  // LPT option (Q18): descending |S|, ties by id
    auto lpt = [&](uint32_t a, uint32_t b) {
      int64_t x = std::llabs(S(od[a])), y = std::llabs(S(od[b]));
      return x != y ? x > y : a < b;
    };
    std::sort(vmem.begin(), vmem.end(), lpt);
    std::sort(vcomp.begin(), vcomp.end(), lpt);
  }
  const size_t nact = vmem.size() + vcomp.size();
  const size_t b = (nact + k - 1) / k;
  std::vector<int64_t> mem_sup(b, 0);        // line 1
  std::vector<uint32_t> fill(b, 0);
  std::vector<uint32_t> members(b * (size_t)k);
  std::vector<uint8_t> alive(b, 1);
  // Phase 1 / phase 2 priority queues.  Packed 4-ary tree when max|mem_sup| and the bucket
  // index fit 63 bits (always for the default parameters), else the generic tree.
  int64_t smax = 0;
  for (uint32_t v : vmem) smax = std::max<int64_t>(smax, std::llabs(S(od[v])));
  for (uint32_t v : vcomp) smax = std::max<int64_t>(smax, std::llabs(S(od[v])));
  const int ib = b > 1 ? 64 - __builtin_clzll((unsigned long long)(b - 1)) : 1;
  const long double bound = (long double)smax * (long double)k * 2.0L + 2.0L;  // |mem_sup| < k smax
  const bool packed = bound * (long double)(1ull << ib) < 9.0e18L;
  auto run = [&](auto &q) {
    q.want_max = false;                      // line 2: min queue
    q.build(b, mem_sup, alive);
    for (uint32_t v : vmem) {                // line 5
      int64_t bk = q.top();                  // line 6
      members[(size_t)bk * k + fill[bk]++] = v;  // line 7
      mem_sup[bk] += S(od[v]);               // line 8
      if (fill[bk] == k) alive[bk] = 0;
      q.update((size_t)bk, mem_sup[bk], alive[bk]);  // line 9
    }
    q.want_max = true;                       // line 10: max queue
    q.build(b, mem_sup, alive);
    for (uint32_t v : vcomp) {               // line 11
      int64_t bk = q.top();                  // line 12
      members[(size_t)bk * k + fill[bk]++] = v;  // line 13
      mem_sup[bk] += S(od[v]);               // line 14
      if (fill[bk] == k) alive[bk] = 0;
      q.update((size_t)bk, mem_sup[bk], alive[bk]);  // line 15
    }
  };
  if (b) {
    if (packed) {
      PackedTournament4 q;
      q.ib = ib;
      q.off = (int64_t)(smax * (int64_t)k + 1);
      run(q);
    } else {
      Tournament q;
      run(q);
    }
  }
  perm.assign(n, 0);
  bucket_off.assign(b + 1, 0);
  uint32_t idx = 0;                          // line 16
  eq3 = 0;
  for (size_t i = 0; i < b; ++i) {           // line 17
    bucket_off[i] = idx;
    for (uint32_t j = 0; j < fill[i]; ++j) perm[members[i * (size_t)k + j]] = idx++;  // line 18-20
    eq3 += std::llabs(mem_sup[i]);           // Eq.3 objective (λ folded into S)
  }
  bucket_off[b] = idx;
  for (size_t v = 0; v < n; ++v)
    if (od[v] == 0) perm[v] = idx++;         // Q16
}

}  // namespace tc
