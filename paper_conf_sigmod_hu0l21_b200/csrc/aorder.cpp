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
struct Tournament {
  // node holds the winning leaf (bucket index) or -1; leaves beyond b are empty
  std::vector<int64_t> node;
  size_t P = 1;
  const std::vector<int64_t> *sup = nullptr;
  bool want_max = false;
  bool better(int64_t a, int64_t b) const {
    if (a < 0) return false;
    if (b < 0) return true;
    int64_t x = (*sup)[a], y = (*sup)[b];
    if (x != y) return want_max ? x > y : x < y;
    return a < b;
  }
  void build(size_t b, const std::vector<uint8_t> &alive) {
    P = 1;
    while (P < b) P <<= 1;
    node.assign(2 * P, -1);
    for (size_t i = 0; i < b; ++i) node[P + i] = alive[i] ? (int64_t)i : -1;
    for (size_t i = P - 1; i >= 1; --i) node[i] = better(node[2 * i], node[2 * i + 1]) ? node[2 * i] : node[2 * i + 1];
  }
  void update(size_t leaf, bool alive) {
    size_t i = P + leaf;
    node[i] = alive ? (int64_t)leaf : -1;
    for (i >>= 1; i >= 1; i >>= 1) node[i] = better(node[2 * i], node[2 * i + 1]) ? node[2 * i] : node[2 * i + 1];
  }
  int64_t top() const { return node[1]; }
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
  Tournament q;
  q.sup = &mem_sup;
  if (b) {
    q.want_max = false;                      // line 2: min queue
    q.build(b, alive);
    for (uint32_t v : vmem) {                // line 5
      int64_t bk = q.top();                  // line 6
      members[(size_t)bk * k + fill[bk]++] = v;  // line 7
      mem_sup[bk] += S(od[v]);               // line 8
      if (fill[bk] == k) alive[bk] = 0;
      q.update((size_t)bk, alive[bk]);       // line 9
    }
    q.want_max = true;                       // line 10: max queue
    q.build(b, alive);
    for (uint32_t v : vcomp) {               // line 11
      int64_t bk = q.top();                  // line 12
      members[(size_t)bk * k + fill[bk]++] = v;  // line 13
      mem_sup[bk] += S(od[v]);               // line 14
      if (fill[bk] == k) alive[bk] = 0;
      q.update((size_t)bk, alive[bk]);       // line 15
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
