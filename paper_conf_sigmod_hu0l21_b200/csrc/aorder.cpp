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
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <cstdint>
#include <memory>
#include <mutex>
#include <stdexcept>
#include <thread>
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

// Sorts a bin's packed keys by (value, bucket index): LSD radix on the value bits below the
// bin boundary only ([lo_bits, shift): the bin fixes the bits above, the low lo_bits are the
// bucket index), stable; then every run of equal values is put in index order (rare, except
// for the initial all-zero bin, which is already in index order).
static void sort_keys(std::vector<uint64_t> &v, std::vector<uint64_t> &tmp, int lo_bits, int shift) {
  const size_t n = v.size();
  if (n < 64) {
    std::sort(v.begin(), v.end());
    return;
  }
  tmp.resize(n);
  uint32_t cnt[256];
  for (int b = lo_bits; b < shift; b += 8) {
    const int w = std::min(8, shift - b);
    const uint64_t mask = (1ull << w) - 1;
    std::fill(cnt, cnt + 256, 0u);
    for (size_t i = 0; i < n; ++i) ++cnt[(v[i] >> b) & mask];
    uint32_t acc = 0;
    for (uint64_t d = 0; d <= mask; ++d) {
      const uint32_t c = cnt[d];
      cnt[d] = acc;
      acc += c;
    }
    for (size_t i = 0; i < n; ++i) tmp[cnt[(v[i] >> b) & mask]++] = v[i];
    v.swap(tmp);
  }
  for (size_t i = 0; i < n;) {
    size_t j = i + 1;
    while (j < n && (v[j] >> lo_bits) == (v[i] >> lo_bits)) ++j;
    if (j - i > 1 && !std::is_sorted(v.begin() + i, v.begin() + j)) std::sort(v.begin() + i, v.begin() + j);
    i = j;
  }
}

// Helper thread that sorts a copy of the NEXT bin while the greedy consumes the current
// one (the bin sorts are ~30% of the sequential greedy).  Keys pushed into that bin after the
// copy was taken (its tail) are sorted and merged in when the bin becomes current, so the
// consumed order is exactly the single-threaded one.
struct PreSorter {
  std::thread th;
  std::atomic<uint64_t> req{0}, done{0};
  std::atomic<bool> stop{false};
  std::vector<uint64_t> keys, tmp;  // the copy, sorted in place by the helper
  int lo_bits = 0, shift = 0;
  size_t bin = SIZE_MAX;            // bin of the submitted copy
  PreSorter() {
    th = std::thread([this] {
      uint64_t seen = 0;
      for (;;) {
        uint64_t r;
        unsigned spins = 0;
        while ((r = req.load(std::memory_order_acquire)) == seen) {
          if (stop.load(std::memory_order_acquire)) return;
          if (++spins > 4096) std::this_thread::yield();
        }
        seen = r;
        sort_keys(keys, tmp, lo_bits, shift);
        done.store(r, std::memory_order_release);
      }
    });
  }
  ~PreSorter() {
    stop.store(true, std::memory_order_release);
    th.join();
  }
  void submit(size_t b, const std::vector<uint64_t> &src, int lo, int sh) {
    keys.assign(src.begin(), src.end());
    lo_bits = lo;
    shift = sh;
    bin = b;
    req.fetch_add(1, std::memory_order_acq_rel);
  }
  void wait() const {
    const uint64_t r = req.load(std::memory_order_relaxed);
    while (done.load(std::memory_order_acquire) != r) {
    }
  }
};

// Monotone bucketed priority queue on the same packed keys.  In both phases only the
// top bucket changes and its packed key only grows (phase 1 adds S > 0 to the min; phase
// 2 adds S <= 0 to the max, i.e. its negated key grows), so the extracted minimum never
// decreases: keys are binned by their high bits, only the lowest non-empty bin is kept as
// an exact binary min-heap (small, cache-resident), higher bins are plain vectors.
struct MonoQueue {
  int shift = 0;
  int lo_bits = 0;  // low key bits below the value (the bucket index)
  uint64_t bin0 = 0;
  std::vector<std::vector<uint64_t>> bins;
  // the current (lowest non-empty) bin, sorted once when it becomes current: it is then
  // consumed in order; keys re-inserted into the current bin (increments smaller than the
  // bin width) go to a small heap beside it.  Exact: the queue pops the same strictly
  // increasing sequence of unique packed keys as a single heap would.
  std::vector<uint64_t> run, tmp;
  size_t rpos = 0;
  std::vector<uint64_t> heap;
  size_t cur = 0;
  double *trace_ns = nullptr;  // TC_AORDER_TRACE: time spent sorting bins
  size_t bin_of(uint64_t pk) const { return (size_t)((pk >> shift) - bin0); }
  static constexpr size_t D = 4;  // 4-ary min-heap, children 4i+1 .. 4i+4
  void sift_down(size_t i) {
    const size_t n = heap.size();
    uint64_t *h = heap.data();
    const uint64_t x = h[i];
    for (;;) {
      const size_t c = D * i + 1;
      if (c >= n) break;
      size_t best = c;
      uint64_t bv = h[c];
      for (size_t j = c + 1; j < n && j < c + D; ++j)
        if (h[j] < bv) {
          bv = h[j];
          best = j;
        }
      if (bv >= x) break;
      h[i] = bv;
      i = best;
    }
    h[i] = x;
  }
  void push(uint64_t x) {
    heap.push_back(x);
    size_t i = heap.size() - 1;
    while (i > 0) {
      const size_t p = (i - 1) / D;
      if (heap[p] <= x) break;
      heap[i] = heap[p];
      i = p;
    }
    heap[i] = x;
  }
  // Sort of the current bin: LSD radix on the value bits below the bin boundary only
  // ([lo_bits, shift): the bin fixes the bits above, the low lo_bits are the bucket index),
  // stable; then every run of equal values is put in index order (rare, except for the
  // initial all-zero bin, which is already in index order)
  void sort_run() { sort_keys(run, tmp, lo_bits, shift); }
  PreSorter *ps = nullptr;  // optional helper thread (large queues)
  std::vector<uint64_t> tail;
  void activate() {  // bin `cur` becomes the sorted run
    if (ps && ps->bin == cur) {
      ps->wait();
      std::vector<uint64_t> &B = bins[cur];
      const size_t P = ps->keys.size();
      tail.assign(B.begin() + P, B.end());
      sort_keys(tail, tmp, lo_bits, shift);
      run.resize(P + tail.size());
      std::merge(ps->keys.begin(), ps->keys.end(), tail.begin(), tail.end(), run.begin());
      B.clear();
      ps->bin = SIZE_MAX;
    } else {
      run.clear();
      run.swap(bins[cur]);
      sort_run();
    }
    rpos = 0;
    if (ps && cur + 1 < bins.size() && bins[cur + 1].size() >= 256) ps->submit(cur + 1, bins[cur + 1], lo_bits, shift);
  }
  void refill() {
    while (rpos == run.size() && heap.empty() && cur + 1 < bins.size()) {
      ++cur;
      if (trace_ns) {
        const auto t0 = std::chrono::steady_clock::now();
        activate();
        *trace_ns += std::chrono::duration<double, std::nano>(std::chrono::steady_clock::now() - t0).count();
      } else {
        activate();
      }
    }
  }
  // keys: packed keys of the alive buckets; max_pk: upper bound of any key ever inserted;
  // step: smallest key increment (packed units).  Bins ~step/8 wide (<= 2^16 bins).
  void build(const std::vector<uint64_t> &keys, uint64_t max_pk, uint64_t step, int low_bits) {
    lo_bits = low_bits;
    uint64_t mn = UINT64_MAX;
    for (uint64_t k : keys) mn = std::min(mn, k);
    if (keys.empty()) mn = 0;
    const int span_bits = 64 - __builtin_clzll((max_pk - mn) | 1);
    const int step_bits = step >= 8 ? 63 - __builtin_clzll(step / 8) : 0;
    shift = std::max(step_bits, std::max(0, span_bits - 16));
    bin0 = mn >> shift;
    bins.assign(((max_pk >> shift) - bin0) + 2, {});
    for (uint64_t k : keys) bins[bin_of(k)].push_back(k);
    cur = 0;
    heap.clear();
    if (ps) {
      ps->wait();
      ps->bin = SIZE_MAX;
    }
    activate();
    refill();
  }
  bool empty() const { return rpos == run.size() && heap.empty(); }
  template <class F>
  void for_each(F f) const {  // every key still in the queue
    for (size_t i = rpos; i < run.size(); ++i) f(run[i]);
    for (uint64_t x : heap) f(x);
    for (size_t b = cur + 1; b < bins.size(); ++b)
      for (uint64_t x : bins[b]) f(x);
  }
  uint64_t top() const {
    const uint64_t a = rpos < run.size() ? run[rpos] : UINT64_MAX;
    const uint64_t b = heap.empty() ? UINT64_MAX : heap[0];
    return a < b ? a : b;
  }
  // the top's key grew to `pk` (alive) or its bucket left the queue (!alive)
  void replace_top(uint64_t pk, bool alive) {
    if (rpos < run.size() && (heap.empty() || run[rpos] < heap[0])) {
      ++rpos;
    } else {
      heap[0] = heap.back();
      heap.pop_back();
      if (!heap.empty()) sift_down(0);
    }
    if (alive) {
      const size_t bi = bin_of(pk);
      if (bi == cur) push(pk);
      else bins[bi].push_back(pk);
    }
    refill();
  }
};
}  // namespace

// Algorithm 2 over arbitrary units (vertices, or the edge units of the per-edge schedule,
// P:638-640): unit i has superiority S[i] (fixed point, λ folded in) and takes part iff
// active[i]; pos[i] = its new index (buckets in index order, members in insertion order;
// inactive units last, in unit order); bucket_off[b+1]; eq3 = Eq.3 objective.
// The O(n) passes around the sequential greedy (classification, relabel) run on all host
// cores: f(lo, hi, t) over T contiguous chunks of [0, n).
template <class F>
static void par_chunks(size_t n, unsigned T, F f) {
  if (T <= 1) {
    f((size_t)0, n, 0u);
    return;
  }
  std::vector<std::thread> th;
  for (unsigned t = 0; t < T; ++t) th.emplace_back([&, t] { f(n * t / T, n * (t + 1) / T, t); });
  for (auto &x : th) x.join();
}
static unsigned host_threads(size_t n) {
  if (n < (1u << 20)) return 1;
  unsigned h = std::thread::hardware_concurrency();
  return std::max(1u, std::min(h ? h : 1u, 32u));
}

// Host workspace of the greedy, kept across calls (grow-only; first-touch page faults of
// ~10 B per unit otherwise cost as much as the greedy itself).  One A-order at a time.
struct AOrderWorkspace {
  std::mutex mu;
  std::vector<uint32_t> vmem, vcomp, bmem, bcomp, rmem, rcomp;  // bucket / rank of vmem[i], vcomp[i]
  std::vector<int64_t> smem, scomp;  // S of vmem[i] / vcomp[i]
};
static AOrderWorkspace &workspace() {
  static AOrderWorkspace w;
  return w;
}
template <class T>
static T *grow(std::vector<T> &v, size_t n) {
  if (v.size() < n) v.resize(n);
  return v.data();
}

// phase timing to stderr when TC_AORDER_TRACE is set (tools/aorder_bench.cpp)
static bool trace_on() {
  static const bool on = std::getenv("TC_AORDER_TRACE") != nullptr;
  return on;
}
static double now_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

// Lines 1-20 of Algorithm 2 after the classification (lines 3-4): memory-dominated units
// (superiority SMEM(i) > 0, i < nmem, in placement order) then computing-dominated ones
// (SCOMP(i) <= 0); records bucket / rank per placement, bucket_off (buckets in index order,
// members in insertion order) and the Eq.3 objective.  smax = max |S|, smin1 = least S > 0,
// smin2 = least nonzero |S| of the computing-dominated units (INT64_MAX when none).
template <class SMF, class SCF>
static void aorder_greedy(size_t nmem, SMF SMEM, size_t ncomp, SCF SCOMP, int64_t smax, int64_t smin1, int64_t smin2,
                          uint32_t k, uint32_t *bmem, uint32_t *rmem, uint32_t *bcomp, uint32_t *rcomp,
                          std::vector<uint32_t> &bucket_off, int64_t &eq3, double *tr) {
  double t2 = 0, sort_ns = 0;
  const size_t nact = nmem + ncomp;
  const size_t b = (nact + k - 1) / k;
  std::vector<int64_t> mem_sup(b, 0);        // line 1
  std::vector<uint32_t> fill(b, 0);
  // insertion record per placement index (sequential writes; the relabel scatters them)
  const int ib = b > 1 ? 64 - __builtin_clzll((unsigned long long)(b - 1)) : 1;
  const long double bound = (long double)smax * (long double)k * 2.0L + 2.0L;  // |mem_sup| < k smax
  const bool packed = bound * (long double)(1ull << ib) < 9.0e18L;
  if (b && packed) {
    // Packed keys ((±mem_sup + off) << ib) | index: a bucket's mem_sup lives only in its key
    // (the popped key plus S << ib is the updated key), so a placement touches the queue,
    // the bucket's fill count and sequential per-unit arrays only.
    const int64_t off = (int64_t)(smax * (int64_t)k + 1);
    const uint64_t imask = (1ull << ib) - 1;
    const uint64_t max_pk = ((uint64_t)(2 * off) << ib) | imask;
    auto pack = [&](size_t i, int64_t sup, bool want_max) {
      return ((uint64_t)((want_max ? -sup : sup) + off) << ib) | (uint64_t)i;
    };
    MonoQueue q;
    if (trace_on()) q.trace_ns = &sort_ns;
    // bin pre-sorting on a helper thread for large queues (identical output)
    std::unique_ptr<PreSorter> presorter;
    if (b >= 4096 && std::thread::hardware_concurrency() >= 2 && !std::getenv("TC_AORDER_NOPRESORT")) {
      presorter.reset(new PreSorter());
      q.ps = presorter.get();
    }
    std::vector<uint64_t> keys;
    keys.reserve(b);
    // One phase of the greedy: unit i takes the bucket at the top of the queue and the
    // bucket's key grows by inc[i] (packed units).  While no re-entered key is pending, the
    // top is the next key of the sorted current bin, so a run of placements is a straight
    // loop over that bin (a grown key lands in a later bin whenever the bin is narrower
    // than the smallest increment); a key re-entering the current bin goes through the
    // queue's small heap and the step-by-step path.  full(pk) records a bucket that left.
    // fill counts as bytes when k < 256 (the bucket counters stay cache-resident)
    std::vector<uint8_t> fill8(k < 256 ? b : 0, 0);
    auto phase = [&](size_t nu, auto inc, uint32_t *brec, uint32_t *rrec, auto full, auto *fl) {
      size_t i = 0;
      while (i < nu) {
        if (q.heap.empty() && q.rpos < q.run.size()) {
          const uint64_t *rp = q.run.data();
          const size_t rsz = q.run.size();
          const size_t jend = std::min(rsz, q.rpos + (nu - i));
          size_t j = q.rpos;
          bool reentered = false;
          for (; j < jend; ++j, ++i) {
            if (j + 16 < rsz) __builtin_prefetch(&fl[rp[j + 16] & imask], 1);
            const uint64_t pk = rp[j];
            const size_t bk = (size_t)(pk & imask);
            const uint32_t r = fl[bk]++;
            brec[i] = (uint32_t)bk;
            rrec[i] = r;
            const uint64_t npk = pk + inc(i);
            if (r + 1 < k) {
              const size_t bi = q.bin_of(npk);
              if (bi == q.cur) {
                q.push(npk);
                reentered = true;
                ++j;
                ++i;
                break;
              }
              q.bins[bi].push_back(npk);
            } else {
              full(bk, npk);
            }
          }
          q.rpos = j;
          if (!reentered) q.refill();
          continue;
        }
        const uint64_t pk = q.top();
        const size_t bk = (size_t)(pk & imask);
        const uint32_t r = fl[bk]++;
        brec[i] = (uint32_t)bk;
        rrec[i] = r;
        const uint64_t npk = pk + inc(i);
        const bool live = r + 1 < k;
        if (!live) full(bk, npk);
        q.replace_top(npk, live);
        ++i;
      }
    };
    for (size_t i = 0; i < b; ++i) keys.push_back(pack(i, 0, false));
    q.build(keys, max_pk, smin1 == INT64_MAX ? 0 : (uint64_t)smin1 << ib, ib);  // line 2: min queue
    // lines 5-9: memory-dominated v -> min bucket (line 6-7), mem_sup += S(v) (line 8), re-queue (line 9)
    auto run_phase = [&](size_t nu, auto inc, uint32_t *brec, uint32_t *rrec, auto full) {
      if (k < 256) phase(nu, inc, brec, rrec, full, fill8.data());
      else phase(nu, inc, brec, rrec, full, fill.data());
    };
    run_phase(
        nmem, [&](size_t i) { return (uint64_t)SMEM(i) << ib; }, bmem, rmem,
        [&](size_t bk, uint64_t npk) { mem_sup[bk] = (int64_t)(npk >> ib) - off; });
    if (k < 256)
      for (size_t i = 0; i < b; ++i) fill[i] = fill8[i];
    q.for_each([&](uint64_t pk) { mem_sup[pk & imask] = (int64_t)(pk >> ib) - off; });
    if (trace_on()) t2 = now_ms();
    keys.clear();
    for (size_t i = 0; i < b; ++i)
      if (fill[i] < k) keys.push_back(pack(i, mem_sup[i], true));
    q.build(keys, max_pk, smin2 == INT64_MAX ? 0 : (uint64_t)smin2 << ib, ib);  // line 10: max queue
    // lines 11-15: computing-dominated v -> max bucket, mem_sup += S(v) <= 0 (its negated key grows)
    run_phase(
        ncomp, [&](size_t i) { return (uint64_t)(-SCOMP(i)) << ib; }, bcomp, rcomp,
        [&](size_t bk, uint64_t npk) { mem_sup[bk] = off - (int64_t)(npk >> ib); });
    if (k < 256)
      for (size_t i = 0; i < b; ++i) fill[i] = fill8[i];
    q.for_each([&](uint64_t pk) { mem_sup[pk & imask] = off - (int64_t)(pk >> ib); });
  } else if (b) {
    // generic tournament tree (mem_sup beyond the packed range)
    std::vector<uint8_t> alive(b, 1);
    Tournament q;
    q.want_max = false;                          // line 2: min queue
    q.build(b, mem_sup, alive);
    for (size_t i = 0; i < nmem; ++i) {          // line 5
      const int64_t bk = q.top();                // line 6
      bmem[i] = (uint32_t)bk;                    // line 7
      rmem[i] = fill[bk]++;
      mem_sup[bk] += SMEM(i);                    // line 8
      if (fill[bk] == k) alive[bk] = 0;
      q.update((size_t)bk, mem_sup[bk], alive[bk]);  // line 9
    }
    q.want_max = true;                           // line 10: max queue
    q.build(b, mem_sup, alive);
    for (size_t i = 0; i < ncomp; ++i) {         // line 11
      const int64_t bk = q.top();                // line 12
      bcomp[i] = (uint32_t)bk;                   // line 13
      rcomp[i] = fill[bk]++;
      mem_sup[bk] += SCOMP(i);                   // line 14
      if (fill[bk] == k) alive[bk] = 0;
      q.update((size_t)bk, mem_sup[bk], alive[bk]);  // line 15
    }
  }
  if (tr) {
    tr[0] = t2;
    tr[1] = sort_ns;
  }
  // line 16-20: bucket offsets; Eq.3 objective (λ folded into S)
  bucket_off.assign(b + 1, 0);
  eq3 = 0;
  for (size_t i = 0; i < b; ++i) {
    bucket_off[i + 1] = bucket_off[i] + fill[i];
    eq3 += std::llabs(mem_sup[i]);
  }
}

template <class SF, class AF>
static void aorder_core(size_t n, SF S, AF active, uint32_t k, int order, uint32_t *perm,
                        std::vector<uint32_t> &bucket_off, int64_t &eq3) {
  AOrderWorkspace &W = workspace();
  std::lock_guard<std::mutex> lock(W.mu);
  const double t0 = trace_on() ? now_ms() : 0;
  double t1 = 0, t3 = 0;
  // line 3-4: V_mem / V_comp in ascending unit index: per-chunk counts (with max |S| and
  // the least nonzero |S| of each class, for the queue's key packing), then placement of
  // each unit and its S, all on the host cores
  const unsigned T = host_threads(n);
  std::vector<size_t> cm(T + 1, 0), cc(T + 1, 0), ci(T + 1, 0);
  std::vector<int64_t> tmax(T, 0), tmin1(T, INT64_MAX), tmin2(T, INT64_MAX);
  par_chunks(n, T, [&](size_t lo, size_t hi, unsigned t) {
    size_t a = 0, c = 0, z = 0;
    int64_t mx = 0, m1 = INT64_MAX, m2 = INT64_MAX;
    for (size_t v = lo; v < hi; ++v) {
      if (!active(v)) {
        ++z;
        continue;
      }
      const int64_t sv = S(v), av = std::llabs(sv);
      mx = std::max(mx, av);
      if (sv > 0) {
        ++a;
        m1 = std::min(m1, av);
      } else {
        ++c;
        if (av) m2 = std::min(m2, av);
      }
    }
    cm[t + 1] = a;
    cc[t + 1] = c;
    ci[t + 1] = z;
    tmax[t] = mx;
    tmin1[t] = m1;
    tmin2[t] = m2;
  });
  int64_t smax = 0, smin1 = INT64_MAX, smin2 = INT64_MAX;  // max |S|; min nonzero |S| per phase
  for (unsigned t = 0; t < T; ++t) {
    cm[t + 1] += cm[t];
    cc[t + 1] += cc[t];
    ci[t + 1] += ci[t];
    smax = std::max(smax, tmax[t]);
    smin1 = std::min(smin1, tmin1[t]);
    smin2 = std::min(smin2, tmin2[t]);
  }
  const size_t nmem = cm[T], ncomp = cc[T];
  uint32_t *vmem = grow(W.vmem, nmem), *vcomp = grow(W.vcomp, ncomp);
  int64_t *smem = grow(W.smem, nmem), *scomp = grow(W.scomp, ncomp);
  par_chunks(n, T, [&](size_t lo, size_t hi, unsigned t) {
    size_t a = cm[t], c = cc[t];
    for (size_t v = lo; v < hi; ++v) {
      if (!active(v)) continue;
      const int64_t sv = S(v);
      if (sv > 0) {
        smem[a] = sv;
        vmem[a++] = (uint32_t)v;
      } else {
        scomp[c] = sv;
        vcomp[c++] = (uint32_t)v;
      }
    }
  });
  if (order == 1) {  // LPT option (Q18): descending |S|, ties by index
    auto lpt = [&](uint32_t a, uint32_t b) {
      int64_t x = std::llabs(S(a)), y = std::llabs(S(b));
      return x != y ? x > y : a < b;
    };
    std::sort(vmem, vmem + nmem, lpt);
    std::sort(vcomp, vcomp + ncomp, lpt);
    for (size_t i = 0; i < nmem; ++i) smem[i] = S(vmem[i]);
    for (size_t i = 0; i < ncomp; ++i) scomp[i] = S(vcomp[i]);
  }
  if (trace_on()) t1 = now_ms();
  uint32_t *bmem = grow(W.bmem, nmem), *rmem = grow(W.rmem, nmem);
  uint32_t *bcomp = grow(W.bcomp, ncomp), *rcomp = grow(W.rcomp, ncomp);
  double tr[2] = {0, 0};
  aorder_greedy(
      nmem, [&](size_t i) { return smem[i]; }, ncomp, [&](size_t i) { return scomp[i]; }, smax, smin1, smin2, k, bmem,
      rmem, bcomp, rcomp, bucket_off, eq3, trace_on() ? tr : nullptr);
  const double t2 = tr[0], sort_ns = tr[1];
  const size_t b = bucket_off.size() - 1;
  if (trace_on()) t3 = now_ms();
  // line 16-20: buckets in index order, members in insertion order (bucket start + rank);
  // inactive units last in unit order (Q16)
  const uint32_t inactive0 = bucket_off[b];
  par_chunks(nmem, T, [&](size_t lo, size_t hi, unsigned) {
    for (size_t i = lo; i < hi; ++i) perm[vmem[i]] = bucket_off[bmem[i]] + rmem[i];
  });
  par_chunks(ncomp, T, [&](size_t lo, size_t hi, unsigned) {
    for (size_t i = lo; i < hi; ++i) perm[vcomp[i]] = bucket_off[bcomp[i]] + rcomp[i];
  });
  par_chunks(n, T, [&](size_t lo, size_t hi, unsigned t) {
    uint32_t idx = inactive0 + (uint32_t)ci[t];
    for (size_t v = lo; v < hi; ++v)
      if (!active(v)) perm[v] = idx++;
  });
  if (trace_on())
    fprintf(stderr, "aorder n=%zu mem=%zu comp=%zu b=%zu: classify %.1f ms, phase1 %.1f, phase2 %.1f (bin sorts %.1f), relabel %.1f\n",
            n, nmem, ncomp, b, t1 - t0, t2 - t1, t3 - t2, sort_ns / 1e6, now_ms() - t3);
}


void aorder_units(const std::vector<int64_t> &Sv, const std::vector<uint8_t> &act, uint32_t k, int order,
                  std::vector<uint32_t> &perm, std::vector<uint32_t> &bucket_off, int64_t &eq3) {
  perm.resize(Sv.size());
  aorder_core(
      Sv.size(), [&](size_t v) -> int64_t { return Sv[v]; }, [&](size_t v) { return act[v] != 0; }, k, order,
      perm.data(), bucket_off, eq3);
}

void aorder_host(const uint32_t *od, size_t n, const tc_aorder_params &p, uint32_t *perm,
                 std::vector<uint32_t> &bucket_off, int64_t &eq3) {
  uint32_t maxd = 0;
  for (size_t v = 0; v < n; ++v) maxd = std::max(maxd, od[v]);
  // superiority per degree value: a table over the degrees up to max d~ when the range is
  // modest (S is evaluated once per degree value, Q20)
  const bool use_table = maxd <= (1u << 24);
  std::vector<int64_t> table;
  if (use_table) {
    table.assign((size_t)maxd + 1, 0);
    for (uint32_t d = 1; d <= maxd; ++d) table[d] = memory_superiority(d, p);
  }
  // d~ = 0: no work, F_c(0) undefined (Q16) -> not active
  aorder_core(
      n, [&](size_t v) -> int64_t { return use_table ? table[od[v]] : memory_superiority(od[v], p); },
      [&](size_t v) { return od[v] != 0; }, p.k, p.order, perm, bucket_off, eq3);
}

// Algorithm 2 over vertices classified on the device (reorder.cu: aorder_device): odm[i] /
// odc[i] = d~ of the i-th memory- / computing-dominated vertex in ascending vertex order
// (lines 3-4), table[d] = S(d).  Records bucket / rank per placement; the relabel (lines
// 16-20) runs on the device.
void aorder_classified(const uint32_t *odm, size_t nmem, const uint32_t *odc, size_t ncomp,
                       const std::vector<int64_t> &table, int64_t smax, int64_t smin1, int64_t smin2, uint32_t k,
                       uint32_t *bmem, uint32_t *rmem, uint32_t *bcomp, uint32_t *rcomp,
                       std::vector<uint32_t> &bucket_off, int64_t &eq3) {
  AOrderWorkspace &W = workspace();
  std::lock_guard<std::mutex> lock(W.mu);
  const double t0 = trace_on() ? now_ms() : 0;
  double tr[2] = {0, 0};
  const int64_t *tab = table.data();
  aorder_greedy(
      nmem, [&](size_t i) { return tab[odm[i]]; }, ncomp, [&](size_t i) { return tab[odc[i]]; }, smax, smin1, smin2,
      k, bmem, rmem, bcomp, rcomp, bucket_off, eq3, trace_on() ? tr : nullptr);
  if (trace_on())
    fprintf(stderr, "aorder (device-classified) mem=%zu comp=%zu b=%zu: phase1 %.1f ms, phase2 %.1f (bin sorts %.1f)\n",
            nmem, ncomp, bucket_off.size() - 1, tr[0] - t0, now_ms() - tr[0], tr[1] / 1e6);
}

std::vector<int64_t> superiority_table(uint32_t maxd, const tc_aorder_params &p) {
  std::vector<int64_t> table((size_t)maxd + 1, 0);
  for (uint32_t d = 1; d <= maxd; ++d) table[d] = memory_superiority(d, p);
  return table;
}

}  // namespace tc
