#include <mutex>
// reorder.cu — steps a6-a7: vertex ordering and the oriented CSR in the new labels.
//
//   NONE    identity ("Original")
//   DEGREE  D-order: descending out-degree d~, ties by id (Q14) — one radix sort of
//           ((max d~ - d~(v)) << bits(n)) | v
//   PAPER   A-order (Algorithm 2) on the host (aorder.cpp), perm and bucket offsets uploaded
// Oriented CSR: each undirected edge {u,v} becomes (π(src), π(dst)) with src the earlier
// endpoint in the directing order; keys (π(src) << b) | π(dst) are radix-sorted,
// giving ascending lists N+(x) (the layout binary search needs); offsets come
// from the run boundaries of π(s) in the same pass that extracts the column array.
#include <vector>

#include "internal.h"
#include "prims.cuh"

namespace tc {

int g_opt_split = 1;

namespace {

__global__ void dorder_keys_kernel(const uint32_t *__restrict__ od, uint32_t n, uint32_t maxod, int bn,
                                   uint64_t *__restrict__ keys) {
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
    keys[v] = ((uint64_t)(maxod - od[v]) << bn) | v;
}

__global__ void perm_from_sorted_kernel(const uint64_t *__restrict__ keys, uint32_t n, uint64_t mask,
                                        uint32_t *__restrict__ perm) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    perm[keys[i] & mask] = (uint32_t)i;
}

template <bool IDENT>
__global__ void orient_keys_kernel(const uint64_t *__restrict__ edges, uint64_t m, int bits,
                                   const uint64_t *__restrict__ prim, const uint32_t *__restrict__ perm,
                                   uint64_t *__restrict__ keys) {
  uint64_t mask = (1ull << bits) - 1;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t k = edges[i];
    uint32_t u = (uint32_t)(k >> bits), v = (uint32_t)(k & mask);  // u < v
    bool ufirst = prim[u] <= prim[v];
    uint32_t s = ufirst ? u : v, t = ufirst ? v : u;
    if (!IDENT) { s = perm[s]; t = perm[t]; }
    keys[i] = ((uint64_t)s << bits) | t;
  }
}

// col[i] = low bits of the sorted (π(s) << b) | π(t) keys; offs from the run boundaries of
// π(s) (every label in a gap gets the boundary index) — no out-degree pass needed.
__global__ void extract_csr_kernel(const uint64_t *__restrict__ keys, uint64_t m, int bits, uint32_t n,
                                   uint32_t *__restrict__ col, uint64_t *__restrict__ offs) {
  const uint64_t mask = (1ull << bits) - 1;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t k = keys[i];
    col[i] = (uint32_t)(k & mask);
    const uint64_t s = k >> bits;
    const uint64_t sp = i ? (keys[i - 1] >> bits) : 0;
    if (i > 0 && s != sp)
      for (uint64_t x = sp + 1; x <= s; ++x) offs[x] = i;  // interior gaps are short
  }
}

// Labels before the first source get 0, after the last source m (long tails, e.g. the
// d~ = 0 vertices that D-order / A-order put last, are filled grid-wide).
__global__ void csr_ends_kernel(const uint64_t *__restrict__ keys, uint64_t m, int bits, uint32_t n,
                                uint64_t *__restrict__ offs) {
  const uint64_t s_first = keys[0] >> bits, s_last = keys[m - 1] >> bits;
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x <= n; x += (uint64_t)gridDim.x * blockDim.x) {
    if (x <= s_first) offs[x] = 0;
    else if (x > s_last) offs[x] = m;
  }
}

// ---- original labels: CSR from the orientation split (forward run F, sorted reversed run R)
// lb[x] = first index of a key with source >= x in a source-sorted key array (x in [0, n]);
// fused with the column fill of the same array: R entry i (source s) lands at
// col[i + LF[s]] (R entries before it + F entries of smaller sources), F entry j at
// col[j + LR[s + 1]] (all R entries of sources <= s precede it: they are smaller targets).
template <bool IS_R>
__global__ void lb_fill_kernel(const uint64_t *__restrict__ keys, uint64_t len, int bits, uint64_t *__restrict__ lb,
                               const uint64_t *__restrict__ other_lb, uint32_t *__restrict__ col) {
  const uint64_t mask = (1ull << bits) - 1;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < len; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t k = keys[i];
    const uint64_t s = k >> bits;
    const uint64_t x0 = i ? (keys[i - 1] >> bits) + 1 : 0;
    for (uint64_t x = x0; x <= s; ++x) lb[x] = i;  // interior gaps are short
    if (IS_R) col[i + other_lb[s]] = (uint32_t)(k & mask);
  }
}
__global__ void lb_tail_kernel(const uint64_t *__restrict__ keys, uint64_t len, int bits, uint32_t n,
                               uint64_t *__restrict__ lb) {
  const uint64_t first = len ? (keys[len - 1] >> bits) + 1 : 0;
  for (uint64_t x = first + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x <= n; x += (uint64_t)gridDim.x * blockDim.x)
    lb[x] = len;
}
__global__ void fill_fwd_kernel(const uint64_t *__restrict__ F, uint64_t nf, int bits,
                                const uint64_t *__restrict__ LR, uint32_t *__restrict__ col) {
  const uint64_t mask = (1ull << bits) - 1;
  for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nf; j += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t k = F[j];
    col[j + LR[(k >> bits) + 1]] = (uint32_t)(k & mask);
  }
}
__global__ void offs_sum_kernel(uint64_t *__restrict__ offs, const uint64_t *__restrict__ LR, uint32_t n) {
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x <= n; x += (uint64_t)gridDim.x * blockDim.x)
    offs[x] += LR[x];
}

}  // namespace

static void alloc_csr(Graph &g) {
  cudaStream_t s = g.stream;
  // [offs | col] in one allocation; col gets 32 words of tail padding (TMA bulk copies may
  // over-read by < 16 B) and starts 16-B aligned
  const uint64_t offs_words = ((uint64_t)g.n + 1 + 1) & ~1ull;
  g.offs.release();
  g.col.release();
  g.csr_mem.alloc(offs_words + (g.m + 32 + 1) / 2, s);
  g.offs = View<uint64_t>{g.csr_mem.get(), (size_t)g.n + 1};
  g.col = View<uint32_t>{reinterpret_cast<uint32_t *>(g.csr_mem.get() + offs_words), (size_t)(g.m + 32)};
  TC_CUDA(cudaMemsetAsync(g.col.get() + g.m, 0xff, 32 * sizeof(uint32_t), s));
}

// Original labels, any non-ID rule: the unique edge keys (a << b) | c, a < c, are already
// sorted; the forward edges (a -> c) stay in that order, and only the reversed ones (c -> a)
// need a STABLE sort on their source bits (b bits of |R| keys instead of all m keys).
// N+(x) = R(x) ++ F(x): every reversed target is < x < every forward target, each run
// ascending, so the lists come out sorted without a merge.
static void build_csr_split(Graph &g) {
  cudaStream_t s = g.stream;
  const uint32_t n = g.n;
  const uint64_t m = g.m;
  const int b = g.bits;
  DevBuf<uint64_t> F, R, tmp;
  F.alloc(m, s);
  R.alloc(m, s);
  const uint64_t nf = split_oriented(g.edges.get(), m, b, g.prim.get(), F.get(), R.get(), s);
  const uint64_t nr = m - nf;
  uint64_t *Rs = R.get();
  if (nr > 1) {
    tmp.alloc(nr, s);
    Rs = radix_sort_u64(R.get(), tmp.get(), nr, b, 2 * b, s);
  }
  alloc_csr(g);
  DevBuf<uint64_t> LR;
  LR.alloc((uint64_t)n + 1, s);
  uint64_t *LF = g.offs.get();
  ProfScope prof("csr_fill", s, 8.0 * m + 4.0 * m + 16.0 * ((double)n + 1));
  if (nf) {
    lb_fill_kernel<false><<<grid_for(nf, 256), 256, 0, s>>>(F.get(), nf, b, LF, nullptr, nullptr);
    TC_LAUNCH_CHECK();
  }
  lb_tail_kernel<<<grid_for((uint64_t)n + 1, 256), 256, 0, s>>>(F.get(), nf, b, n, LF);
  TC_LAUNCH_CHECK();
  if (nr) {
    lb_fill_kernel<true><<<grid_for(nr, 256), 256, 0, s>>>(Rs, nr, b, LR.get(), LF, g.col.get());
    TC_LAUNCH_CHECK();
  }
  lb_tail_kernel<<<grid_for((uint64_t)n + 1, 256), 256, 0, s>>>(Rs, nr, b, n, LR.get());
  TC_LAUNCH_CHECK();
  if (nf) {
    fill_fwd_kernel<<<grid_for(nf, 256), 256, 0, s>>>(F.get(), nf, b, LR.get(), g.col.get());
    TC_LAUNCH_CHECK();
  }
  offs_sum_kernel<<<grid_for((uint64_t)n + 1, 256), 256, 0, s>>>(LF, LR.get(), n);
  TC_LAUNCH_CHECK();
  g.csr_ready = true;
  g.units_ready = false;
}

void build_oriented_csr(Graph &g) {
  cudaStream_t s = g.stream;
  const uint32_t n = g.n;
  const uint64_t m = g.m;
  const int b = g.bits;
  const bool ident = g.identity_perm;
  if (ident && g.direct_rule != TC_DIRECT_ID && m && g_opt_split) {
    build_csr_split(g);
    return;
  }
  DevBuf<uint64_t> keys, tmp;
  keys.alloc(m ? m : 1, s);
  if (m) {
    ProfScope prof("orient_keys", s, 24.0 * m);
    if (ident)
      orient_keys_kernel<true><<<grid_for(m, 256), 256, 0, s>>>(g.edges.get(), m, b, g.prim.get(), nullptr, keys.get());
    else
      orient_keys_kernel<false><<<grid_for(m, 256), 256, 0, s>>>(g.edges.get(), m, b, g.prim.get(), g.perm.get(),
                                                                  keys.get());
    TC_LAUNCH_CHECK();
  }
  uint64_t *sorted = keys.get();
  if (ident && g.direct_rule == TC_DIRECT_ID) {
    // ID order + identity labels: the edge array is already the sorted oriented list
  } else if (ident) {
    // Original labels: the keys are in (min, max) order.  For a source s, its reversed
    // edges (t < s) precede its forward block (t > s) and each group is ascending in t, so a
    // STABLE sort on the source bits alone yields ascending N+(s): b bits instead of 2b.
    tmp.alloc(m ? m : 1, s);
    sorted = radix_sort_u64(keys.get(), tmp.get(), m, b, 2 * b, s);
  } else {
    tmp.alloc(m ? m : 1, s);
    sorted = radix_sort_u64(keys.get(), tmp.get(), m, 0, 2 * b, s);
  }
  alloc_csr(g);
  if (m) {
    ProfScope prof("extract_csr", s, 12.0 * m);
    extract_csr_kernel<<<grid_for(m, 256), 256, 0, s>>>(sorted, m, b, n, g.col.get(), g.offs.get());
    TC_LAUNCH_CHECK();
    csr_ends_kernel<<<grid_for((uint64_t)n + 1, 256), 256, 0, s>>>(sorted, m, b, n, g.offs.get());
    TC_LAUNCH_CHECK();
  } else {
    TC_CUDA(cudaMemsetAsync(g.offs.get(), 0, g.offs.bytes(), s));
  }
  g.csr_ready = true;
  g.units_ready = false;
}

// Pinned host staging buffers for the A-order round trip (grow-only; the driver keeps
// them for the process lifetime).
std::mutex g_pinned_mu;
uint32_t *pinned_u32(size_t n, int slot) {
  static uint32_t *buf[8] = {nullptr};
  static size_t cap[8] = {0};
  if (cap[slot] < n) {
    if (buf[slot]) TC_CUDA(cudaFreeHost(buf[slot]));
    buf[slot] = nullptr;
    cap[slot] = 0;
    TC_CUDA(cudaMallocHost((void **)&buf[slot], n * sizeof(uint32_t)));
    cap[slot] = n;
  }
  return buf[slot];
}

namespace {
// ---- A-order classification / relabel on the device (Algorithm 2 lines 3-4 and 16-20)
constexpr uint32_t AO_SH_BINS = 2048;  // d~ histogram: shared-memory bins, global above
__global__ void ao_hist_kernel(const uint32_t *__restrict__ od, uint32_t n, uint32_t maxd,
                               unsigned long long *__restrict__ hist) {
  __shared__ unsigned s_h[AO_SH_BINS];
  for (uint32_t i = threadIdx.x; i < AO_SH_BINS; i += blockDim.x) s_h[i] = 0;
  __syncthreads();
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t d = od[v];
    if (d < AO_SH_BINS) atomicAdd(&s_h[d], 1u);
    else atomicAdd(&hist[d], 1ull);
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < AO_SH_BINS && i <= maxd; i += blockDim.x)
    if (s_h[i]) atomicAdd(&hist[i], (unsigned long long)s_h[i]);
}
// class flags: fm = memory-dominated (S > 0), fc = computing-dominated (S <= 0), fi = d~ = 0
__global__ void ao_class_kernel(const uint32_t *__restrict__ od, uint32_t n, const int64_t *__restrict__ tab,
                                uint32_t *__restrict__ fm, uint32_t *__restrict__ fc, uint32_t *__restrict__ fi) {
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t d = od[v];
    const bool act = d != 0;
    const bool mem = act && tab[d] > 0;
    fm[v] = mem;
    fc[v] = act && !mem;
    fi[v] = !act;
  }
}
// odm / odc: d~ of the memory- / computing-dominated vertices in ascending vertex order
__global__ void ao_compact_kernel(const uint32_t *__restrict__ od, uint32_t n, const uint32_t *__restrict__ fm,
                                  const uint32_t *__restrict__ fc, const uint64_t *__restrict__ pm,
                                  const uint64_t *__restrict__ pc, uint32_t *__restrict__ odm,
                                  uint32_t *__restrict__ odc) {
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    if (fm[v]) odm[pm[v]] = od[v];
    else if (fc[v]) odc[pc[v]] = od[v];
  }
}
// pi: bucket start + insertion rank of every placed vertex; inactive vertices last, in id order
__global__ void ao_relabel_kernel(uint32_t n, const uint32_t *__restrict__ fm, const uint32_t *__restrict__ fc,
                                  const uint64_t *__restrict__ pm, const uint64_t *__restrict__ pc,
                                  const uint64_t *__restrict__ pi, const uint32_t *__restrict__ bmem,
                                  const uint32_t *__restrict__ rmem, const uint32_t *__restrict__ bcomp,
                                  const uint32_t *__restrict__ rcomp, const uint32_t *__restrict__ boff,
                                  uint32_t inactive0, uint32_t *__restrict__ perm) {
  for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t r;
    if (fm[v]) {
      const uint64_t i = pm[v];
      r = boff[bmem[i]] + rmem[i];
    } else if (fc[v]) {
      const uint64_t i = pc[v];
      r = boff[bcomp[i]] + rcomp[i];
    } else {
      r = inactive0 + (uint32_t)pi[v];
    }
    perm[v] = r;
  }
}
}  // namespace

bool aorder_device(Graph &g, const tc_aorder_params &p) {
  if (p.order != 0 || g.n < 2) return false;
  cudaStream_t s = g.stream;
  const uint32_t n = g.n;
  ensure_od(g);
  const uint32_t maxd = g.max_outdeg;
  if (maxd > (1u << 24)) return false;  // S per degree value as a table (as aorder_host)
  const std::vector<int64_t> table = superiority_table(maxd, p);
  DevBuf<int64_t> dtab;
  dtab.alloc((size_t)maxd + 1, s);
  TC_CUDA(cudaMemcpyAsync(dtab.get(), table.data(), sizeof(int64_t) * table.size(), cudaMemcpyHostToDevice, s));
  DevBuf<unsigned long long> hist;
  hist.alloc((size_t)maxd + 1, s);
  TC_CUDA(cudaMemsetAsync(hist.get(), 0, hist.bytes(), s));
  ao_hist_kernel<<<grid_for(n, 256, 4), 256, 0, s>>>(g.od.get(), n, maxd, hist.get());
  TC_LAUNCH_CHECK();
  DevBuf<uint32_t> fm, fc, fi;
  DevBuf<uint64_t> pm, pc, pi;
  fm.alloc(n, s);
  fc.alloc(n, s);
  fi.alloc(n, s);
  pm.alloc((uint64_t)n + 1, s);
  pc.alloc((uint64_t)n + 1, s);
  pi.alloc((uint64_t)n + 1, s);
  ao_class_kernel<<<grid_for(n, 256), 256, 0, s>>>(g.od.get(), n, dtab.get(), fm.get(), fc.get(), fi.get());
  TC_LAUNCH_CHECK();
  scan_u32_to_u64(fm.get(), pm.get(), n, s);
  scan_u32_to_u64(fc.get(), pc.get(), n, s);
  scan_u32_to_u64(fi.get(), pi.get(), n, s);
  // class sizes and the superiority range from the d~ histogram (S is a function of d~)
  std::vector<unsigned long long> h(maxd + 1);
  TC_CUDA(cudaMemcpyAsync(h.data(), hist.get(), sizeof(unsigned long long) * h.size(), cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  uint64_t nmem = 0, ncomp = 0;
  int64_t smax = 0, smin1 = INT64_MAX, smin2 = INT64_MAX;
  for (uint32_t d = 1; d <= maxd; ++d) {
    if (!h[d]) continue;
    const int64_t sv = table[d], av = sv < 0 ? -sv : sv;
    smax = std::max(smax, av);
    if (sv > 0) {
      nmem += h[d];
      smin1 = std::min(smin1, av);
    } else {
      ncomp += h[d];
      if (av) smin2 = std::min(smin2, av);
    }
  }
  DevBuf<uint32_t> odm, odc;
  odm.alloc(nmem ? nmem : 1, s);
  odc.alloc(ncomp ? ncomp : 1, s);
  ao_compact_kernel<<<grid_for(n, 256), 256, 0, s>>>(g.od.get(), n, fm.get(), fc.get(), pm.get(), pc.get(), odm.get(),
                                                      odc.get());
  TC_LAUNCH_CHECK();
  uint32_t *h_odm = pinned_u32(nmem ? nmem : 1, 2), *h_odc = pinned_u32(ncomp ? ncomp : 1, 3);
  uint32_t *h_bm = pinned_u32(nmem ? nmem : 1, 4), *h_rm = pinned_u32(nmem ? nmem : 1, 5);
  uint32_t *h_bc = pinned_u32(ncomp ? ncomp : 1, 6), *h_rc = pinned_u32(ncomp ? ncomp : 1, 7);
  if (nmem) TC_CUDA(cudaMemcpyAsync(h_odm, odm.get(), 4 * nmem, cudaMemcpyDeviceToHost, s));
  if (ncomp) TC_CUDA(cudaMemcpyAsync(h_odc, odc.get(), 4 * ncomp, cudaMemcpyDeviceToHost, s));
  TC_CUDA(cudaStreamSynchronize(s));
  // lines 1-15 on the host (sequential greedy)
  aorder_classified(h_odm, nmem, h_odc, ncomp, table, smax, smin1, smin2, p.k, h_bm, h_rm, h_bc, h_rc,
                    g.h_bucket_off, g.eq3);
  // lines 16-20 on the device
  DevBuf<uint32_t> bm, rm, bc, rc;
  bm.alloc(nmem ? nmem : 1, s);
  rm.alloc(nmem ? nmem : 1, s);
  bc.alloc(ncomp ? ncomp : 1, s);
  rc.alloc(ncomp ? ncomp : 1, s);
  if (nmem) {
    TC_CUDA(cudaMemcpyAsync(bm.get(), h_bm, 4 * nmem, cudaMemcpyHostToDevice, s));
    TC_CUDA(cudaMemcpyAsync(rm.get(), h_rm, 4 * nmem, cudaMemcpyHostToDevice, s));
  }
  if (ncomp) {
    TC_CUDA(cudaMemcpyAsync(bc.get(), h_bc, 4 * ncomp, cudaMemcpyHostToDevice, s));
    TC_CUDA(cudaMemcpyAsync(rc.get(), h_rc, 4 * ncomp, cudaMemcpyHostToDevice, s));
  }
  g.bucket_off.alloc(g.h_bucket_off.size(), s);
  TC_CUDA(cudaMemcpyAsync(g.bucket_off.get(), g.h_bucket_off.data(), sizeof(uint32_t) * g.h_bucket_off.size(),
                          cudaMemcpyHostToDevice, s));
  g.perm.alloc(n, s);
  ao_relabel_kernel<<<grid_for(n, 256), 256, 0, s>>>(n, fm.get(), fc.get(), pm.get(), pc.get(), pi.get(), bm.get(),
                                                      rm.get(), bc.get(), rc.get(), g.bucket_off.get(),
                                                      g.h_bucket_off.back(), g.perm.get());
  TC_LAUNCH_CHECK();
  TC_CUDA(cudaStreamSynchronize(s));  // pinned buffers are reused by the next A-order
  g.identity_perm = false;
  return true;
}

void reorder_graph(Graph &g, int rule, const tc_aorder_params &p, AOrderSource *src) {
  cudaStream_t s = g.stream;
  const uint32_t n = g.n;
  if (rule != TC_REORDER_NONE) ensure_od(g);  // D-order / A-order read d~
  g.perm.release();
  g.bucket_off.release();
  g.h_bucket_off.clear();
  g.eq3 = -1;
  g.identity_perm = true;
  if (rule == TC_REORDER_DEGREE && n > 1) {
    int bn = bits_for(n - 1);
    uint32_t maxod = g.max_outdeg;
    int kb = bits_for(maxod) + bn;
    DevBuf<uint64_t> keys, tmp;
    keys.alloc(n, s);
    tmp.alloc(n, s);
    dorder_keys_kernel<<<grid_for(n, 256), 256, 0, s>>>(g.od.get(), n, maxod, bn, keys.get());
    TC_LAUNCH_CHECK();
    uint64_t *sorted = radix_sort_u64(keys.get(), tmp.get(), n, 0, kb, s);
    g.perm.alloc(n, s);
    perm_from_sorted_kernel<<<grid_for(n, 256), 256, 0, s>>>(sorted, n, (1ull << bn) - 1, g.perm.get());
    TC_LAUNCH_CHECK();
    g.identity_perm = false;
  } else if (rule == TC_REORDER_PAPER) {
    // d~ down and pi up through pinned staging buffers (kept across calls, one A-order at a
    // time: the host greedy holds the lock anyway)
    std::lock_guard<std::mutex> lock(g_pinned_mu);
    if (!src && g_opt_aorder_device && aorder_device(g, p)) {
      g.reorder_rule = rule;
      build_oriented_csr(g);
      g.state = G_ORDERED;
      return;
    }
    uint32_t *h_od = pinned_u32(n ? n : 1, 0), *h_perm = pinned_u32(n ? n : 1, 1);
    if (n) TC_CUDA(cudaMemcpyAsync(h_od, g.od.get(), sizeof(uint32_t) * n, cudaMemcpyDeviceToHost, s));
    TC_CUDA(cudaStreamSynchronize(s));
    if (src && src->produce(g, h_od, h_perm, p)) {
      g.identity_perm = n == 0;
      g.reorder_rule = rule;
      build_oriented_csr(g);
      g.state = G_ORDERED;
      return;
    }
    aorder_host(h_od, n, p, h_perm, g.h_bucket_off, g.eq3);
    if (n) {
      g.perm.alloc(n, s);
      TC_CUDA(cudaMemcpyAsync(g.perm.get(), h_perm, sizeof(uint32_t) * n, cudaMemcpyHostToDevice, s));
      g.identity_perm = false;
    }
    g.bucket_off.alloc(g.h_bucket_off.size(), s);
    TC_CUDA(cudaMemcpyAsync(g.bucket_off.get(), g.h_bucket_off.data(), sizeof(uint32_t) * g.h_bucket_off.size(),
                            cudaMemcpyHostToDevice, s));
    TC_CUDA(cudaStreamSynchronize(s));  // host buffers must outlive the copies
  }
  g.reorder_rule = rule;
  build_oriented_csr(g);
  g.state = G_ORDERED;
}

}  // namespace tc
