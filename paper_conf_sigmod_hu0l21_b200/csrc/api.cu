// api.cu — the C-ABI of include/tc.h: argument checks, the state machine, stage timing,
// host/device pointer handling, exports, and the NCCL plumbing of tc_count_dist (a11).
#include <dlfcn.h>

#include <algorithm>
#include <cstring>
#include <map>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "internal.h"

struct tc_graph : tc::Graph {
  std::map<uint32_t, std::vector<uint32_t>> partitions;  // world -> bounds
};

namespace tc {

int g_opt_profile = 1;
int g_opt_aorder_device = 1;
static thread_local std::string t_err;

void cuda_fail(cudaError_t e, const char *what, const char *file, int line) {
  std::string msg = std::string(cudaGetErrorName(e)) + ": " + cudaGetErrorString(e) + " at " + what + " (" + file +
                    ":" + std::to_string(line) + ")";
  cudaGetLastError();
  throw Error(e == cudaErrorMemoryAllocation ? ST_OOM : ST_CUDA, msg);
}

int num_sms() {
  static int cached[64] = {0};
  int dev = 0;
  TC_CUDA(cudaGetDevice(&dev));
  if (dev < 64 && cached[dev]) return cached[dev];
  int sms = 0;
  TC_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  if (dev < 64) cached[dev] = sms;
  return sms;
}

template <class F>
static tc_status guard(F &&f) {
  try {
    f();
    return TC_OK;
  } catch (const Error &e) {
    t_err = e.what();
    return (tc_status)e.status;
  } catch (const std::bad_alloc &) {
    t_err = "host allocation failed";
    return TC_ERR_OOM;
  } catch (const std::exception &e) {
    t_err = e.what();
    return TC_ERR_CUDA;
  }
}

static void select_device(int device) {
  int count = 0;
  cudaError_t e = cudaGetDeviceCount(&count);
  if (e != cudaSuccess || count == 0) {
    cudaGetLastError();
    throw Error(ST_CUDA, "no CUDA device available (libtc_b200 has no CPU fallback)");
  }
  TC_REQUIRE(device >= 0 && device < count, ST_INVALID, "device ordinal out of range");
  TC_CUDA(cudaSetDevice(device));
  static std::once_flag pool_once[64];
  if (device < 64)
    std::call_once(pool_once[device], [device] {
      cudaMemPool_t pool;
      if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) {
        uint64_t thr = UINT64_MAX;  // keep freed blocks cached across graphs
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
      }
      cudaGetLastError();
    });
}

static bool is_device_ptr(const void *p) {
  if (!p) return false;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

struct StageTimer {
  cudaEvent_t a = nullptr, b = nullptr;
  cudaStream_t s;
  bool on;
  explicit StageTimer(cudaStream_t st) : s(st), on(g_opt_profile != 0) {
    if (!on) return;
    TC_CUDA(cudaEventCreate(&a));
    TC_CUDA(cudaEventCreate(&b));
    TC_CUDA(cudaEventRecord(a, s));
  }
  double stop() {
    if (!on) return 0.0;
    TC_CUDA(cudaEventRecord(b, s));
    TC_CUDA(cudaEventSynchronize(b));
    float ms = 0;
    TC_CUDA(cudaEventElapsedTime(&ms, a, b));
    return ms;
  }
  ~StageTimer() {
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
  }
};

static void copy_out(void *dst, const void *src, size_t bytes, cudaStream_t s) {
  if (!bytes || !dst) return;
  TC_REQUIRE(src != nullptr, ST_STATE, "requested data does not exist for this graph state");
  TC_CUDA(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDefault, s));
}

static Graph &checked(tc_graph *g, GraphState need) {
  TC_REQUIRE(g != nullptr, ST_INVALID, "graph is NULL");
  TC_REQUIRE(g->state >= need, ST_STATE,
             need == G_DIRECTED ? "call tc_direct first" : "graph not ready for this call");
  TC_CUDA(cudaSetDevice(g->device));
  return *g;
}

// ------------------------------------------------------------------ NCCL (dlopen)
namespace nccl {
typedef int Result;
typedef struct Comm *Comm_t;
struct UniqueId { char internal[128]; };
enum { Uint32 = 3, Uint64 = 5 };
enum { Sum = 0 };
struct Api {
  void *h = nullptr;
  Result (*GetUniqueId)(UniqueId *) = nullptr;
  Result (*CommInitRank)(Comm_t *, int, UniqueId, int) = nullptr;
  Result (*AllReduce)(const void *, void *, size_t, int, int, Comm_t, cudaStream_t) = nullptr;
  Result (*Broadcast)(const void *, void *, size_t, int, int, Comm_t, cudaStream_t) = nullptr;
  Result (*CommDestroy)(Comm_t) = nullptr;
  const char *(*GetErrorString)(Result) = nullptr;
};
static Api &api() {
  static Api a;
  static std::once_flag once;
  std::call_once(once, [] {
    a.h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!a.h) a.h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!a.h) return;
    a.GetUniqueId = (Result(*)(UniqueId *))dlsym(a.h, "ncclGetUniqueId");
    a.CommInitRank = (Result(*)(Comm_t *, int, UniqueId, int))dlsym(a.h, "ncclCommInitRank");
    a.AllReduce = (Result(*)(const void *, void *, size_t, int, int, Comm_t, cudaStream_t))dlsym(a.h, "ncclAllReduce");
    a.Broadcast = (Result(*)(const void *, void *, size_t, int, int, Comm_t, cudaStream_t))dlsym(a.h, "ncclBroadcast");
    a.CommDestroy = (Result(*)(Comm_t))dlsym(a.h, "ncclCommDestroy");
    a.GetErrorString = (const char *(*)(Result))dlsym(a.h, "ncclGetErrorString");
  });
  TC_REQUIRE(a.h && a.GetUniqueId && a.CommInitRank && a.AllReduce && a.Broadcast && a.CommDestroy, ST_NCCL,
             "libnccl.so.2 not loadable");
  return a;
}
static void check(Result r, const char *what) {
  if (r != 0) {
    const char *m = api().GetErrorString ? api().GetErrorString(r) : "?";
    throw Error(ST_NCCL, std::string(what) + ": " + m);
  }
}
}  // namespace nccl

}  // namespace tc

using namespace tc;

extern "C" {

const char *tc_last_error(void) { return t_err.c_str(); }
const char *tc_version(void) { return "tc_b200 0.1 (sm_100a)"; }

tc_status tc_set_option(const char *key, int64_t value) {
  return guard([&] {
    TC_REQUIRE(key != nullptr, ST_INVALID, "key is NULL");
    std::string k(key);
    if (k == "profile") g_opt_profile = value ? 1 : 0;
    else if (k == "kernel_profile") g_opt_kernel_profile = value ? 1 : 0;
    else if (k == "l2_persist") g_opt_l2_persist = value ? 1 : 0;
    else if (k == "trim_memory") dev_trim();
    else if (k == "bracket") g_opt_bracket = value ? 1 : 0;
    else if (k == "lean") g_opt_lean = value ? 1 : 0;
    else if (k == "extra_compute") {
      TC_REQUIRE(value >= -1 && value <= 1024, ST_INVALID, "extra_compute: -1 (off) or 0..1024");
      g_opt_extra = (int)value;
    }
    else if (k == "intersect") {
      TC_REQUIRE(value >= 0 && value <= 2, ST_INVALID, "intersect: 0 = binary search, 1 = sort-merge, 2 = bitmap");
      g_opt_intersect = (int)value;
    }
    else if (k == "peel_coop") g_opt_peel_coop = value ? 1 : 0;
    else if (k == "peel_red") g_opt_peel_red = value < 0 ? -1 : (value ? 1 : 0);
    else if (k == "split") g_opt_split = value ? 1 : 0;
    else if (k == "shorter") g_opt_shorter = value ? 1 : 0;
    else if (k == "owner_span") {
      TC_REQUIRE(value >= 32 && value <= (1 << 20) && value % 32 == 0, ST_INVALID, "owner_span: multiple of 32");
      g_opt_owner_span = (int)value;
    } else if (k == "vtiles") {
      TC_REQUIRE(value >= 1 && value <= 1024, ST_INVALID, "vtiles: 1 .. 1024");
      g_opt_vtiles = (int)value;
    } else if (k == "owner_lspan") {
      TC_REQUIRE(value >= 8 && value <= (1 << 24), ST_INVALID, "owner_lspan: 8 .. 2^24");
      g_opt_owner_lspan = (int)value;
    } else if (k == "aorder_device") {
      g_opt_aorder_device = value ? 1 : 0;
    } else if (k == "cuckoo") {
      TC_REQUIRE(value >= 0 && value <= 1024, ST_INVALID, "cuckoo: 0 (off) .. 1024 evictions");
      g_opt_cuckoo = (int)value;
    } else if (k == "e2sort") {
      g_opt_e2sort = value < 0 ? -1 : (value ? 1 : 0);
    } else if (k == "otiles") {
      TC_REQUIRE(value >= 0 && value <= 255, ST_INVALID, "otiles: 0 (auto) .. 255");
      g_opt_otiles = (int)value;
    } else if (k == "otile_mb") {
      TC_REQUIRE(value >= 1 && value <= 4096, ST_INVALID, "otile_mb: 1 .. 4096");
      g_opt_otile_mb = (int)value;
    } else if (k == "otile_min") {
      TC_REQUIRE(value >= 0 && value <= 1 << 20, ST_INVALID, "otile_min: 0 .. 2^20");
      g_opt_otile_min = (int)value;
    }
    else if (k == "small_cap") {
      TC_REQUIRE(value >= 32 && value <= 2048 && (value & (value - 1)) == 0, ST_INVALID,
                 "small_cap must be a power of two in [32, 2048]");
      g_opt_small_cap = (int)value;
    } else throw Error(ST_INVALID, "unknown option " + k);
  });
}

tc_status tc_graph_from_edges(const uint32_t *src, const uint32_t *dst, uint64_t num_edges, uint32_t num_vertices,
                              int device, void *cuda_stream, tc_graph **out) {
  return guard([&] {
    TC_REQUIRE(out != nullptr, ST_INVALID, "out is NULL");
    TC_REQUIRE(num_edges == 0 || (src && dst), ST_INVALID, "src/dst NULL with num_edges > 0");
    select_device(device);
    tc_graph *g = new tc_graph();
    try {
      g->device = device;
      g->stream = (cudaStream_t)cuda_stream;
      g->n = num_vertices;
      StageTimer t(g->stream);
      DevBuf<uint32_t> hs, hd;
      const uint32_t *ds = src, *dd = dst;
      if (num_edges && !is_device_ptr(src)) {
        hs.alloc(num_edges, g->stream);
        TC_CUDA(cudaMemcpyAsync(hs.get(), src, num_edges * 4, cudaMemcpyHostToDevice, g->stream));
        ds = hs.get();
      }
      if (num_edges && !is_device_ptr(dst)) {
        hd.alloc(num_edges, g->stream);
        TC_CUDA(cudaMemcpyAsync(hd.get(), dst, num_edges * 4, cudaMemcpyHostToDevice, g->stream));
        dd = hd.get();
      }
      build_graph(*g, ds, dd, num_edges);
      hs.release();
      hd.release();
      g->ms_build = t.stop();
      TC_CUDA(cudaStreamSynchronize(g->stream));
    } catch (...) {
      cudaStreamSynchronize(g->stream);
      delete g;
      throw;
    }
    *out = g;
  });
}

tc_status tc_direct(tc_graph *gp, tc_direct_rule rule) {
  return guard([&] {
    Graph &g = checked(gp, G_BUILT);
    TC_REQUIRE(rule >= TC_DIRECT_ID && rule <= TC_DIRECT_PAPER, ST_INVALID, "unknown directing rule");
    StageTimer t(g.stream);
    direct_graph(g, rule);
    g.ms_direct = t.stop();
    gp->partitions.clear();
  });
}

static tc_aorder_params defaults_or(const tc_aorder_params *p) {
  tc_aorder_params d;
  d.lambda = 9.682;
  d.alpha = 0.5;
  d.beta = 0.5;
  d.bw = nullptr;
  d.bw_len = 0;
  d.k = 32;
  d.order = 0;
  if (!p) return d;
  TC_REQUIRE(p->k >= 1, ST_INVALID, "A-order: k must be >= 1");
  TC_REQUIRE(p->bw == nullptr || p->bw_len >= 1, ST_INVALID, "A-order: bw_len must be >= 1");
  TC_REQUIRE(p->order == 0 || p->order == 1, ST_INVALID, "A-order: order must be 0 or 1");
  TC_REQUIRE(p->alpha > 0 && p->beta > 0, ST_INVALID, "A-order: alpha, beta must be > 0 (Eq.19-20)");
  return *p;
}

tc_status tc_reorder(tc_graph *gp, tc_reorder_rule rule, const tc_aorder_params *p) {
  return guard([&] {
    Graph &g = checked(gp, G_DIRECTED);
    TC_REQUIRE(rule >= TC_REORDER_NONE && rule <= TC_REORDER_PAPER, ST_INVALID, "unknown reorder rule");
    tc_aorder_params prm = defaults_or(p);
    // keep the parameters (bw copied) for the edge-unit schedule
    g.abw.assign(prm.bw ? prm.bw : nullptr, prm.bw ? prm.bw + prm.bw_len : nullptr);
    g.aparams = prm;
    g.aparams.bw = g.abw.empty() ? nullptr : g.abw.data();
    g.aparams_set = true;
    StageTimer t(g.stream);
    reorder_graph(g, rule, prm);
    g.ms_reorder = t.stop();
    gp->partitions.clear();
  });
}

namespace {
// A-order computed once (rank `root`) and broadcast: a 2-word header [b + 1, eq3], then pi
// (n u32) and bucket_off (b + 1 u32), all on the graph's stream (a11 plumbing).
struct BroadcastAOrder : AOrderSource {
  nccl::Comm_t comm;
  int rank, root = 0;
  bool produce(Graph &g, const uint32_t *h_od, uint32_t *h_perm, const tc_aorder_params &p) override {
    nccl::Api &a = nccl::api();
    cudaStream_t s = g.stream;
    const uint32_t n = g.n;
    uint64_t hdr[2] = {0, 0};
    bool on_device = false;  // root: pi already in g.perm (device classification / relabel)
    if (rank == root) {
      on_device = g_opt_aorder_device && aorder_device(g, p);
      if (!on_device) aorder_host(h_od, n, p, h_perm, g.h_bucket_off, g.eq3);
      hdr[0] = g.h_bucket_off.size();
      hdr[1] = (uint64_t)g.eq3;
    }
    DevBuf<uint64_t> dh;
    dh.alloc(2, s);
    TC_CUDA(cudaMemcpyAsync(dh.get(), hdr, sizeof(hdr), cudaMemcpyHostToDevice, s));
    nccl::check(a.Broadcast(dh.get(), dh.get(), 2, nccl::Uint64, root, comm, s), "ncclBroadcast(header)");
    TC_CUDA(cudaMemcpyAsync(hdr, dh.get(), sizeof(hdr), cudaMemcpyDeviceToHost, s));
    TC_CUDA(cudaStreamSynchronize(s));
    const size_t nb1 = (size_t)hdr[0];
    TC_REQUIRE(nb1 >= 1, ST_NCCL, "A-order broadcast: empty bucket table");
    if (rank != root) {
      g.h_bucket_off.assign(nb1, 0);
      g.eq3 = (int64_t)hdr[1];
    }
    if (!on_device) {
      if (n) g.perm.alloc(n, s);
      g.bucket_off.alloc(nb1, s);
    }
    if (rank == root && !on_device) {
      if (n) TC_CUDA(cudaMemcpyAsync(g.perm.get(), h_perm, sizeof(uint32_t) * n, cudaMemcpyHostToDevice, s));
      TC_CUDA(cudaMemcpyAsync(g.bucket_off.get(), g.h_bucket_off.data(), sizeof(uint32_t) * nb1,
                              cudaMemcpyHostToDevice, s));
    }
    if (n) nccl::check(a.Broadcast(g.perm.get(), g.perm.get(), n, nccl::Uint32, root, comm, s), "ncclBroadcast(pi)");
    nccl::check(a.Broadcast(g.bucket_off.get(), g.bucket_off.get(), nb1, nccl::Uint32, root, comm, s),
                "ncclBroadcast(bucket_off)");
    if (rank != root)
      TC_CUDA(cudaMemcpyAsync(g.h_bucket_off.data(), g.bucket_off.get(), sizeof(uint32_t) * nb1,
                              cudaMemcpyDeviceToHost, s));
    TC_CUDA(cudaStreamSynchronize(s));  // host vectors must outlive the copies
    return true;
  }
};
}  // namespace

tc_status tc_reorder_dist(tc_graph *gp, tc_reorder_rule rule, const tc_aorder_params *p, void *comm, int rank,
                          int world) {
  return guard([&] {
    Graph &g = checked(gp, G_DIRECTED);
    TC_REQUIRE(rule >= TC_REORDER_NONE && rule <= TC_REORDER_PAPER, ST_INVALID, "unknown reorder rule");
    TC_REQUIRE(comm != nullptr, ST_INVALID, "comm is NULL");
    TC_REQUIRE(world >= 1 && rank >= 0 && rank < world, ST_INVALID, "bad rank/world");
    tc_aorder_params prm = defaults_or(p);
    g.abw.assign(prm.bw ? prm.bw : nullptr, prm.bw ? prm.bw + prm.bw_len : nullptr);
    g.aparams = prm;
    g.aparams.bw = g.abw.empty() ? nullptr : g.abw.data();
    g.aparams_set = true;
    StageTimer t(g.stream);
    BroadcastAOrder src;
    src.comm = (nccl::Comm_t)comm;
    src.rank = rank;
    reorder_graph(g, rule, prm, rule == TC_REORDER_PAPER ? &src : nullptr);
    g.ms_reorder = t.stop();
    gp->partitions.clear();
  });
}

tc_status tc_set_schedule(tc_graph *gp, tc_schedule s) {
  return guard([&] {
    TC_REQUIRE(gp != nullptr, ST_INVALID, "graph is NULL");
    TC_REQUIRE(s >= TC_SCHED_AUTO && s <= TC_SCHED_EDGE_AORDER, ST_INVALID, "unknown schedule");
    gp->schedule = s;
    if (s == TC_SCHED_EDGE_AORDER && gp->state >= G_DIRECTED && gp->csr_ready && !gp->units_ready) {
      // the edge-unit A-order is preprocessing: built here (timed with the reorder stage)
      // when the CSR exists, else lazily by the first count
      TC_CUDA(cudaSetDevice(gp->device));
      StageTimer t(gp->stream);
      build_units(*gp);
      gp->ms_reorder += t.stop();
    }
  });
}

static void ensure_csr(Graph &g) {
  if (!g.csr_ready) {
    tc_aorder_params prm = defaults_or(nullptr);
    reorder_graph(g, TC_REORDER_NONE, prm);
  }
}

static uint64_t do_count(tc_graph *gp, uint32_t ub, uint32_t ue, uint64_t *per_vertex, void *comm, bool reduce) {
  Graph &g = *gp;
  StageTimer t(g.stream);
  ensure_csr(g);
  DevBuf<uint64_t> tnew;
  if (per_vertex) {
    tnew.alloc(g.n ? g.n : 1, g.stream);
    TC_CUDA(cudaMemsetAsync(tnew.get(), 0, tnew.bytes(), g.stream));
  }
  float kms = 0;
  uint64_t launches = 0;
  uint64_t T = 0;
  DevBuf<unsigned long long> dT;  // a11: the allreduce consumes the device partial directly
  if (reduce) {
    dT.alloc(1, g.stream);
    TC_CUDA(cudaMemsetAsync(dT.get(), 0, 8, g.stream));
  }
  T = count_graph(g, ub, ue, per_vertex ? tnew.get() : nullptr, g_opt_profile ? &kms : nullptr, &launches, -1,
                  reduce ? dT.get() : nullptr);
  if (reduce) {
    nccl::Api &a = nccl::api();
    nccl::check(a.AllReduce(dT.get(), dT.get(), 1, nccl::Uint64, nccl::Sum, (nccl::Comm_t)comm, g.stream),
                "ncclAllReduce(T)");
    if (per_vertex && g.n)
      nccl::check(a.AllReduce(tnew.get(), tnew.get(), g.n, nccl::Uint64, nccl::Sum, (nccl::Comm_t)comm, g.stream),
                  "ncclAllReduce(per_vertex)");
    TC_CUDA(cudaMemcpyAsync(&T, dT.get(), 8, cudaMemcpyDeviceToHost, g.stream));
    TC_CUDA(cudaStreamSynchronize(g.stream));
  }
  if (per_vertex && g.n) {
    if (is_device_ptr(per_vertex)) {
      gather_per_vertex(g, tnew.get(), per_vertex);
    } else {
      DevBuf<uint64_t> tmp;
      tmp.alloc(g.n, g.stream);
      gather_per_vertex(g, tnew.get(), tmp.get());
      TC_CUDA(cudaMemcpyAsync(per_vertex, tmp.get(), 8ull * g.n, cudaMemcpyDeviceToHost, g.stream));
      TC_CUDA(cudaStreamSynchronize(g.stream));
    }
  }
  TC_CUDA(cudaStreamSynchronize(g.stream));
  g.ms_count = t.stop();
  g.ms_count_kernel = kms;
  g.count_launches = launches;
  g.triangles = T;
  return T;
}

tc_status tc_count(tc_graph *gp, uint64_t *triangles, uint64_t *per_vertex) {
  return guard([&] {
    checked(gp, G_DIRECTED);
    TC_REQUIRE(triangles != nullptr, ST_INVALID, "triangles is NULL");
    uint64_t T = do_count(gp, 0, gp->n, per_vertex, nullptr, false);
    *triangles = T;
  });
}

tc_status tc_count_edges(tc_graph *gp, uint64_t *triangles, uint64_t *per_edge) {
  return guard([&] {
    Graph &g = checked(gp, G_DIRECTED);
    TC_REQUIRE(triangles != nullptr, ST_INVALID, "triangles is NULL");
    TC_REQUIRE(per_edge != nullptr || g.m == 0, ST_INVALID, "per_edge is NULL");
    StageTimer t(g.stream);
    ensure_csr(g);
    cudaStream_t s = g.stream;
    DevBuf<uint64_t> te, out;
    te.alloc(g.m ? g.m : 1, s);
    TC_CUDA(cudaMemsetAsync(te.get(), 0, te.bytes(), s));
    float kms = 0;
    uint64_t launches = 0;
    const uint64_t T = count_graph(g, 0, g.n, te.get(), g_opt_profile ? &kms : nullptr, &launches, 2);
    if (g.m) {
      const bool dev = is_device_ptr(per_edge);
      if (!dev) out.alloc(g.m, s);
      map_edges_canonical(g, te.get(), dev ? per_edge : out.get());
      if (!dev) TC_CUDA(cudaMemcpyAsync(per_edge, out.get(), 8ull * g.m, cudaMemcpyDeviceToHost, s));
    }
    TC_CUDA(cudaStreamSynchronize(s));
    g.ms_count = t.stop();
    g.ms_count_kernel = kms;
    g.count_launches = launches;
    g.triangles = T;
    *triangles = T;
  });
}

tc_status tc_count_range(tc_graph *gp, uint32_t u_begin, uint32_t u_end, uint64_t *triangles,
                         uint64_t *per_vertex) {
  return guard([&] {
    checked(gp, G_DIRECTED);
    TC_REQUIRE(triangles != nullptr, ST_INVALID, "triangles is NULL");
    TC_REQUIRE(u_begin <= u_end && u_end <= gp->n, ST_INVALID, "bad vertex range");
    uint64_t T = do_count(gp, u_begin, u_end, per_vertex, nullptr, false);
    *triangles = T;
  });
}

tc_status tc_partition(tc_graph *gp, uint32_t world, uint32_t *bounds) {
  return guard([&] {
    Graph &g = checked(gp, G_DIRECTED);
    TC_REQUIRE(world >= 1 && bounds != nullptr, ST_INVALID, "world >= 1 and bounds required");
    ensure_csr(g);
    auto it = gp->partitions.find(world);
    if (it == gp->partitions.end()) {
      std::vector<uint32_t> b(world + 1);
      partition_graph(g, world, b.data());
      // RANGE schedule after A-order: snap to bucket starts so buckets stay whole
      if (!g.h_bucket_off.empty()) {
        const auto &hb = g.h_bucket_off;
        for (uint32_t r = 1; r < world; ++r) {
          auto pos = std::lower_bound(hb.begin(), hb.end(), b[r]);
          if (pos != hb.end()) b[r] = *pos;
          else b[r] = g.n;
          b[r] = std::max(b[r], b[r - 1]);
        }
      }
      it = gp->partitions.emplace(world, std::move(b)).first;
    }
    std::memcpy(bounds, it->second.data(), sizeof(uint32_t) * (world + 1));
  });
}

tc_status tc_nccl_get_unique_id(void *unique_id) {
  return guard([&] {
    TC_REQUIRE(unique_id != nullptr, ST_INVALID, "unique_id is NULL");
    nccl::UniqueId id;
    nccl::check(nccl::api().GetUniqueId(&id), "ncclGetUniqueId");
    std::memcpy(unique_id, &id, sizeof(id));
  });
}

tc_status tc_nccl_comm_init(const void *unique_id, int rank, int world, int device, void **comm) {
  return guard([&] {
    TC_REQUIRE(unique_id && comm && world >= 1 && rank >= 0 && rank < world, ST_INVALID, "bad NCCL init args");
    select_device(device);
    nccl::UniqueId id;
    std::memcpy(&id, unique_id, sizeof(id));
    nccl::Comm_t c = nullptr;
    nccl::check(nccl::api().CommInitRank(&c, world, id, rank), "ncclCommInitRank");
    *comm = c;
  });
}

tc_status tc_nccl_comm_destroy(void *comm) {
  return guard([&] {
    if (comm) nccl::check(nccl::api().CommDestroy((nccl::Comm_t)comm), "ncclCommDestroy");
  });
}

tc_status tc_count_dist(tc_graph *gp, void *comm, int rank, int world, uint64_t *triangles, uint64_t *per_vertex) {
  return guard([&] {
    checked(gp, G_DIRECTED);
    TC_REQUIRE(triangles != nullptr && comm != nullptr, ST_INVALID, "triangles/comm NULL");
    TC_REQUIRE(world >= 1 && rank >= 0 && rank < world, ST_INVALID, "bad rank/world");
    std::vector<uint32_t> b(world + 1);
    tc_status st = tc_partition(gp, (uint32_t)world, b.data());
    if (st != TC_OK) throw Error(st, t_err);
    uint64_t T = do_count(gp, b[rank], b[rank + 1], per_vertex, comm, true);
    *triangles = T;
  });
}

tc_status tc_analyze(tc_graph *gp) {
  return guard([&] {
    Graph &g = checked(gp, G_DIRECTED);
    ensure_csr(g);
    analyze_graph(g);
  });
}

tc_status tc_get_stats(const tc_graph *gp, tc_stats_t *o) {
  return guard([&] {
    TC_REQUIRE(gp && o, ST_INVALID, "NULL argument");
    Graph &g = *const_cast<tc_graph *>(gp);  // lazily filled statistics (no logical change)
    TC_CUDA(cudaSetDevice(g.device));
    ensure_max_degree(g);
    if (g.state >= G_DIRECTED) ensure_od(g);
    std::memset(o, 0, sizeof(*o));
    o->n = g.n;
    o->m = g.m;
    o->samples = g.samples;
    o->max_degree = g.max_degree;
    o->max_outdeg = g.max_outdeg;
    o->eq1_lo = g.eq1_lo;
    o->eq1_hi = g.eq1_hi;
    o->eq3 = g.eq3;
    o->levels = g.levels;
    o->subrounds = g.subrounds;
    o->nbuckets = g.h_bucket_off.empty() ? 0 : (uint32_t)g.h_bucket_off.size() - 1;
    o->direct_rule = (uint32_t)g.direct_rule;
    o->reorder_rule = (uint32_t)g.reorder_rule;
    o->schedule = (uint32_t)g.schedule;
    o->triangles = g.triangles;
    o->wedges = g.wedges;
    o->alg_bytes = g.alg_bytes;
    o->ms_build = g.ms_build;
    o->ms_direct = g.ms_direct;
    o->ms_reorder = g.ms_reorder;
    o->ms_count = g.ms_count;
    o->ms_count_kernel = g.ms_count_kernel;
    o->count_launches = g.count_launches;
    o->eq3_units = g.units_ready ? g.eq3_units : -1;
    o->nunits = g.units_ready && !g.h_unit_off.empty() ? g.h_unit_off.back() : 0;
    o->unit_buckets = g.units_ready && !g.h_unit_off.empty() ? g.h_unit_off.size() - 1 : 0;
  });
}

tc_status tc_export(tc_graph *gp, uint64_t *offs, uint32_t *col, uint32_t *perm) {
  return guard([&] {
    Graph &g = checked(gp, G_DIRECTED);
    ensure_csr(g);
    copy_out(offs, g.offs.get(), 8ull * (g.n + 1ull), g.stream);
    copy_out(col, g.col.get(), 4ull * g.m, g.stream);
    if (perm && g.n) {
      if (g.identity_perm) {
        std::vector<uint32_t> id(g.n);
        for (uint32_t i = 0; i < g.n; ++i) id[i] = i;
        copy_out(perm, id.data(), 4ull * g.n, g.stream);
        TC_CUDA(cudaStreamSynchronize(g.stream));
      } else {
        copy_out(perm, g.perm.get(), 4ull * g.n, g.stream);
      }
    }
    TC_CUDA(cudaStreamSynchronize(g.stream));
  });
}

__global__ void unpack_edges_kernel(const uint64_t *in, uint64_t m, int bits, uint64_t *out) {
  uint64_t mask = (1ull << bits) - 1;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = ((in[i] >> bits) << 32) | (in[i] & mask);
}

tc_status tc_export_graph(tc_graph *gp, uint64_t *edges, uint32_t *degree) {
  return guard([&] {
    Graph &g = checked(gp, G_BUILT);
    if (edges && g.m) {
      DevBuf<uint64_t> tmp;
      tmp.alloc(g.m, g.stream);
      unpack_edges_kernel<<<grid_for(g.m, 256), 256, 0, g.stream>>>(g.edges.get(), g.m, g.bits, tmp.get());
      TC_LAUNCH_CHECK();
      copy_out(edges, tmp.get(), 8ull * g.m, g.stream);
      TC_CUDA(cudaStreamSynchronize(g.stream));
    }
    copy_out(degree, g.deg.get(), 4ull * g.n, g.stream);
    TC_CUDA(cudaStreamSynchronize(g.stream));
  });
}

tc_status tc_export_direct(tc_graph *gp, uint32_t *outdeg, uint32_t *sub, uint32_t *dsnap) {
  return guard([&] {
    Graph &g = checked(gp, G_DIRECTED);
    TC_REQUIRE(!(sub || dsnap) || g.direct_rule == TC_DIRECT_PAPER, ST_STATE, "sub/dsnap exist only for PAPER");
    if (outdeg) ensure_od(g);
    copy_out(outdeg, g.od.get(), 4ull * g.n, g.stream);
    copy_out(sub, g.sub.get(), 4ull * g.n, g.stream);
    copy_out(dsnap, g.dsnap.get(), 4ull * g.n, g.stream);
    TC_CUDA(cudaStreamSynchronize(g.stream));
  });
}

tc_status tc_export_buckets(tc_graph *gp, uint32_t *bucket_off) {
  return guard([&] {
    Graph &g = checked(gp, G_DIRECTED);
    TC_REQUIRE(!g.h_bucket_off.empty(), ST_STATE, "no A-order buckets (tc_reorder PAPER first)");
    copy_out(bucket_off, g.h_bucket_off.data(), 4ull * g.h_bucket_off.size(), g.stream);
    TC_CUDA(cudaStreamSynchronize(g.stream));
  });
}

tc_status tc_export_units(tc_graph *gp, uint64_t *units, uint32_t *unit_off) {
  return guard([&] {
    Graph &g = checked(gp, G_DIRECTED);
    ensure_csr(g);
    build_units(g);
    const uint64_t nu = g.h_unit_off.back();
    if (nu) copy_out(units, g.units.get(), 8ull * nu, g.stream);
    copy_out(unit_off, g.h_unit_off.data(), 4ull * g.h_unit_off.size(), g.stream);
    TC_CUDA(cudaStreamSynchronize(g.stream));
  });
}

void tc_graph_free(tc_graph *gp) {
  if (!gp) return;
  cudaSetDevice(gp->device);
  cudaStream_t s = gp->stream;
  delete gp;  // DevBufs free stream-ordered
  cudaStreamSynchronize(s);
  cudaGetLastError();
}

}  // extern "C"
