// prof.cu — optional per-kernel CUDA-event profiling (option "kernel_profile").
//
// Each instrumented launch records an event pair on the launching stream plus the
// kernel's algorithmic bytes; tc_profile_report() resolves the pairs (after the caller's
// synchronisation) and aggregates time / launches / bytes per kernel name.  bench.py uses
// it to obtain the dominant kernel's live per-launch duration inside the timed region.
#include <cstdio>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/tc.h"
#include "common.cuh"

namespace tc {

int g_opt_kernel_profile = 0;
unsigned long long g_launch_count = 0;

namespace {
struct Rec {
  const char *name;
  cudaEvent_t a, b;
  double bytes;
};
std::mutex g_mu;
std::vector<Rec> g_recs;
std::vector<cudaEvent_t> g_free;

cudaEvent_t take_event() {
  if (!g_free.empty()) {
    cudaEvent_t e = g_free.back();
    g_free.pop_back();
    return e;
  }
  cudaEvent_t e;
  TC_CUDA(cudaEventCreate(&e));
  return e;
}
}  // namespace

ProfScope::ProfScope(const char *name, cudaStream_t s, double bytes) : name_(name), s_(s), bytes_(bytes) {
  if (!g_opt_kernel_profile) return;
  std::lock_guard<std::mutex> lk(g_mu);
  a_ = take_event();
  b_ = take_event();
  TC_CUDA(cudaEventRecord((cudaEvent_t)a_, s_));
}

ProfScope::~ProfScope() {
  if (!a_) return;
  std::lock_guard<std::mutex> lk(g_mu);
  cudaEventRecord((cudaEvent_t)b_, s_);
  g_recs.push_back({name_, (cudaEvent_t)a_, (cudaEvent_t)b_, bytes_});
}

}  // namespace tc

using namespace tc;

extern "C" tc_status tc_profile_report(char *buf, uint64_t cap, int reset) {
  try {
    std::lock_guard<std::mutex> lk(g_mu);
    struct Agg {
      double ms = 0, bytes = 0;
      uint64_t launches = 0;
    };
    std::map<std::string, Agg> agg;
    for (auto &r : g_recs) {
      TC_CUDA(cudaEventSynchronize(r.b));
      float ms = 0;
      TC_CUDA(cudaEventElapsedTime(&ms, r.a, r.b));
      Agg &x = agg[r.name];
      x.ms += ms;
      x.bytes += r.bytes;
      x.launches += 1;
    }
    std::string out = "{\"_launches\": " + std::to_string(g_launch_count);
    bool first = false;
    for (auto &kv : agg) {
      char tmp[256];
      snprintf(tmp, sizeof tmp, "%s\"%s\": {\"ms\": %.6f, \"launches\": %llu, \"bytes\": %.0f}", first ? "" : ", ",
               kv.first.c_str(), kv.second.ms, (unsigned long long)kv.second.launches, kv.second.bytes);
      out += tmp;
      first = false;
    }
    out += "}";
    if (reset) {
      for (auto &r : g_recs) {
        g_free.push_back(r.a);
        g_free.push_back(r.b);
      }
      g_recs.clear();
      g_launch_count = 0;
    }
    if (buf && cap) {
      size_t n = out.size() < cap - 1 ? out.size() : cap - 1;
      memcpy(buf, out.data(), n);
      buf[n] = 0;
    }
    return out.size() < cap ? TC_OK : TC_ERR_INVALID;
  } catch (const Error &e) {
    return (tc_status)e.status;
  }
}
