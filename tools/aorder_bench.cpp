// Host micro-benchmark of the library's A-order greedy (csrc/aorder.cpp) on a raw u32
// out-degree file:  g++ -O3 -std=c++17 -pthread tools/aorder_bench.cpp -o /tmp/aorder_bench
//                    /tmp/aorder_bench od.u32 [reps]
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../paper_conf_sigmod_hu0l21_b200/csrc/aorder.cpp"

int main(int argc, char **argv) {
  if (argc < 2) return 1;
  FILE *f = fopen(argv[1], "rb");
  if (!f) return 1;
  fseek(f, 0, SEEK_END);
  size_t n = ftell(f) / 4;
  fseek(f, 0, SEEK_SET);
  std::vector<uint32_t> od(n);
  if (fread(od.data(), 4, n, f) != n) return 1;
  fclose(f);
  int reps = argc > 2 ? atoi(argv[2]) : 3;
  tc_aorder_params p{9.682, 0.5, 0.5, nullptr, 0, 32, 0};
  std::vector<uint32_t> perm(n), boff;
  int64_t eq3 = 0;
  uint64_t h = 0;
  for (int r = 0; r < reps; ++r) {
    auto t0 = std::chrono::steady_clock::now();
    tc::aorder_host(od.data(), n, p, perm.data(), boff, eq3);
    auto t1 = std::chrono::steady_clock::now();
    h = 1469598103934665603ull;
    for (uint32_t x : perm) h = (h ^ x) * 1099511628211ull;
    for (uint32_t x : boff) h = (h ^ x) * 1099511628211ull;
    printf("n=%zu buckets=%zu eq3=%lld  %.1f ms  hash=%016llx\n", n, boff.size() - 1, (long long)eq3,
           std::chrono::duration<double, std::milli>(t1 - t0).count(), (unsigned long long)h);
  }
  return 0;
}
