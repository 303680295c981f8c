// count_small.cu — instantiations of the warp-item count kernels (bucketed schedule, d~ below
// the small cap) and of the RANGE-schedule kernel; device code in count_dev.cuh, host driver
// in count.cu.  A translation unit of its own so the kernel families compile in parallel.
#include "count_dev.cuh"
#include "internal.h"

namespace tc {
namespace cnt {

const void *small_kernel(int mode, bool own) {
  if (own) return mode == 4 ? (const void *)count_small_kernel<4, true> : (const void *)count_small_kernel<0, true>;
  switch (mode) {
    case 1: return (const void *)count_small_kernel<1>;
    case 2: return (const void *)count_small_kernel<2>;
    case 3: return (const void *)count_small_kernel<3>;
    case 4: return (const void *)count_small_kernel<4>;
    default: return (const void *)count_small_kernel<0>;
  }
}

const void *range_kernel(int mode) {
  switch (mode) {
    case 1: return (const void *)count_range_kernel<1>;
    case 2: return (const void *)count_range_kernel<2>;
    default: return (const void *)count_range_kernel<0>;
  }
}

void small_set_constants(int bracket, int merge, int extra, int cuckoo) {
  TC_CUDA(cudaMemcpyToSymbol(g_cuckoo, &cuckoo, sizeof(int)));
  TC_CUDA(cudaMemcpyToSymbol(g_bracket, &bracket, sizeof(int)));
  TC_CUDA(cudaMemcpyToSymbol(g_merge, &merge, sizeof(int)));
  TC_CUDA(cudaMemcpyToSymbol(g_extra, &extra, sizeof(int)));
}

}  // namespace cnt
}  // namespace tc
