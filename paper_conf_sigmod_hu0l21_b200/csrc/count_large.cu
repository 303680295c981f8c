// count_large.cu — instantiations of the CTA-item count kernels (bucketed schedule, d~ at or
// above the small cap; N+(u) staged piece by piece with TMA bulk copies); device code in
// count_dev.cuh, host driver in count.cu.
#include "count_dev.cuh"
#include "internal.h"

namespace tc {
namespace cnt {

const void *large_kernel(int mode, bool own) {
  if (own) return (const void *)count_large_kernel<0, true>;
  switch (mode) {
    case 1: return (const void *)count_large_kernel<1>;
    case 2: return (const void *)count_large_kernel<2>;
    default: return (const void *)count_large_kernel<0>;
  }
}

void large_set_constants(int bracket, int merge, int extra, int cuckoo) {
  TC_CUDA(cudaMemcpyToSymbol(g_cuckoo, &cuckoo, sizeof(int)));
  TC_CUDA(cudaMemcpyToSymbol(g_bracket, &bracket, sizeof(int)));
  TC_CUDA(cudaMemcpyToSymbol(g_merge, &merge, sizeof(int)));
  TC_CUDA(cudaMemcpyToSymbol(g_extra, &extra, sizeof(int)));
}

}  // namespace cnt
}  // namespace tc
