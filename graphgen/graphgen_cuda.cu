// graphgen_cuda.cu — CUDA implementation of the seeded synthetic-graph generators.
//
// Input generator only (no triangle-counting arithmetic).  Used by bench.py and
// the large-size GPU tests to materialise BASELINE.json's inputs directly in
// HBM; bit-identical to graphgen_cpu.c (tests/test_gpu_graphgen.py samples it).
#include <cuda_runtime.h>
#include <stdint.h>

#include "philox.h"

__global__ void gg_rmat_kernel(uint64_t seed, uint32_t scale, uint32_t ta, uint32_t tab,
                               uint32_t tabc, int scramble, uint64_t e0, uint64_t count,
                               uint32_t *__restrict__ src, uint32_t *__restrict__ dst) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride) {
    uint32_t u, v;
    gg_rmat_sample(seed, e0 + i, scale, ta, tab, tabc, &u, &v);
    if (scramble) {
      u = gg_scramble(u, scale, seed);
      v = gg_scramble(v, scale, seed);
    }
    src[i] = u;
    dst[i] = v;
  }
}

__global__ void gg_er_kernel(uint64_t seed, uint32_t n, uint64_t e0, uint64_t count,
                             uint32_t *__restrict__ src, uint32_t *__restrict__ dst) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride) {
    uint32_t u, v;
    gg_er_sample(seed, e0 + i, n, &u, &v);
    src[i] = u;
    dst[i] = v;
  }
}

static int gg_grid(uint64_t count) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  uint64_t want = (count + 255) / 256;
  uint64_t cap = (uint64_t)sms * 8;
  return (int)(want < cap ? (want ? want : 1) : cap);
}

extern "C" int gg_rmat_cuda(uint64_t seed, uint32_t scale, uint32_t ta, uint32_t tab,
                            uint32_t tabc, int scramble, uint64_t e0, uint64_t count,
                            uint32_t *src, uint32_t *dst, void *stream) {
  if (scale > 32) return -1;
  if (count == 0) return 0;
  gg_rmat_kernel<<<gg_grid(count), 256, 0, (cudaStream_t)stream>>>(seed, scale, ta, tab, tabc,
                                                                     scramble, e0, count, src, dst);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

extern "C" int gg_er_cuda(uint64_t seed, uint32_t n, uint64_t e0, uint64_t count, uint32_t *src,
                          uint32_t *dst, void *stream) {
  if (count == 0) return 0;
  gg_er_kernel<<<gg_grid(count), 256, 0, (cudaStream_t)stream>>>(seed, n, e0, count, src, dst);
  return cudaGetLastError() == cudaSuccess ? 0 : -2;
}
