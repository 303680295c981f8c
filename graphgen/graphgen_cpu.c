/* graphgen_cpu.c — CPU implementation of the seeded synthetic-graph generators.
 *
 * Input generator only (no triangle-counting arithmetic).  Emits the raw edge
 * samples (src[e], dst[e]) of BASELINE.json's configs; duplicates, both
 * directions and self-loops are left in, as in Graph500 (the method's ingest
 * step normalises them).  Bit-identical to graphgen_cuda.cu.
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>

#include "philox.h"

typedef struct {
  int kind; /* 0 = rmat, 1 = er */
  uint64_t seed, e0, count;
  uint32_t scale, ta, tab, tabc, scramble, n;
  uint32_t *src, *dst;
} gg_job;

static void *gg_worker(void *arg) {
  gg_job *j = (gg_job *)arg;
  for (uint64_t i = 0; i < j->count; ++i) {
    uint64_t e = j->e0 + i;
    uint32_t u, v;
    if (j->kind == 0) {
      gg_rmat_sample(j->seed, e, j->scale, j->ta, j->tab, j->tabc, &u, &v);
      if (j->scramble) {
        u = gg_scramble(u, j->scale, j->seed);
        v = gg_scramble(v, j->scale, j->seed);
      }
    } else {
      gg_er_sample(j->seed, e, j->n, &u, &v);
    }
    j->src[i] = u;
    j->dst[i] = v;
  }
  return NULL;
}

static int gg_run(gg_job proto, int threads) {
  if (threads < 1) threads = 1;
  if (threads > 256) threads = 256;
  if ((uint64_t)threads > proto.count) threads = proto.count ? (int)proto.count : 1;
  pthread_t tid[256];
  gg_job jobs[256];
  uint64_t per = (proto.count + threads - 1) / threads;
  int started = 0;
  for (int t = 0; t < threads; ++t) {
    uint64_t b = per * t;
    if (b >= proto.count) break;
    uint64_t c = proto.count - b < per ? proto.count - b : per;
    jobs[t] = proto;
    jobs[t].e0 = proto.e0 + b;
    jobs[t].count = c;
    jobs[t].src = proto.src + b;
    jobs[t].dst = proto.dst + b;
    if (pthread_create(&tid[t], NULL, gg_worker, &jobs[t]) != 0) {
      gg_worker(&jobs[t]);
      tid[t] = 0;
    }
    started = t + 1;
  }
  for (int t = 0; t < started; ++t)
    if (tid[t]) pthread_join(tid[t], NULL);
  return 0;
}

/* Samples e in [e0, e0+count) of an R-MAT/Kronecker graph on 2^scale vertices. */
int gg_rmat_cpu(uint64_t seed, uint32_t scale, uint32_t ta, uint32_t tab, uint32_t tabc,
                int scramble, uint64_t e0, uint64_t count, uint32_t *src, uint32_t *dst,
                int threads) {
  if (scale > 32) return -1;
  gg_job j = {0, seed, e0, count, scale, ta, tab, tabc, (uint32_t)scramble, 0, src, dst};
  return gg_run(j, threads);
}

/* Samples e in [e0, e0+count) of an Erdos-Renyi G(n, M) multigraph. */
int gg_er_cpu(uint64_t seed, uint32_t n, uint64_t e0, uint64_t count, uint32_t *src,
              uint32_t *dst, int threads) {
  gg_job j = {1, seed, e0, count, 0, 0, 0, 0, 0, n, src, dst};
  return gg_run(j, threads);
}

/* Known-answer hook for tests: one Philox4x32-10 block. */
void gg_philox_block(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  gg_u32x4 c = {{ctr[0], ctr[1], ctr[2], ctr[3]}};
  gg_u32x4 r = gg_philox4x32_10(c, key[0], key[1]);
  for (int i = 0; i < 4; ++i) out[i] = r.v[i];
}
