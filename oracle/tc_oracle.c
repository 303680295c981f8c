/* oracle/tc_oracle.c — plain, slow, obviously-correct CPU oracle.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code
 * with the CUDA path (paper_conf_sigmod_hu0l21_b200/) and neither imports the other.
 *
 * Citations "P:N" are /root/reference/PAPER.md line N (the paper "Accelerating
 * Triangle Counting on GPU"); "Qk" are the readings listed in DESIGN.md §Readings
 * (taken from SURVEY.md §8(c)) where the paper is silent, ambiguous or garbled.
 *
 * What each function computes and what pins it (tests/test_oracle*.py):
 *   orc_canonical_keys / O1  simple undirected graph (Q1): (min,max) keys,
 *   orc_unique_sorted        sorted by a library sort (numpy), duplicates dropped
 *                            pinned: brute-force set semantics on random inputs
 *   orc_sym_csr          symmetric adjacency N(v), ascending ("nbrList")
 *   orc_direct_id        ID-based directing, u->v iff u<v (Q12)
 *   orc_direct_degree    degree-based directing (Q11 tie by id)
 *   orc_direct_paper     Algorithm 1 "A-direction", sequential, in the
 *                        paper's line order, readings Q3-Q10.  PARITY VS AUTHORS'
 *                        CODE UNPINNED (no worked example survives, Figs.1-3
 *                        missing); pinned by: hand cases in tests/golden/,
 *                        Lemma 4.1, acyclicity, Eq.11 lower
 *                        bound, per-level out-degree bound.
 *   orc_outdeg           out-degree d~(u) of the directed graph (Eq.4)
 *   orc_reorder_none     original order
 *   orc_reorder_degree   D-order: descending d~, ties by id (Q14)
 *   orc_reorder_paper    Algorithm 2 "A-order", Eq.19-22,
 *                        readings Q15-Q21.  PARITY VS AUTHORS' CODE UNPINNED (Fig.8
 *                        BW curve not printed); pinned by: hand cases in
 *                        tests/golden/, bijection, bucket capacity, Eq.3 >= |sum S|.
 *   orc_oriented_keys /  oriented + relabelled CSR, lists ascending: (pi(s), pi(t)) keys,
 *   orc_csr_from_sorted_keys    sorted by a library sort, then counted into offsets
 *   orc_count_forward    T = sum_u sum_{v in N+(u)} |N+(u) ∩ N+(v)| by two-pointer
 *                        merge (forward algorithm); per-vertex t(v).
 *                        pinned: closed forms (K_n, K_{a,b}, wheels, K_{a,b,c},
 *                        friendship/book graphs, cycles, cocktail party),
 *                        brute-force trace(A^3)/6, node-iterator, Σt = 3T,
 *                        invariance over all 3x3 rules and relabelings.
 *   orc_edge_support     per-edge triangle counts (support):
 *                        support(a,b) = |N(a) ∩ N(b)| for every edge of the simple graph,
 *                        by two-pointer merge of the two ascending SYMMETRIC lists (the
 *                        plain definition: a triangle through {a,b} is a common
 *                        neighbour).  pinned: Σ support = 3T, closed forms (K_n: n-2;
 *                        wheel: spokes 2, rim 1; book: spine k, pages 1; friendship: 1;
 *                        K_{a,b}: 0), brute force (A²∘A), t(v) = Σ_{e∋v} support(e) / 2.
 *   orc_aorder_units     Algorithm 2 over arbitrary units with given superiorities (the
 *                        vertex A-order calls it; the edge-unit variant of P:638-640 passes
 *                        the per-edge schedule's work items, Q26).  pinned
 *                        through orc_reorder_paper's pins, and directly: with all S equal
 *                        it fills buckets round-robin; a unit-by-unit brute-force check
 *                        of lines 6/12 (min / max mem_sup, smallest index) on random S.
 *   orc_cost_eq1         Eq.1 numerator Σ_u |n·d~(u) − m|, exact 128-bit
 *   orc_superiority      S(d) = llround(2^20 (F_m(d) − λ F_c(d))) (Eq.22; Q20)
 *   orc_objective_eq3    Eq.3 Σ_i |Σ_{v∈B_i} S(v)| with λ folded into S
 *
 * Build: gcc -O2 -std=c11 -ffp-contract=off -pthread (Makefile).  Single-threaded except
 * orc_count_forward_mt (sources split over threads, per-thread uint64 partials, SURVEY
 * §8(c) O4).
 */
#define _GNU_SOURCE
#include <math.h>
#include <pthread.h>
#include <unistd.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------ */
/* helpers                                                                   */
/* ------------------------------------------------------------------------ */

static int cmp_u64(const void *a, const void *b) {
  uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b;
  return (x > y) - (x < y);
}

static int cmp_u32(const void *a, const void *b) {
  uint32_t x = *(const uint32_t *)a, y = *(const uint32_t *)b;
  return (x > y) - (x < y);
}

static uint64_t edge_key(uint32_t u, uint32_t v) {
  uint32_t lo = u < v ? u : v, hi = u < v ? v : u;
  return ((uint64_t)lo << 32) | hi;
}

/* ------------------------------------------------------------------------ */
/* O1: simple undirected graph ("undirected graph G=(V,E)")     */
/* ------------------------------------------------------------------------ */

/* Drops self-loops u==v and maps each sample to its unordered pair (min,max) as the key
 * (min << 32) | max (Q1).  keys[] needs room for M keys; returns the number of keys k, or
 * -1 if some id >= n.  The keys are then sorted (a library sort, oracle/__init__.py) and
 * orc_unique_sorted removes the duplicates. */
int64_t orc_canonical_keys(const uint32_t *src, const uint32_t *dst, uint64_t M, uint32_t n,
                           uint64_t *keys) {
  uint64_t k = 0;
  for (uint64_t i = 0; i < M; ++i) {
    if (src[i] >= n || dst[i] >= n) return -1;
    if (src[i] == dst[i]) continue;
    keys[k++] = edge_key(src[i], dst[i]);
  }
  return (int64_t)k;
}

/* Keeps the first of every run of equal keys of an ascending array (in place); returns the
 * number kept. */
uint64_t orc_unique_sorted(uint64_t *keys, uint64_t k) {
  uint64_t m = 0;
  for (uint64_t i = 0; i < k; ++i)
    if (m == 0 || keys[m - 1] != keys[i]) keys[m++] = keys[i];
  return m;
}

/* O1 in one call (qsort as the sort step; small inputs). */
int64_t orc_simple_graph(const uint32_t *src, const uint32_t *dst, uint64_t M, uint32_t n,
                         uint64_t *edges) {
  int64_t k = orc_canonical_keys(src, dst, M, n, edges);
  if (k < 0) return -1;
  qsort(edges, (size_t)k, sizeof(uint64_t), cmp_u64);
  return (int64_t)orc_unique_sorted(edges, (uint64_t)k);
}

/* Undirected degree d(v) (Table 1). */
void orc_degrees(const uint64_t *edges, uint64_t m, uint32_t n, uint32_t *deg) {
  memset(deg, 0, sizeof(uint32_t) * n);
  for (uint64_t i = 0; i < m; ++i) {
    deg[edges[i] >> 32]++;
    deg[(uint32_t)edges[i]]++;
  }
}

/* Symmetric adjacency: offs[n+1], adj[2m], each N(v) ascending. */
void orc_sym_csr(const uint64_t *edges, uint64_t m, uint32_t n, uint64_t *offs, uint32_t *adj) {
  uint32_t *deg = (uint32_t *)malloc(sizeof(uint32_t) * (n ? n : 1));
  orc_degrees(edges, m, n, deg);
  offs[0] = 0;
  for (uint32_t v = 0; v < n; ++v) offs[v + 1] = offs[v] + deg[v];
  uint64_t *fill = (uint64_t *)malloc(sizeof(uint64_t) * (n ? n : 1));
  for (uint32_t v = 0; v < n; ++v) fill[v] = offs[v];
  for (uint64_t i = 0; i < m; ++i) {
    uint32_t u = (uint32_t)(edges[i] >> 32), v = (uint32_t)edges[i];
    adj[fill[u]++] = v;
    adj[fill[v]++] = u;
  }
  for (uint32_t v = 0; v < n; ++v)
    qsort(adj + offs[v], offs[v + 1] - offs[v], sizeof(uint32_t), cmp_u32);
  free(fill);
  free(deg);
}

/* ------------------------------------------------------------------------ */
/* O2: edge directing.  dir[i] for edge i=(lo,hi): 0 => lo->hi, 1 => hi->lo.  */
/* ------------------------------------------------------------------------ */

/* ID-based: "directed edge from small vertex id to large vertex id". */
void orc_direct_id(uint64_t m, uint8_t *dir) { memset(dir, 0, m); }

/* Degree-based: "from the small degree vertex to the large degree vertex"
 * (P:19); equal degrees -> smaller id first (Q11). */
void orc_direct_degree(const uint64_t *edges, uint64_t m, const uint32_t *deg, uint8_t *dir) {
  for (uint64_t i = 0; i < m; ++i) {
    uint32_t u = (uint32_t)(edges[i] >> 32), v = (uint32_t)edges[i]; /* u < v */
    int u_first = deg[u] < deg[v] || (deg[u] == deg[v] && u < v);
    dir[i] = u_first ? 0 : 1;
  }
}

static void set_edge(const uint64_t *edges, uint8_t *dir, uint8_t *isset, uint64_t e, uint32_t from) {
  uint32_t lo = (uint32_t)(edges[e] >> 32);
  dir[e] = (from == lo) ? 0 : 1;
  isset[e] = 1;
}

/* Algorithm 1, A-direction, sequential, in the paper's line order.
 *
 * threshold: d <= threshold  <=>  d·|V| <= |E|·2^l      (Q3, Q4; d~avg=|E|/|V| Q2)
 * d(.):      residual degree = still-undirected incident edges     (Q5)
 * line 4-6:  only unpeeled vertices join the frontier              (Q6)
 * line 9-11: both ends in the frontier: compare degrees snapshotted when the
 *            frontier was formed, ties by id, smaller -> larger   (Q7)
 * line 8-16: each edge is set once ("(v,nbr) is unset")           (Q8)
 * line 15-16: a vertex enters nextFrontier once                     (Q9)
 * loop ends when every vertex is peeled; an empty level only doubles the
 *            threshold (line 19)                                    (Q10)
 * Outputs dir[m]; optional sub[n] (subround in which v was peeled), dsnap[n]
 * (snapshot degree), and counters levels / subrounds.  Returns 0. */
int orc_direct_paper(const uint64_t *edges, uint64_t m, uint32_t n, const uint64_t *offs,
                     uint8_t *dir, uint32_t *sub_out, uint32_t *dsnap_out,
                     uint32_t *levels_out, uint32_t *subrounds_out) {
  if (m > UINT32_MAX) return -1; /* edge indices are kept in 32 bits (every config has m < 2^32) */
  size_t nn = n ? n : 1;
  uint32_t *d = (uint32_t *)malloc(sizeof(uint32_t) * nn);        /* residual degree */
  uint32_t *dsnap = (uint32_t *)malloc(sizeof(uint32_t) * nn);
  uint8_t *peeled = (uint8_t *)calloc(nn, 1);
  uint8_t *in_frontier = (uint8_t *)calloc(nn, 1);
  uint8_t *queued = (uint8_t *)calloc(nn, 1);
  uint8_t *isset = (uint8_t *)calloc(m ? m : 1, 1);
  uint32_t *frontier = (uint32_t *)malloc(sizeof(uint32_t) * nn);
  uint32_t *next = (uint32_t *)malloc(sizeof(uint32_t) * nn);
  for (uint32_t v = 0; v < n; ++v) d[v] = (uint32_t)(offs[v + 1] - offs[v]);
  /* N(v) as the indices of its incident undirected edges, in edge order: the neighbour is
   * the other end of edges[e], and the "(v,nbr) is unset" test is a direct lookup (the
   * list order does not matter: frontier members are processed as a set, readings Q7/Q9). */
  uint64_t *cur = (uint64_t *)malloc(sizeof(uint64_t) * nn);
  uint32_t *eid = (uint32_t *)malloc(sizeof(uint32_t) * (2 * m + 1));
  for (uint32_t v = 0; v < n; ++v) cur[v] = offs[v];
  for (uint64_t i = 0; i < m; ++i) {
    uint32_t u = (uint32_t)(edges[i] >> 32), w = (uint32_t)edges[i];
    eid[cur[u]++] = (uint32_t)i;
    eid[cur[w]++] = (uint32_t)i;
  }
  free(cur);

  uint64_t npeeled = 0;
  uint32_t level = 0, subround = 0;
  /* line 2: threshold <- d~avg = |E|/|V| ; kept as the pair (|E|·2^level, |V|). */
  while (npeeled < n) {                                   /* line 3 */
    unsigned __int128 thr_num = (unsigned __int128)m << level; /* |E|·2^level */
    uint64_t nf = 0;
    for (uint32_t v = 0; v < n; ++v)                      /* line 4 */
      if (!peeled[v] && (unsigned __int128)d[v] * n <= thr_num) /* line 5 */
        frontier[nf++] = v;                               /* line 6 */
    while (nf > 0) {                                      /* line 7 */
      for (uint64_t i = 0; i < nf; ++i) {
        uint32_t v = frontier[i];
        in_frontier[v] = 1;
        dsnap[v] = d[v];
        if (sub_out) sub_out[v] = subround;
      }
      uint64_t nn_next = 0;
      for (uint64_t i = 0; i < nf; ++i) {                 /* line 8 */
        uint32_t v = frontier[i];
        for (uint64_t p = offs[v]; p < offs[v + 1]; ++p) {
          uint64_t e = eid[p];
          uint32_t lo = (uint32_t)(edges[e] >> 32), hi = (uint32_t)edges[e];
          uint32_t nbr = lo == v ? hi : lo;
          if (isset[e]) continue;
          if (in_frontier[nbr]) {                         /* line 9 */
            int v_first = dsnap[v] < dsnap[nbr] || (dsnap[v] == dsnap[nbr] && v < nbr);
            uint32_t from = v_first ? v : nbr, to = v_first ? nbr : v;
            set_edge(edges, dir, isset, e, from);         /* line 10 */
            d[to]--;                                      /* line 11 */
          } else if (!peeled[nbr]) {                      /* line 12 */
            set_edge(edges, dir, isset, e, v);            /* line 13 */
            d[nbr]--;                                     /* line 14 */
            if ((unsigned __int128)d[nbr] * n <= thr_num && !queued[nbr]) { /* line 15 */
              queued[nbr] = 1;
              next[nn_next++] = nbr;                      /* line 16 */
            }
          }
        }
      }
      for (uint64_t i = 0; i < nf; ++i) {
        uint32_t v = frontier[i];
        peeled[v] = 1;
        in_frontier[v] = 0;
      }
      npeeled += nf;
      subround++;
      uint32_t *t = frontier; frontier = next; next = t; /* line 17-18 */
      nf = nn_next;
    }
    level++;                                              /* line 19: threshold *= 2 */
  }
  if (dsnap_out) memcpy(dsnap_out, dsnap, sizeof(uint32_t) * n);
  if (levels_out) *levels_out = level;
  if (subrounds_out) *subrounds_out = subround;
  free(d); free(dsnap); free(peeled); free(in_frontier); free(queued); free(isset);
  free(frontier); free(next); free(eid);
  return 0;
}

/* d~(u): out-degree in the directed graph (Eq.4). */
void orc_outdeg(const uint64_t *edges, uint64_t m, uint32_t n, const uint8_t *dir, uint32_t *od) {
  memset(od, 0, sizeof(uint32_t) * n);
  for (uint64_t i = 0; i < m; ++i) {
    uint32_t u = (uint32_t)(edges[i] >> 32), v = (uint32_t)edges[i];
    od[dir[i] ? v : u]++;
  }
}

/* ------------------------------------------------------------------------ */
/* O3: vertex ordering.  perm[old] = new label.                              */
/* ------------------------------------------------------------------------ */

void orc_reorder_none(uint32_t n, uint32_t *perm) {
  for (uint32_t v = 0; v < n; ++v) perm[v] = v;
}

static const uint32_t *g_sort_od; /* qsort has no context argument in C11 */
static int cmp_degree_desc(const void *a, const void *b) {
  uint32_t x = *(const uint32_t *)a, y = *(const uint32_t *)b;
  if (g_sort_od[x] != g_sort_od[y]) return g_sort_od[x] > g_sort_od[y] ? -1 : 1;
  return (x > y) - (x < y);
}

/* D-order: "reordering vertices in the degree descending ... order",
 * on the out-degree d~ of the directed graph, ties by id (Q14). */
void orc_reorder_degree(uint32_t n, const uint32_t *od, uint32_t *perm) {
  uint32_t *order = (uint32_t *)malloc(sizeof(uint32_t) * (n ? n : 1));
  for (uint32_t v = 0; v < n; ++v) order[v] = v;
  g_sort_od = od;
  qsort(order, n, sizeof(uint32_t), cmp_degree_desc);
  for (uint32_t i = 0; i < n; ++i) perm[order[i]] = i;
  free(order);
}

/* Memory superiority of a vertex with out-degree d >= 1:
 *   F_m(d) - λ F_c(d),  F_m = BW(d)^α (Eq.19), F_c = 1/d^β (Eq.20),
 * with Eq.22 (α = β = 1/2) written literally as sqrt(BW(d)) and sqrt(1/d).
 * BW(d) = bw[min(d, bw_len-1)], or d when bw == NULL (Q15).
 * Fixed point: S = llround(2^20 · s) (Q20). */
int64_t orc_superiority(uint32_t d, double lambda, double alpha, double beta, const double *bw,
                        uint32_t bw_len) {
  double b = bw ? bw[d < bw_len ? d : bw_len - 1] : (double)d;
  double fm, fc;
  if (alpha == 0.5) fm = sqrt(b);
  else fm = pow(b, alpha);
  if (beta == 0.5) fc = sqrt(1.0 / (double)d);
  else fc = 1.0 / pow((double)d, beta);
  return llround(ldexp(fm - lambda * fc, 20));
}

/* Binary heap of buckets (Alg.2 lines 2, 10: B.make_min_queue / make_max_queue).
 * Priority: min-queue orders by (mem_sup, index); max-queue by (-mem_sup, index). */
typedef struct {
  uint32_t *h;
  uint32_t size;
  const int64_t *mem_sup;
  int is_max;
} bheap;

static int bh_before(const bheap *q, uint32_t a, uint32_t b) {
  int64_t x = q->mem_sup[a], y = q->mem_sup[b];
  if (x != y) return q->is_max ? x > y : x < y;
  return a < b;
}

static void bh_up(bheap *q, uint32_t i) {
  while (i > 0) {
    uint32_t p = (i - 1) / 2;
    if (!bh_before(q, q->h[i], q->h[p])) break;
    uint32_t t = q->h[i]; q->h[i] = q->h[p]; q->h[p] = t;
    i = p;
  }
}

static void bh_down(bheap *q, uint32_t i) {
  for (;;) {
    uint32_t l = 2 * i + 1, r = l + 1, best = i;
    if (l < q->size && bh_before(q, q->h[l], q->h[best])) best = l;
    if (r < q->size && bh_before(q, q->h[r], q->h[best])) best = r;
    if (best == i) break;
    uint32_t t = q->h[i]; q->h[i] = q->h[best]; q->h[best] = t;
    i = best;
  }
}

static uint32_t bh_pop(bheap *q) {
  uint32_t top = q->h[0];
  q->h[0] = q->h[--q->size];
  if (q->size) bh_down(q, 0);
  return top;
}

static void bh_insert(bheap *q, uint32_t b) {
  q->h[q->size++] = b;
  bh_up(q, q->size - 1);
}

/* Algorithm 2, A-order, readings Q15-Q21:
 *  - d~(v) = 0: no work, F_c(0) undefined -> excluded, appended last by id (Q16)
 *  - V_mem = {S > 0}, V_comp = {S <= 0} among d~ >= 1 (line 3-4; Q19)
 *  - b = ceil(n_active / k) buckets of capacity k; a full bucket is not
 *    re-inserted into the queue (Q17)
 *  - iteration over V_mem / V_comp in ascending id (order = 0, literal "for
 *    all", Q18) or by descending |S| then id (order = 1, LPT option)
 *  - mem_sup sums in int64 fixed point (Q20); relabel buckets in index order,
 *    vertices in insertion order (line 16-20; Q21).
 * Outputs perm[n] (perm[old] = new), bucket_off[b+1]; *nbuckets = b. */
static const int64_t *g_sort_S;
static int cmp_lpt(const void *a, const void *b) {
  uint32_t x = *(const uint32_t *)a, y = *(const uint32_t *)b;
  int64_t sx = g_sort_S[x] < 0 ? -g_sort_S[x] : g_sort_S[x];
  int64_t sy = g_sort_S[y] < 0 ? -g_sort_S[y] : g_sort_S[y];
  if (sx != sy) return sx > sy ? -1 : 1;
  return (x > y) - (x < y);
}

/* Algorithm 2 over n units with given superiorities S[i] (fixed point, λ folded in);
 * unit i takes part iff active[i].  The vertex A-order below calls it with S(d~(v)) and
 * active = (d~(v) > 0); the edge-unit variant (Q26) with the work
 * items of the per-edge schedule.  Outputs pos[i] (new index; inactive units last, in
 * unit order), bucket_off[b+1], *nbuckets = b. */
int orc_aorder_units(uint32_t n, const int64_t *S, const uint8_t *active, uint32_t k, int order,
                     uint32_t *perm, uint32_t *bucket_off, uint32_t *nbuckets) {
  if (k == 0) return -1;
  size_t nn = n ? n : 1;
  uint32_t *vmem = (uint32_t *)malloc(sizeof(uint32_t) * nn);
  uint32_t *vcomp = (uint32_t *)malloc(sizeof(uint32_t) * nn);
  uint32_t nmem = 0, ncomp = 0;
  for (uint32_t v = 0; v < n; ++v) {
    if (!active[v]) continue;
    if (S[v] > 0) vmem[nmem++] = v;   /* line 3: memory dominated */
    else vcomp[ncomp++] = v;           /* line 4: computing dominated */
  }
  if (order == 1) {
    g_sort_S = S;
    qsort(vmem, nmem, sizeof(uint32_t), cmp_lpt);
    qsort(vcomp, ncomp, sizeof(uint32_t), cmp_lpt);
  }
  uint64_t nactive = (uint64_t)nmem + ncomp;
  uint32_t b = (uint32_t)((nactive + k - 1) / k);
  size_t bb = b ? b : 1;
  int64_t *mem_sup = (int64_t *)calloc(bb, sizeof(int64_t));   /* line 1 */
  uint32_t *cnt = (uint32_t *)calloc(bb, sizeof(uint32_t));
  uint32_t *members = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)bb * k);
  bheap q = {(uint32_t *)malloc(sizeof(uint32_t) * bb), 0, mem_sup, 0};
  for (uint32_t i = 0; i < b; ++i) bh_insert(&q, i);            /* line 2 */
  for (uint32_t i = 0; i < nmem; ++i) {                         /* line 5 */
    uint32_t v = vmem[i];
    uint32_t bk = bh_pop(&q);                                   /* line 6 */
    members[(size_t)bk * k + cnt[bk]++] = v;                    /* line 7 */
    mem_sup[bk] += S[v];                                        /* line 8 */
    if (cnt[bk] < k) bh_insert(&q, bk);                         /* line 9 */
  }
  /* line 10: rebuild the (non-full) buckets as a max queue */
  uint32_t *rest = (uint32_t *)malloc(sizeof(uint32_t) * bb);
  uint32_t nrest = 0;
  for (uint32_t i = 0; i < b; ++i)
    if (cnt[i] < k) rest[nrest++] = i;
  q.size = 0;
  q.is_max = 1;
  for (uint32_t i = 0; i < nrest; ++i) bh_insert(&q, rest[i]);
  for (uint32_t i = 0; i < ncomp; ++i) {                        /* line 11 */
    uint32_t v = vcomp[i];
    uint32_t bk = bh_pop(&q);                                   /* line 12 */
    members[(size_t)bk * k + cnt[bk]++] = v;                    /* line 13 */
    mem_sup[bk] += S[v];                                        /* line 14 */
    if (cnt[bk] < k) bh_insert(&q, bk);                         /* line 15 */
  }
  uint32_t idx = 0;                                             /* line 16 */
  for (uint32_t i = 0; i < b; ++i) {                            /* line 17 */
    if (bucket_off) bucket_off[i] = idx;
    for (uint32_t j = 0; j < cnt[i]; ++j)                       /* line 18 */
      perm[members[(size_t)i * k + j]] = idx++;                 /* line 19-20 */
  }
  if (bucket_off) bucket_off[b] = idx;
  for (uint32_t v = 0; v < n; ++v)                              /* Q16: inactive last */
    if (!active[v]) perm[v] = idx++;
  if (nbuckets) *nbuckets = b;
  free(vmem); free(vcomp); free(mem_sup); free(cnt); free(members); free(q.h);
  free(rest);
  return 0;
}

int orc_reorder_paper(uint32_t n, const uint32_t *od, double lambda, double alpha, double beta,
                      const double *bw, uint32_t bw_len, uint32_t k, int order, uint32_t *perm,
                      uint32_t *bucket_off, uint32_t *nbuckets) {
  if (k == 0) return -1;
  size_t nn = n ? n : 1;
  int64_t *S = (int64_t *)calloc(nn, sizeof(int64_t));
  uint8_t *active = (uint8_t *)calloc(nn, 1);
  for (uint32_t v = 0; v < n; ++v) {
    if (od[v] == 0) continue;          /* Q16: d~ = 0 does no work, F_c(0) undefined */
    S[v] = orc_superiority(od[v], lambda, alpha, beta, bw, bw_len);
    active[v] = 1;
  }
  int r = orc_aorder_units(n, S, active, k, order, perm, bucket_off, nbuckets);
  free(S);
  free(active);
  return r;
}

/* Eq.3 objective, with λ folded into S: Σ_i |Σ_{v∈B_i} S(v)| where bucket i
 * holds new labels [bucket_off[i], bucket_off[i+1]).  inv_perm[new] = old. */
int64_t orc_objective_eq3(uint32_t nb, const uint32_t *bucket_off, const uint32_t *inv_perm,
                          const uint32_t *od, double lambda, double alpha, double beta,
                          const double *bw, uint32_t bw_len) {
  int64_t total = 0;
  for (uint32_t i = 0; i < nb; ++i) {
    int64_t s = 0;
    for (uint32_t p = bucket_off[i]; p < bucket_off[i + 1]; ++p) {
      uint32_t v = inv_perm[p];
      if (od[v]) s += orc_superiority(od[v], lambda, alpha, beta, bw, bw_len);
    }
    total += s < 0 ? -s : s;
  }
  return total;
}

/* Eq.1 numerator: n·C(P) = Σ_u |n·d~(u) − m| (exact, 128-bit). */
void orc_cost_eq1(uint32_t n, uint64_t m, const uint32_t *od, uint64_t *lo, uint64_t *hi) {
  unsigned __int128 s = 0;
  for (uint32_t u = 0; u < n; ++u) {
    unsigned __int128 a = (unsigned __int128)n * od[u];
    s += a >= m ? a - m : (unsigned __int128)m - a;
  }
  *lo = (uint64_t)s;
  *hi = (uint64_t)(s >> 64);
}

/* ------------------------------------------------------------------------ */
/* Oriented, relabelled CSR (directed graph G; relabel P:450 line 16-20) */
/* ------------------------------------------------------------------------ */

/* Directed edge i as the key (perm[source] << 32) | perm[target]: sorting these keys
 * (a library sort, oracle/__init__.py) groups every out-list N+(x) by its new label x, each
 * list ascending. */
void orc_oriented_keys(const uint64_t *edges, uint64_t m, const uint8_t *dir, const uint32_t *perm,
                       uint64_t *keys) {
  for (uint64_t i = 0; i < m; ++i) {
    uint32_t u = (uint32_t)(edges[i] >> 32), v = (uint32_t)edges[i];
    uint32_t s = dir[i] ? v : u, t = dir[i] ? u : v;
    keys[i] = ((uint64_t)perm[s] << 32) | perm[t];
  }
}

/* CSR of ascending (source << 32) | target keys: offs[x] = number of keys with source < x,
 * col[i] = target of key i. */
void orc_csr_from_sorted_keys(const uint64_t *keys, uint64_t m, uint32_t n, uint64_t *offs,
                              uint32_t *col) {
  memset(offs, 0, sizeof(uint64_t) * ((size_t)n + 1));
  for (uint64_t i = 0; i < m; ++i) {
    offs[(keys[i] >> 32) + 1]++;
    col[i] = (uint32_t)keys[i];
  }
  for (uint32_t x = 0; x < n; ++x) offs[x + 1] += offs[x];
}

/* ------------------------------------------------------------------------ */
/* Local (per-vertex) triangle counts straight from raw samples, by definition: */
/* t(v) = number of edges among the neighbours N(v) of v in the simple graph    */
/* (P:15).  For full-size parity on sampled vertices; needs no graph build.     */
/* ------------------------------------------------------------------------ */

typedef struct {
  uint64_t *slot; /* key + 1, 0 = empty */
  uint64_t cap;
  uint64_t size;
} u64set;

static uint64_t mix64(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
  return x;
}

static void set_init(u64set *s, uint64_t want) {
  uint64_t cap = 16;
  while (cap < 2 * want + 16) cap <<= 1;
  s->cap = cap;
  s->size = 0;
  s->slot = (uint64_t *)calloc(cap, sizeof(uint64_t));
}

static int set_has(const u64set *s, uint64_t k) {
  uint64_t i = mix64(k) & (s->cap - 1);
  while (s->slot[i]) {
    if (s->slot[i] == k + 1) return 1;
    i = (i + 1) & (s->cap - 1);
  }
  return 0;
}

static void set_add(u64set *s, uint64_t k);

static void set_grow(u64set *s) { /* keep the load factor <= 1/2 */
  u64set t;
  set_init(&t, s->cap);
  for (uint64_t i = 0; i < s->cap; ++i)
    if (s->slot[i]) set_add(&t, s->slot[i] - 1);
  free(s->slot);
  *s = t;
}

static void set_add(u64set *s, uint64_t k) {
  if (2 * (s->size + 1) > s->cap) set_grow(s);
  uint64_t i = mix64(k) & (s->cap - 1);
  while (s->slot[i]) {
    if (s->slot[i] == k + 1) return;
    i = (i + 1) & (s->cap - 1);
  }
  s->slot[i] = k + 1;
  s->size++;
}

/* vs[0..nv): sampled vertices (each with degree <= max_deg in the simple graph, else
 * t = UINT64_MAX is reported).  Two passes over the raw samples. */
int orc_local_triangles(const uint32_t *src, const uint32_t *dst, uint64_t M, const uint32_t *vs,
                        uint32_t nv, uint32_t max_deg, uint64_t *t_out) {
  u64set S, X, E;
  set_init(&S, nv);
  for (uint32_t i = 0; i < nv; ++i) set_add(&S, vs[i]);
  /* pass 1: neighbour sets of the sampled vertices, as (v << 32 | w) pairs */
  uint64_t np = 0, cap = 1024;
  uint64_t *pairs = (uint64_t *)malloc(cap * sizeof(uint64_t));
  for (uint64_t i = 0; i < M; ++i) {
    uint32_t a = src[i], b = dst[i];
    if (a == b) continue;
    for (int side = 0; side < 2; ++side) {
      uint32_t v = side ? b : a, w = side ? a : b;
      if (!set_has(&S, v)) continue;
      if (np == cap) { cap *= 2; pairs = (uint64_t *)realloc(pairs, cap * sizeof(uint64_t)); }
      pairs[np++] = ((uint64_t)v << 32) | w;
    }
  }
  qsort(pairs, np, sizeof(uint64_t), cmp_u64);
  uint64_t k = 0;
  for (uint64_t i = 0; i < np; ++i)
    if (k == 0 || pairs[k - 1] != pairs[i]) pairs[k++] = pairs[i];
  np = k;
  set_init(&X, np);
  for (uint64_t i = 0; i < np; ++i) set_add(&X, (uint32_t)pairs[i]);
  /* pass 2: every edge with both ends in X = ∪ N(v) */
  set_init(&E, 4 * np + 1024);
  for (uint64_t i = 0; i < M; ++i) {
    uint32_t a = src[i], b = dst[i];
    if (a == b || !set_has(&X, a) || !set_has(&X, b)) continue;
    set_add(&E, edge_key(a, b));
  }
  /* t(v) = Σ over pairs x < y in N(v) of [ {x,y} ∈ E ] */
  for (uint32_t q = 0; q < nv; ++q) {
    uint32_t v = vs[q];
    /* N(v) is the run of pairs with high word v (pairs sorted) */
    uint64_t lo = 0, hi = np;
    while (lo < hi) {
      uint64_t mid = lo + (hi - lo) / 2;
      if ((pairs[mid] >> 32) < v) lo = mid + 1;
      else hi = mid;
    }
    uint64_t e = lo;
    while (e < np && (pairs[e] >> 32) == v) ++e;
    if (e - lo > max_deg) { t_out[q] = UINT64_MAX; continue; }
    uint64_t t = 0;
    for (uint64_t i = lo; i < e; ++i)
      for (uint64_t j = i + 1; j < e; ++j)
        t += set_has(&E, edge_key((uint32_t)pairs[i], (uint32_t)pairs[j]));
    t_out[q] = t;
  }
  free(pairs); free(S.slot); free(X.slot); free(E.slot);
  return 0;
}

/* ------------------------------------------------------------------------ */
/* O4: count (forward algorithm): every triangle of the undirected graph */
/* is counted once at its unique source u with u->v, u->w, v->w.       */
/* ------------------------------------------------------------------------ */

/* The triangles counted at one source u: for every v in N+(u), |N+(u) ∩ N+(v)| by a
 * two-pointer merge of the two ascending lists.  tv (per label of the CSR, may be NULL)
 * gets +1 at all three corners of every triangle found (atomically: sources run on
 * several threads). */
static uint64_t count_source(uint32_t u, const uint64_t *offs, const uint32_t *col, uint64_t *tv) {
  uint64_t T = 0;
  for (uint64_t p = offs[u]; p < offs[u + 1]; ++p) {
    uint32_t v = col[p];
    uint64_t i = offs[u], ie = offs[u + 1], j = offs[v], je = offs[v + 1];
    while (i < ie && j < je) {
      if (col[i] < col[j]) ++i;
      else if (col[i] > col[j]) ++j;
      else {
        ++T;
        if (tv) {
          __atomic_fetch_add(&tv[u], 1, __ATOMIC_RELAXED);
          __atomic_fetch_add(&tv[v], 1, __ATOMIC_RELAXED);
          __atomic_fetch_add(&tv[col[i]], 1, __ATOMIC_RELAXED);
        }
        ++i; ++j;
      }
    }
  }
  return T;
}

/* Sources u in [u_begin, u_end) are handed out in chunks of COUNT_CHUNK from a shared
 * counter; every thread sums its own uint64 partial and the partials are added at the
 * end (integer addition: the result does not depend on the split). */
#define COUNT_CHUNK 256
typedef struct {
  const uint64_t *offs;
  const uint32_t *col;
  uint64_t *tv;
  uint32_t u_begin, u_end;
  uint64_t next_chunk; /* shared, atomic */
} count_job;

typedef struct {
  count_job *job;
  uint64_t T;
} count_worker_arg;

static void *count_worker(void *p) {
  count_worker_arg *a = (count_worker_arg *)p;
  count_job *J = a->job;
  uint64_t T = 0;
  for (;;) {
    uint64_t c = __atomic_fetch_add(&J->next_chunk, 1, __ATOMIC_RELAXED);
    uint64_t lo = (uint64_t)J->u_begin + c * COUNT_CHUNK;
    if (lo >= J->u_end) break;
    uint64_t hi = lo + COUNT_CHUNK < J->u_end ? lo + COUNT_CHUNK : J->u_end;
    for (uint64_t u = lo; u < hi; ++u) T += count_source((uint32_t)u, J->offs, J->col, J->tv);
  }
  a->T = T;
  return NULL;
}

/* T over sources [u_begin, u_end) on `threads` threads (<= 0: all online cores). */
uint64_t orc_count_forward_mt(uint32_t n, const uint64_t *offs, const uint32_t *col, uint32_t u_begin,
                              uint32_t u_end, uint64_t *tv, int threads) {
  if (u_end > n) u_end = n;
  if (u_begin >= u_end) return 0;
  if (threads <= 0) threads = (int)sysconf(_SC_NPROCESSORS_ONLN);
  if (threads < 1) threads = 1;
  count_job J = {offs, col, tv, u_begin, u_end, 0};
  pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * threads);
  count_worker_arg *args = (count_worker_arg *)malloc(sizeof(count_worker_arg) * threads);
  int started = 0;
  for (int t = 0; t < threads; ++t) {
    args[t].job = &J;
    args[t].T = 0;
    if (t > 0 && pthread_create(&th[t], NULL, count_worker, &args[t]) == 0) ++started;
    else if (t > 0) args[t].job = NULL; /* not started: its share is taken by the others */
  }
  count_worker(&args[0]);
  uint64_t T = args[0].T;
  for (int t = 1; t < threads; ++t) {
    if (!args[t].job) continue;
    pthread_join(th[t], NULL);
    T += args[t].T;
  }
  (void)started;
  free(th);
  free(args);
  return T;
}

/* Single-threaded entry point (small graphs, range checks). */
uint64_t orc_count_forward(uint32_t n, const uint64_t *offs, const uint32_t *col, uint32_t u_begin,
                           uint32_t u_end, uint64_t *tv) {
  uint64_t T = 0;
  if (u_end > n) u_end = n;
  for (uint32_t u = u_begin; u < u_end; ++u) T += count_source(u, offs, col, tv);
  return T;
}

/* ------------------------------------------------------------------------ */
/* per-edge triangle counts (support)                                        */
/* ------------------------------------------------------------------------ */
/* edges: m sorted keys (min << 32) | max; offs/adj: the symmetric CSR of orc_sym_csr
 * (ascending lists).  out[e] = |N(a) ∩ N(b)| for edge e = {a, b}. */
void orc_edge_support(const uint64_t *edges, uint64_t m, const uint64_t *offs, const uint32_t *adj,
                      uint64_t *out) {
  for (uint64_t e = 0; e < m; ++e) {
    uint32_t a = (uint32_t)(edges[e] >> 32), b = (uint32_t)(edges[e] & 0xffffffffu);
    uint64_t i = offs[a], ie = offs[a + 1], j = offs[b], je = offs[b + 1], c = 0;
    while (i < ie && j < je) {
      if (adj[i] < adj[j]) ++i;
      else if (adj[i] > adj[j]) ++j;
      else { ++c; ++i; ++j; }
    }
    out[e] = c;
  }
}
