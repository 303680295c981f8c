/* tc.h — C-ABI of the B200-native exact triangle-counting library (libtc_b200.so).
 *
 * The path:
 *   tc_graph_from_edges  a1-a3  simple undirected graph G=(V,E) from raw samples
 *                                 ("undirected graph";
 *                                 self-loops dropped, duplicates merged, Q1)
 *   tc_direct            a4-a5  edge directing: ID-based / degree-based /
 *                                 A-direction, Algorithm 1
 *   tc_reorder           a6-a7  vertex ordering: original / D-order /
 *                                 A-order, Algorithm 2 (Eq.19-22);
 *                                 then the oriented CSR in the new labels
 *   tc_count             a8-a10 T = sum_u sum_{v in N+(u)} |N+(u) ∩ N+(v)| by
 *                                 binary-search list intersection (P:31, P:118,
 *                                 P:154-170), optional per-vertex counts t(v)
 *   tc_count_dist        a11    the same on a work-balanced slice per GPU, partials
 *                                 combined with one ncclAllReduce (uint64, sum)
 *
 * Conventions (all entry points):
 *   - Every call returns tc_status; TC_OK = 0.  On error the message is in
 *     tc_last_error() (thread-local, valid until the next call on that thread) and
 *     no output argument is written.  There is NO CPU fallback: without a CUDA
 *     device every call that needs one returns TC_ERR_CUDA.
 *   - Pointers may be host or device memory unless stated otherwise; the library
 *     detects which (cudaPointerGetAttributes).  The caller keeps ownership of every
 *     pointer it passes; the library copies what it needs and never frees caller
 *     memory.  A tc_graph owns all device buffers it allocates (stream-ordered
 *     allocations on its stream) and releases them in tc_graph_free.
 *   - All work is enqueued on the graph's stream; every call is synchronous on
 *     return (results are readable by the host) unless stated otherwise.
 *   - Vertex ids are uint32 (n <= 2^32-1); edge counts / offsets / triangle counts are
 *     uint64 (Q24: twitter_rv alone has 34.8e9 triangles).
 *   - A tc_graph is not thread-safe; distinct graphs may be used from distinct threads.
 *
 * State machine: from_edges -> direct -> [reorder] -> count (repeatable).
 *   tc_reorder or tc_count before tc_direct -> TC_ERR_STATE; calling tc_direct again
 *   discards any reordering.  tc_count without tc_reorder counts in original order.
 */
#ifndef TC_B200_H
#define TC_B200_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct tc_graph tc_graph; /* opaque */

typedef enum {
  TC_OK = 0,
  TC_ERR_INVALID = 1, /* bad argument (id >= n, NULL where required, bad rule/params) */
  TC_ERR_OOM = 2,     /* device allocation failed */
  TC_ERR_CUDA = 3,    /* CUDA error or no CUDA device */
  TC_ERR_NCCL = 4,    /* NCCL unavailable or failed */
  TC_ERR_STATE = 5    /* call out of order (see state machine) */
} tc_status;

typedef enum { TC_DIRECT_ID = 0, TC_DIRECT_DEGREE = 1, TC_DIRECT_PAPER = 2 } tc_direct_rule;
typedef enum { TC_REORDER_NONE = 0, TC_REORDER_DEGREE = 1, TC_REORDER_PAPER = 2 } tc_reorder_rule;

/* Counting schedule (step a8).  BUCKETED: (u, 32-v chunk) work items, heaviest
 * ⌊log2 d~⌋ bin first, fetched dynamically.  RANGE: CTA i takes the k consecutive labels
 * of bucket i — the block model A-order optimises ("every consecutive k vertices are
 * grouped into a bucket ... assigned to one block").  AUTO = BUCKETED (measured
 * faster on B200 for every ordering). */
/* EDGE_AORDER: A-order with edge units (the paper's variant for per-edge schedules,
 * P:638-640 "edge is reorder unit ... resource usage tense of edges instead of vertices"):
 * every directed edge u->v of the oriented CSR is a unit whose task streams N+(v) and
 * binary-searches it in N+(u); its superiority is S(d~(v)) of the streamed list, d~(v) = 0
 * -> no work, not a unit (Q26).  Algorithm 2 puts the units in buckets of k
 * (tc_aorder_params of the last tc_reorder, else defaults), CTA i takes bucket i, a warp per
 * unit.  Built by tc_set_schedule when the oriented CSR exists (its device time added to
 * ms_reorder), else by the first count after the CSR changes. */
typedef enum { TC_SCHED_AUTO = 0, TC_SCHED_BUCKETED = 1, TC_SCHED_RANGE = 2, TC_SCHED_EDGE_AORDER = 3 } tc_schedule;

/* A-order parameters (Alg.2 inputs "F_c, F_m, λ"; Eq.19-22).
 *   F_m(d) = BW(d)^alpha (Eq.19), F_c(d) = 1/d^beta (Eq.20); alpha = beta = 1/2 is
 *   evaluated literally as sqrt(BW(d)) and sqrt(1/d) (Eq.22).  BW(d) = bw[min(d,
 *   bw_len-1)], or d when bw == NULL (Q15).  Memory superiority F_m - λ F_c in
 *   fixed point llround(2^20 x) (Q20).  k = bucket capacity = vertices per CTA in
 *   the RANGE schedule (Q17).  order: 0 = ascending id (literal "for all"), 1 =
 *   descending |superiority| (LPT) (Q18). */
typedef struct {
  double lambda;     /* default 9.682 */
  double alpha;      /* default 0.5 */
  double beta;       /* default 0.5 */
  const double *bw;  /* host pointer or NULL */
  uint32_t bw_len;
  uint32_t k;        /* default 32 */
  int32_t order;     /* default 0 */
} tc_aorder_params;

/* Counters and timings of a graph (plain struct, layout fixed). */
typedef struct {
  uint64_t n, m, samples;        /* |V|, |E| after normalisation, raw samples */
  uint64_t max_degree;           /* max undirected degree d */
  uint64_t max_outdeg;           /* max out-degree d~ after directing */
  uint64_t eq1_lo, eq1_hi;       /* Eq.1 numerator n*C(P) = sum_u |n d~(u) - m| (128-bit) */
  int64_t eq3;                   /* Eq.3 objective sum_i |sum_{v in B_i} S(v)| (A-order), else -1 */
  uint32_t levels, subrounds;    /* A-direction threshold doublings and frontier rounds */
  uint32_t nbuckets;             /* A-order buckets b */
  uint32_t direct_rule, reorder_rule, schedule;
  uint64_t triangles;            /* last count */
  uint64_t wedges;               /* sum_u sum_{v in N+(u)} d~(v) (after tc_analyze) */
  uint64_t alg_bytes;            /* count kernel algorithmic DRAM bytes, no-reuse 32-B sector model of
                                    the schedule a plain tc_count runs: per edge the streamed list
                                    (the shorter one, or N+(v) in Hu's pattern) + its offsets, per
                                    source its staged list (tc_analyze) */
  double ms_build, ms_direct, ms_reorder, ms_count; /* device time of the last call of each */
  double ms_count_kernel;        /* device time of the count kernels alone (last tc_count) */
  uint64_t count_launches;       /* kernels launched by the last tc_count */
  int64_t eq3_units;             /* Eq.3 objective of the edge-unit buckets (EDGE_AORDER), else -1 */
  uint64_t nunits;               /* edge units (active edges) in those buckets */
  uint64_t unit_buckets;         /* number of edge-unit buckets (EDGE_AORDER), else 0 */
} tc_stats_t;

/* a1-a3.  Raw samples (src[i], dst[i]), i < num_edges; ids must be < num_vertices.
 * num_vertices = |V| including isolated vertices (Q2).  device: CUDA ordinal;
 * cuda_stream: cudaStream_t to use (NULL = the legacy default stream).
 * On success *out is a new graph. */
tc_status tc_graph_from_edges(const uint32_t *src, const uint32_t *dst, uint64_t num_edges,
                              uint32_t num_vertices, int device, void *cuda_stream,
                              tc_graph **out);

/* a4-a5.  Orient every edge u->v iff key(u) < key(v), a total order, so 𝒢 has no
 * directed 3-cycle: ID key = u; DEGREE key = (d(u), u) (Q11); PAPER key =
 * (subround, snapshot residual degree, u) from the bulk-synchronous peeling of
 * Algorithm 1 (readings Q3-Q10). */
tc_status tc_direct(tc_graph *g, tc_direct_rule rule);

/* a6-a7.  p may be NULL (defaults above) and is ignored unless rule == PAPER.
 * Builds the oriented CSR in the new labels (lists ascending). */
tc_status tc_reorder(tc_graph *g, tc_reorder_rule rule, const tc_aorder_params *p);

/* a6-a7 on N ranks holding replicas of the same directed graph (a11 plumbing):
 * identical result to tc_reorder on every rank, but for rule == PAPER the Algorithm 2
 * greedy (sequential host work) runs on rank 0 only and pi / bucket_off / the Eq.3
 * objective reach the other ranks by ncclBroadcast on the graph's stream (instead of N
 * concurrent host greedies); other rules run locally.  nccl_comm: ncclComm_t from
 * tc_nccl_comm_init, rank in [0, world).  Collective: every rank must call it.  Errors:
 * TC_ERR_INVALID (bad comm/rank/world/params), TC_ERR_STATE (before tc_direct),
 * TC_ERR_NCCL. */
tc_status tc_reorder_dist(tc_graph *g, tc_reorder_rule rule, const tc_aorder_params *p, void *nccl_comm,
                          int rank, int world);

/* Schedule used by subsequent counts (TC_SCHED_AUTO by default). */
tc_status tc_set_schedule(tc_graph *g, tc_schedule s);

/* a8-a10.  *triangles = T.  per_vertex: NULL, or n entries (host or device) that
 * receive t(v) indexed by ORIGINAL vertex id (Q23). */
tc_status tc_count(tc_graph *g, uint64_t *triangles, uint64_t *per_vertex);

/* Per-edge triangle counts ("support", the input of k-truss; P:15 and
 * P:61 name TC's uses).  per_edge[e] = number of triangles containing the e-th edge of the
 * simple undirected graph in canonical order — the order of tc_export_graph's `edges`
 * (keys (min << 32) | max over the caller's vertex ids, ascending) — so it does not depend
 * on the directing or ordering rule.  m entries, host or device memory (caller-owned);
 * *triangles receives T.  Same kernels as tc_count, with three aggregated increments per
 * triangle (edges (u,v), (u,w), (v,w) of u -> v -> w).  Requires tc_direct; errors as
 * tc_count (TC_ERR_INVALID when per_edge is NULL and m > 0). */
tc_status tc_count_edges(tc_graph *g, uint64_t *triangles, uint64_t *per_edge);

/* Count only triangles whose source vertex (the lowest in the orientation) has a
 * new label in [u_begin, u_end); per_vertex (optional, n entries) receives this
 * slice's contributions (original ids).  The sum over a partition of [0,n) is T. */
tc_status tc_count_range(tc_graph *g, uint32_t u_begin, uint32_t u_end, uint64_t *triangles,
                         uint64_t *per_vertex);

/* Work-balanced contiguous ranges for `world` GPUs: bounds[0..world], bounds[0]=0,
 * bounds[world]=n (host memory).  Work model = the elements the count streams for the
 * source's edges: w(u) = d~(u) + sum_{v in N+(u)} min(d~(u), d~(v)) when a plain count runs
 * the shorter-list schedule (option "shorter", max d~ >= 64), else d~(u) + sum d~(v). */
tc_status tc_partition(tc_graph *g, uint32_t world, uint32_t *bounds);

/* a11.  NCCL plumbing (libnccl.so.2 is dlopen'ed; TC_ERR_NCCL if absent).
 * unique_id: 128 bytes (ncclUniqueId), host memory.  The id is produced on rank 0
 * and shared out of band (torch.distributed in the Python binding). */
tc_status tc_nccl_get_unique_id(void *unique_id);
tc_status tc_nccl_comm_init(const void *unique_id, int rank, int world, int device, void **comm);
tc_status tc_nccl_comm_destroy(void *comm);

/* Rank `rank` counts its tc_partition slice, then one ncclAllReduce(sum, uint64)
 * over `comm` (and one over n uint64 when per_vertex != NULL).  Every rank gets T. */
tc_status tc_count_dist(tc_graph *g, void *comm, int rank, int world, uint64_t *triangles,
                        uint64_t *per_vertex);

/* Extra statistics (wedges, algorithmic bytes of the count kernel); not on the hot path. */
tc_status tc_analyze(tc_graph *g);
tc_status tc_get_stats(const tc_graph *g, tc_stats_t *out);

/* Parity exports (host or device buffers).  offs: n+1, col: m (final labels),
 * perm: n (perm[old] = new; identity for NONE).  Any pointer may be NULL. */
tc_status tc_export(tc_graph *g, uint64_t *offs, uint32_t *col, uint32_t *perm);
/* Undirected simple graph: edges (m keys (min<<32)|max ascending), degree d (n). */
tc_status tc_export_graph(tc_graph *g, uint64_t *edges, uint32_t *degree);
/* Directing internals: out-degree d~ (n, original ids); for PAPER also sub[n]
 * (peeling subround) and dsnap[n] (snapshot residual degree). */
tc_status tc_export_direct(tc_graph *g, uint32_t *outdeg, uint32_t *sub, uint32_t *dsnap);
/* A-order buckets: bucket_off[nbuckets+1] (host or device). */
tc_status tc_export_buckets(tc_graph *g, uint32_t *bucket_off);
/* Edge-unit A-order (TC_SCHED_EDGE_AORDER, built on demand): units[nunits] = the active
 * edge units in bucket order, each (u << 32) | j (source u in final labels, the edge
 * u -> col[offs[u] + j]); unit_off[unit_buckets+1] (tc_stats_t).  Host or device pointers. */
tc_status tc_export_units(tc_graph *g, uint64_t *units, uint32_t *unit_off);

/* Library options: "profile" (0/1: per-stage CUDA-event timing in tc_stats_t, default 1),
 * "kernel_profile" (0/1: per-kernel event pairs for tc_profile_report, default 0),
 * "small_cap" (power of two in [32, 2048]; d~(u) below it is counted with N+(u) in a
 * per-warp shared-memory slice, default 256), "l2_persist" (0/1: L2 access-policy window
 * over the CSR during counts, default 0), "split" (0/1: with original labels, build the
 * oriented CSR by splitting the sorted edge list into forward and reversed runs and sorting
 * only the reversed run, default 1; 0 = sort every oriented key), "intersect" (0 = binary
 * search, the paper's kernel, default; 1 = sort-merge: each lane two-pointer-merges N+(u)
 * with its N+(v), the strategy of the paper's §6.2 comparison; 2 = bitmap:
 * Bisson's block-per-vertex pattern, N+(u) marked in a |V|-bit bitmap, one thread per v
 * per barrier-closed superstep, the kernel of Fig.13; 1 and 2 apply to
 * tc_count / tc_count_range / tc_count_dist without per-vertex output), "peel_coop" (0/1:
 * run the whole A-direction peel as one cooperative launch with grid-wide barriers instead
 * of 5 launches and a host round trip per subround, default 1), "peel_red" (-1 = auto, the
 * default: from 2^25 vertices the cooperative peel decrements residual degrees with
 * fire-and-forget reductions and finds the next frontier by a scan of the unpeeled
 * vertices, the same set as the per-decrement crossing test of Alg.1; 0 / 1 force it), "lean" (0/1: when every
 * warp-item list of a count has < 32 entries, run the 32-register short-list instantiation
 * of the warp-item kernel, 8 CTAs per SM; default 1), "trim_memory" (any
 * value: release the library's cached device blocks), "extra_compute" (-1 = off, the
 * default; q in 0..1024: counts run an instrumented copy of the warp-item kernel that
 * performs p_c = q/8 extra searches of the staged N+(u) per wedge (whole 32-wedge warp
 * steps, spread evenly), results discarded — the
 * balance-point experiment of §5.3, used to re-fit the A-order model on B200
 * (tools/refit.py); counts are unchanged), "shorter" (0/1, default 1: in the counts without
 * per-vertex/per-edge output of the bucketed schedule, every directed edge u->v streams the
 * SHORTER of N+(u), N+(v) and binary-searches its elements in the other, staged once for
 * all edges that search it — SURVEY.md §8(a) a9 "the shorter of the two lists per edge ...
 * probed into the longer list"; 0 = always stream N+(v) against the staged N+(u), Hu's
 * pattern), "owner_span" / "owner_lspan" (streamed lists per warp / CTA work item of
 * that schedule, defaults 128 / 2048), "otiles" (0 = auto, 1 = off (default), 2..255: the CTA work
 * items of that schedule run in this many owner-label tiles — the owners of each long
 * staged list grouped by the label tile of the owner, items listed tile by tile, so the
 * lists streamed at any moment lie in one tile of col and are re-read from L2 instead of
 * HBM; auto = ceil(col bytes / "otile_mb" MB), default 48), "otile_min" (a long list is
 * tiled when it has >= otile_min x tiles owners, default 4), "cuckoo" (count-only CTA work
 * items: the staged list is held as a cuckoo hash set — two tables of 2^b slots, probe =
 * two independent shared loads — instead of the sorted piece with its bracket table; the
 * value is the eviction limit per insertion, default 64, 0 = off; an insertion that fails
 * falls back to the sorted piece, counts are unchanged), "aorder_device" (1 = default: the
 * A-order classification into memory- / computing-dominated vertices (Alg.2 lines 3-4) and
 * the relabel (lines 16-20) run on the device around the host's sequential greedy; 0 = all
 * on the host; identical pi), "e2sort" (shorter-list schedule: the owners an edge gives
 * to the endpoint with the longer list grouped by a radix sort of (x, u) pairs instead of
 * per-x cursor atomics; -1 = auto (from 2^28 edges), 0 / 1). */
tc_status tc_set_option(const char *key, int64_t value);

/* Per-kernel profile since the last reset, as JSON text into buf (host, cap bytes):
 * {"kernel": {"ms": total, "launches": L, "bytes": algorithmic bytes}, ...}.
 * Synchronises on the recorded events.  reset != 0 clears the records. */
tc_status tc_profile_report(char *buf, uint64_t cap, int reset);

void tc_graph_free(tc_graph *g);
const char *tc_last_error(void);
const char *tc_version(void);

#ifdef __cplusplus
}
#endif
#endif /* TC_B200_H */
