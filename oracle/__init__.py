"""CPU oracle for exact triangle counting with the paper's directing / ordering rules.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It wraps ``oracle/liboracle.so`` (plain C, single-threaded, see
``tc_oracle.c`` for the per-function citations of PAPER.md and the list of
pins).  It shares no code with ``paper_conf_sigmod_hu0l21_b200`` and never
imports it.

Parity status:
  * count T, per-vertex t(v), per-edge support, simple graph, ID/degree directing, D-order: pinned
    (closed forms, brute force, invariants).
  * A-direction (Alg.1) and A-order (Alg.2): "parity unpinned" against the
    authors' code (no worked example survives in PAPER.md); pinned only by hand
    cases (tests/golden/) and the invariants the paper states.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

DIRECT = {"id": 0, "degree": 1, "paper": 2}
REORDER = {"none": 0, "degree": 1, "paper": 2}

# Eq.22 / P:487 defaults: F_c = sqrt(1/d), F_m = sqrt(BW(d)), lambda = 9.682; BW(d)=d (Q15)
DEFAULT_LAMBDA = 9.682
DEFAULT_ALPHA = 0.5
DEFAULT_BETA = 0.5
DEFAULT_K = 32


def _p(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else ctypes.c_void_p(0)


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make` (or __graft_entry__.build())")
        L = ctypes.CDLL(path)
        u64, u32, i32, i64, d, p = (ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int,
                                    ctypes.c_int64, ctypes.c_double, ctypes.c_void_p)
        L.orc_simple_graph.argtypes = [p, p, u64, u32, p]
        L.orc_simple_graph.restype = i64
        L.orc_canonical_keys.argtypes = [p, p, u64, u32, p]
        L.orc_canonical_keys.restype = i64
        L.orc_unique_sorted.argtypes = [p, u64]
        L.orc_unique_sorted.restype = u64
        L.orc_oriented_keys.argtypes = [p, u64, p, p, p]
        L.orc_csr_from_sorted_keys.argtypes = [p, u64, u32, p, p]
        L.orc_degrees.argtypes = [p, u64, u32, p]
        L.orc_sym_csr.argtypes = [p, u64, u32, p, p]
        L.orc_direct_id.argtypes = [u64, p]
        L.orc_direct_degree.argtypes = [p, u64, p, p]
        L.orc_direct_paper.argtypes = [p, u64, u32, p, p, p, p, p, p]
        L.orc_direct_paper.restype = i32
        L.orc_outdeg.argtypes = [p, u64, u32, p, p]
        L.orc_reorder_none.argtypes = [u32, p]
        L.orc_reorder_degree.argtypes = [u32, p, p]
        L.orc_superiority.argtypes = [u32, d, d, d, p, u32]
        L.orc_superiority.restype = i64
        L.orc_reorder_paper.argtypes = [u32, p, d, d, d, p, u32, u32, i32, p, p, p]
        L.orc_reorder_paper.restype = i32
        L.orc_aorder_units.argtypes = [u32, p, p, u32, i32, p, p, p]
        L.orc_aorder_units.restype = i32
        L.orc_objective_eq3.argtypes = [u32, p, p, p, d, d, d, p, u32]
        L.orc_objective_eq3.restype = i64
        L.orc_cost_eq1.argtypes = [u32, u64, p, p, p]
        L.orc_count_forward.argtypes = [u32, p, p, u32, u32, p]
        L.orc_count_forward.restype = u64
        L.orc_count_forward_mt.argtypes = [u32, p, p, u32, u32, p, i32]
        L.orc_count_forward_mt.restype = u64
        L.orc_local_triangles.argtypes = [p, p, u64, p, u32, u32, p]
        L.orc_local_triangles.restype = i32
        L.orc_edge_support.argtypes = [p, u64, p, p, p]
        _LIB = L
    return _LIB


# ---------------------------------------------------------------- primitives


def simple_graph(src, dst, n):
    """O1: sorted unique undirected edges as uint64 keys (min<<32 | max).  The sort step is
    numpy's (a library sort)."""
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    keys = np.empty(max(len(src), 1), dtype=np.uint64)
    k = lib().orc_canonical_keys(_p(src), _p(dst), len(src), n, _p(keys))
    if k < 0:
        raise ValueError("vertex id >= n")
    keys[:k].sort()
    m = lib().orc_unique_sorted(_p(keys), k)
    return keys[:m]  # a view: no second M-sized buffer at full-size configs


def degrees(edges, n):
    deg = np.zeros(max(n, 1), dtype=np.uint32)
    lib().orc_degrees(_p(edges), len(edges), n, _p(deg))
    return deg[:n]


def sym_csr(edges, n):
    offs = np.zeros(n + 1, dtype=np.uint64)
    adj = np.zeros(max(2 * len(edges), 1), dtype=np.uint32)
    lib().orc_sym_csr(_p(edges), len(edges), n, _p(offs), _p(adj))
    return offs, adj[: 2 * len(edges)]


def direct(edges, n, rule):
    """O2: returns (dir[m] uint8, info dict)."""
    m = len(edges)
    d = np.zeros(max(m, 1), dtype=np.uint8)
    info = {}
    if rule == "id":
        lib().orc_direct_id(m, _p(d))
    elif rule == "degree":
        deg = degrees(edges, n)
        lib().orc_direct_degree(_p(edges), m, _p(deg), _p(d))
    elif rule == "paper":
        # list offsets of N(v): exclusive prefix sum of the degrees
        offs = np.zeros(n + 1, dtype=np.uint64)
        np.cumsum(degrees(edges, n), dtype=np.uint64, out=offs[1:])
        sub = np.zeros(max(n, 1), dtype=np.uint32)
        dsnap = np.zeros(max(n, 1), dtype=np.uint32)
        lv = np.zeros(1, dtype=np.uint32)
        sr = np.zeros(1, dtype=np.uint32)
        if lib().orc_direct_paper(_p(edges), m, n, _p(offs), _p(d), _p(sub), _p(dsnap),
                                  _p(lv), _p(sr)) != 0:
            raise ValueError("orc_direct_paper: m >= 2^32 not supported")
        del offs
        info = {"sub": sub[:n], "dsnap": dsnap[:n], "levels": int(lv[0]), "subrounds": int(sr[0])}
    else:
        raise ValueError(rule)
    return d[:m], info


def outdeg(edges, n, dirs):
    od = np.zeros(max(n, 1), dtype=np.uint32)
    lib().orc_outdeg(_p(edges), len(edges), n, _p(dirs), _p(od))
    return od[:n]


def superiority(d, lam=DEFAULT_LAMBDA, alpha=DEFAULT_ALPHA, beta=DEFAULT_BETA, bw=None):
    bwa = None if bw is None else np.ascontiguousarray(bw, dtype=np.float64)
    return int(lib().orc_superiority(d, lam, alpha, beta, _p(bwa), 0 if bwa is None else len(bwa)))


def reorder(od, rule, k=DEFAULT_K, lam=DEFAULT_LAMBDA, alpha=DEFAULT_ALPHA, beta=DEFAULT_BETA,
            bw=None, order=0):
    """O3: returns (perm[n] with perm[old]=new, bucket_off or None)."""
    n = len(od)
    od = np.ascontiguousarray(od, dtype=np.uint32)
    perm = np.zeros(max(n, 1), dtype=np.uint32)
    if rule == "none":
        lib().orc_reorder_none(n, _p(perm))
        return perm[:n], None
    if rule == "degree":
        lib().orc_reorder_degree(n, _p(od), _p(perm))
        return perm[:n], None
    if rule == "paper":
        bwa = None if bw is None else np.ascontiguousarray(bw, dtype=np.float64)
        boff = np.zeros(n + 2, dtype=np.uint32)
        nb = np.zeros(1, dtype=np.uint32)
        rc = lib().orc_reorder_paper(n, _p(od), lam, alpha, beta, _p(bwa),
                                     0 if bwa is None else len(bwa), k, order, _p(perm), _p(boff),
                                     _p(nb))
        if rc != 0:
            raise ValueError("reorder_paper failed")
        return perm[:n], boff[: int(nb[0]) + 1].copy()
    raise ValueError(rule)


def aorder_units(S, active, k=DEFAULT_K, order=0):
    """Algorithm 2 over units with given superiorities (the edge-unit variant of
    P:638-640): returns (pos[i] = new index of unit i, bucket_off)."""
    S = np.ascontiguousarray(S, dtype=np.int64)
    act = np.ascontiguousarray(active, dtype=np.uint8)
    n = len(S)
    pos = np.zeros(max(n, 1), dtype=np.uint32)
    boff = np.zeros(n + 2, dtype=np.uint32)
    nb = np.zeros(1, dtype=np.uint32)
    if lib().orc_aorder_units(n, _p(S), _p(act), k, order, _p(pos), _p(boff), _p(nb)) != 0:
        raise ValueError("aorder_units failed")
    return pos[:n], boff[: int(nb[0]) + 1].copy()


def edge_unit_superiority(offs, col, lam=DEFAULT_LAMBDA, alpha=DEFAULT_ALPHA, beta=DEFAULT_BETA,
                          bw=None):
    """Edge units (Q26): every directed edge u->v of the oriented CSR,
    in CSR order, is a unit whose task streams N+(v) and binary-searches it in N+(u); its
    superiority is that of the streamed list, S(d~(v)) (Eq.19-22 with the vertex model's
    parameters); d~(v) = 0 means no work: not a unit (as Q16 for vertices).
    Returns (S[m] int64, active[m] uint8), indexed by CSR position."""
    offs = np.asarray(offs, dtype=np.int64)
    od = np.diff(offs)
    dv = od[np.asarray(col, dtype=np.int64)] if len(col) else np.zeros(0, np.int64)
    table = {int(d): superiority(int(d), lam, alpha, beta, bw) for d in np.unique(dv) if d > 0}
    S = np.array([table.get(int(d), 0) for d in dv], dtype=np.int64)
    return S, (dv > 0).astype(np.uint8)


def edge_units(offs, col, k=DEFAULT_K, lam=DEFAULT_LAMBDA, alpha=DEFAULT_ALPHA, beta=DEFAULT_BETA,
               bw=None, order=0):
    """Edge-unit A-order: Algorithm 2 (orc_aorder_units) over the edge units of
    edge_unit_superiority.  Returns (units in bucket order as (u << 32) | j — the edge
    u -> col[offs[u] + j] — and bucket_off)."""
    offs = np.asarray(offs, dtype=np.int64)
    S, act = edge_unit_superiority(offs, col, lam, alpha, beta, bw)
    pos, boff = aorder_units(S, act, k, order)
    m = len(S)
    src = np.repeat(np.arange(len(offs) - 1, dtype=np.int64), np.diff(offs))
    j = np.arange(m, dtype=np.int64) - offs[src] if m else np.zeros(0, np.int64)
    units = np.zeros(int(boff[-1]) if len(boff) else 0, dtype=np.uint64)
    a = act.astype(bool)
    units[pos[a].astype(np.int64)] = ((src[a] << 32) | j[a]).astype(np.uint64)
    return units, boff


def oriented_csr(edges, n, dirs, perm):
    """Oriented, relabelled CSR: the (pi(source), pi(target)) keys of the directed edges,
    sorted (numpy's sort), counted into offsets."""
    m = len(edges)
    keys = np.empty(max(m, 1), dtype=np.uint64)
    lib().orc_oriented_keys(_p(edges), m, _p(dirs), _p(np.ascontiguousarray(perm, dtype=np.uint32)),
                            _p(keys))
    keys[:m].sort()
    offs = np.zeros(n + 1, dtype=np.uint64)
    col = np.zeros(max(m, 1), dtype=np.uint32)
    lib().orc_csr_from_sorted_keys(_p(keys), m, n, _p(offs), _p(col))
    del keys
    return offs, col[:m]


def count_forward(offs, col, u_begin=0, u_end=None, per_vertex=False, threads=1):
    """O4 forward count over sources [u_begin, u_end); threads > 1 (or 0 = all online
    cores) splits the sources over threads (orc_count_forward_mt)."""
    n = len(offs) - 1
    if u_end is None:
        u_end = n
    tv = np.zeros(max(n, 1), dtype=np.uint64) if per_vertex else None
    col = col if len(col) else np.zeros(1, dtype=np.uint32)
    if threads == 1:
        T = lib().orc_count_forward(n, _p(offs), _p(col), u_begin, u_end, _p(tv))
    else:
        T = lib().orc_count_forward_mt(n, _p(offs), _p(col), u_begin, u_end, _p(tv), threads)
    return (int(T), tv[:n]) if per_vertex else int(T)


def host_cores():
    """Threads orc_count_forward_mt uses with threads=0 (online cores)."""
    return os.cpu_count() or 1


def local_triangles(src, dst, vertices, max_deg=4096):
    """t(v) = #edges among N(v), straight from raw samples; UINT64_MAX when
    d(v) > max_deg.  For sampled full-size parity (no graph build)."""
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    vs = np.ascontiguousarray(vertices, dtype=np.uint32)
    out = np.zeros(max(len(vs), 1), dtype=np.uint64)
    lib().orc_local_triangles(_p(src), _p(dst), len(src), _p(vs), len(vs), max_deg, _p(out))
    return out[: len(vs)]


def edge_support(edges, n, subset=None):
    """Per-edge triangle counts |N(a) ∩ N(b)| in canonical edge order; `subset` (keys of
    edges of the graph) restricts the output to those edges (sampled full-size parity)."""
    offs, adj = sym_csr(edges, n)
    q = edges if subset is None else np.ascontiguousarray(subset, dtype=np.uint64)
    out = np.zeros(max(len(q), 1), dtype=np.uint64)
    adj = adj if len(adj) else np.zeros(1, dtype=np.uint32)
    lib().orc_edge_support(_p(q), len(q), _p(offs), _p(adj), _p(out))
    return out[:len(q)]


def cost_eq1(n, m, od):
    lo = np.zeros(1, dtype=np.uint64)
    hi = np.zeros(1, dtype=np.uint64)
    lib().orc_cost_eq1(n, m, _p(np.ascontiguousarray(od, dtype=np.uint32)), _p(lo), _p(hi))
    return (int(hi[0]) << 64) | int(lo[0])


def objective_eq3(bucket_off, perm, od, lam=DEFAULT_LAMBDA, alpha=DEFAULT_ALPHA,
                  beta=DEFAULT_BETA, bw=None):
    n = len(perm)
    inv = np.empty(max(n, 1), dtype=np.uint32)
    inv[perm] = np.arange(n, dtype=np.uint32)
    boff = np.ascontiguousarray(bucket_off, dtype=np.uint32)
    bwa = None if bw is None else np.ascontiguousarray(bw, dtype=np.float64)
    return int(lib().orc_objective_eq3(len(boff) - 1, _p(boff), _p(inv),
                                       _p(np.ascontiguousarray(od, dtype=np.uint32)), lam, alpha,
                                       beta, _p(bwa), 0 if bwa is None else len(bwa)))


def range_buckets(od, perm, k):
    """Buckets of k consecutive *active* (d~>0) vertices in new-label order (for
    NONE / DEGREE orderings, the block model of P:186)."""
    n = len(perm)
    inv = np.empty(n, dtype=np.uint32)
    inv[perm] = np.arange(n, dtype=np.uint32)
    active = np.nonzero(od[inv] > 0)[0]
    # buckets as label ranges covering consecutive active labels
    starts = active[::k]
    ends = np.append(active[k - 1::k] + 1, [])
    if len(ends) < len(starts):
        ends = np.append(ends, active[-1] + 1)
    return starts.astype(np.uint32), ends.astype(np.uint32)


# ---------------------------------------------------------------- pipeline


def run(src, dst, n, direct_rule="degree", reorder_rule="none", per_vertex=False,
        k=DEFAULT_K, lam=DEFAULT_LAMBDA, alpha=DEFAULT_ALPHA, beta=DEFAULT_BETA, bw=None,
        order=0, per_edge=False):
    """The whole path on the CPU: O1 -> O2 -> O3 -> oriented CSR -> O4.

    Returns a dict: m, edges, deg, dir, od, perm, bucket_off, offs, col, T,
    t (per ORIGINAL vertex id, if per_vertex), direct_info, eq1 numerator.
    """
    edges = simple_graph(src, dst, n)
    m = len(edges)
    deg = degrees(edges, n)
    dirs, info = direct(edges, n, direct_rule)
    od = outdeg(edges, n, dirs)
    perm, boff = reorder(od, reorder_rule, k=k, lam=lam, alpha=alpha, beta=beta, bw=bw,
                         order=order)
    offs, col = oriented_csr(edges, n, dirs, perm)
    res = dict(m=m, edges=edges, deg=deg, dir=dirs, od=od, perm=perm, bucket_off=boff,
               offs=offs, col=col, direct_info=info, eq1=cost_eq1(n, m, od))
    if per_vertex:
        T, tnew = count_forward(offs, col, per_vertex=True)
        res["t"] = tnew[perm] if n else tnew  # t_orig[v] = t_new[perm[v]]
    else:
        T = count_forward(offs, col)
    res["T"] = T
    if per_edge:
        res["te"] = edge_support(edges, n)
    return res
