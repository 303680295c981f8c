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
        L.orc_degrees.argtypes = [p, u64, u32, p]
        L.orc_sym_csr.argtypes = [p, u64, u32, p, p]
        L.orc_direct_id.argtypes = [u64, p]
        L.orc_direct_degree.argtypes = [p, u64, p, p]
        L.orc_direct_paper.argtypes = [p, u64, u32, p, p, p, p, p, p, p]
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
        L.orc_oriented_csr.argtypes = [p, u64, u32, p, p, p, p]
        L.orc_count_forward.argtypes = [u32, p, p, u32, u32, p]
        L.orc_count_forward.restype = u64
        L.orc_local_triangles.argtypes = [p, p, u64, p, u32, u32, p]
        L.orc_local_triangles.restype = i32
        L.orc_edge_support.argtypes = [p, u64, p, p, p]
        _LIB = L
    return _LIB


# ---------------------------------------------------------------- primitives


def simple_graph(src, dst, n):
    """O1: sorted unique undirected edges as uint64 keys (min<<32 | max)."""
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    edges = np.empty(max(len(src), 1), dtype=np.uint64)
    m = lib().orc_simple_graph(_p(src), _p(dst), len(src), n, _p(edges))
    if m < 0:
        raise ValueError("vertex id >= n")
    return edges[:m].copy()


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
        offs, adj = sym_csr(edges, n)
        sub = np.zeros(max(n, 1), dtype=np.uint32)
        dsnap = np.zeros(max(n, 1), dtype=np.uint32)
        lv = np.zeros(1, dtype=np.uint32)
        sr = np.zeros(1, dtype=np.uint32)
        lib().orc_direct_paper(_p(edges), m, n, _p(offs), _p(adj), _p(d), _p(sub), _p(dsnap),
                               _p(lv), _p(sr))
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


def edge_units(offs, col, k=DEFAULT_K, lam=DEFAULT_LAMBDA, alpha=DEFAULT_ALPHA, beta=DEFAULT_BETA,
               bw=None, order=0):
    """Edge-unit A-order (Q26): units are the per-edge schedule's work items
    (u, c0) — 32 consecutive out-edges of u, u ascending, for d~(u) >= 2 — with superiority
    the sum of S(d~(v)) over the item's edges u->v (0 for d~(v) = 0); a unit with no wedge
    (every d~(v) = 0) takes no part.  Returns (units in bucket order as (u << 32) | c0,
    bucket_off)."""
    offs = np.asarray(offs, dtype=np.int64)
    col = np.asarray(col)
    od = np.diff(offs)
    table = {}
    items, sup, act = [], [], []
    for u in range(len(od)):
        d = int(od[u])
        if d < 2:
            continue
        for c0 in range(0, d, 32):
            s, a = 0, False
            for v in col[offs[u] + c0: offs[u] + min(d, c0 + 32)]:
                dv = int(od[v])
                if dv:
                    if dv not in table:
                        table[dv] = superiority(dv, lam, alpha, beta, bw)
                    s += table[dv]
                    a = True
            items.append((u << 32) | c0)
            sup.append(s)
            act.append(1 if a else 0)
    pos, boff = aorder_units(np.array(sup, dtype=np.int64), np.array(act, dtype=np.uint8), k, order)
    units = np.zeros(int(boff[-1]) if len(boff) else 0, dtype=np.uint64)
    for i, it in enumerate(items):
        if act[i]:
            units[pos[i]] = it
    return units, boff


def oriented_csr(edges, n, dirs, perm):
    offs = np.zeros(n + 1, dtype=np.uint64)
    col = np.zeros(max(len(edges), 1), dtype=np.uint32)
    lib().orc_oriented_csr(_p(edges), len(edges), n, _p(dirs), _p(perm), _p(offs), _p(col))
    return offs, col[: len(edges)]


def count_forward(offs, col, u_begin=0, u_end=None, per_vertex=False):
    n = len(offs) - 1
    if u_end is None:
        u_end = n
    tv = np.zeros(max(n, 1), dtype=np.uint64) if per_vertex else None
    col = col if len(col) else np.zeros(1, dtype=np.uint32)
    T = lib().orc_count_forward(n, _p(offs), _p(col), u_begin, u_end, _p(tv))
    return (int(T), tv[:n]) if per_vertex else int(T)


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
