"""Closed-form test graphs and brute-force references (test utilities only).

Each builder returns (edges as list of (u, v), n, T, t) where T is the number of
triangles known in closed form and t the per-vertex triangle counts (PAPER.md:15
"total number of triangles"; t(v) = triangles containing v).
"""
from __future__ import annotations

import itertools
from math import comb

import numpy as np


def complete(n):
    e = list(itertools.combinations(range(n), 2))
    return e, n, comb(n, 3), [comb(n - 1, 2)] * n


def complete_bipartite(a, b):
    e = [(i, a + j) for i in range(a) for j in range(b)]
    return e, a + b, 0, [0] * (a + b)


def wheel(r):
    """Hub 0 + rim cycle 1..r. r>=4: r triangles; r=3 is K_4."""
    e = [(0, i) for i in range(1, r + 1)] + [(i, i % r + 1) for i in range(1, r + 1)]
    if r == 3:
        return e, 4, 4, [3, 3, 3, 3]
    return e, r + 1, r, [r] + [2] * r


def complete_tripartite(a, b, c):
    parts = [list(range(a)), list(range(a, a + b)), list(range(a + b, a + b + c))]
    e = []
    for p, q in ((0, 1), (0, 2), (1, 2)):
        e += [(x, y) for x in parts[p] for y in parts[q]]
    t = [b * c] * a + [a * c] * b + [a * b] * c
    return e, a + b + c, a * b * c, t


def friendship(k):
    """k triangles sharing vertex 0."""
    e = []
    for i in range(k):
        x, y = 1 + 2 * i, 2 + 2 * i
        e += [(0, x), (0, y), (x, y)]
    return e, 2 * k + 1, k, [k] + [1] * (2 * k)


def book(k):
    """k triangles sharing the spine edge (0,1)."""
    e = [(0, 1)] + [(0, 2 + i) for i in range(k)] + [(1, 2 + i) for i in range(k)]
    return e, k + 2, k, [k, k] + [1] * k


def cycle(n):
    e = [(i, (i + 1) % n) for i in range(n)]
    T = 1 if n == 3 else 0
    return e, n, T, [T] * n


def star(r):
    return [(0, i) for i in range(1, r + 1)], r + 1, 0, [0] * (r + 1)


def cocktail_party(t):
    """K_{2t} minus the perfect matching {(2i, 2i+1)}: C(2t,3) - t(2t-2)."""
    n = 2 * t
    e = [(u, v) for u, v in itertools.combinations(range(n), 2) if not (u % 2 == 0 and v == u + 1)]
    T = comb(n, 3) - t * (n - 2)
    # each vertex: C(n-2, 2) pairs among its n-2 neighbours minus the (t-1) removed pairs
    tv = comb(n - 2, 2) - (t - 1)
    return e, n, T, [tv] * n


def petersen():
    outer = [(i, (i + 1) % 5) for i in range(5)]
    spokes = [(i, i + 5) for i in range(5)]
    inner = [(5 + i, 5 + (i + 2) % 5) for i in range(5)]
    return outer + spokes + inner, 10, 0, [0] * 10


CLOSED_FORMS = {
    "K3": complete(3), "K4": complete(4), "K7": complete(7), "K12": complete(12),
    "K3_4": complete_bipartite(3, 4), "K6_9": complete_bipartite(6, 9),
    "W3": wheel(3), "W4": wheel(4), "W9": wheel(9),
    "K2_3_4": complete_tripartite(2, 3, 4), "K5_5_5": complete_tripartite(5, 5, 5),
    "F1": friendship(1), "F8": friendship(8), "B1": book(1), "B10": book(10),
    "C3": cycle(3), "C4": cycle(4), "C11": cycle(11), "star9": star(9),
    "CP2": cocktail_party(2), "CP3": cocktail_party(3), "CP6": cocktail_party(6),
    "petersen": petersen(),
}


def noisy_samples(edges, n, rng, pad=0, dup=0.5, loops=3, relabel=True):
    """Turn a simple edge list into raw samples: random relabel onto n+pad ids,
    random endpoint order, duplicated edges and self-loops (Q1 normalisation)."""
    N = n + pad
    perm = rng.permutation(N) if relabel else np.arange(N)
    e = np.array(edges, dtype=np.int64).reshape(-1, 2)
    k = int(len(e) * dup)
    if len(e):
        e = np.concatenate([e, e[rng.integers(0, len(e), size=k)]])
    flip = rng.random(len(e)) < 0.5
    e[flip] = e[flip][:, ::-1]
    if loops:
        lv = rng.integers(0, N, size=loops)
        e = np.concatenate([e, np.stack([lv, lv], 1)])
    rng.shuffle(e)
    src = perm[e[:, 0]] if len(e) else np.zeros(0, dtype=np.int64)
    dst = perm[e[:, 1]] if len(e) else np.zeros(0, dtype=np.int64)
    return src.astype(np.uint32), dst.astype(np.uint32), N, perm


def brute_force(src, dst, n):
    """trace(A^3)/6 and diag(A^3)/2 on the dense adjacency matrix (n <= ~200)."""
    A = np.zeros((n, n), dtype=np.int64)
    for u, v in zip(src.tolist(), dst.tolist()):
        if u != v:
            A[u, v] = A[v, u] = 1
    A3 = A @ A @ A
    return int(np.trace(A3)) // 6, np.diag(A3) // 2


def node_iterator(src, dst, n):
    """Node-iterator: for every vertex, test each neighbour pair for adjacency."""
    adj = [set() for _ in range(n)]
    for u, v in zip(src.tolist(), dst.tolist()):
        if u != v:
            adj[u].add(v)
            adj[v].add(u)
    t = np.zeros(n, dtype=np.int64)
    for v in range(n):
        nb = sorted(adj[v])
        c = 0
        for i in range(len(nb)):
            ai = adj[nb[i]]
            for j in range(i + 1, len(nb)):
                if nb[j] in ai:
                    c += 1
        t[v] = c
    return int(t.sum()) // 3, t


def random_graph(rng, n, m_samples, kind="er"):
    if kind == "er":
        src = rng.integers(0, n, size=m_samples)
        dst = rng.integers(0, n, size=m_samples)
    else:  # skewed: preferential endpoints
        w = 1.0 / np.arange(1, n + 1) ** 0.8
        w /= w.sum()
        src = rng.choice(n, size=m_samples, p=w)
        dst = rng.choice(n, size=m_samples, p=w)
    return src.astype(np.uint32), dst.astype(np.uint32)


# Per-edge triangle counts ("support") in closed form, as a function of
# the builder's own labels (u < v not assumed).
def _support_wheel(r):
    if r == 3:
        return lambda u, v: 2
    return lambda u, v: 2 if 0 in (u, v) else 1


def _support_tripartite(a, b, c):
    def part(x):
        return 0 if x < a else (1 if x < a + b else 2)
    sizes = (a, b, c)
    return lambda u, v: sizes[3 - part(u) - part(v)]


SUPPORT = {
    "K3": lambda u, v: 1, "K4": lambda u, v: 2, "K7": lambda u, v: 5, "K12": lambda u, v: 10,
    "K3_4": lambda u, v: 0, "K6_9": lambda u, v: 0,
    "W3": _support_wheel(3), "W4": _support_wheel(4), "W9": _support_wheel(9),
    "K2_3_4": _support_tripartite(2, 3, 4), "K5_5_5": _support_tripartite(5, 5, 5),
    "F1": lambda u, v: 1, "F8": lambda u, v: 1,
    "B1": lambda u, v: 1, "B10": lambda u, v: 10 if {u, v} == {0, 1} else 1,
    "C3": lambda u, v: 1, "C4": lambda u, v: 0, "C11": lambda u, v: 0, "star9": lambda u, v: 0,
    # K_2t minus a perfect matching: common neighbours of u, v = all but u, v and their partners
    "CP2": lambda u, v: 0, "CP3": lambda u, v: 2, "CP6": lambda u, v: 8,
    "petersen": lambda u, v: 0,
}


def expected_support(name, edges, n, perm):
    """Closed-form support in canonical order of the relabelled simple graph (keys
    (min << 32) | max over perm[]-labels, ascending)."""
    f = SUPPORT[name]
    d = {}
    for u, v in edges:
        a, b = int(perm[u]), int(perm[v])
        d[(min(a, b) << 32) | max(a, b)] = f(u, v)
    keys = sorted(d)
    return np.array(keys, dtype=np.uint64), np.array([d[k] for k in keys], dtype=np.uint64)


def brute_force_support(src, dst, n):
    """(A @ A) ∘ A on the dense adjacency: common neighbours of every adjacent pair, in
    canonical (min, max) order."""
    A = np.zeros((n, n), dtype=np.int64)
    for u, v in zip(src.tolist(), dst.tolist()):
        if u != v:
            A[u, v] = A[v, u] = 1
    A2 = A @ A
    iu, iv = np.nonzero(np.triu(A, 1))
    return ((iu.astype(np.uint64) << np.uint64(32)) | iv.astype(np.uint64)), A2[iu, iv].astype(np.uint64)
