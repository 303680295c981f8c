"""Pins for the oracle's preprocessing rules: simple-graph normalisation (O1),
ID / degree / A-direction (O2, Alg.1), D-order and
A-order (O3, Alg.2), Eq.1 / Eq.3 statistics.  CPU only.

A-direction and A-order have no surviving worked example in PAPER.md, so they
are pinned by hand-traced cases (tests/golden/) and by the invariants the paper
states (Lemma 4.1, acyclicity P:220, Eq.11 bound P:319-323)."""
import itertools
import math
import os

import numpy as np
import pytest

import graphgen
import oracle
from tests import graphs
from tests.conftest import GOLDEN, read_golden


def _edge_dirs(res_edges, dirs):
    """Directed pairs (from, to) of the oracle's orientation."""
    lo = (res_edges >> np.uint64(32)).astype(np.int64)
    hi = (res_edges & np.uint64(0xFFFFFFFF)).astype(np.int64)
    fr = np.where(dirs == 0, lo, hi)
    to = np.where(dirs == 0, hi, lo)
    return set(zip(fr.tolist(), to.tolist()))


def test_simple_graph_matches_set_semantics():
    rng = np.random.default_rng(1)
    for _ in range(20):
        n = int(rng.integers(1, 50))
        M = int(rng.integers(0, 300))
        src = rng.integers(0, n, M).astype(np.uint32)
        dst = rng.integers(0, n, M).astype(np.uint32)
        want = sorted({(min(a, b), max(a, b)) for a, b in zip(src.tolist(), dst.tolist()) if a != b})
        got = oracle.simple_graph(src, dst, n)
        pairs = [(int(k) >> 32, int(k) & 0xFFFFFFFF) for k in got]
        assert pairs == want
        deg = oracle.degrees(got, n)
        want_deg = np.zeros(n, np.int64)
        for a, b in want:
            want_deg[a] += 1
            want_deg[b] += 1
        assert np.array_equal(deg.astype(np.int64), want_deg)


def test_sym_csr_lists_sorted_and_complete():
    src, dst = graphgen.generate_cpu(graphgen.rmat_spec(9, 8, 11))
    e = oracle.simple_graph(src, dst, 512)
    offs, adj = oracle.sym_csr(e, 512)
    S = {(int(k) >> 32, int(k) & 0xFFFFFFFF) for k in e}
    for v in range(512):
        lst = adj[offs[v]:offs[v + 1]].tolist()
        assert lst == sorted(lst)
        for w in lst:
            assert (min(v, w), max(v, w)) in S


@pytest.mark.parametrize("seed", range(5))
def test_id_and_degree_rules_by_definition(seed):
    rng = np.random.default_rng(seed)
    n = 80
    src, dst = graphs.random_graph(rng, n, 400, "skew")
    e = oracle.simple_graph(src, dst, n)
    deg = oracle.degrees(e, n)
    d_id, _ = oracle.direct(e, n, "id")
    d_dg, _ = oracle.direct(e, n, "degree")
    for (fr, to) in _edge_dirs(e, d_id):
        assert fr < to  # P:19 ID-based
    for (fr, to) in _edge_dirs(e, d_dg):
        assert (deg[fr], fr) < (deg[to], to)  # P:19 degree-based, Q11
    od = oracle.outdeg(e, n, d_dg)
    # degree rule bound: max out-degree <= sqrt(2m)
    assert od.max() <= math.sqrt(2 * len(e))


@pytest.mark.parametrize("name", ["adirection_hand7.txt", "adirection_star.txt",
                                  "adirection_k4.txt"])
def test_adirection_golden(name):
    g = read_golden(name)
    n = g["n"]
    src = np.array([a for a, b in g["edge"]], np.uint32)
    dst = np.array([b for a, b in g["edge"]], np.uint32)
    e = oracle.simple_graph(src, dst, n)
    dirs, info = oracle.direct(e, n, "paper")
    assert _edge_dirs(e, dirs) == set(g["dir"])
    assert info["sub"].tolist() == g["sub"]
    assert info["dsnap"].tolist() == g["dsnap"]
    assert info["levels"] == g["levels"]
    assert info["subrounds"] == g["subrounds"]
    assert oracle.run(src, dst, n, "paper", "none")["T"] == g["T"]


def _adirection_invariants(src, dst, n):
    e = oracle.simple_graph(src, dst, n)
    m = len(e)
    deg = oracle.degrees(e, n).astype(np.int64)
    dirs, info = oracle.direct(e, n, "paper")
    od = oracle.outdeg(e, n, dirs).astype(np.int64)
    sub, dsnap = info["sub"].astype(np.int64), info["dsnap"].astype(np.int64)
    pairs = _edge_dirs(e, dirs)
    assert len(pairs) == m  # every edge set exactly once
    for fr, to in pairs:
        # orientation is the total order (sub, dsnap, id): acyclic
        assert (sub[fr], dsnap[fr], fr) < (sub[to], dsnap[to], to)
        # Lemma 4.1 first phase: d*n <= m (first frontier) -> d*n > m
        if deg[fr] * n > m:
            assert not (deg[to] * n <= m)
    # out-degree never exceeds the snapshot, which respects its level threshold
    assert np.all(od <= dsnap)
    assert np.all(dsnap * n <= m * 2 ** max(info["levels"] - 1, 0))
    # Eq.11 lower bound: n*C >= sum_{n d(v) < m} (m - n d(v))
    lb = int(np.sum(np.maximum(m - n * deg, 0)))
    assert oracle.cost_eq1(n, m, od) >= lb
    return e, dirs, od


@pytest.mark.parametrize("seed", range(8))
def test_adirection_invariants_random(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(5, 300))
    src, dst = graphs.random_graph(rng, n, int(rng.integers(n, 8 * n)), "skew" if seed % 2 else "er")
    _adirection_invariants(src, dst, n)


def test_adirection_invariants_rmat():
    spec = graphgen.rmat_spec(12, 16, 1)
    src, dst = graphgen.generate_cpu(spec)
    e, dirs, od = _adirection_invariants(src, dst, spec.n)
    # on R-MAT, A-direction lowers the max out-degree vs degree directing
    d_dg, _ = oracle.direct(e, spec.n, "degree")
    assert od.max() <= oracle.outdeg(e, spec.n, d_dg).max()


def test_superiority_sign_boundary():
    """With BW(d)=d, s(d) = sqrt(d) - λ/sqrt(d) > 0  <=>  d > λ = 9.682 (Eq.22, Q15)."""
    for d in range(1, 200):
        S = oracle.superiority(d)
        assert (S > 0) == (d >= 10), d
    vals = [oracle.superiority(d) for d in range(1, 500)]
    assert all(a < b for a, b in zip(vals, vals[1:]))  # increasing in d
    # λ = 0: s(d) = sqrt(d) exactly representable for squares: S = 2^20 * sqrt(d)
    for r in range(1, 40):
        assert oracle.superiority(r * r, lam=0.0) == r << 20


def test_aorder_golden():
    g = read_golden("aorder_hand7.txt")
    od = np.array(g["od"], np.uint32)
    perm, boff = oracle.reorder(od, "paper", k=g["k"])
    assert perm.tolist() == g["perm"] and boff.tolist() == g["bucket_off"]
    perm, boff = oracle.reorder(od, "paper", k=g["k"], order=1)
    assert perm.tolist() == g["perm_lpt"] and boff.tolist() == g["bucket_off_lpt"]
    perm, _ = oracle.reorder(od, "degree")
    assert perm.tolist() == g["perm_dorder"]
    # hand-computed superiorities and Eq.3 objectives
    assert [oracle.superiority(int(d)) if d else 0 for d in od] == g["S"]
    for order, key in ((0, "eq3"), (1, "eq3_lpt")):
        perm, boff = oracle.reorder(od, "paper", k=g["k"], order=order)
        assert oracle.objective_eq3(boff, perm, od) == g[key]


def read_superiority_golden():
    rows = []
    with open(os.path.join(GOLDEN, "superiority_hand.txt")) as f:
        for line in f:
            line = line.split("#", 1)[0].split()
            if not line:
                continue
            assert line[0] == "sup"
            d, lam, alpha, beta, S, bw = line[1:]
            bw = None if bw == "-" else [float(x) for x in bw.split(",")]
            rows.append((int(d), float(lam), float(alpha), float(beta), int(S), bw))
    return rows


def test_superiority_golden():
    """S(d) with a BW table and alpha, beta != 1/2, worked by hand (Eq.19-20, Q15, Q20)."""
    rows = read_superiority_golden()
    assert len(rows) >= 10
    for d, lam, alpha, beta, S, bw in rows:
        assert oracle.superiority(d, lam=lam, alpha=alpha, beta=beta, bw=bw) == S, (d, lam, alpha, beta, bw)


@pytest.mark.parametrize("k", [1, 3, 8, 32, 128])
def test_aorder_invariants(k):
    spec = graphgen.rmat_spec(12, 16, 2)
    src, dst = graphgen.generate_cpu(spec)
    res = oracle.run(src, dst, spec.n, "degree", "paper", k=k)
    perm, boff, od = res["perm"], res["bucket_off"], res["od"]
    n = spec.n
    assert np.array_equal(np.sort(perm), np.arange(n))  # bijection
    sizes = np.diff(boff.astype(np.int64))
    assert np.all(sizes <= k) and np.all(sizes >= 1)
    nact = int((od > 0).sum())
    assert boff[-1] == nact and len(sizes) == -(-nact // k)
    assert np.all(od[perm >= nact] == 0)  # d~ = 0 vertices last (Q16)
    S = np.array([oracle.superiority(int(d)) if d else 0 for d in od], np.int64)
    obj = oracle.objective_eq3(boff, perm, od)
    assert obj >= abs(int(S.sum()))  # Eq.3 objective >= |Σ S| (triangle inequality)
    # A-order beats (or ties) D-order on the Eq.3 objective with the same k-blocks
    pd, _ = oracle.reorder(od, "degree")
    inv = np.empty(n, np.int64)
    inv[pd] = np.arange(n)
    Sd = S[inv][:nact]
    obj_d = sum(abs(int(Sd[i:i + k].sum())) for i in range(0, nact, k))
    assert obj <= obj_d


def test_dorder_sorted_desc():
    rng = np.random.default_rng(3)
    od = rng.integers(0, 20, 500).astype(np.uint32)
    perm, _ = oracle.reorder(od, "degree")
    inv = np.empty(500, np.int64)
    inv[perm] = np.arange(500)
    seq = [(-int(od[v]), int(v)) for v in inv]
    assert seq == sorted(seq)


def test_cost_eq1_closed_form():
    """Degree rule on K_n gives out-degrees 0..n-1: Σ|n·i - m| with m = C(n,2)."""
    for n in (3, 4, 9, 20):
        edges, _, _, _ = graphs.complete(n)
        src = np.array([a for a, b in edges], np.uint32)
        dst = np.array([b for a, b in edges], np.uint32)
        res = oracle.run(src, dst, n, "degree", "none")
        m = n * (n - 1) // 2
        assert sorted(res["od"].tolist()) == list(range(n))
        assert res["eq1"] == sum(abs(n * i - m) for i in range(n))


def test_reorder_preserves_orientation():
    """Relabeling only changes labels: the relabelled directed edge set is
    the image of the original one."""
    spec = graphgen.rmat_spec(9, 16, 4)
    src, dst = graphgen.generate_cpu(spec)
    base = oracle.run(src, dst, spec.n, "paper", "none")
    for r in ("degree", "paper"):
        res = oracle.run(src, dst, spec.n, "paper", r)
        p = res["perm"]
        got = set()
        for u in range(spec.n):
            for v in res["col"][res["offs"][u]:res["offs"][u + 1]].tolist():
                got.add((u, v))
        want = set()
        for u in range(spec.n):
            for v in base["col"][base["offs"][u]:base["offs"][u + 1]].tolist():
                want.add((int(p[u]), int(p[v])))
        assert got == want


# ---------------------------------------------------------------- Algorithm 2 over units (f3)
def _greedy_scan(S, active, k, order=0):
    """Algorithm 2 by exhaustive scan (no priority queue): line 6 takes the non-full bucket
    of least (mem_sup, index), line 12 the non-full bucket of greatest mem_sup, ties by the
    smallest index (P:424-438 with readings Q17-Q21)."""
    idx = [i for i in range(len(S)) if active[i]]
    mem = [i for i in idx if S[i] > 0]
    comp = [i for i in idx if S[i] <= 0]
    if order == 1:
        key = lambda i: (-abs(int(S[i])), i)
        mem.sort(key=key)
        comp.sort(key=key)
    b = (len(idx) + k - 1) // k
    sup, members = [0] * b, [[] for _ in range(b)]
    for v in mem:
        bk = min((j for j in range(b) if len(members[j]) < k), key=lambda j: (sup[j], j))
        members[bk].append(v)
        sup[bk] += int(S[v])
    for v in comp:
        bk = min((j for j in range(b) if len(members[j]) < k), key=lambda j: (-sup[j], j))
        members[bk].append(v)
        sup[bk] += int(S[v])
    pos, p = {}, 0
    for j in range(b):
        for v in members[j]:
            pos[v] = p
            p += 1
    for i in range(len(S)):
        if not active[i]:
            pos[i] = p
            p += 1
    return [pos[i] for i in range(len(S))]


@pytest.mark.parametrize("seed", range(12))
def test_aorder_units_vs_exhaustive_scan(seed):
    rng = np.random.default_rng(700 + seed)
    n = int(rng.integers(1, 200))
    S = rng.integers(-50, 50, size=n) * int(rng.integers(1, 1 << 20))
    S[rng.random(n) < 0.1] = 0
    active = (rng.random(n) < 0.85).astype(np.uint8)
    k = int(rng.integers(1, 9))
    order = seed % 2
    pos, boff = oracle.aorder_units(S, active, k, order)
    assert list(pos) == _greedy_scan(S, active, k, order)
    assert boff[-1] == int(active.sum()) and np.all(np.diff(boff.astype(np.int64)) <= k)


def test_aorder_units_equal_superiority_round_robin():
    # all S equal and positive: phase 1 always takes the least-index bucket among those with
    # the fewest members, i.e. unit i -> bucket i mod b, insertion order i // b
    for b, k in ((5, 4), (7, 3), (1, 6)):
        n = b * k
        pos, boff = oracle.aorder_units(np.full(n, 3 << 20), np.ones(n, np.uint8), k)
        assert list(pos) == [(i % b) * k + i // b for i in range(n)]
        assert list(boff) == [j * k for j in range(b + 1)]


def test_edge_units_cover_every_edge_with_work():
    """Edge units of a CSR: every directed edge u->v with d~(v) >= 1 appears once."""
    src, dst = graphgen.generate_cpu(graphgen.rmat_spec(9, 8, 31))
    res = oracle.run(src, dst, 1 << 9, "degree", "none")
    offs, col = res["offs"].astype(np.int64), res["col"]
    units, boff = oracle.edge_units(offs, col, k=4)
    od = np.diff(offs)
    want = set()
    for u in range(len(od)):
        for j in range(int(od[u])):
            if od[col[offs[u] + j]] > 0:
                want.add((u << 32) | j)
    assert sorted(units.tolist()) == sorted(want) and len(units) == len(want)
    assert boff[-1] == len(units)


def test_edge_units_golden():
    """Hand-traced edge-unit A-order (tests/golden/edge_units_hand7.txt)."""
    g = read_golden("edge_units_hand7.txt")
    offs, col = np.array(g["offs"], np.int64), np.array(g["col"], np.uint32)
    lam = g["lambda_milli"] / 1000.0
    S, act = oracle.edge_unit_superiority(offs, col, lam=lam)
    assert S.tolist() == g["S"] and act.tolist() == g["active"]
    units, boff = oracle.edge_units(offs, col, k=g["k"], lam=lam)
    assert [int(x) >> 32 for x in units] == g["unit_u"]
    assert [int(x) & 0xFFFFFFFF for x in units] == g["unit_j"]
    assert boff.tolist() == g["bucket_off"]
    # Eq.3 over the unit buckets
    pos = {int(x): i for i, x in enumerate(units)}
    src = np.repeat(np.arange(len(offs) - 1), np.diff(offs))
    per_unit = {(int(src[p]) << 32) | int(p - offs[src[p]]): int(S[p]) for p in range(len(S)) if act[p]}
    eq3 = sum(abs(sum(per_unit[int(units[i])] for i in range(boff[b], boff[b + 1])))
              for b in range(len(boff) - 1))
    assert eq3 == g["eq3"] and len(pos) == len(units)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_oriented_csr_by_definition(seed):
    """The oriented, relabelled CSR holds exactly the directed edges (pi(s), pi(t)), each
    out-list ascending; the one-call O1 (qsort) equals the library-sort O1."""
    rng = np.random.default_rng(seed)
    n = 300
    src = rng.integers(0, n, 4000).astype(np.uint32)
    dst = rng.integers(0, n, 4000).astype(np.uint32)
    e = oracle.simple_graph(src, dst, n)
    buf = np.zeros(len(src), np.uint64)
    m1 = oracle.lib().orc_simple_graph(oracle._p(src), oracle._p(dst), len(src), n, oracle._p(buf))
    assert np.array_equal(buf[:m1], e)
    dirs, _ = oracle.direct(e, n, "degree")
    perm = rng.permutation(n).astype(np.uint32)
    offs, col = oracle.oriented_csr(e, n, dirs, perm)
    want = {}
    for (fr, to) in _edge_dirs(e, dirs):
        want.setdefault(int(perm[fr]), []).append(int(perm[to]))
    for x in range(n):
        assert col[offs[x]:offs[x + 1]].tolist() == sorted(want.get(x, []))
    assert offs[-1] == len(e)
