"""Pins for the oracle's count (O4): closed forms, brute force, node-iterator,
invariance over all directing x ordering rules and relabelings (PAPER.md:15,
P:65).  CPU only."""
import itertools
import zlib

import numpy as np
import pytest

import oracle
from tests import graphs

RULES = list(itertools.product(["id", "degree", "paper"], ["none", "degree", "paper"]))


@pytest.mark.parametrize("name", sorted(graphs.CLOSED_FORMS))
def test_closed_forms_all_rules(name):
    edges, n, T, t = graphs.CLOSED_FORMS[name]
    rng = np.random.default_rng(zlib.crc32(name.encode()))
    src, dst, N, perm = graphs.noisy_samples(edges, n, rng, pad=3)
    t_expect = np.zeros(N, dtype=np.int64)
    t_expect[perm[:n]] = t
    for d, r in RULES:
        res = oracle.run(src, dst, N, d, r, per_vertex=True, k=3)
        assert res["T"] == T, (name, d, r)
        assert np.array_equal(res["t"].astype(np.int64), t_expect), (name, d, r)
        assert int(res["t"].sum()) == 3 * T


@pytest.mark.parametrize("seed", range(12))
def test_brute_force_trace(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(2, 64))
    M = int(rng.integers(0, 4 * n))
    kind = "er" if seed % 2 else "skew"
    src, dst = graphs.random_graph(rng, n, M, kind)
    T, tv = graphs.brute_force(src, dst, n)
    for d, r in RULES:
        res = oracle.run(src, dst, n, d, r, per_vertex=True, k=1 + seed % 5)
        assert res["T"] == T
        assert np.array_equal(res["t"].astype(np.int64), tv)


@pytest.mark.parametrize("seed", range(3))
def test_node_iterator_medium(seed):
    rng = np.random.default_rng(100 + seed)
    n = 600
    src, dst = graphs.random_graph(rng, n, 6000, "skew")
    T, tv = graphs.node_iterator(src, dst, n)
    res = oracle.run(src, dst, n, "paper", "paper", per_vertex=True)
    assert res["T"] == T
    assert np.array_equal(res["t"].astype(np.int64), tv)


def test_relabel_invariance_rmat():
    import graphgen
    spec = graphgen.rmat_spec(11, 16, 7)
    src, dst = graphgen.generate_cpu(spec)
    Ts = set()
    rng = np.random.default_rng(5)
    for d, r in RULES:
        Ts.add(oracle.run(src, dst, spec.n, d, r)["T"])
        p = rng.permutation(spec.n).astype(np.uint32)
        Ts.add(oracle.run(p[src], p[dst], spec.n, d, r)["T"])
    assert len(Ts) == 1


def test_empty_and_degenerate():
    z = np.zeros(0, dtype=np.uint32)
    assert oracle.run(z, z, 0)["T"] == 0
    assert oracle.run(z, z, 5, "paper", "paper")["T"] == 0
    loops = np.array([1, 2, 3], dtype=np.uint32)
    res = oracle.run(loops, loops, 4, "paper", "paper", per_vertex=True)
    assert res["m"] == 0 and res["T"] == 0 and res["t"].sum() == 0
    with pytest.raises(ValueError):
        oracle.run(np.array([0], np.uint32), np.array([9], np.uint32), 4)


def test_count_range_partition_sums():
    """Sum of per-range counts equals the total (the multi-GPU slice invariant)."""
    import graphgen
    spec = graphgen.rmat_spec(10, 8, 3)
    src, dst = graphgen.generate_cpu(spec)
    res = oracle.run(src, dst, spec.n, "degree", "none")
    cuts = [0, 100, 101, 500, 1000, spec.n]
    parts = [oracle.count_forward(res["offs"], res["col"], a, b) for a, b in zip(cuts, cuts[1:])]
    assert sum(parts) == res["T"]


def test_local_triangles_matches_per_vertex():
    """The sampled-vertex definition t(v) = #edges among N(v) agrees with the count's
    per-vertex output (and brute force) on R-MAT with duplicates and self-loops."""
    import graphgen
    spec = graphgen.rmat_spec(12, 16, 9)
    src, dst = graphgen.generate_cpu(spec)
    res = oracle.run(src, dst, spec.n, "degree", "none", per_vertex=True)
    rng = np.random.default_rng(0)
    vs = rng.choice(spec.n, 300, replace=False).astype(np.uint32)
    loc = oracle.local_triangles(src, dst, vs)
    assert np.array_equal(loc, res["t"][vs])
    rng = np.random.default_rng(1)
    n = 50
    s2, d2 = graphs.random_graph(rng, n, 300, "skew")
    _, tv = graphs.brute_force(s2, d2, n)
    assert np.array_equal(oracle.local_triangles(s2, d2, np.arange(n)).astype(np.int64), tv)


# ---------------------------------------------------------------- per-edge support (f1)
@pytest.mark.parametrize("name", sorted(graphs.CLOSED_FORMS))
def test_edge_support_closed_forms(name):
    """support(e) = #triangles containing e, against the closed form of every family."""
    edges, n, T, t = graphs.CLOSED_FORMS[name]
    rng = np.random.default_rng(zlib.crc32(name.encode()) + 1)
    src, dst, N, perm = graphs.noisy_samples(edges, n, rng, pad=2)
    keys, expect = graphs.expected_support(name, edges, n, perm)
    res = oracle.run(src, dst, N, "degree", "none", per_edge=True)
    assert np.array_equal(res["edges"], keys)
    assert np.array_equal(res["te"], expect), name
    assert int(res["te"].sum()) == 3 * T


@pytest.mark.parametrize("seed", range(10))
def test_edge_support_brute_force(seed):
    """(A @ A) ∘ A on tiny random graphs (a dropped or double-counted triangle edge fails)."""
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(2, 60))
    src, dst = graphs.random_graph(rng, n, int(rng.integers(0, 5 * n)), "er" if seed % 2 else "skew")
    keys, sup = graphs.brute_force_support(src, dst, n)
    res = oracle.run(src, dst, n, "id", "none", per_edge=True)
    assert np.array_equal(res["edges"], keys)
    assert np.array_equal(res["te"], sup)


def test_edge_support_vertex_identity():
    """Each triangle at v contains exactly two edges at v: t(v) = Σ_{e ∋ v} support(e) / 2,
    and Σ_e support(e) = 3T (R-MAT scale 10, skewed)."""
    import graphgen
    spec = graphgen.rmat_spec(10, 16, 7)
    src, dst = graphgen.generate_cpu(spec)
    res = oracle.run(src, dst, spec.n, "degree", "none", per_vertex=True, per_edge=True)
    te = res["te"].astype(np.int64)
    assert int(te.sum()) == 3 * res["T"]
    a = (res["edges"] >> np.uint64(32)).astype(np.int64)
    b = (res["edges"] & np.uint64(0xffffffff)).astype(np.int64)
    acc = np.zeros(spec.n, dtype=np.int64)
    np.add.at(acc, a, te)
    np.add.at(acc, b, te)
    assert np.array_equal(acc // 2, res["t"].astype(np.int64)) and not (acc % 2).any()
