"""GPU path vs the CPU oracle, element by element, through the C-ABI (libtc_b200.so).

Bar: bit-exact for everything — T, per-vertex t(v), the
simple graph, the orientation (out-degrees, A-direction subround/snapshot), the
permutation, the A-order buckets and the oriented CSR.  Sizes span many radix
tiles (4096 keys) with ragged tails; full-size configs are covered in
test_gpu_configs.py.
"""
import itertools
import zlib

import numpy as np
import pytest

import graphgen
import oracle
import paper_conf_sigmod_hu0l21_b200 as tc
from tests import graphs

pytestmark = pytest.mark.gpu

RULES = list(itertools.product(["id", "degree", "paper"], ["none", "degree", "paper"]))


def _oracle_edges_u64(res):
    return res["edges"]


def check_against_oracle(src, dst, n, d, r, k=32, per_vertex=True, sched=None, order=0):
    ref = oracle.run(src, dst, n, d, r, per_vertex=per_vertex, k=k, order=order)
    g = tc.Graph(src, dst, n)
    try:
        edges, deg = g.export_graph()
        assert np.array_equal(edges, ref["edges"]), "simple graph"
        assert np.array_equal(deg, ref["deg"]), "degrees"
        g.direct(d)
        if d == "paper":
            od, sub, dsnap = g.export_direct(internals=True)
            assert np.array_equal(sub, ref["direct_info"]["sub"]), "A-direction subround"
            assert np.array_equal(dsnap, ref["direct_info"]["dsnap"]), "A-direction snapshot"
        else:
            od = g.export_direct()
        assert np.array_equal(od, ref["od"]), "out-degree"
        g.reorder(r, k=k, order=order)
        if sched:
            g.set_schedule(sched)
        offs, col, perm = g.export()
        assert np.array_equal(perm, ref["perm"]), "permutation"
        assert np.array_equal(offs, ref["offs"]), "CSR offsets"
        assert np.array_equal(col, ref["col"]), "CSR columns"
        if r == "paper":
            assert np.array_equal(g.export_buckets(), ref["bucket_off"]), "A-order buckets"
        if per_vertex:
            T, t = g.count(per_vertex=True)
            assert np.array_equal(t, ref["t"]), "per-vertex counts"
        else:
            T = g.count()
        assert T == ref["T"], "triangle count"
        st = g.stats()
        assert st["m"] == ref["m"]
        assert st["eq1"] == ref["eq1"]
        return T, g.stats()
    finally:
        g.free()


@pytest.mark.parametrize("name", sorted(graphs.CLOSED_FORMS))
def test_closed_forms(name):
    edges, n, T, t = graphs.CLOSED_FORMS[name]
    rng = np.random.default_rng(zlib.crc32(name.encode()))
    src, dst, N, perm = graphs.noisy_samples(edges, n, rng, pad=3)
    t_expect = np.zeros(N, dtype=np.uint64)
    t_expect[perm[:n]] = t
    for d, r in RULES:
        got, _ = check_against_oracle(src, dst, N, d, r, k=3)
        assert got == T
        g = tc.Graph(src, dst, N)
        g.direct(d).reorder(r, k=3)
        T2, tv = g.count(per_vertex=True)
        assert T2 == T and np.array_equal(tv, t_expect)
        g.free()


@pytest.mark.parametrize("seed", range(40))
def test_random_small(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 3000))
    M = int(rng.integers(0, 12 * n))
    src, dst = graphs.random_graph(rng, n, M, "skew" if seed % 3 else "er")
    d, r = RULES[seed % len(RULES)]
    check_against_oracle(src, dst, n, d, r, k=int(rng.integers(1, 64)), order=seed % 2)


@pytest.mark.parametrize("d,r", RULES)
def test_config1_rmat_s16(d, r):
    spec = graphgen.CONFIGS[1]
    src, dst = graphgen.generate_cpu(spec)
    check_against_oracle(src, dst, spec.n, d, r)


@pytest.mark.parametrize("sched", ["bucketed", "range"])
@pytest.mark.parametrize("cap", [32, 64, 256, 2048])
def test_schedules_and_caps(sched, cap):
    """Every kernel path (warp slice, global-search fallback, CTA+TMA pieces) counts the same."""
    spec = graphgen.rmat_spec(13, 16, 77)
    src, dst = graphgen.generate_cpu(spec)
    ref = oracle.run(src, dst, spec.n, "id", "none", per_vertex=True)
    tc.tc_set_option("small_cap", cap)
    try:
        for d in ("id", "degree"):
            g = tc.Graph(src, dst, spec.n).direct(d).reorder("none").set_schedule(sched)
            T, t = g.count(per_vertex=True)
            assert T == ref["T"] and np.array_equal(t, ref["t"])
            g.free()
    finally:
        tc.tc_set_option("small_cap", 256)


def test_large_kernel_multi_piece():
    """A star-heavy graph with ID directing: one source list spans several TMA pieces."""
    rng = np.random.default_rng(9)
    n = 40000
    hub = 0
    leaves = np.arange(1, n, dtype=np.uint32)
    # hub -> every leaf, plus random leaf-leaf edges to make triangles through the hub
    a = rng.integers(1, n, 60000).astype(np.uint32)
    b = rng.integers(1, n, 60000).astype(np.uint32)
    src = np.concatenate([np.full(n - 1, hub, np.uint32), a])
    dst = np.concatenate([leaves, b])
    ref = oracle.run(src, dst, n, "id", "none", per_vertex=True)
    for sched in ("bucketed", "range"):
        g = tc.Graph(src, dst, n).direct("id").reorder("none").set_schedule(sched)
        T, t = g.count(per_vertex=True)
        assert T == ref["T"] and np.array_equal(t, ref["t"])
        g.free()


def test_count_range_partition():
    spec = graphgen.rmat_spec(14, 16, 5)
    src, dst = graphgen.generate_cpu(spec)
    for r in ("none", "paper"):
        g = tc.Graph(src, dst, spec.n).direct("degree").reorder(r)
        T = g.count()
        for world in (1, 2, 3, 8):
            b = g.partition(world)
            assert b[0] == 0 and b[-1] == spec.n and np.all(np.diff(b.astype(np.int64)) >= 0)
            parts = [g.count_range(int(b[i]), int(b[i + 1])) for i in range(world)]
            assert sum(parts) == T
        # per-vertex over a partition sums to the full per-vertex vector
        T2, t = g.count(per_vertex=True)
        b = g.partition(3)
        acc = np.zeros(spec.n, np.uint64)
        for i in range(3):
            _, ti = g.count_range(int(b[i]), int(b[i + 1]), per_vertex=True)
            acc += ti
        assert np.array_equal(acc, t) and T2 == T
        g.free()


def test_device_and_host_inputs_agree():
    import torch
    spec = graphgen.rmat_spec(12, 16, 3)
    src, dst = graphgen.generate_cpu(spec)
    T_host = tc.count_triangles(src, dst, spec.n)
    ds = torch.from_numpy(src.view(np.int32)).cuda()
    dd = torch.from_numpy(dst.view(np.int32)).cuda()
    g = tc.Graph(ds, dd, spec.n).direct("paper").reorder("paper")
    assert g.count() == T_host
    tv = torch.zeros(spec.n, dtype=torch.int64, device="cuda")
    T_dev = tc.tc_count(g.handle, tv)
    _, t_host = g.count(per_vertex=True)
    assert T_dev == T_host and np.array_equal(tv.cpu().numpy().view(np.uint64), t_host)
    g.free()


def test_edge_cases():
    z = np.zeros(0, np.uint32)
    for n in (0, 1, 5):
        g = tc.Graph(z, z, n).direct("paper").reorder("paper")
        assert g.count() == 0
        T, t = g.count(per_vertex=True)
        assert T == 0 and (len(t) == 0 or t.sum() == 0)
        g.free()
    loops = np.array([1, 2, 2, 3], np.uint32)
    assert tc.count_triangles(loops, loops, 4, "paper", "paper") == 0
    one = np.array([0], np.uint32), np.array([1], np.uint32)
    assert tc.count_triangles(*one, 2) == 0
    tri = np.array([0, 1, 2], np.uint32), np.array([1, 2, 0], np.uint32)
    assert tc.count_triangles(*tri, 3, "paper", "paper", per_vertex=True)[0] == 1


def test_errors():
    bad = np.array([0, 7], np.uint32)
    with pytest.raises(tc.TCError) as e:
        tc.Graph(bad, np.array([1, 1], np.uint32), 4)
    assert e.value.status == tc.TC_ERR_INVALID
    g = tc.Graph(np.array([0], np.uint32), np.array([1], np.uint32), 2)
    with pytest.raises(tc.TCError) as e:
        g.reorder("none")
    assert e.value.status == tc.TC_ERR_STATE
    with pytest.raises(tc.TCError) as e:
        g.count()
    assert e.value.status == tc.TC_ERR_STATE
    g.direct("degree")
    with pytest.raises(tc.TCError) as e:
        g.reorder("paper", k=0)
    assert e.value.status == tc.TC_ERR_INVALID
    with pytest.raises(tc.TCError):
        g.export_direct(internals=True)  # sub/dsnap only for PAPER
    with pytest.raises(tc.TCError):
        g.count_range(0, 5)
    g.free()


def test_redirect_resets_reorder():
    spec = graphgen.rmat_spec(11, 16, 4)
    src, dst = graphgen.generate_cpu(spec)
    g = tc.Graph(src, dst, spec.n).direct("degree").reorder("paper")
    T = g.count()
    g.direct("paper")  # discards the reordering
    offs, col, perm = g.export()
    assert np.array_equal(perm, np.arange(spec.n))
    assert g.count() == T
    g.free()


def test_aorder_params_bw_table_and_lpt():
    spec = graphgen.rmat_spec(12, 16, 8)
    src, dst = graphgen.generate_cpu(spec)
    bw = np.linspace(1.0, 50.0, 64)
    ref = oracle.run(src, dst, spec.n, "degree", "paper", k=16, lam=3.0, bw=bw, order=1)
    g = tc.Graph(src, dst, spec.n).direct("degree").reorder("paper", k=16, lam=3.0, bw=bw, order=1)
    offs, col, perm = g.export()
    assert np.array_equal(perm, ref["perm"])
    assert np.array_equal(g.export_buckets(), ref["bucket_off"])
    assert g.stats()["eq3"] == oracle.objective_eq3(ref["bucket_off"], ref["perm"], ref["od"], lam=3.0, bw=bw)
    assert g.count() == ref["T"]
    g.free()


@pytest.mark.parametrize("device_side", [0, 1])
def test_aorder_host_and_device_classification(device_side):
    """A-order with the classification / relabel on the host (aorder_device=0) and on the
    device (1): pi, bucket_off and Eq.3 equal the oracle's, incl. a BW table, k != 32 and
    graphs with isolated vertices."""
    tc.tc_set_option("aorder_device", device_side)
    try:
        for seed, (sc, ef, d, k, lam, bw) in enumerate(((12, 16, "degree", 32, 9.682, None),
                                                       (11, 8, "paper", 16, 3.0, np.linspace(1.0, 50.0, 64)),
                                                       (13, 4, "id", 7, 9.682, None))):
            spec = graphgen.rmat_spec(sc, ef, 400 + seed)
            src, dst = graphgen.generate_cpu(spec)
            ref = oracle.run(src, dst, spec.n, d, "paper", k=k, lam=lam, bw=bw)
            g = tc.Graph(src, dst, spec.n).direct(d).reorder("paper", k=k, lam=lam, bw=bw)
            offs, col, perm = g.export()
            assert np.array_equal(perm, ref["perm"]), (seed, device_side)
            assert np.array_equal(g.export_buckets(), ref["bucket_off"]), (seed, device_side)
            assert g.stats()["eq3"] == oracle.objective_eq3(ref["bucket_off"], ref["perm"], ref["od"], lam=lam, bw=bw)
            assert g.count() == ref["T"]
            g.free()
    finally:
        tc.tc_set_option("aorder_device", 1)


@pytest.mark.parametrize("red", [0, 1])
def test_adirection_peel_red_and_atomic(red):
    """A-direction peel with returning atomics (crossing test per decrement) and with RED
    decrements + a frontier scan: sub / dsnap / d~ and T equal the oracle's (Alg.1)."""
    tc.tc_set_option("peel_red", red)
    try:
        for seed, (sc, ef) in enumerate(((12, 16), (13, 8), (10, 48))):
            spec = graphgen.rmat_spec(sc, ef, 600 + seed)
            src, dst = graphgen.generate_cpu(spec)
            ref = oracle.run(src, dst, spec.n, "paper", "none")
            g = tc.Graph(src, dst, spec.n).direct("paper")
            od, sub, dsnap = g.export_direct(internals=True)
            info = ref["direct_info"]
            assert np.array_equal(sub, info["sub"]) and np.array_equal(dsnap, info["dsnap"]), (seed, red)
            assert np.array_equal(od, ref["od"]), (seed, red)
            assert g.count() == ref["T"]
            g.free()
    finally:
        tc.tc_set_option("peel_red", -1)


def test_gpu_generator_matches_cpu():
    import torch
    for spec in (graphgen.rmat_spec(16, 4, 11), graphgen.er_spec(100003, 1 << 18, 12)):
        s = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
        d = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
        graphgen.generate_cuda(spec, s.data_ptr(), d.data_ptr())
        torch.cuda.synchronize()
        cs, cd = graphgen.generate_cpu(spec)
        assert np.array_equal(s.cpu().numpy().view(np.uint32), cs)
        assert np.array_equal(d.cpu().numpy().view(np.uint32), cd)


def test_count_dist_single_rank_nccl():
    """a11 through the real NCCL path on one GPU: unique id, comm init, the slice count and
    the ncclAllReduce of the uint64 partial (and of the per-vertex vector)."""
    spec = graphgen.rmat_spec(13, 16, 21)
    src, dst = graphgen.generate_cpu(spec)
    ref = oracle.run(src, dst, spec.n, "paper", "paper", per_vertex=True)
    uid = tc.tc_nccl_get_unique_id()
    comm = tc.tc_nccl_comm_init(uid, 0, 1, 0)
    try:
        g = tc.Graph(src, dst, spec.n).direct("paper").reorder("paper")
        assert tc.tc_count_dist(g.handle, comm, 0, 1) == ref["T"]
        t = np.zeros(spec.n, np.uint64)
        assert tc.tc_count_dist(g.handle, comm, 0, 1, t) == ref["T"]
        assert np.array_equal(t, ref["t"])
        g.free()
    finally:
        tc.tc_nccl_comm_destroy(comm)


def test_bench_under_torchrun_single_process():
    """bench.py's N>1 code path (torch.distributed NCCL + library comm) with one rank."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "1",
           "--master-addr", "127.0.0.1", "--master-port", "29533", os.path.join(root, "bench.py"),
           "--gpus", "1", "--steps", "2", "--warmup", "1", "--config", "1", "--reorder", "paper", "--no-e2e",
           "--no-cpu-baseline"]
    env = dict(os.environ, WORLD_SIZE="1")
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env, cwd=root)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads(out.stdout.strip().splitlines()[-1])
    assert line["config"]["triangles"] > 0 and line["value"] > 0
    # t = max over ranks of (count + allreduce); A-order broadcast from rank 0
    assert "allreduce" in line["value_def"] and "ncclBroadcast" in line["config"]["parallelism"]


# ---------------------------------------------------------------- per-edge support (f1)
def _edges_parity(src, dst, n, d, r, ref_te=None, sched=None, k=32):
    ref = oracle.run(src, dst, n, d, r, per_edge=True, k=k)
    g = tc.Graph(src, dst, n).direct(d).reorder(r, k=k)
    try:
        if sched:
            g.set_schedule(sched)
        T, te = g.count_edges()
        assert T == ref["T"], (d, r)
        assert np.array_equal(te, ref["te"]), (d, r)
        if ref_te is not None:
            assert np.array_equal(te, ref_te)
    finally:
        g.free()


@pytest.mark.parametrize("name", sorted(graphs.CLOSED_FORMS))
def test_count_edges_closed_forms(name):
    edges, n, T, t = graphs.CLOSED_FORMS[name]
    rng = np.random.default_rng(zlib.crc32(name.encode()) + 1)
    src, dst, N, perm = graphs.noisy_samples(edges, n, rng, pad=2)
    keys, expect = graphs.expected_support(name, edges, n, perm)
    for d, r in RULES:
        _edges_parity(src, dst, N, d, r, ref_te=expect, k=3)


@pytest.mark.parametrize("seed", range(6))
def test_count_edges_random(seed):
    rng = np.random.default_rng(500 + seed)
    n = int(rng.integers(50, 3000))
    src, dst = graphs.random_graph(rng, n, int(rng.integers(n, 12 * n)), "er" if seed % 2 else "skew")
    for d, r in RULES:
        _edges_parity(src, dst, n, d, r, k=1 + seed)


@pytest.mark.parametrize("sched", ["bucketed", "range"])
@pytest.mark.parametrize("cap", [32, 256, 2048])
def test_count_edges_schedules_and_caps(sched, cap):
    """Warp slices, the global-memory search fallback and CTA+TMA pieces all place the
    three edge increments of every triangle at the right CSR positions."""
    spec = graphgen.rmat_spec(13, 16, 78)
    src, dst = graphgen.generate_cpu(spec)
    tc.tc_set_option("small_cap", cap)
    try:
        for d in ("id", "degree"):
            _edges_parity(src, dst, spec.n, d, "none", sched=sched)
    finally:
        tc.tc_set_option("small_cap", 256)


def test_count_edges_large_kernel_multi_piece():
    rng = np.random.default_rng(19)
    n = 30000
    a = rng.integers(1, n, 50000).astype(np.uint32)
    b = rng.integers(1, n, 50000).astype(np.uint32)
    src = np.concatenate([np.zeros(n - 1, np.uint32), a])
    dst = np.concatenate([np.arange(1, n, dtype=np.uint32), b])
    _edges_parity(src, dst, n, "id", "none")
    _edges_parity(src, dst, n, "id", "degree")


def test_count_edges_config1_and_device_output():
    import torch
    spec = graphgen.CONFIGS[1]
    src, dst = graphgen.generate_cpu(spec)
    _edges_parity(src, dst, spec.n, "degree", "none")
    _edges_parity(src, dst, spec.n, "paper", "paper")
    ref = oracle.run(src, dst, spec.n, "degree", "none", per_edge=True)
    g = tc.Graph(src, dst, spec.n).direct("degree")
    try:
        out = torch.zeros(len(ref["te"]), dtype=torch.int64, device="cuda")
        T = tc.tc_count_edges(g.handle, out)
        assert T == ref["T"]
        assert np.array_equal(out.cpu().numpy().astype(np.uint64), ref["te"])
    finally:
        g.free()


# ---------------------------------------------------------------- sort-merge intersection (§6.2)
@pytest.mark.parametrize("sched", ["bucketed", "range"])
@pytest.mark.parametrize("cap", [32, 256, 2048])
def test_sort_merge_intersection(sched, cap):
    """The sort-merge variant of the paper's §6.2 comparison (option "intersect"=1) counts
    the same T on every kernel path (warp slices, global lists, CTA pieces)."""
    tc.tc_set_option("small_cap", cap)
    tc.tc_set_option("intersect", 1)
    try:
        for seed, (sc, ef) in enumerate(((12, 16), (13, 8))):
            spec = graphgen.rmat_spec(sc, ef, 90 + seed)
            src, dst = graphgen.generate_cpu(spec)
            ref = oracle.run(src, dst, spec.n, "id", "none")
            for d, r in (("id", "none"), ("degree", "degree"), ("paper", "paper")):
                g = tc.Graph(src, dst, spec.n).direct(d).reorder(r).set_schedule(sched)
                assert g.count() == ref["T"], (d, r)
                T, t = g.count(per_vertex=True)  # per-vertex stays on binary search
                assert T == ref["T"]
                g.free()
        for name in ("K12", "W9", "B10", "CP6", "petersen"):
            edges, n, T, t = graphs.CLOSED_FORMS[name]
            src, dst, N, perm = graphs.noisy_samples(edges, n, np.random.default_rng(3), pad=2)
            g = tc.Graph(src, dst, N).direct("degree").set_schedule(sched)
            assert g.count() == T, name
            g.free()
    finally:
        tc.tc_set_option("intersect", 0)
        tc.tc_set_option("small_cap", 256)


# ---------------------------------------------------------------- bitmap intersection (Bisson, Fig.13)
def test_bitmap_intersection():
    """Option "intersect"=2 (Bisson's block-per-vertex bitmap pattern) counts the
    oracle's T under every directing / ordering rule, with the bitmap in shared memory
    (|V| <= 2^20) and in per-CTA global slices (|V| > 2^20: isolated padding vertices)."""
    tc.tc_set_option("intersect", 2)
    try:
        for seed, (sc, ef) in enumerate(((12, 16), (13, 8))):
            spec = graphgen.rmat_spec(sc, ef, 95 + seed)
            src, dst = graphgen.generate_cpu(spec)
            ref = oracle.run(src, dst, spec.n, "id", "none")
            for N in (spec.n, (1 << 20) + 77):
                for d, r in (("id", "none"), ("degree", "degree"), ("paper", "paper"), ("degree", "none")):
                    g = tc.Graph(src, dst, N).direct(d).reorder(r)
                    assert g.count() == ref["T"], (N, d, r)
                    g.free()
        for name in ("K12", "W9", "B10", "CP6", "petersen"):
            edges, n, T, t = graphs.CLOSED_FORMS[name]
            src, dst, N, perm = graphs.noisy_samples(edges, n, np.random.default_rng(4), pad=2)
            g = tc.Graph(src, dst, N).direct("paper")
            assert g.count() == T, name
            g.free()
    finally:
        tc.tc_set_option("intersect", 0)


# ---------------------------------------------------------------- edge-unit A-order (f3)
@pytest.mark.parametrize("d,r", [("degree", "none"), ("paper", "paper"), ("id", "degree")])
def test_edge_aorder_schedule(d, r):
    """Schedule "edge_aorder": the units and buckets equal the oracle's Algorithm 2 over the
    edge units (same superiorities, same greedy), and every count mode gives the oracle's
    T / t(v) / support on every slice."""
    for seed, (sc, ef) in enumerate(((10, 8), (12, 16))):
        spec = graphgen.rmat_spec(sc, ef, 300 + seed)
        src, dst = graphgen.generate_cpu(spec)
        for k, order in ((32, 0), (5, 1)):
            ref = oracle.run(src, dst, spec.n, d, r, per_vertex=True, k=k, order=order)
            g = tc.Graph(src, dst, spec.n).direct(d).reorder(r, k=k, order=order).set_schedule("edge_aorder")
            try:
                units, uoff = g.export_units()
                want_u, want_off = oracle.edge_units(ref["offs"], ref["col"], k=k, order=order)
                assert np.array_equal(units, want_u) and np.array_equal(uoff, want_off)
                assert g.stats()["eq3_units"] >= 0
                assert g.count() == ref["T"]
                T, t = g.count(per_vertex=True)
                assert T == ref["T"] and np.array_equal(t, ref["t"])
                bounds = [0, spec.n // 3, spec.n // 2, spec.n]
                assert sum(g.count_range(a, b) for a, b in zip(bounds, bounds[1:])) == ref["T"]
                T, te = g.count_edges()
                assert T == ref["T"] and int(te.sum()) == 3 * T
                assert np.array_equal(te, oracle.edge_support(ref["edges"], spec.n))
            finally:
                g.free()
    for name in ("K12", "W9", "B10", "petersen"):
        edges, n, T, t = graphs.CLOSED_FORMS[name]
        src, dst, N, perm = graphs.noisy_samples(edges, n, np.random.default_rng(8), pad=2)
        g = tc.Graph(src, dst, N).direct(d).reorder(r).set_schedule("edge_aorder")
        assert g.count() == T, name
        g.free()


# ---------------------------------------------------------------- shorter-list schedule, options
@pytest.mark.parametrize("cap", [32, 256])
@pytest.mark.parametrize("spans", [(32, 8), (128, 2048), (1 << 12, 1 << 16)])
def test_shorter_list_schedule(cap, spans):
    """Count with the shorter-list owner schedule (default for count-only calls) and with the
    classic Hu pattern: every warp / CTA owner-item shape gives the oracle's T, whole and on
    work-balanced slices (the owners of a slice are its sources' edges, counted at either end)."""
    span, lspan = spans
    tc.tc_set_option("small_cap", cap)
    tc.tc_set_option("owner_span", span)
    tc.tc_set_option("owner_lspan", lspan)
    try:
        for seed, (sc, ef, d, r) in enumerate(((13, 16, "degree", "none"), (12, 32, "paper", "paper"),
                                               (12, 16, "id", "degree"))):
            spec = graphgen.rmat_spec(sc, ef, 900 + seed)
            src, dst = graphgen.generate_cpu(spec)
            ref = oracle.run(src, dst, spec.n, d, r)
            g = tc.Graph(src, dst, spec.n).direct(d).reorder(r)
            for shorter in (1, 0):
                tc.tc_set_option("shorter", shorter)
                assert g.count() == ref["T"], (d, r, shorter)
                b = g.partition(3).tolist()
                assert sum(g.count_range(a, c) for a, c in zip(b, b[1:])) == ref["T"]
            g.free()
    finally:
        tc.tc_set_option("shorter", 1)
        tc.tc_set_option("small_cap", 256)
        tc.tc_set_option("owner_span", 128)
        tc.tc_set_option("owner_lspan", 2048)


@pytest.mark.parametrize("cap", [32, 256])
def test_owner_tiles(cap):
    """CTA items of the shorter-list schedule in owner-label L2 tiles (option otiles): every
    tile count / tiling threshold / item span gives the oracle's T, whole and on slices."""
    tc.tc_set_option("small_cap", cap)
    try:
        for seed, (sc, ef, d, r) in enumerate(((13, 32, "degree", "paper"), (12, 16, "paper", "none"),
                                               (11, 48, "id", "degree"))):
            spec = graphgen.rmat_spec(sc, ef, 950 + seed)
            src, dst = graphgen.generate_cpu(spec)
            ref = oracle.run(src, dst, spec.n, d, r)
            g = tc.Graph(src, dst, spec.n).direct(d).reorder(r)
            for nt, tmin, lspan in ((2, 0, 2048), (7, 0, 8), (7, 4, 64), (255, 0, 2048), (255, 1, 16)):
                tc.tc_set_option("otiles", nt)
                tc.tc_set_option("otile_min", tmin)
                tc.tc_set_option("owner_lspan", lspan)
                assert g.count() == ref["T"], (seed, nt, tmin, lspan)
                b = g.partition(3).tolist()
                assert sum(g.count_range(a, c) for a, c in zip(b, b[1:])) == ref["T"], (seed, nt, tmin, lspan)
            g.free()
    finally:
        tc.tc_set_option("otiles", 1)
        tc.tc_set_option("otile_min", 4)
        tc.tc_set_option("owner_lspan", 2048)
        tc.tc_set_option("small_cap", 256)


@pytest.mark.parametrize("evictions", [0, 1, 2, 64])
def test_cuckoo_piece_sets(evictions):
    """Count-only CTA items with the staged list as a cuckoo set (option cuckoo = eviction
    limit): off (0), mostly failing inserts that fall back to the sorted piece (1, 2) and the
    default (64) all give the oracle's T, on both the owner and the classic schedule, with
    single- and multi-piece lists."""
    tc.tc_set_option("cuckoo", evictions)
    tc.tc_set_option("small_cap", 32)
    try:
        for seed, (sc, ef, d, r) in enumerate(((13, 32, "degree", "paper"), (12, 16, "id", "none"))):
            spec = graphgen.rmat_spec(sc, ef, 970 + seed)
            src, dst = graphgen.generate_cpu(spec)
            ref = oracle.run(src, dst, spec.n, d, r)
            g = tc.Graph(src, dst, spec.n).direct(d).reorder(r)
            for shorter in (1, 0):
                tc.tc_set_option("shorter", shorter)
                assert g.count() == ref["T"], (seed, evictions, shorter)
            g.free()
    finally:
        tc.tc_set_option("cuckoo", 64)
        tc.tc_set_option("shorter", 1)
        tc.tc_set_option("small_cap", 256)


@pytest.mark.parametrize("e2sort", [0, 1])
def test_owner_e2_grouping_sort_and_atomics(e2sort):
    """E2 owners grouped by cursor atomics (0) or by a sort of the (x, u) pairs (1): T equal
    to the oracle's, whole and on work-balanced slices (the owners of a slice's sources)."""
    tc.tc_set_option("e2sort", e2sort)
    tc.tc_set_option("small_cap", 32)
    try:
        for seed, (sc, ef, d, r) in enumerate(((13, 32, "degree", "paper"), (12, 16, "paper", "none"),
                                               (12, 8, "id", "degree"))):
            spec = graphgen.rmat_spec(sc, ef, 990 + seed)
            src, dst = graphgen.generate_cpu(spec)
            ref = oracle.run(src, dst, spec.n, d, r)
            g = tc.Graph(src, dst, spec.n).direct(d).reorder(r)
            assert g.count() == ref["T"], (seed, e2sort)
            b = g.partition(4).tolist()
            assert sum(g.count_range(a, c) for a, c in zip(b, b[1:])) == ref["T"], (seed, e2sort)
            g.free()
    finally:
        tc.tc_set_option("e2sort", -1)
        tc.tc_set_option("small_cap", 256)


def test_extra_compute_instrumented_kernel_counts_unchanged():
    """The §5.3 balance-point instrumentation (option extra_compute, MODE 3: p_c extra
    searches per wedge, results discarded) leaves T and t(v) equal to the oracle's."""
    spec = graphgen.rmat_spec(12, 16, 31)
    src, dst = graphgen.generate_cpu(spec)
    ref = oracle.run(src, dst, spec.n, "degree", "paper", per_vertex=True)
    g = tc.Graph(src, dst, spec.n).direct("degree").reorder("paper")
    try:
        for q in (0, 1, 8, 24):
            tc.tc_set_option("extra_compute", q)
            assert g.count() == ref["T"], q
            T, t = g.count(per_vertex=True)
            assert T == ref["T"] and np.array_equal(t, ref["t"]), q
    finally:
        tc.tc_set_option("extra_compute", -1)
        g.free()


def test_reorder_dist_single_rank_equals_reorder():
    """tc_reorder_dist (A-order on rank 0, pi / bucket_off / Eq.3 broadcast over NCCL) gives
    the same graph as tc_reorder, and the count through tc_count_dist equals the oracle's."""
    spec = graphgen.rmat_spec(13, 16, 41)
    src, dst = graphgen.generate_cpu(spec)
    ref = oracle.run(src, dst, spec.n, "degree", "paper")
    uid = tc.tc_nccl_get_unique_id()
    comm = tc.tc_nccl_comm_init(uid, 0, 1, 0)
    try:
        g = tc.Graph(src, dst, spec.n).direct("degree")
        prm, keep = tc.make_aorder_params()
        tc.tc_reorder_dist(g.handle, "paper", prm, comm, 0, 1)
        offs, col, perm = g.export()
        assert np.array_equal(perm, ref["perm"]) and np.array_equal(col, ref["col"])
        assert np.array_equal(g.export_buckets(), ref["bucket_off"])
        assert g.stats()["eq3"] == oracle.objective_eq3(ref["bucket_off"], ref["perm"], ref["od"])
        assert tc.tc_count_dist(g.handle, comm, 0, 1) == ref["T"]
        g.free()
    finally:
        tc.tc_nccl_comm_destroy(comm)
