"""Full-size BASELINE.json configs on the GPU, in the launch configuration bench.py times.

Every config x rule pair BASELINE.json lists is compared, whole, against the oracle's
goldens tests/golden/cfg{C}_{direct}_{reorder}.json (written by tools/oracle_golden.py,
which calls only oracle/ and the seeded generator): m, T, the A-direction subround /
snapshot arrays, d~, pi, the A-order bucket offsets, the oriented CSR and t(v) of every
vertex (per original id) — bit-exact via sha256 of the exported arrays, and the t(v) of the
200 highest-degree vertices (the hubs that run the CTA-item / TMA-piece count path) value
by value.  The GPU side draws the same raw samples with the CUDA build of the generator
(bit-identical to the CPU build, test_gpu_parity.py::test_gpu_generator_matches_cpu).

Besides the goldens:
* configs[1] (ER, 67M edges): whole oracle vs GPU — oriented CSR, T, per-edge support.
* configs[2] (R-MAT s22): per-edge support on sampled edges vs the oracle's
  common-neighbour merge, Σ = 3T; partition bounds vs the restated work rule; count_range
  on sampled label ranges vs the oracle's merge on the (bit-identical) CSR.
"""
import functools
import glob
import hashlib
import json
import os

import numpy as np
import pytest

import graphgen
import oracle
import paper_conf_sigmod_hu0l21_b200 as tc
from tests.test_dist_gloo import work_bounds

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
GOLDENS = sorted(glob.glob(os.path.join(GOLDEN, "cfg*_*_*.json")))


def sha(a, dtype):
    a = np.ascontiguousarray(a, dtype=dtype)
    return hashlib.sha256(memoryview(a).cast("B")).hexdigest()


@functools.lru_cache(maxsize=1)
def device_samples(cfg):
    """Raw samples of a config drawn on the device (kept for the config's tests)."""
    import torch
    spec = graphgen.CONFIGS[cfg]
    src = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
    dst = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
    graphgen.generate_cuda(spec, src.data_ptr(), dst.data_ptr(),
                           torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    return src, dst


@functools.lru_cache(maxsize=1)
def host_samples(cfg):
    return graphgen.generate_cpu(graphgen.CONFIGS[cfg])


def _golden_id(path):
    return os.path.basename(path)[:-5]


@pytest.mark.parametrize("path", GOLDENS, ids=_golden_id)
def test_config_golden(path):
    with open(path) as f:
        rec = json.load(f)
    cfg, d, r = rec["config"], rec["direct"], rec["reorder"]
    spec = graphgen.CONFIGS[cfg]
    assert (spec.name, spec.n, spec.samples, spec.seed) == (rec["workload"], rec["n"], rec["samples"],
                                                            rec["seed"])
    hs = rec["sha256"]
    src, dst = device_samples(cfg)
    g = tc.Graph(src, dst, spec.n)
    try:
        g.direct(d)
        if d == "paper":
            od, sub, dsnap = g.export_direct(internals=True)
            assert sha(sub, np.uint32) == hs["sub"], "A-direction subround"
            assert sha(dsnap, np.uint32) == hs["dsnap"], "A-direction snapshot"
            st = g.stats()
            assert (st["levels"], st["subrounds"]) == (rec["levels"], rec["subrounds"])
            del sub, dsnap
        else:
            od = g.export_direct()
        assert sha(od, np.uint32) == hs["od"], "out-degree d~"
        assert int(od.max()) == rec["max_outdeg"]
        del od
        prm = rec["aorder_params"]
        g.reorder(r, k=prm["k"], lam=prm["lambda"], alpha=prm["alpha"], beta=prm["beta"],
                  order=prm["order"])
        st = g.stats()
        assert st["m"] == rec["m"]
        assert str(st["eq1"]) == rec["eq1"], "Eq.1 cost"
        offs, col, perm = g.export()
        assert sha(perm, np.uint32) == hs["perm"], "permutation pi"
        assert sha(offs, np.uint64) == hs["offs"], "oriented CSR offsets"
        assert sha(col, np.uint32) == hs["col"], "oriented CSR columns"
        del offs, col, perm
        if r == "paper":
            b = g.export_buckets()
            assert len(b) - 1 == rec["buckets"]
            assert sha(b, np.uint32) == hs["bucket_off"], "A-order bucket offsets"
        if "t" in hs:
            T, t = g.count(per_vertex=True)
            top = np.array(rec["top_t"], dtype=np.int64)
            assert np.array_equal(t[top[:, 0]].astype(np.int64), top[:, 2]), "hub t(v)"
            assert sha(t, np.uint64) == hs["t"], "per-vertex t(v)"
            del t
        else:
            T = g.count()
        assert T == rec["T"], "triangle count T"
        assert g.count() == T  # repeatable, no per-vertex instantiation
    finally:
        g.free()


def test_config2_er_full_oracle():
    spec = graphgen.CONFIGS[2]
    src, dst = host_samples(2)
    ref = oracle.run(src, dst, spec.n, "degree", "none")
    g = tc.Graph(src, dst, spec.n).direct("degree").reorder("none")
    offs, col, perm = g.export()
    assert np.array_equal(offs, ref["offs"]) and np.array_equal(col, ref["col"])
    assert g.count() == ref["T"]
    # per-edge support (f1), every edge: the oracle's common-neighbour merge on the
    # symmetric lists vs the GPU's three aggregated increments per triangle
    T, te = g.count_edges()
    assert T == ref["T"]
    assert np.array_equal(te, oracle.edge_support(ref["edges"], spec.n))
    g.free()


def test_config3_rmat_s22_ranges_partition_support():
    spec = graphgen.CONFIGS[3]
    n = spec.n
    src, dst = host_samples(3)
    edges = oracle.simple_graph(src, dst, n)
    dirs, _ = oracle.direct(edges, n, "paper")
    od = oracle.outdeg(edges, n, dirs)
    perm, _ = oracle.reorder(od, "none")
    offs, col = oracle.oriented_csr(edges, n, dirs, perm)
    g = tc.Graph(src, dst, n).direct("paper").reorder("none")
    T = g.count()
    # sampled label ranges of the CSR counted by the oracle's merge
    rng = np.random.default_rng(3)
    for a in rng.integers(0, n - 40000, 3):
        a = int(a)
        assert g.count_range(a, a + 40000) == oracle.count_forward(offs, col, a, a + 40000)
    # work-balanced partition = the restated rule (tests/test_dist_gloo.py)
    for world in (2, 4, 8):  # max d~ >= 64: the shorter-list work model
        assert g.partition(world).tolist() == work_bounds_fast(offs, col, world, shorter=True)
    # per-edge support (f1): Σ = 3T, and uniformly sampled edges (chosen without looking at
    # the GPU output) against the oracle's common-neighbour merge
    Te, te = g.count_edges()
    assert Te == T and int(te.sum()) == 3 * T
    idx = np.sort(rng.choice(len(edges), size=3000, replace=False))
    assert np.array_equal(te[idx], oracle.edge_support(edges, n, subset=edges[idx]))
    g.free()


def work_bounds_fast(offs, col, world, shorter=False):
    od = np.diff(offs.astype(np.int64))
    s = np.zeros(len(od), np.int64)
    nz = od > 0
    dv = od[col.astype(np.int64)]
    if shorter:  # the shorter-list schedule streams min(d~(u), d~(v)) per edge
        dv = np.minimum(dv, np.repeat(od, od))
    s[nz] = np.add.reduceat(dv, offs[:-1][nz].astype(np.int64))
    pre = np.concatenate([[0], np.cumsum(od + s)])
    n = len(od)
    b = [0] + [int(np.searchsorted(pre, (int(pre[-1]) * g) // world, side="left")) for g in range(1, world)] + [n]
    return b


def test_work_bounds_fast_matches_rule():
    spec = graphgen.rmat_spec(11, 16, 3)
    src, dst = graphgen.generate_cpu(spec)
    res = oracle.run(src, dst, spec.n, "degree", "none")
    for w in (2, 3, 8):
        for sh in (False, True):
            assert work_bounds_fast(res["offs"], res["col"], w, sh) == work_bounds(res["offs"], res["col"], w,
                                                                                   shorter=sh)
