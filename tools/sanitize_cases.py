"""Small cases covering every kernel path of the library, for compute-sanitizer
(memcheck / racecheck / synccheck): each result is checked against the oracle.

    compute-sanitizer --tool racecheck python tools/sanitize_cases.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import graphgen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sigmod_hu0l21_b200 as tc  # noqa: E402


def case(spec, d, r, sched=None, opts=(), per_vertex=True, per_edge=False):
    src, dst = graphgen.generate_cpu(spec)
    ref = oracle.run(src, dst, spec.n, d, r, per_vertex=per_vertex, per_edge=per_edge)
    for k, v in opts:
        tc.tc_set_option(k, v)
    try:
        g = tc.Graph(src, dst, spec.n).direct(d).reorder(r)
        if sched:
            g.set_schedule(sched)
        assert g.count() == ref["T"], (d, r, sched, opts)
        if per_vertex:
            T, t = g.count(per_vertex=True)
            assert T == ref["T"] and np.array_equal(t, ref["t"])
        if per_edge:
            T, te = g.count_edges()
            assert T == ref["T"] and np.array_equal(te, ref["te"])
        b = g.partition(3).tolist()
        assert sum(g.count_range(a, c) for a, c in zip(b, b[1:])) == ref["T"]
        g.free()
    finally:
        for k, _ in opts:
            tc.tc_set_option(k, {"small_cap": 256, "shorter": 1, "intersect": 0, "peel_coop": 1,
                                 "owner_span": 128, "owner_lspan": 2048, "extra_compute": -1,
                                 "otiles": 1, "otile_min": 4}[k])
    print("ok", spec.name, d, r, sched, opts, flush=True)


def multi_piece():
    """ID directing on a hub graph: the hub's N+ spans two TMA pieces (> 4096 entries)."""
    rng = np.random.default_rng(9)
    n = 6000
    a = rng.integers(1, n, 12000).astype(np.uint32)
    b = rng.integers(1, n, 12000).astype(np.uint32)
    src = np.concatenate([np.zeros(n - 1, np.uint32), a])
    dst = np.concatenate([np.arange(1, n, dtype=np.uint32), b])
    ref = oracle.run(src, dst, n, "id", "none", per_vertex=True, per_edge=True)
    for shorter in (1, 0):
        tc.tc_set_option("shorter", shorter)
        g = tc.Graph(src, dst, n).direct("id").reorder("none")
        assert g.count() == ref["T"]
        T, t = g.count(per_vertex=True)
        assert T == ref["T"] and np.array_equal(t, ref["t"])
        T, te = g.count_edges()
        assert T == ref["T"] and np.array_equal(te, ref["te"])
        g.free()
    tc.tc_set_option("shorter", 1)
    print("ok multi-piece hub", flush=True)


def main():
    multi_piece()
    s10 = graphgen.rmat_spec(10, 16, 5)
    s11 = graphgen.rmat_spec(11, 16, 6)
    er = graphgen.er_spec(3000, 1 << 15, 7)
    case(s10, "degree", "none", per_edge=True)
    case(s11, "paper", "paper", per_edge=True)
    case(s11, "id", "degree")
    case(er, "degree", "none", per_edge=True)
    case(s11, "degree", "none", opts=(("small_cap", 32),), per_edge=True)          # CTA items + TMA pieces
    case(s11, "id", "none", opts=(("small_cap", 32), ("owner_span", 32), ("owner_lspan", 8)))
    case(s11, "degree", "paper", sched="range", per_edge=True)
    case(s11, "degree", "paper", sched="edge_aorder", per_edge=True)
    case(s10, "degree", "none", opts=(("intersect", 1),), per_vertex=False)       # sort-merge
    case(s10, "degree", "none", opts=(("intersect", 2),), per_vertex=False)       # bitmap
    case(s11, "paper", "none", opts=(("peel_coop", 0),))                          # multi-launch peel
    case(s10, "degree", "none", opts=(("extra_compute", 8), ("shorter", 0)))      # §5.3 instrumented
    case(s11, "degree", "paper", opts=(("small_cap", 32), ("otiles", 7), ("otile_min", 0), ("owner_lspan", 8)),
         per_vertex=False)                                                          # owner-label tiles
    print("all sanitizer cases passed")


if __name__ == "__main__":
    main()
