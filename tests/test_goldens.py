"""The full-size oracle goldens (tests/golden/cfg*_*.json, tools/oracle_golden.py) cover
every config x rule pair BASELINE.json lists and are mutually consistent.  CPU only: the
GPU comparison is tests/test_gpu_configs.py::test_config_golden."""
import glob
import json
import os

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _load():
    out = {}
    for p in sorted(glob.glob(os.path.join(GOLDEN, "cfg*_*_*.json"))):
        with open(p) as f:
            rec = json.load(f)
        out[(rec["config"], rec["direct"], rec["reorder"])] = rec
    return out


def test_goldens_cover_baseline_rule_pairs():
    # BASELINE.json configs (1-based): 1 degree x none; 2 degree x none;
    # 3 {id, degree, paper} x none; 4 degree x {none, degree, paper}; 5 paper x paper
    # (+ degree x none)
    want = {(1, "degree", "none"), (2, "degree", "none"), (3, "id", "none"),
            (3, "degree", "none"), (3, "paper", "none"), (4, "degree", "none"),
            (4, "degree", "degree"), (4, "degree", "paper"), (5, "paper", "paper"),
            (5, "degree", "none")}
    have = set(_load())
    assert want <= have, sorted(want - have)


def test_goldens_consistent():
    recs = _load()
    by_cfg = {}
    for (c, d, r), rec in recs.items():
        by_cfg.setdefault(c, []).append(rec)
        hs = rec["sha256"]
        for k in ("od", "perm", "offs", "col"):
            assert len(hs[k]) == 64
        assert (r == "paper") == ("bucket_off" in hs)
        assert (d == "paper") == ("sub" in hs)
        if "top_t" in rec:
            assert len(rec["top_t"]) == 200
            degs = [x[1] for x in rec["top_t"]]
            assert degs == sorted(degs, reverse=True)
            # a vertex of degree d is in at most C(d, 2) triangles
            assert all(t <= dd * (dd - 1) // 2 for _, dd, t in rec["top_t"])
    for c, rs in by_cfg.items():
        # T and m do not depend on the rules; t(v) per original id neither
        assert len({r["T"] for r in rs}) == 1, c
        assert len({r["m"] for r in rs}) == 1, c
        ts = {r["sha256"]["t"] for r in rs if "t" in r["sha256"]}
        assert len(ts) == 1, c
        # the undirected degree is rule-free, so the hub list is too
        tops = {json.dumps(r["top_t"]) for r in rs if "top_t" in r}
        assert len(tops) <= 1, c
