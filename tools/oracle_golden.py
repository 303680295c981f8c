#!/usr/bin/env python
"""Write the full-size oracle goldens tests/golden/cfg{C}_{direct}_{reorder}.json.

Calls ONLY oracle/ (and the seeded input generator graphgen/, which holds none of the
method's arithmetic): no value here comes from the CUDA path.  For each rule pair that
BASELINE.json lists for a config it records what the oracle computes on the config's full
raw samples:

    m, T ("the total number of triangles"), levels / subrounds (A-direction),
    sha256 of the oriented CSR offs (u64 LE) and col (u32 LE), of pi (u32, perm[old] = new),
    of bucket_off (u32, A-order), of d~ (u32), of the A-direction sub / dsnap (u32),
    of t(v) per original id (u64), and t(v) of the 200 highest-degree vertices (hubs).

    python tools/oracle_golden.py --config 3 [--threads 0] [--pairs paper:none,...]

configs (1-based as SURVEY.md §8 / graphgen.CONFIGS) and their rule pairs:
    3  R-MAT s22 ef16      {id, degree, paper} x none           (BASELINE configs[2])
    4  R-MAT s24 ef32      degree x {none, degree, paper}       (BASELINE configs[3])
    5  Kronecker s27 ef16  paper x paper (+ degree x none: CSR only, T from paper x paper)
                                                                (BASELINE configs[4])
T is unique (any acyclic orientation counts each triangle once at its source), so
where a pair is marked "csr only" its T is not recounted.
"""
from __future__ import annotations

import argparse
import gc
import hashlib
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import graphgen  # noqa: E402
import oracle  # noqa: E402

PAIRS = {
    1: [("degree", "none", True)],
    2: [("degree", "none", True)],
    3: [("id", "none", True), ("degree", "none", True), ("paper", "none", True)],
    4: [("degree", "none", True), ("degree", "degree", True), ("degree", "paper", True)],
    5: [("paper", "paper", True), ("degree", "none", False)],
}
TOP = 200


def sha(a, dtype):
    a = np.ascontiguousarray(a, dtype=dtype)
    return hashlib.sha256(memoryview(a).cast("B")).hexdigest()


def log(msg):
    print(f"[{time.strftime('%H:%M:%S')}] {msg}", flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, required=True, choices=sorted(PAIRS))
    ap.add_argument("--threads", type=int, default=0, help="count threads (0 = all cores)")
    ap.add_argument("--pairs", default=None, help="subset, e.g. paper:none,degree:none")
    ap.add_argument("--out", default=os.path.join(ROOT, "tests", "golden"))
    args = ap.parse_args()
    cfg = args.config
    spec = graphgen.CONFIGS[cfg]
    pairs = PAIRS[cfg]
    if args.pairs:
        want = {tuple(p.split(":")) for p in args.pairs.split(",")}
        pairs = [p for p in pairs if (p[0], p[1]) in want]
    n = spec.n
    secs = {}
    t0 = time.perf_counter()
    src, dst = graphgen.generate_cpu(spec)
    log(f"cfg{cfg} {spec.name}: {spec.samples} samples generated")
    t1 = time.perf_counter()
    edges = oracle.simple_graph(src, dst, n)
    secs["simple_graph"] = time.perf_counter() - t1
    del src, dst
    gc.collect()
    m = len(edges)
    deg = oracle.degrees(edges, n)
    top = np.lexsort((np.arange(n), -deg.astype(np.int64)))[:TOP].astype(np.uint32)
    log(f"m={m} ({secs['simple_graph']:.0f} s)")
    T_known = None
    for d, r, count in pairs:
        rec = {"config": cfg, "baseline_index": cfg - 1, "workload": spec.name, "n": n,
               "samples": spec.samples, "seed": spec.seed, "direct": d, "reorder": r, "m": m,
               "generated_by": "tools/oracle_golden.py (oracle/ + graphgen/ only)",
               "aorder_params": {"k": oracle.DEFAULT_K, "lambda": oracle.DEFAULT_LAMBDA,
                                 "alpha": oracle.DEFAULT_ALPHA, "beta": oracle.DEFAULT_BETA,
                                 "bw": None, "order": 0}}
        hs = {}
        t1 = time.perf_counter()
        dirs, info = oracle.direct(edges, n, d)
        rec["seconds_direct"] = time.perf_counter() - t1
        if d == "paper":
            hs["sub"] = sha(info["sub"], np.uint32)
            hs["dsnap"] = sha(info["dsnap"], np.uint32)
            rec["levels"], rec["subrounds"] = info["levels"], info["subrounds"]
        del info
        od = oracle.outdeg(edges, n, dirs)
        hs["od"] = sha(od, np.uint32)
        rec["max_outdeg"] = int(od.max()) if n else 0
        rec["eq1"] = str(oracle.cost_eq1(n, m, od))
        t1 = time.perf_counter()
        perm, boff = oracle.reorder(od, r)
        rec["seconds_reorder"] = time.perf_counter() - t1
        hs["perm"] = sha(perm, np.uint32)
        if boff is not None:
            hs["bucket_off"] = sha(boff, np.uint32)
            rec["buckets"] = len(boff) - 1
            rec["eq3"] = oracle.objective_eq3(boff, perm, od)
        t1 = time.perf_counter()
        offs, col = oracle.oriented_csr(edges, n, dirs, perm)
        rec["seconds_csr"] = time.perf_counter() - t1
        del dirs
        gc.collect()
        hs["offs"] = sha(offs, np.uint64)
        hs["col"] = sha(col, np.uint32)
        log(f"{d}x{r}: directed ({rec['seconds_direct']:.0f} s), reordered "
            f"({rec['seconds_reorder']:.0f} s), CSR ({rec['seconds_csr']:.0f} s), max d~ {rec['max_outdeg']}")
        if count:
            t1 = time.perf_counter()
            T, tnew = oracle.count_forward(offs, col, per_vertex=True, threads=args.threads)
            rec["seconds_count"] = time.perf_counter() - t1
            rec["count_threads"] = args.threads or oracle.host_cores()
            t = tnew[perm]  # per original id
            del tnew
            rec["T"] = T
            hs["t"] = sha(t, np.uint64)
            rec["top_t"] = [[int(v), int(deg[v]), int(t[v])] for v in top]
            assert int(t.sum()) == 3 * T
            del t
            if T_known is not None:
                assert T == T_known, (T, T_known)
            T_known = T
            log(f"{d}x{r}: T={T} ({rec['seconds_count']:.0f} s on {rec['count_threads']} threads)")
        else:
            rec["T"] = T_known
            rec["T_from"] = "the first pair of this config (T does not depend on the rules, P:220)"
        rec["sha256"] = hs
        del offs, col, perm, boff, od
        gc.collect()
        path = os.path.join(args.out, f"cfg{cfg}_{d}_{r}.json")
        with open(path, "w") as f:  # one key per line, values compact
            f.write("{\n" + ",\n".join(f" {json.dumps(k)}: {json.dumps(v)}" for k, v in rec.items())
                    + "\n}\n")
        log(f"wrote {path}")
    log(f"total {time.perf_counter() - t0:.0f} s")


if __name__ == "__main__":
    main()
