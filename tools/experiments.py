"""Paper-experiment analogs on B200: every directing x ordering
x schedule variant of one config, device time per stage (CUDA events, median of 3 after a
warm-up), with the paper's Eq.1 / Eq.3 statistics.  Prints a markdown table.

    python tools/experiments.py --config 3 [--rules id:none,degree:none,paper:none]
"""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import graphgen
import paper_conf_sigmod_hu0l21_b200 as tc


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--rules", default="id:none,degree:none,paper:none,degree:degree,degree:paper,paper:paper")
    ap.add_argument("--schedules", default="bucketed,range")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--intersect", default="0", help="comma list: 0 binary search, 1 sort-merge (§6.2), 2 bitmap (Bisson, Fig.13)")
    a = ap.parse_args()
    spec = graphgen.CONFIGS[a.config]
    src = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
    dst = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
    graphgen.generate_cuda(spec, src.data_ptr(), dst.data_ptr(), torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    print(f"### {spec.name} (BASELINE configs[{a.config - 1}]), device ms (median of {a.reps})\n")
    print("| directing | ordering | schedule | intersect | build | direct | reorder | count | total | count GTEPS "
          "| total GTEPS | max d~ | Eq.1 n*C | Eq.3 | T |")
    print("|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|")
    prm, keep = tc.make_aorder_params()
    for rule in a.rules.split(","):
        d, r = rule.split(":")
        for sched, isect in [(x, y) for x in a.schedules.split(",") for y in a.intersect.split(",")]:
            tc.tc_set_option("intersect", int(isect))
            rows = []
            for rep in range(a.reps + 1):
                g = tc.Graph(src, dst, spec.n)
                g.direct(d)
                tc.tc_reorder(g.handle, r, prm)
                g.set_schedule(sched)
                T = g.count()
                st = g.stats()
                g.free()
                if rep:
                    rows.append(st)
            med = {k: statistics.median(x[k] for x in rows) for k in ("ms_build", "ms_direct", "ms_reorder", "ms_count")}
            tot = sum(med.values())
            m = st["m"]
            print(f"| {d} | {r} | {sched} | { {'0': 'binary search', '1': 'sort-merge', '2': 'bitmap'}[isect]} | {med['ms_build']:.2f} | {med['ms_direct']:.2f} | {med['ms_reorder']:.2f} | "
                  f"{med['ms_count']:.2f} | {tot:.2f} | {m / med['ms_count'] / 1e6:.2f} | {m / tot / 1e6:.2f} | "
                  f"{st['max_outdeg']} | {st['eq1']} | {st['eq3']} | {T} |", flush=True)


if __name__ == "__main__":
    main()
