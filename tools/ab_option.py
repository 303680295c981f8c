"""A/B one library option on one config: device ms of each stage (median of --reps after a
warm-up) and T for every value of the option (T must not change).

    python tools/ab_option.py --config 2 --option bloom --values 0,1 [--rule degree:none]
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
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--option", required=True)
    ap.add_argument("--values", default="0,1")
    ap.add_argument("--rule", default="degree:none")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--set", default="", help="fixed options k=v,k=v applied first")
    a = ap.parse_args()
    for kv in filter(None, a.set.split(",")):
        k, v = kv.split("=")
        tc.tc_set_option(k, int(v))
    spec = graphgen.CONFIGS[a.config]
    src = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
    dst = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
    graphgen.generate_cuda(spec, src.data_ptr(), dst.data_ptr(), torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    d, r = a.rule.split(":")
    prm, keep = tc.make_aorder_params()
    print(f"{spec.name} {a.rule} option {a.option}")
    Ts = set()
    for val in a.values.split(","):
        tc.tc_set_option(a.option, int(val))
        rows = []
        for rep in range(a.reps + 1):
            g = tc.Graph(src, dst, spec.n)
            g.direct(d)
            tc.tc_reorder(g.handle, r, prm)
            T = g.count()
            st = g.stats()
            g.free()
            Ts.add(T)
            if rep:
                rows.append(st)
        med = {k: statistics.median(x[k] for x in rows) for k in ("ms_build", "ms_direct", "ms_reorder", "ms_count")}
        print(f"  {a.option}={val}: " + " ".join(f"{k[3:]}={v:.3f}" for k, v in med.items()) + f" T={T}", flush=True)
    assert len(Ts) == 1, Ts


if __name__ == "__main__":
    main()
