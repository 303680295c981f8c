"""Per-kernel device ms (library ProfScope events) of one directing/ordering run, averaged
over --reps after a warm-up, for each value of an option.

    python tools/kprof.py --config 3 [--rule degree:none] [--option group_build --values 0,1]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import graphgen
import paper_conf_sigmod_hu0l21_b200 as tc


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--rule", default="degree:none")
    ap.add_argument("--option", default=None)
    ap.add_argument("--values", default="1")
    ap.add_argument("--reps", type=int, default=3)
    a = ap.parse_args()
    spec = graphgen.CONFIGS[a.config]
    src = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
    dst = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
    graphgen.generate_cuda(spec, src.data_ptr(), dst.data_ptr(), torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    d, r = a.rule.split(":")
    prm, keep = tc.make_aorder_params()
    for val in a.values.split(","):
        if a.option:
            tc.tc_set_option(a.option, int(val))
        for rep in range(a.reps + 1):
            if rep == 1:
                tc.tc_set_option("kernel_profile", 1)
                tc.tc_profile_report(reset=True)
            g = tc.Graph(src, dst, spec.n)
            g.direct(d)
            tc.tc_reorder(g.handle, r, prm)
            g.count()
            g.free()
        tc.tc_set_option("kernel_profile", 0)
        prof = tc.tc_profile_report(reset=True)
        if isinstance(prof, str):
            prof = json.loads(prof)
        prof.pop("_launches", None)
        print(f"{spec.name} {a.rule} {a.option}={val}")
        for k, v in sorted(prof.items(), key=lambda kv: -kv[1]["ms"]):
            print(f"  {k:16s} {v['ms'] / a.reps:8.3f} ms  x{v['launches'] // a.reps}")


if __name__ == "__main__":
    main()
