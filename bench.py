#!/usr/bin/env python
"""bench.py — triangle-count edges/s on B200 (BASELINE.json metric), one JSON line.

A step is one pass of the whole hot path over the workload's
raw edge samples, which are resident in HBM before the timed region:
    tc_graph_from_edges -> tc_direct -> tc_reorder -> tc_count[_dist] -> tc_graph_free
value = m (undirected edges after normalisation) / step time, in GTEPS (1e9 edges/s);
N>1: every rank builds the replicated oriented CSR and counts its work-balanced slice,
partials combined with one ncclAllReduce inside tc_count_dist; time = max over ranks.

    python bench.py [--gpus N --steps K --warmup W] [--config C] [--impl reference]

Default workload: BASELINE.json configs[1] (ER n=2^22, 2^26 samples, degree directing,
original order).  `--impl reference` times the CPU oracle (the reference arm of this
tier: the paper ships no code) on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "triangle-count edges/s (GTEPS)"
UNIT = "GTEPS"
# (directing, ordering) per BASELINE.json config (1-based)
CONFIG_RULES = {1: ("degree", "none"), 2: ("degree", "none"), 3: ("paper", "none"),
                4: ("degree", "paper"), 5: ("paper", "paper")}
DEFAULT_CONFIG = 2
L2_BYTES = 126 * 1024 * 1024


def env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get("hbm_gbs", 6650.0), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 100 ms during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")
    NAMES = ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "100", "-i", str(self.gpu)],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except (OSError, ValueError):
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        time.sleep(0.15)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, mx, reasons = [], None, set()
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[1]))
                mx = float(parts[2])
            except ValueError:
                continue
            for name, val in zip(self.NAMES, parts[3:7]):
                if val.lower().startswith("active"):
                    reasons.add(name)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def cpu_cores_used():
    return 1  # the oracle is single-threaded plain C


def oracle_sample(spec, d, r, n_samples):
    """Run the oracle's whole path (O1-O4) on the first n_samples raw samples."""
    import graphgen
    import oracle
    src, dst = graphgen.generate_cpu(spec, count=n_samples)
    t0 = time.perf_counter()
    res = oracle.run(src, dst, spec.n, d, r)
    dt = time.perf_counter() - t0
    return res["m"], res["T"], dt


def sample_size(spec, target):
    s = 1
    while s * 2 <= min(spec.samples, target):
        s *= 2
    return min(spec.samples, s)


def run_reference(args, rank, world):
    """Reference arm: the CPU oracle as it stands, rank 0 only, bounded samples."""
    if rank != 0:
        return
    import graphgen
    cfg = args.config
    spec = graphgen.CONFIGS[cfg]
    d, r = args.direct or CONFIG_RULES[cfg][0], args.reorder or CONFIG_RULES[cfg][1]
    S = sample_size(spec, 1 << 22)
    for _ in range(args.warmup):
        oracle_sample(spec, d, r, S)
    times, m = [], 0
    for _ in range(args.steps):
        m, T, dt = oracle_sample(spec, d, r, S)
        times.append(dt)
    ms = 1e3 * statistics.mean(times)
    value = m / (ms / 1e3) / 1e9
    sample = (f"first {S} of {spec.samples} raw samples of {spec.name} (n={spec.n}), whole oracle "
              f"path O1-O4 ({d} directing, {r} order), per step")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": f"{spec.name} (BASELINE.json configs[{cfg - 1}])", "direct": d,
                       "reorder": r, "sample_edges": m},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cpu_cores_used(), "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=DEFAULT_CONFIG, choices=sorted(CONFIG_RULES))
    ap.add_argument("--direct", choices=["id", "degree", "paper"])
    ap.add_argument("--reorder", choices=["none", "degree", "paper"])
    ap.add_argument("--schedule", default="auto", choices=["auto", "bucketed", "range"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    rank, world, local_rank = env_int("RANK", 0), env_int("WORLD_SIZE", 1), env_int("LOCAL_RANK", 0)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist

    import graphgen
    import paper_conf_sigmod_hu0l21_b200 as tc
    from paper_conf_sigmod_hu0l21_b200 import dist as tdist

    cfg = args.config
    spec = graphgen.CONFIGS[cfg]
    d = args.direct or CONFIG_RULES[cfg][0]
    r = args.reorder or CONFIG_RULES[cfg][1]
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    # under torchrun (even with one rank) the count goes through tc_count_dist + NCCL
    distributed = world > 1 or "LOCAL_RANK" in os.environ
    if distributed:
        dist.init_process_group("nccl", device_id=dev)
    stream = torch.cuda.current_stream(dev)
    sptr = stream.cuda_stream

    # inputs resident in HBM before the timed region
    src = torch.empty(spec.samples, dtype=torch.int32, device=dev)
    dst = torch.empty(spec.samples, dtype=torch.int32, device=dev)
    graphgen.generate_cuda(spec, src.data_ptr(), dst.data_ptr(), sptr)
    torch.cuda.synchronize()
    in_bytes = 8 * spec.samples
    flush = None
    if in_bytes < 2 * L2_BYTES:  # small inputs: flush L2 between timed steps
        flush = torch.empty(2 * L2_BYTES // 4, dtype=torch.int32, device=dev)

    comm = None
    if distributed:
        comm = tdist.init_nccl_comm(rank, world, local_rank)

    prm, keep = tc.make_aorder_params()

    def step(s_in, d_in, keep=False):
        """One pass of the path; keep=True returns the live graph (caller frees it)."""
        g = tc.tc_graph_from_edges(s_in, d_in, spec.n, local_rank, sptr)
        try:
            tc.tc_direct(g, d)
            tc.tc_reorder(g, r, prm)
            if args.schedule != "auto":
                tc.tc_set_schedule(g, args.schedule)
            if comm is not None:
                T = tc.tc_count_dist(g, comm, rank, world)
            else:
                T = tc.tc_count(g)
        except BaseException:
            tc.tc_graph_free(g)
            raise
        if keep:
            return T, g
        tc.tc_graph_free(g)
        return T, None

    for _ in range(args.warmup):
        step(src, dst)
    torch.cuda.synchronize()

    # ---------------------------------------------------------------- timed region
    # per-stage event pairs (option "profile") stay off in the timed region (they add a
    # measured ~1%); the per-kernel events the roofline needs stay on
    tc.tc_set_option("profile", 0)
    tc.tc_set_option("kernel_profile", 1)
    tc.tc_profile_report(reset=True)
    if distributed:
        dist.barrier()
    torch.cuda.synchronize()
    clocks = ClockSampler(local_rank)
    clocks.start()
    times, T, st = [], 0, {}
    for i in range(args.steps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        T, _ = step(src, dst)
        e1.record(stream)
        if flush is not None:
            flush.fill_(1)
        times.append((e0, e1))
    torch.cuda.synchronize()
    if distributed:
        dist.barrier()
    clk = clocks.stop()
    tc.tc_set_option("kernel_profile", 0)
    prof = tc.tc_profile_report(reset=True)
    # stage timings from one extra (untimed) step with the stage events on
    tc.tc_set_option("profile", 1)
    _, g_last = step(src, dst, keep=True)
    st = tc.tc_get_stats(g_last)
    tc.tc_graph_free(g_last)
    step_ms = [a.elapsed_time(b) for a, b in times]
    ms = tdist.max_over_ranks(statistics.mean(step_ms), dev)
    m = st["m"]
    value = m / (ms / 1e3) / 1e9

    # ---------------------------------------------------------------- roofline
    launches = prof.pop("_launches", 0)
    g = tc.tc_graph_from_edges(src, dst, spec.n, local_rank, sptr)
    tc.tc_direct(g, d)
    tc.tc_reorder(g, r, prm)
    tc.tc_analyze(g)
    ast = tc.tc_get_stats(g)
    tc.tc_graph_free(g)
    for k in ("count_small", "count_large", "count_range"):
        if k in prof and world == 1:
            prof[k]["bytes_note"] = "sector model shared by the count kernels"
    count_ms = sum(prof[k]["ms"] for k in ("count_small", "count_large", "count_range") if k in prof)
    kernels = {k: v for k, v in prof.items()}
    if count_ms > 0:
        kernels["count"] = {"ms": count_ms, "launches": args.steps, "bytes": float(ast["alg_bytes"]) * args.steps}
        for k in ("count_small", "count_large", "count_range"):
            kernels.pop(k, None)
    dom = max(kernels, key=lambda k: kernels[k]["ms"]) if kernels else None
    peak, peak_src = measured_peaks()
    roof = None
    if dom:
        kd = kernels[dom]
        per_launch_ms = kd["ms"] / max(kd["launches"], 1)
        per_launch_bytes = kd["bytes"] / max(kd["launches"], 1)
        achieved = per_launch_bytes / (per_launch_ms / 1e3) / 1e9 if per_launch_ms > 0 else 0.0
        traffic = None
        tpath = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tpath):
            with open(tpath) as f:
                traffic = json.load(f).get(f"cfg{cfg}:{d}:{r}", {}).get(dom)
        roof = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                "share_of_step": kd["ms"] / (ms * args.steps),
                "per_launch_ms": per_launch_ms, "alg_bytes_per_launch": per_launch_bytes}

    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": f"{spec.name} (BASELINE.json configs[{cfg - 1}])", "direct": d,
                       "reorder": r, "n": spec.n, "samples": spec.samples, "m": m, "triangles": T,
                       "l2": ("inputs %.0f MiB > L2: no flush" % (in_bytes / 2**20)) if flush is None
                       else "L2 flushed (252 MiB write) between timed steps",
                       "parallelism": "replicated CSR, work-sliced count, 1 NCCL allreduce" if world > 1
                       else "single GPU"},
            "roofline": roof, "clocks": clk, "gpu_launches": launches,
            "stages_ms": {k: st[k] for k in ("ms_build", "ms_direct", "ms_reorder", "ms_count",
                                              "ms_count_kernel")},
            "count_only_gteps": m / (st["ms_count"] / 1e3) / 1e9 if st["ms_count"] else None,
            "kernels_ms_per_step": {k: v["ms"] / args.steps for k, v in kernels.items()},
            "analysis": {"wedges": ast["wedges"], "count_alg_bytes": ast["alg_bytes"],
                         "max_outdeg": ast["max_outdeg"], "levels": ast["levels"],
                         "subrounds": ast["subrounds"], "eq1": ast["eq1"], "eq3": ast["eq3"]}}

    # ---------------------------------------------------------------- e2e (host buffers)
    if not args.no_e2e:
        hs = torch.empty(spec.samples, dtype=torch.int32, pin_memory=True)
        hd = torch.empty(spec.samples, dtype=torch.int32, pin_memory=True)
        hs.copy_(src)
        hd.copy_(dst)
        step(hs, hd)
        torch.cuda.synchronize()
        if distributed:
            dist.barrier()
        ev = []
        for _ in range(args.steps):
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            step(hs, hd)
            e1.record(stream)
            ev.append((e0, e1))
        torch.cuda.synchronize()
        e_ms = tdist.max_over_ranks(statistics.mean(a.elapsed_time(b) for a, b in ev), dev)
        line["e2e"] = {"value": m / (e_ms / 1e3) / 1e9, "unit": UNIT, "h2d_bytes_per_step": in_bytes,
                       "d2h_bytes_per_step": 8, "ms_per_step": e_ms,
                       "api": "tc_graph_from_edges(pinned host src/dst) -> tc_direct -> tc_reorder -> tc_count"}

    # ---------------------------------------------------------------- CPU oracle baseline
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        S = sample_size(spec, 1 << 24)
        m_s, _, dt = oracle_sample(spec, d, r, S)
        line["cpu_baseline"] = {"value": m_s / dt / 1e9, "unit": UNIT, "cores": cpu_cores_used(),
                                "kind": "oracle",
                                "sample": f"first {S} of {spec.samples} raw samples of {spec.name} "
                                          f"(n={spec.n}, m={m_s}), whole oracle path O1-O4, {dt:.1f} s"}
    if comm is not None:
        tc.tc_nccl_comm_destroy(comm)
    del keep
    if rank == 0:
        print(json.dumps(line), flush=True)
    if distributed:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
