#!/usr/bin/env python
"""bench.py — triangle-count edges/s on B200 (BASELINE.json metric), one JSON line.

A step is one pass of the whole hot path over the workload's
raw edge samples, which are resident in HBM before the timed region:
    tc_graph_from_edges -> tc_direct -> tc_reorder -> tc_count[_dist] -> tc_graph_free
value = m (undirected edges after normalisation) / t_count in GTEPS (1e9 edges/s), where
t_count = the CUDA-event time of tc_count (schedule + count kernels + reduction; at N>1
tc_count_dist incl. its ncclAllReduce), median over the timed steps, max over ranks
(SURVEY.md §8(d)/(e)).  The whole-path throughput (build + direct + reorder + count) is
reported beside it as "whole_path" and, from pinned host buffers, as "e2e".

    python bench.py [--gpus N --steps K --warmup W] [--config C] [--impl reference]

Default workload: BASELINE.json configs[3] (R-MAT s24 ef32, 2^29 samples, degree directing,
A-order), the config BASELINE's "1/2/4/8 B200" metric is quoted on.  N>1: every rank builds
the replicated CSR, rank 0 runs the A-order greedy and broadcasts pi (tc_reorder_dist), each
rank counts its work-balanced slice, one ncclAllReduce.  `cpu_baseline` and
`--impl reference` time the CPU oracle (the reference arm of this tier: the paper ships no
code) on the SAME graph: the oracle builds it once (untimed), then its forward count runs
on a uniform random sample of source-label chunks on all host cores.
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
DEFAULT_CONFIG = 4
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


def oracle_graph(spec, d, r):
    """The oracle's own oriented CSR of the whole workload (O1-O3 + CSR), untimed setup."""
    import gc

    import graphgen
    import oracle
    t0 = time.perf_counter()
    src, dst = graphgen.generate_cpu(spec)
    edges = oracle.simple_graph(src, dst, spec.n)
    del src, dst
    gc.collect()
    dirs, _ = oracle.direct(edges, spec.n, d)
    od = oracle.outdeg(edges, spec.n, dirs)
    perm, _ = oracle.reorder(od, r)
    offs, col = oracle.oriented_csr(edges, spec.n, dirs, perm)
    m = len(edges)
    del edges, dirs, od, perm
    gc.collect()
    return offs, col, m, time.perf_counter() - t0


class OracleSampler:
    """The oracle's forward count (O4, orc_count_forward_mt on all host cores) over a
    uniform random sample of source-label chunks of the same graph the GPU counts.
    Throughput = edges whose intersections were computed (Σ d~(u) over the sampled u) / t."""

    CHUNK = 4096

    def __init__(self, offs, col, seed=20210):
        import numpy as np
        self.offs, self.col = offs, col
        n = len(offs) - 1
        nch = max(1, (n + self.CHUNK - 1) // self.CHUNK)
        self.order = np.random.default_rng(seed).permutation(nch)
        self.pos = 0

    def run(self, budget_s):
        import oracle
        t0 = time.perf_counter()
        edges, chunks = 0, 0
        n = len(self.offs) - 1
        while True:
            c = int(self.order[self.pos % len(self.order)])
            self.pos += 1
            a, b = c * self.CHUNK, min(n, (c + 1) * self.CHUNK)
            oracle.count_forward(self.offs, self.col, a, b, threads=0)
            edges += int(self.offs[b] - self.offs[a])
            chunks += 1
            if time.perf_counter() - t0 >= budget_s or chunks >= len(self.order):
                break
        return edges, time.perf_counter() - t0, chunks


def cpu_baseline_line(spec, d, r, budget_s, steps=1):
    """(per-step values, description) of the oracle on the same graph."""
    import oracle
    offs, col, m, build_s = oracle_graph(spec, d, r)
    smp = OracleSampler(offs, col)
    vals, desc = [], None
    for _ in range(steps):
        e, dt, ch = smp.run(budget_s)
        vals.append((e, dt))
        desc = (f"{spec.name} (n={spec.n}, m={m}), {d} directing x {r} order, the oracle's own CSR "
                f"(built once, {build_s:.0f} s, untimed); per step its forward count (two-pointer "
                f"merge, orc_count_forward_mt) over {ch} random chunks of {OracleSampler.CHUNK} source "
                f"labels = {e} directed edges, {dt:.1f} s on {oracle.host_cores()} threads")
    return vals, desc, oracle.host_cores()


def run_reference(args, rank, world):
    """Reference arm: the CPU oracle as it stands on the same workload, rank 0 only."""
    if rank != 0:
        return
    import graphgen
    cfg = args.config
    spec = graphgen.CONFIGS[cfg]
    d, r = args.direct or CONFIG_RULES[cfg][0], args.reorder or CONFIG_RULES[cfg][1]
    budget = max(1.0, min(8.0, 150.0 / max(1, args.steps + args.warmup)))
    vals, desc, cores = cpu_baseline_line(spec, d, r, budget, steps=args.warmup + args.steps)
    vals = vals[args.warmup:]
    rates = [e / dt / 1e9 for e, dt in vals]
    value = statistics.median(rates)
    ms = 1e3 * statistics.median(dt for _, dt in vals)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": f"{spec.name} (BASELINE.json configs[{cfg - 1}])", "direct": d,
                       "reorder": r},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": desc},
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
    ap.add_argument("--schedule", default="auto", choices=["auto", "bucketed", "range", "edge_aorder"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=12.0, help="seconds of oracle count sample")
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

    def step(s_in, d_in, keep=False, events=None):
        """One pass of the path; keep=True returns the live graph (caller frees it).
        events = (c0, c1): CUDA events recorded on the stream around the count."""
        g = tc.tc_graph_from_edges(s_in, d_in, spec.n, local_rank, sptr)
        try:
            tc.tc_direct(g, d)
            if comm is not None and r == "paper":
                tc.tc_reorder_dist(g, r, prm, comm, rank, world)  # greedy on rank 0, pi broadcast
            else:
                tc.tc_reorder(g, r, prm)
            if args.schedule != "auto":
                tc.tc_set_schedule(g, args.schedule)
            if events:
                events[0].record(stream)
            if comm is not None:
                T = tc.tc_count_dist(g, comm, rank, world)
            else:
                T = tc.tc_count(g)
            if events:
                events[1].record(stream)
        except BaseException:
            tc.tc_graph_free(g)
            raise
        if keep:
            return T, g
        tc.tc_graph_free(g)
        return T, None

    def ev():
        return torch.cuda.Event(enable_timing=True)

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
    times, T = [], 0
    for i in range(args.steps):
        e0, e1, c0, c1 = ev(), ev(), ev(), ev()
        e0.record(stream)
        T, _ = step(src, dst, events=(c0, c1))
        e1.record(stream)
        if flush is not None:
            flush.fill_(1)
        times.append((e0, e1, c0, c1))
    torch.cuda.synchronize()
    if distributed:
        dist.barrier()
    clk = clocks.stop()
    tc.tc_set_option("kernel_profile", 0)
    prof = tc.tc_profile_report(reset=True)
    step_ms = [a.elapsed_time(b) for a, b, _, _ in times]
    count_ms = [c.elapsed_time(e) for _, _, c, e in times]
    # max over ranks of the per-rank median (count + allreduce)
    t_count = tdist.max_over_ranks(statistics.median(count_ms), dev)
    t_step = tdist.max_over_ranks(statistics.median(step_ms), dev)
    # stage timings from one extra (untimed) step with the stage events on
    tc.tc_set_option("profile", 1)
    _, g_last = step(src, dst, keep=True)
    st = tc.tc_get_stats(g_last)
    tc.tc_graph_free(g_last)
    m = st["m"]
    value = m / (t_count / 1e3) / 1e9

    # ---------------------------------------------------------------- roofline
    launches = prof.pop("_launches", 0)
    g = tc.tc_graph_from_edges(src, dst, spec.n, local_rank, sptr)
    tc.tc_direct(g, d)
    tc.tc_reorder(g, r, prm)
    tc.tc_analyze(g)
    ast = tc.tc_get_stats(g)
    tc.tc_graph_free(g)
    count_keys = ("count_small", "count_large", "count_range", "count_units", "count_bitmap")
    kernels = {k: v for k, v in prof.items()}
    # the count kernels share one algorithmic-bytes model (the no-reuse sector model of the
    # whole count): roofline over their summed time
    kc_ms = sum(prof[k]["ms"] for k in count_keys if k in prof)
    if kc_ms > 0:
        for k in count_keys:
            kernels.pop(k, None)
        kernels["count"] = {"ms": kc_ms, "launches": args.steps,
                            "bytes": float(ast["alg_bytes"]) * args.steps * (1.0 if world == 1 else 1.0 / world)}
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
                "share_of_step": kd["ms"] / (t_step * args.steps),
                "per_launch_ms": per_launch_ms, "alg_bytes_per_launch": per_launch_bytes}
        if dom == "count":
            roof["kernels"] = [k for k in count_keys if k in prof]
            roof["bytes_model"] = ("SURVEY.md §8(d) no-reuse 32-B-sector model of the count's schedule "
                                   "(per edge the streamed list = the shorter of N+(u), N+(v), + its "
                                   "offsets; per source its staged list), computed exactly per graph "
                                   "by tc_analyze")

    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t_step, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": f"{spec.name} (BASELINE.json configs[{cfg - 1}])", "direct": d,
                       "reorder": r, "n": spec.n, "samples": spec.samples, "m": m, "triangles": T,
                       "l2": ("inputs %.0f MiB > L2: no flush" % (in_bytes / 2**20)) if flush is None
                       else "L2 flushed (252 MiB write) between timed steps",
                       "parallelism": ("replicated CSR, A-order on rank 0 + ncclBroadcast, work-sliced "
                                       "count, 1 ncclAllReduce") if distributed else "single GPU"},
            "value_def": "m / t_count, t_count = median CUDA-event time of tc_count"
                         + ("_dist (incl. allreduce), max over ranks" if distributed else ""),
            "count_ms": t_count,
            "whole_path": {"value": m / (t_step / 1e3) / 1e9, "unit": UNIT, "ms_per_step": t_step,
                           "steps": "build -> direct -> reorder -> count -> free, median, max over ranks"},
            "roofline": roof, "clocks": clk, "gpu_launches": launches,
            "stages_ms": {k: st[k] for k in ("ms_build", "ms_direct", "ms_reorder", "ms_count",
                                              "ms_count_kernel")},
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
        evs = []
        for _ in range(args.steps):
            e0, e1 = ev(), ev()
            e0.record(stream)
            step(hs, hd)
            e1.record(stream)
            evs.append((e0, e1))
        torch.cuda.synchronize()
        e_ms = tdist.max_over_ranks(statistics.median(a.elapsed_time(b) for a, b in evs), dev)
        line["e2e"] = {"value": m / (e_ms / 1e3) / 1e9, "unit": UNIT, "h2d_bytes_per_step": in_bytes,
                       "d2h_bytes_per_step": 8, "ms_per_step": e_ms,
                       "api": "tc_graph_from_edges(pinned host src/dst) -> tc_direct -> tc_reorder -> "
                              "tc_count, whole path per step"}
        del hs, hd

    # ---------------------------------------------------------------- CPU oracle baseline
    if comm is not None:
        tc.tc_nccl_comm_destroy(comm)
    del keep, src, dst, flush
    torch.cuda.empty_cache()
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        vals, desc, cores = cpu_baseline_line(spec, d, r, args.cpu_budget, steps=1)
        e, dt = vals[0]
        line["cpu_baseline"] = {"value": e / dt / 1e9, "unit": UNIT, "cores": cores, "kind": "oracle",
                                "sample": desc}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if distributed:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
