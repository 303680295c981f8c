"""Wall-clock per API call vs device time per kernel for one pipeline pass (diagnostics)."""
import sys, time, json
sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
import torch
import graphgen
import paper_conf_sigmod_hu0l21_b200 as tc

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
d = sys.argv[2] if len(sys.argv) > 2 else "degree"
r = sys.argv[3] if len(sys.argv) > 3 else "none"
spec = graphgen.CONFIGS[cfg]
src = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
dst = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
graphgen.generate_cuda(spec, src.data_ptr(), dst.data_ptr(), torch.cuda.current_stream().cuda_stream)
torch.cuda.synchronize()
prm, keep = tc.make_aorder_params()
import os
for kv in filter(None, os.environ.get("TC_OPTS", "").split(",")):
    k, v = kv.split("=")
    tc.tc_set_option(k, int(v))
ITERS = int(os.environ.get("ITERS", "4"))
for it in range(ITERS):
    tc.tc_set_option("kernel_profile", 1)
    tc.tc_profile_report(reset=True)
    t = {}
    t0 = time.perf_counter(); g = tc.tc_graph_from_edges(src, dst, spec.n); t["build"] = time.perf_counter() - t0
    t0 = time.perf_counter(); tc.tc_direct(g, d); t["direct"] = time.perf_counter() - t0
    t0 = time.perf_counter(); tc.tc_reorder(g, r, prm); t["reorder"] = time.perf_counter() - t0
    if os.environ.get("TC_SCHED"):
        tc.tc_set_schedule(g, os.environ["TC_SCHED"])
    t0 = time.perf_counter(); T = tc.tc_count(g); t["count"] = time.perf_counter() - t0
    st = tc.tc_get_stats(g)
    t0 = time.perf_counter(); tc.tc_graph_free(g); t["free"] = time.perf_counter() - t0
    prof = tc.tc_profile_report(reset=True)
    if it == ITERS - 1:
        print("wall ms:", {k: round(v * 1e3, 3) for k, v in t.items()}, "total", round(sum(t.values()) * 1e3, 3))
        print("stage ms:", {k: round(st[k], 3) for k in ("ms_build", "ms_direct", "ms_reorder", "ms_count", "ms_count_kernel")})
        launches = prof.pop("_launches")
        print("kernels ms:", {k: round(v["ms"], 3) for k, v in sorted(prof.items(), key=lambda x: -x[1]["ms"])}, "launches", launches)
        print("T", T, "m", st["m"])
