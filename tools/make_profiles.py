"""Turn gpurun_out/ ncu captures into profiles/ summaries + profiles/traffic.json.

    python tools/make_profiles.py --round r01 --cfg 2 --rules degree:none
"""
import argparse
import collections
import csv
import glob
import io
import json
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
        "smsp__thread_inst_executed_per_inst_executed.ratio",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"]
UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def kernel_short(name):
    m = re.search(r"(\w+_kernel)", name)
    return m.group(1) if m else name[:40]


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr, agg = None, collections.OrderedDict()
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr is None or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(d["Metric Value"].replace(",", ""))
        unit = d["Metric Unit"]
        v *= {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3,
              "second": 1e6, "s": 1e6}.get(unit, 1.0)
        a = agg.setdefault(kernel_short(d["Kernel Name"]), [0, 0.0])
        a[0] += 1
        a[1] += v
    return agg


def full(path):
    """Summary of one `ncu --page raw --csv` page (a .raw.csv file, or a .ncu-rep read with ncu)."""
    if path.endswith(".ncu-rep"):
        out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    else:
        out = open(path).read()
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return None
    h, u = rows[0], rows[1]
    d = dict(zip(h, rows[2]))
    res = {"kernel": kernel_short(d.get("Kernel Name", "?"))}
    for k in KEYS:
        if k in d:
            res[k] = (d[k], u[h.index(k)])
    stalls = [(k, d[k]) for k in h if k.startswith("smsp__average_warps_issue_stalled_")
              and k.endswith("per_issue_active.ratio")]
    res["stalls"] = sorted(((float(v.replace(",", "")), k[len("smsp__average_warps_issue_stalled_"):-len(
        "_per_issue_active.ratio")]) for k, v in stalls if v), reverse=True)[:6]
    rb = float(d["dram__bytes_read.sum"].replace(",", "")) * UNIT_SCALE.get(u[h.index("dram__bytes_read.sum")], 1)
    wb = float(d["dram__bytes_write.sum"].replace(",", "")) * UNIT_SCALE.get(u[h.index("dram__bytes_write.sum")], 1)
    res["traffic_bytes"] = rb + wb
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--round", default="r01")
    ap.add_argument("--cfg", type=int, default=2)
    ap.add_argument("--rules", default="degree:none")
    ap.add_argument("--src", default=os.path.join(ROOT, "gpurun_out"))
    ap.add_argument("--tag", default="", help="file prefix of tools/gpu_round.sh outputs, e.g. r02d_")
    a = ap.parse_args()
    prof = os.path.join(ROOT, "profiles")
    os.makedirs(prof, exist_ok=True)
    lines = [f"# {a.round}: ncu summary, BASELINE configs[{a.cfg - 1}] ({a.rules})", ""]
    lp = os.path.join(a.src, f"{a.tag}launches_cfg{a.cfg}.csv")
    if os.path.exists(lp):
        agg = launches(lp)
        tot = sum(t for _, t in agg.values())
        lines += ["## Launch list (ncu gpu__time_duration.sum, --clock-control none; cold-cache, serialised: shares)",
                  "", "| kernel | launches | total us | share |", "|---|---|---|---|"]
        for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
            lines.append(f"| {k} | {c} | {t:.1f} | {100 * t / tot:.1f}% |")
        lines.append("")
    traffic = {}
    for p in sorted(glob.glob(os.path.join(a.src, f"{a.tag}full_cfg{a.cfg}_*.ncu-rep")) +
                    glob.glob(os.path.join(a.src, f"{a.tag}full_cfg{a.cfg}_*.raw.csv"))):
        r = full(p)
        if not r:
            continue
        lines += [f"## {r['kernel']} (`ncu --set full`, one launch)", ""]
        for k in KEYS:
            if k in r:
                lines.append(f"- {k}: {r[k][0]} {r[k][1]}")
        lines.append("- top stalls (warps per issue): " + ", ".join(f"{n} {v:.2f}" for v, n in r["stalls"]))
        lines.append(f"- DRAM traffic per launch: {r['traffic_bytes'] / 1e6:.1f} MB")
        lines.append("")
        name = {"rs_pass_kernel": "radix_pass", "unique_kernel": "unique",
                "rs_hist_kernel": "radix_hist"}.get(r["kernel"], r["kernel"])
        traffic[name] = r["traffic_bytes"]
        if r["kernel"].startswith("count_"):  # the count kernels share one bytes model (bench "count")
            traffic["count"] = traffic.get("count", 0.0) + r["traffic_bytes"]
    with open(os.path.join(prof, f"{a.round}_ncu_cfg{a.cfg}.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    tj = os.path.join(prof, "traffic.json")
    allt = json.load(open(tj)) if os.path.exists(tj) else {}
    d, r = a.rules.split(":")
    allt[f"cfg{a.cfg}:{d}:{r}"] = traffic
    json.dump(allt, open(tj, "w"), indent=1, sort_keys=True)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
