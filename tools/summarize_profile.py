"""Summarise a tools/profile_round.sh output directory into profiles/<round>/ (tracked)."""
import csv
import collections
import json
import os
import shutil
import subprocess
import sys


def rows(path):
    out, hdr = [], None
    for r in csv.reader(open(path)):
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            out.append(dict(zip(hdr, r)))
    return out


def num(x):
    return float(x.replace(",", ""))


def main(src, dst, workload="c2"):
    os.makedirs(dst, exist_ok=True)
    lines = ["# ncu summary: one bench step of workload %s (`tools/profile_round.sh OUT %s`)" % (workload, workload), "",
             "ncu times are cold-cache and serialised (compare shares, not absolute times).", ""]
    L = rows(os.path.join(src, "launches.csv"))
    agg = collections.defaultdict(lambda: [0, 0.0])
    for d in L:
        name = d["Kernel Name"].split("(")[0].replace("<unnamed>::", "")
        if d["Kernel Name"] == "pgk_eval":
            name += " cta=" + d["Block Size"].split(",")[0].strip("(")
        agg[name][0] += 1
        agg[name][1] += num(d["Metric Value"]) / 1e6
    tot = sum(v[1] for v in agg.values())
    lines += ["## Launch list (gpu__time_duration, cold cache, serialised)", "",
              "| kernel | launches | ms | share |", "|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        lines.append("| %s | %d | %.2f | %.1f%% |" % (k, v[0], v[1], 100 * v[1] / tot))
    lines.append("")
    M = rows(os.path.join(src, "k2_metrics.csv"))
    per = collections.defaultdict(dict)
    for d in M:
        per[d["ID"]][d["Metric Name"]] = num(d["Metric Value"])
        per[d["ID"]]["block"] = d["Block Size"]
        per[d["ID"]]["grid"] = d["Grid Size"]
    t_ns = sum(p.get("gpu__time_duration.sum", 0) for p in per.values())
    rd = sum(p.get("dram__bytes_read.sum", 0) for p in per.values())
    wr = sum(p.get("dram__bytes_write.sum", 0) for p in per.values())
    n = len(per)
    w = lambda key: sum(p.get(key, 0) * p.get("gpu__time_duration.sum", 0) for p in per.values()) / max(t_ns, 1)
    traffic = {"kernel": "pgk_eval", "launches_per_step": n, "bytes_per_step": rd + wr,
               "bytes_per_launch": (rd + wr) / max(n, 1), "dram_read": rd, "dram_write": wr,
               "k2_ms_per_step_ncu": t_ns / 1e6,
               "issue_active_pct_time_weighted": w("smsp__issue_active.avg.pct_of_peak_sustained_active"),
               "alu_pipe_pct_time_weighted": w("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active"),
               "warps_active_pct_time_weighted": w("sm__warps_active.avg.pct_of_peak_sustained_active")}
    json.dump(traffic, open(os.path.join(dst, "k2_traffic.json"), "w"), indent=1)
    lines += ["## Evaluation kernel (pgk_eval), all launches of the step", "",
              "| metric | value |", "|---|---|"]
    for k, v in traffic.items():
        lines.append("| %s | %s |" % (k, ("%.3g" % v) if isinstance(v, float) else v))
    lines.append("")
    rep = os.path.join(src, "k2_top.ncu-rep")
    if os.path.exists(rep):
        det = subprocess.run(["ncu", "-i", rep, "--page", "details"], capture_output=True, text=True).stdout
        keep = [l.rstrip() for l in det.splitlines() if any(s in l for s in (
            "Duration", "Registers Per", "Achieved Occupancy", "Theoretical Occupancy", "Issue Slots Busy",
            "Executed Ipc A", "DRAM Throughput", "Memory Throughput", "Warp Cycles Per Issued", "Block Size",
            "Grid Size", "Dynamic Shared"))]
        lines += ["## Top evaluation-kernel launch (`--set full`)", "", "```"] + keep + ["```", ""]
        shutil.copy(rep, os.path.join(dst, "k2_top.ncu-rep"))
        # where the top launch's instructions and stall samples go, per source line
        here = os.path.dirname(os.path.abspath(__file__))
        for title, env in (("instructions executed", {}), ("stall samples", {"SORT_SAMPLES": "1"})):
            out = subprocess.run([sys.executable, os.path.join(here, "ncu_lines.py"), os.path.abspath(rep), "0", "15",
                                  os.path.abspath(os.path.join(src, "src"))], capture_output=True, text=True,
                                 cwd="/", env=dict(os.environ, **env)).stdout
            lines += ["### Top source lines by %s" % title, "", "```"] + \
                [l[:150] for l in out.splitlines()] + ["```", ""]
    shutil.copy(os.path.join(src, "launches.csv"), os.path.join(dst, "launches.csv"))
    shutil.copy(os.path.join(src, "k2_metrics.csv"), os.path.join(dst, "k2_metrics.csv"))
    open(os.path.join(dst, "SUMMARY.md"), "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else "c2")
