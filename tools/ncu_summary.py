"""Summaries of ncu output for profiles/ (run here, on the CPU box).

    python tools/ncu_summary.py launches <launches.csv>          # per-kernel share of device time
    python tools/ncu_summary.py full <report.ncu-rep> <out.json> [flops_per_launch]
"""
import collections
import csv
import io
import json
import subprocess
import sys


def launches(path):
    lines = [l for l in open(path) if l.startswith('"')]
    rows = list(csv.reader(io.StringIO("".join(lines))))
    hdr = rows[0]
    ki, vi, gi = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Grid Size")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[1:]:
        if len(r) <= vi or r[hdr.index("Metric Name")] != "gpu__time_duration.sum":
            continue
        name = r[ki].split("(")[0].split("::")[-1]
        agg[name][0] += 1
        agg[name][1] += float(r[vi].replace(",", ""))
    tot = sum(v[1] for v in agg.values())
    out = []
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        out.append(f"{k:32s} launches={v[0]:5d} time={v[1] / 1e6:10.3f} ms share={100 * v[1] / tot:5.1f}%")
    return "\n".join(out)


WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_tensor_subpipe_dmma.sum", "sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__grid_size", "sm__cycles_elapsed.avg.per_second",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
        "lts__t_bytes.sum"]


def full(rep, out_json, flops=None):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {"kernel": vals[hdr.index("Kernel Name")]}
        for w in WANT:
            if w in hdr:
                i = hdr.index(w)
                try:
                    d[w] = float(vals[i].replace(",", ""))
                except ValueError:
                    d[w] = vals[i]
                d[w + ".unit"] = units[i]
        res.append(d)
    d = res[0]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    rb = d["dram__bytes_read.sum"] * scale.get(d["dram__bytes_read.sum.unit"], 1)
    wb = d["dram__bytes_write.sum"] * scale.get(d["dram__bytes_write.sum.unit"], 1)
    summary = {"report": rep, "metrics": d, "dram_bytes_per_launch": rb + wb}
    if flops:
        t = d["gpu__time_duration.sum"] * (1e-3 if d["gpu__time_duration.sum.unit"] == "us" else 1.0)
        t_s = t * 1e-3 if d["gpu__time_duration.sum.unit"] in ("ms", "us") else t * 1e-9
        summary["flops_per_launch"] = float(flops)
        summary["tflops_under_ncu"] = float(flops) / t_s / 1e12
    with open(out_json, "w") as f:
        json.dump(summary, f, indent=1)
    return summary


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        print(launches(sys.argv[2]))
    else:
        print(json.dumps(full(sys.argv[2], sys.argv[3], sys.argv[4] if len(sys.argv) > 4 else None), indent=1))
