"""Summarize ncu captures (run here, no GPU needed) into profiles/.

  python scripts/ncu_summary.py TAG gpurun_out/prof_a.ncu-rep[:name] ... [--launches gpurun_out/launches.csv]

Writes profiles/ncu_full_<TAG>.json (key metrics per capture, base units),
profiles/ncu_traffic.json (DRAM and L2->L1 bytes per launch per kernel, read by bench.py
for roofline.traffic and roofline.l2) and, with --launches, profiles/launches_<TAG>.txt (per-kernel launch
count, mean device time, and share of the total, from the gpu__time_duration pass).
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
    "l1tex__t_sector_hit_rate.pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
    "launch__occupancy_limit_registers", "launch__shared_mem_per_block_static",
    "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum",
    "smsp__thread_inst_executed_per_inst_executed.ratio",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "lts__t_sectors_srcunit_tex_op_read.sum",
    "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "smsp__pcsamp_warps_issue_stalled_long_scoreboard", "smsp__pcsamp_warps_issue_stalled_wait",
    "smsp__pcsamp_warps_issue_stalled_selected", "smsp__pcsamp_warps_issue_stalled_barrier",
    "smsp__pcsamp_warps_issue_stalled_math_pipe_throttle",
    "smsp__pcsamp_warps_issue_stalled_short_scoreboard",
]


def raw(rep):
    """Key metrics of every launch in a .ncu-rep (or in its exported `--page raw --csv
    --print-units base` CSV)."""
    if rep.endswith(".csv"):
        out = open(rep).read()
    else:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--print-units", "base"],
                             capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = dict(zip(hdr, vals))
        m = {"kernel": d.get("Kernel Name", "")[:200]}
        for k in KEYS:
            if k in d:
                try:
                    m[k] = float(d[k].replace(",", ""))
                except ValueError:
                    m[k] = d[k]
        res.append(m)
    return res


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr, agg = None, {}
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d.get("Metric Name") != "gpu__time_duration.sum":
                continue
            v = float(d["Metric Value"].replace(",", ""))
            unit = d.get("Metric Unit", "nsecond")
            v *= {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3, "second": 1e6}.get(unit, 1e-3)
            k = d["Kernel Name"].split("(")[0]
            agg.setdefault(k, []).append(v)
    tot = sum(sum(v) for v in agg.values())
    lines = [f"# {path}: per-kernel launches under ncu (cold, serialized); us", "# n  mean_us  total_us  share  kernel"]
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        lines.append(f"{len(v):4d} {sum(v)/len(v):12.1f} {sum(v):12.1f} {sum(v)/tot:6.3f}  {k}")
    return "\n".join(lines) + "\n"


def main():
    tag = sys.argv[1]
    args = sys.argv[2:]
    lfile = None
    if "--launches" in args:
        i = args.index("--launches")
        lfile = args[i + 1]
        args = args[:i] + args[i + 2:]
    summary = {}
    traffic_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    for a in args:
        rep, _, name = a.partition(":")
        for m in raw(rep):
            nm = name or m["kernel"]
            summary[nm] = m
            if "dram__bytes_read.sum" in m:
                traffic[nm] = {"dram_bytes_per_launch": m["dram__bytes_read.sum"] + m["dram__bytes_write.sum"],
                               "time_ns": m.get("gpu__time_duration.sum"), "source": os.path.basename(rep),
                               "tag": tag}
                if "lts__t_sectors_srcunit_tex_op_read.sum" in m:  # L2 -> L1 read bytes
                    traffic[nm]["l2_read_bytes_per_launch"] = 32.0 * m["lts__t_sectors_srcunit_tex_op_read.sum"]
                    traffic[nm]["lts_throughput_pct"] = m.get("lts__throughput.avg.pct_of_peak_sustained_elapsed")
                    traffic[nm]["l1tex_throughput_pct"] = m.get("l1tex__throughput.avg.pct_of_peak_sustained_elapsed")
                    traffic[nm]["lts_hit_rate_pct"] = m.get("lts__t_sector_hit_rate.pct")
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", f"ncu_full_{tag}.json"), "w") as f:
        json.dump(summary, f, indent=1)
    with open(traffic_path, "w") as f:
        json.dump(traffic, f, indent=1)
    if lfile:
        with open(os.path.join(ROOT, "profiles", f"launches_{tag}.txt"), "w") as f:
            f.write(launches(lfile))
    print(json.dumps({k: {kk: v.get(kk) for kk in ("gpu__time_duration.sum", "dram__bytes_read.sum",
                                                     "launch__registers_per_thread")}
                      for k, v in summary.items()}, indent=1))


if __name__ == "__main__":
    main()
