#!/usr/bin/env python
"""Summarise ncu outputs for profiles/ (run here, no GPU needed).

  python tools/ncu_summary.py full  <report.ncu-rep> <out.json>
      key metrics per profiled launch of an `ncu --set full` capture, plus
      dram read+write bytes per launch (-> bench.py roofline.traffic)
  python tools/ncu_summary.py launches <launches.csv> <out.json>
      per-kernel-name launch counts and device-time shares from a
      `--metrics gpu__time_duration.sum` launch list
"""
import csv
import io
import json
import subprocess
import sys
from collections import defaultdict

KEYS = [
    "Kernel Name", "Grid Size", "Block Size", "gpu__time_duration.sum",
    "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__occupancy_limit_registers",
    "launch__shared_mem_per_block_dynamic", "launch__waves_per_multiprocessor",
    "lts__t_bytes.sum", "l1tex__t_bytes.sum",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__pcsamp_warps_issue_stalled_long_scoreboard",
    "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_drain_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_sleeping_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
    "smsp__average_warp_latency_per_inst_issued.ratio",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "nvltx__bytes.sum", "nvlrx__bytes.sum",
]

SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9,
         "ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3, "nsecond": 1e-9}


def _num(v, unit):
    try:
        x = float(v.replace(",", ""))
    except ValueError:
        return v
    return x * SCALE.get(unit, 1)


def full(rep, out):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    idx = {h: i for i, h in enumerate(hdr)}
    launches = []
    for r in rows[2:]:
        d = {}
        for k in KEYS:
            if k in idx:
                d[k] = _num(r[idx[k]], units[idx[k]]) if k not in ("Kernel Name", "Grid Size", "Block Size") else r[idx[k]]
        launches.append(d)
    per = [x.get("dram__bytes_read.sum", 0) + x.get("dram__bytes_write.sum", 0) for x in launches]
    res = {"report": rep, "units": "bytes and seconds", "launches": launches,
           "dram_bytes_per_launch": sum(per) / len(per) if per else None}
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
    for x in launches:
        print(x.get("Kernel Name"), x.get("Grid Size"), x.get("gpu__time_duration.sum"),
              x.get("dram__bytes_read.sum"), x.get("dram__bytes_write.sum"))


def launches(path, out):
    text = open(path).read()
    start = text.index('"ID"')
    rows = list(csv.DictReader(io.StringIO(text[start:])))
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        t = _num(r["Metric Value"], r["Metric Unit"])
        agg[r["Kernel Name"]][0] += 1
        agg[r["Kernel Name"]][1] += t
    total = sum(v[1] for v in agg.values())
    res = {k: {"launches": v[0], "time_s": v[1], "share": v[1] / total} for k, v in
           sorted(agg.items(), key=lambda kv: -kv[1][1])}
    with open(out, "w") as f:
        json.dump({"source": path, "total_time_s": total, "kernels": res}, f, indent=1)
    for k, v in res.items():
        print("%6d  %8.3f ms  %5.1f%%  %s" % (v["launches"], v["time_s"] * 1e3, 100 * v["share"], k[:100]))


if __name__ == "__main__":
    {"full": full, "launches": launches}[sys.argv[1]](sys.argv[2], sys.argv[3])
