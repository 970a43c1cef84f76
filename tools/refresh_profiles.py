#!/usr/bin/env python
"""Copy one tools/profile_round.sh run (gpurun_out/<tag>/) into profiles/<round>/
(run here, no GPU needed): bench line, ncu launch list + its summary, the two
ncu --set full captures as JSON summaries and details pages, the GPU test
log, and the bulk path's DRAM bytes per launch into profiles/traffic.json
(bench.py's roofline.traffic).

  python tools/refresh_profiles.py gpurun_out/r01k [profiles/r01]
"""
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main():
    src = sys.argv[1]
    dst = sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, "profiles", "r01")
    summ = os.path.join(ROOT, "tools", "ncu_summary.py")
    for f in ("bench.json", "launches.csv", "pytest_gpu.log"):
        if os.path.exists(os.path.join(src, f)):
            shutil.copy(os.path.join(src, f), os.path.join(dst, f))
    subprocess.run([sys.executable, summ, "launches", os.path.join(src, "launches.csv"),
                    os.path.join(dst, "launches_summary.json")], check=True, stdout=subprocess.DEVNULL)
    for rep, js, det in (("prof_swap.ncu-rep", "ncu_full_swap.json", "ncu_full_details.txt"),
                         ("prof_swap_capped.ncu-rep", "ncu_full_swap_capped.json", "ncu_full_capped_details.txt")):
        r = os.path.join(src, rep)
        if not os.path.exists(r):
            continue
        subprocess.run([sys.executable, summ, "full", r, os.path.join(dst, js)], check=True,
                       stdout=subprocess.DEVNULL)
        with open(os.path.join(dst, det), "w") as f:
            subprocess.run(["ncu", "-i", r, "--page", "details"], stdout=f, stderr=subprocess.STDOUT, check=False)
    d = json.load(open(os.path.join(dst, "ncu_full_swap.json")))
    bulk = [x for x in d["launches"] if "bulk" in x["Kernel Name"]]
    if bulk:
        t_path = os.path.join(ROOT, "profiles", "traffic.json")
        t = json.load(open(t_path))
        t["per_path"]["bulk"]["dram_bytes_per_launch"] = sum(
            x["dram__bytes_read.sum"] + x["dram__bytes_write.sum"] for x in bulk) / len(bulk)
        with open(t_path, "w") as f:
            json.dump(t, f, indent=1)
    b = json.load(open(os.path.join(dst, "bench.json")))
    print(json.dumps({"value": b["value"], "frac": b["roofline"]["frac"],
                      "kernel": b["roofline"]["kernel"], "e2e": b["e2e"]["value"],
                      "gemm": (b.get("gemm_slowdown") or {}).get("slowdown"),
                      "gemm_ce": (b.get("gemm_slowdown_ce") or {}).get("slowdown")}))


if __name__ == "__main__":
    main()
