#!/usr/bin/env python
"""Copy one tools/profile_round.sh run (gpurun_out/<tag>/, already summarised
on the GPU box: the .ncu-rep files stay there) into profiles/<round>/ (run
here, no GPU needed): bench line, ncu launch list (gzipped) + its summary,
the two ncu --set full summaries and details pages, the GPU test log and
smoke log, and the bulk path's DRAM bytes per launch into
profiles/traffic.json (bench.py's roofline.traffic).

  python tools/refresh_profiles.py gpurun_out/r02e profiles/r02
"""
import gzip
import json
import os
import shutil
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
FILES = ("bench.json", "bench_wall.txt", "launches_summary.json", "ncu_full_swap.json",
         "ncu_full_swap_capped.json", "ncu_full_details.txt", "ncu_full_capped_details.txt",
         "pytest_gpu.log", "smoke.log")


def main():
    src, dst = sys.argv[1], sys.argv[2]
    os.makedirs(dst, exist_ok=True)
    for f in FILES:
        if os.path.exists(os.path.join(src, f)):
            shutil.copy(os.path.join(src, f), os.path.join(dst, f))
    csv = os.path.join(src, "launches.csv")
    if os.path.exists(csv):
        with open(csv, "rb") as i, gzip.open(os.path.join(dst, "launches.csv.gz"), "wb") as o:
            shutil.copyfileobj(i, o)
    d = json.load(open(os.path.join(dst, "ncu_full_swap.json")))
    bulk = [x for x in d["launches"] if "bulk" in x["Kernel Name"]]
    if bulk:
        t_path = os.path.join(ROOT, "profiles", "traffic.json")
        t = json.load(open(t_path))
        per = sum(x["dram__bytes_read.sum"] + x["dram__bytes_write.sum"] for x in bulk) / len(bulk)
        t["per_path"]["bulk"] = {"dram_bytes_per_launch": per,
                                 "source": "%s/ncu_full_swap.json (bulk shape 3, full grid; mean of the "
                                           "swap-out and swap-in launch)" % os.path.relpath(dst, ROOT)}
        with open(t_path, "w") as f:
            json.dump(t, f, indent=1)
    print("copied", src, "->", dst)


if __name__ == "__main__":
    main()
