#!/usr/bin/env python
"""A/B of MPRESS_OPT_SPLIT (blocked vs dynamic claims, optionally strided) on
one B200, loopback peers: for each case, runs of R back-to-back swap-out
launches then R swap-in launches on one stream (the bench's timing: events
only around the runs, so PDL chains the launches), splits alternating round
by round.  Prints one JSON row per case with the median per-launch time and
GB/s of each split.

  python tools/split_ab.py [rounds]     # env SPLITS=0,2  PATHS=bulk,direct  VARIANTS=-1  CAPS=0  CASES=0,1
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_hpca_zhouwylbyx23_b200 as mp  # noqa: E402
from synth import device as synth_dev  # noqa: E402
from synth import workloads  # noqa: E402

PATHS = {"direct": mp.PATH_DIRECT, "bulk": mp.PATH_BULK, "auto": mp.PATH_AUTO}
CASES = [  # name, sizes, peers, launches per run
    ("cfg2 micro-batch 900 MiB -> 3", workloads.cfg2_sizes(1), 3, 8),
    ("cfg1 64 MiB (16 x 4 MiB) -> 1", workloads.cfg1_sizes(), 1, 16),
    ("16 MiB -> 3", [16 << 20], 3, 32),
    ("256 MiB -> 7", [256 << 20], 7, 8),
    ("4 GiB -> 7", [4 << 30], 7, 2),
    ("4 MiB -> 7", [4 << 20], 7, 64),
    ("32 MiB (8 x 4 MiB) -> 3", [4 << 20] * 8, 3, 32),
    ("128 MiB -> 3", [128 << 20], 3, 16),
    ("1 MiB -> 3", [1 << 20], 3, 64),
]


def run_case(sizes, peers_n, R, path, splits, rounds, cap, variant=-1):
    world = peers_n + 1
    peers = list(range(1, world))
    spare = workloads.spare_vector(world, 0, peers, spare=64 << 30)
    bw = workloads.bw_vector(world, 0, peers)
    pl = mp.plan(world, 0, spare, bw, sizes)
    part = [[0] * world for _ in range(world)]
    part[0] = [R * u * mp.DEFAULT_GRANULE for u in pl.units]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    ctx.set_option(mp.OPT_PATH, PATHS[path])
    ctx.set_option(mp.OPT_VARIANT, variant)
    ctx.set_option(mp.OPT_MAX_CTAS, cap)
    src = [torch.empty(s, dtype=torch.uint8, device="cuda") for s in sizes]
    for i, t in enumerate(src):
        synth_dev.fill(t, 77, i)
    dst = [torch.empty(s, dtype=torch.uint8, device="cuda") for s in sizes]
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    res = {sp: ([], []) for sp in splits}
    ok = True
    for r in range(rounds + 1):
        for sp in (splits if r % 2 == 0 else splits[::-1]):
            ctx.set_option(mp.OPT_SPLIT, sp)
            e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
            hs = [ctx.swap_out(pl, src, stream=s)]     # warm the stream (PDL predecessor)
            ctx.swap_in(hs[0], dst, stream=s)
            e[0].record(s)
            hs = hs + [ctx.swap_out(pl, src, stream=s) for _ in range(R - 1)]
            e[1].record(s)
            for h in hs[1:]:
                ctx.swap_in(h, dst, stream=s)
            e[2].record(s)
            torch.cuda.synchronize()
            for h in hs:
                h.free()
            if r > 0:
                res[sp][0].append(e[0].elapsed_time(e[1]) / (R - 1))
                res[sp][1].append(e[1].elapsed_time(e[2]) / (R - 1))
    ok = all(synth_dev.check(t, 77, i) == 0 for i, t in enumerate(dst))
    ctx.finalize()
    nbytes = sum(sizes)
    row = {"bit_exact": ok}
    for sp, (to, ti) in res.items():
        mo, mi = statistics.median(to), statistics.median(ti)
        row["split%d" % sp] = {"out_ms": mo, "in_ms": mi, "out_gbs": nbytes / mo / 1e6, "in_gbs": nbytes / mi / 1e6,
                               "hbm_frac_out": 2 * nbytes / mo / 1e6 / 6537.6,
                               "hbm_frac_in": 2 * nbytes / mi / 1e6 / 6537.6}
    return row


def main():
    rounds = int(sys.argv[1]) if len(sys.argv) > 1 else 6
    splits = [int(x) for x in os.environ.get("SPLITS", "0,2").split(",")]
    caps = [int(x) for x in os.environ.get("CAPS", "0").split(",")]
    only = os.environ.get("CASES")
    variants = [int(x) for x in os.environ.get("VARIANTS", "-1").split(",")]
    for path in os.environ.get("PATHS", "bulk,direct").split(","):
        for ci, (name, sizes, peers_n, R) in enumerate(CASES):
            if only and str(ci) not in only.split(","):
                continue
            for cap in caps:
                for var in variants:
                    row = run_case(sizes, peers_n, R, path, splits, rounds, cap, var)
                    print(json.dumps({"case": name, "path": path, "variant": var, "max_ctas": cap, **row}),
                          flush=True)


if __name__ == "__main__":
    main()
