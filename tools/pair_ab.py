#!/usr/bin/env python
"""Round trips (swap-out + swap-in pairs, as a pipeline issues them) per
kernel shape: single pair (host latency included) and R pairs back to back.
  python tools/pair_ab.py        # env SIZES_MIB=4,16,64 PEERS=7 SHAPES=bulk:-1,bulk:3,bulk:0,direct:5,direct:1
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


def main():
    peers_n = int(os.environ.get("PEERS", "7"))
    shapes = [x.split(":") for x in os.environ.get("SHAPES", "bulk:-1,bulk:3,bulk:0,direct:5,direct:1").split(",")]
    world = peers_n + 1
    peers = list(range(1, world))
    for mib in [float(x) for x in os.environ.get("SIZES_MIB", "4,16,64").split(",")]:
        sizes = [int(mib * (1 << 20))]
        spare = workloads.spare_vector(world, 0, peers, spare=8 << 30)
        bw = workloads.bw_vector(world, 0, peers)
        pl = mp.plan(world, 0, spare, bw, sizes)
        part = [[0] * world for _ in range(world)]
        part[0] = [40 * u * mp.DEFAULT_GRANULE for u in pl.units]
        ctx = mp.Context.local(world, 0, [0] * world, part)
        src = [torch.empty(b, dtype=torch.uint8, device="cuda") for b in sizes]
        dst = [torch.empty(b, dtype=torch.uint8, device="cuda") for b in sizes]
        for i, t in enumerate(src):
            synth_dev.fill(t, 5, i)
        torch.cuda.synchronize()
        s = torch.cuda.Stream()
        for name, var in shapes:
            ctx.set_option(mp.OPT_PATH, PATHS[name])
            if name != "auto":
                ctx.set_option(mp.OPT_VARIANT, int(var))
            single, b2b = [], []
            for r in range(8):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                h = ctx.swap_out(pl, src, stream=s)
                ctx.swap_in(h, dst, stream=s)
                e1.record(s)
                torch.cuda.synchronize()
                h.free()
                if r >= 2:
                    single.append(e0.elapsed_time(e1))
                R = 32
                h0 = ctx.swap_out(pl, src, stream=s)
                ctx.swap_in(h0, dst, stream=s)
                hs = [h0]
                e0.record(s)
                for _ in range(R):
                    h = ctx.swap_out(pl, src, stream=s)
                    ctx.swap_in(h, dst, stream=s)
                    hs.append(h)
                e1.record(s)
                torch.cuda.synchronize()
                for h in hs:
                    h.free()
                if r >= 2:
                    b2b.append(e0.elapsed_time(e1) / R)
            ok = all(synth_dev.check(t, 5, i) == 0 for i, t in enumerate(dst))
            n = 2 * sum(sizes)
            print(json.dumps({"mib": mib, "peers": peers_n, "shape": "%s:%s" % (name, var),
                              "single_us": statistics.median(single) * 1e3,
                              "b2b_us": statistics.median(b2b) * 1e3,
                              "single_gbs": n / statistics.median(single) / 1e6,
                              "b2b_gbs": n / statistics.median(b2b) / 1e6, "bit_exact": ok}), flush=True)
        ctx.finalize()


if __name__ == "__main__":
    main()
