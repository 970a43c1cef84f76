#!/usr/bin/env python
"""A/B of two libmpress builds on the same GPU: cfg2 micro-batch over 3
loopback peers at several grid caps, alternating builds (each in a fresh
process) so drift hits both.  usage: tools/ab.py libA.so libB.so [rounds]"""
import json
import os
import subprocess
import sys

CHILD = r'''
import json, os, statistics, sys, torch
sys.path.insert(0, os.getcwd())
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import device as synth_dev, workloads
sizes = workloads.cfg2_sizes(1); nbytes = sum(sizes)
world, peers = 4, [1, 2, 3]
spare = workloads.spare_vector(world, 0, peers, spare=64 << 30)
bw = workloads.bw_vector(world, 0, peers)
pl = mp.plan(world, 0, spare, bw, sizes)
part = [[0] * world for _ in range(world)]; part[0] = [u * 65536 for u in pl.units]
ctx = mp.Context.local(world, 0, [0] * world, part)
if os.environ.get("AB_PATH"):   # e.g. "bulk:5" (path:variant); default = AUTO
    nm, var = os.environ["AB_PATH"].split(":")
    ctx.set_option(mp.OPT_PATH, {"direct": mp.PATH_DIRECT, "bulk": mp.PATH_BULK}[nm])
    ctx.set_option(mp.OPT_VARIANT, int(var))
src = [torch.empty(s, dtype=torch.uint8, device="cuda") for s in sizes]
for i, t in enumerate(src): synth_dev.fill(t, 1, i)
dst = [torch.empty(s, dtype=torch.uint8, device="cuda") for s in sizes]
s = torch.cuda.Stream(); out = {}
for cap in [int(x) for x in os.environ["CAPS"].split(",")]:
    ctx.set_option(mp.OPT_MAX_CTAS, cap)
    ts = []
    for r in range(14):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s); h = ctx.swap_out(pl, src, stream=s); ctx.swap_in(h, dst, stream=s); e1.record(s); h.free()
        ts.append((e0, e1))
    torch.cuda.synchronize()
    out[cap] = 2 * nbytes / statistics.median(a.elapsed_time(b) for a, b in ts[4:]) / 1e6
print(json.dumps(out))
ctx.finalize()
'''


def main():
    libs = sys.argv[1:3]
    rounds = int(sys.argv[3]) if len(sys.argv) > 3 else 3
    env = dict(os.environ, CAPS=os.environ.get("CAPS", "0,8,32,64,148,296"))
    res = {l: [] for l in libs}
    for _ in range(rounds):
        for l in libs:
            r = subprocess.run([sys.executable, "-c", CHILD], env=dict(env, MPRESS_LIB=l),
                               capture_output=True, text=True)
            if r.returncode != 0:
                print(r.stderr[-2000:])
                continue
            res[l].append(json.loads(r.stdout.strip().splitlines()[-1]))
    for l in libs:
        caps = res[l][0].keys() if res[l] else []
        print(os.path.basename(l), {c: round(max(x[c] for x in res[l])) for c in caps})


if __name__ == "__main__":
    main()
