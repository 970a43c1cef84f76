#!/usr/bin/env python
"""Diagnostic: one large tensor over P loopback peers; after swap-in, count
mismatched bytes per stripe (device check against the generator)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import device as synth_dev, workloads

size = int(sys.argv[1]) if len(sys.argv) > 1 else 4 << 30
P = int(sys.argv[2]) if len(sys.argv) > 2 else 7
mode = sys.argv[3] if len(sys.argv) > 3 else "del"
world = P + 1
peers = list(range(1, world))
spare = workloads.spare_vector(world, 0, peers, spare=8 << 30)
bw = workloads.bw_vector(world, 0, peers)
pl = mp.plan(world, 0, spare, bw, [size])
part = [[0] * world for _ in range(world)]
part[0] = [u * 65536 for u in pl.units]
ctx = mp.Context.local(world, 0, [0] * world, part)
src = torch.empty(size, dtype=torch.uint8, device="cuda")
synth_dev.fill(src, 4000, 0)
s = torch.cuda.Stream()
torch.cuda.synchronize()
h = ctx.swap_out(pl, [src], stream=s)
s.synchronize()
print("src ok before:", synth_dev.check(src, 4000, 0))
if mode == "del":
    del src
    torch.cuda.empty_cache()
dst = torch.empty(size, dtype=torch.uint8, device="cuda")
ctx.swap_in(h, [dst], stream=s)
s.synchronize()
print("mode", mode, "launches", ctx.last_launches)
for (i, p, so, do, ln) in pl.stripes:
    bad = synth_dev.check(dst[so:so + ln], 4000, 0, so)
    print("stripe peer", p, "src_off", so, "len", ln, "bad", bad)
