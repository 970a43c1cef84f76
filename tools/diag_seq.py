#!/usr/bin/env python
"""Diagnostic: run the config-3 round trip, then config 4 (4 GiB, 7 peers) in
one process, as tests/test_gpu_fullsize.py does; report per-stripe errors."""
import os, sys, random
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import device as synth_dev, workloads, splitmix64_bytes


def run(world, spare, bw, sizes, seed, reads=True):
    pl = mp.plan(world, 0, spare, bw, sizes)
    part = [[0] * world for _ in range(world)]
    part[0] = [u * 65536 for u in pl.units]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    src = []
    for i, n in enumerate(sizes):
        t = torch.empty(n, dtype=torch.uint8, device="cuda")
        synth_dev.fill(t, seed, i)
        src.append(t)
    torch.cuda.synchronize()   # fills ran on the current stream
    s = torch.cuda.Stream()
    h = ctx.swap_out(pl, src, stream=s)
    s.synchronize()
    sl = h.slices()
    if reads:
        for (i, p, so, do, ln) in pl.stripes[:20]:
            got = np.frombuffer(ctx.peer_read(p, sl[p] + do, min(4096, ln)), dtype=np.uint8)
            assert np.array_equal(got, splitmix64_bytes(seed, i, so, min(4096, ln)))
    del src
    torch.cuda.empty_cache()
    dst = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
    ctx.swap_in(h, dst, stream=s)
    s.synchronize()
    tot = 0
    for (i, p, so, do, ln) in pl.stripes:
        bad = synth_dev.check(dst[i][so:so + ln], seed, i, so)
        tot += bad
        if bad:
            print("  BAD stripe t%d peer %d off %d len %d: %d" % (i, p, so, ln, bad))
    whole = sum(synth_dev.check(d, seed, i) for i, d in enumerate(dst))
    print("seed", seed, "stripe-bad", tot, "whole-bad", whole, flush=True)
    h.free()
    ctx.finalize()


c = workloads.CONFIGS[3]
run(8, workloads.spare_vector(8, 0, c["peers"], spare_by_peer=c["spare_by_peer"]),
    workloads.bw_vector(8, 0, c["peers"]), workloads.cfg3_sizes(), 3000)
peers = list(range(1, 8))
run(8, workloads.spare_vector(8, 0, peers, spare=8 << 30), workloads.bw_vector(8, 0, peers), [4 << 30], 4000)
run(8, workloads.spare_vector(8, 0, peers, spare=8 << 30), workloads.bw_vector(8, 0, peers), [4 << 30], 4001)
