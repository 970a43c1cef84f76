"""Helpers for the GPU parity tests: run a swap through the C ABI on seeded
inputs and compare with the oracle byte model element by element."""
import numpy as np
import torch

import oracle
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import device as synth_dev
from synth import splitmix64_bytes


def loopback_ctx(world, source, pl_units, G, copies=1, extra=0):
    """1-GPU loopback context with room for `copies` handles of a plan."""
    part = [[0] * world for _ in range(world)]
    for p in range(world):
        if pl_units[p]:
            part[source][p] = copies * pl_units[p] * G + extra
    return mp.Context.local(world, source, [0] * world, part)


def make_inputs(sizes, seed):
    ts = []
    for i, s in enumerate(sizes):
        t = torch.empty(s, dtype=torch.uint8, device="cuda")
        synth_dev.fill(t, seed, i)
        ts.append(t)
    torch.cuda.synchronize()
    return ts


def host_inputs(sizes, seed):
    return [splitmix64_bytes(seed, i, 0, s) for i, s in enumerate(sizes)]


def check_stash(ctx, handle, o_plan, host_tensors):
    """Every defined stash byte equals the oracle byte model's."""
    model = oracle.swap_out(o_plan, host_tensors)
    slices = handle.slices()
    for p, (buf, defined) in model.items():
        got = np.frombuffer(ctx.peer_read(p, slices[p], len(buf)), dtype=np.uint8)
        bad = np.nonzero((got != buf) & defined)[0]
        assert bad.size == 0, "peer %d: %d stash bytes differ, first at %d" % (p, bad.size, bad[0])


def run_roundtrip(sizes, world, source, spare, bw, G=0, seed=1, path=mp.PATH_DIRECT,
                  max_ctas=0, check_stash_bytes=True):
    o = oracle.plan(world, source, spare, bw, sizes, G)
    pl = mp.plan(world, source, spare, bw, sizes, G)
    assert pl.stripes == [tuple(s) for s in o["stripes"]]
    ctx = loopback_ctx(world, source, pl.units, o["G"])
    try:
        ctx.set_option(mp.OPT_PATH, path)
        ctx.set_option(mp.OPT_MAX_CTAS, max_ctas)
        src = make_inputs(sizes, seed)
        host = host_inputs(sizes, seed)
        s = torch.cuda.Stream()
        h = ctx.swap_out(pl, src, stream=s)
        s.synchronize()
        assert ctx.query(h) and h.state == mp.STATE_OUT
        if check_stash_bytes:
            check_stash(ctx, h, o, host)
        for t in src:  # poison the sources: the data must come back from the stash
            t.fill_(0xA5)
        dst = [torch.full((n,), 0x5A, dtype=torch.uint8, device="cuda") for n in sizes]
        ctx.swap_in(h, dst, stream=s)
        ctx.wait(h, torch.cuda.current_stream())
        torch.cuda.synchronize()
        assert ctx.query(h) and h.state == mp.STATE_IN
        for i, (d, e) in enumerate(zip(dst, host)):
            got = d.cpu().numpy()
            assert np.array_equal(got, e), "tensor %d differs after the round trip" % i
        h.free()
    finally:
        ctx.finalize()
    return o
